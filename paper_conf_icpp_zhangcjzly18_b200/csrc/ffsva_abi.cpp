// ffsva_abi.cpp — the extern "C" entry points of include/ffsva.h: argument validation (always before any GPU
// work), per-device locking, and dispatch into the runtime.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <memory>
#include <vector>

#include "ffsva_runtime.h"

using namespace ffsva;

namespace ffsva {
const char* last_error();
}

namespace {

ffsva_status validate_desc(const ffsva_stream_desc* d) {
  if (!d) return fail(FFSVA_EINVAL, "desc is NULL");
  if (d->sdd_w < 2 || d->sdd_h < 2 || d->sdd_w > 4096 || d->sdd_h > 4096 || (d->sdd_w & 1) || (d->sdd_h & 1))
    return fail(FFSVA_EINVAL, "sdd grid must be even and in [2, 4096]");
  if (d->snm_w * 2 != d->sdd_w || d->snm_h * 2 != d->sdd_h)
    return fail(FFSVA_EINVAL, "snm grid must be half the sdd grid (50x50 vs 100x100)");
  if (d->width < d->sdd_w || d->height < d->sdd_h) return fail(FFSVA_EINVAL, "frame smaller than the SDD grid");
  if (d->width > 16384) return fail(FFSVA_EINVAL, "width > 16384");
  if ((int64_t)d->height > 256LL * d->sdd_h) return fail(FFSVA_EINVAL, "height > 256 * sdd_h");
  if (d->height > 65535) return fail(FFSVA_EINVAL, "height > 65535");
  if (d->row_pitch < 3LL * d->width) return fail(FFSVA_EINVAL, "row_pitch < 3 * width");
  if (!(d->delta_diff >= 0.0) || !std::isfinite(d->delta_diff)) return fail(FFSVA_EINVAL, "delta_diff < 0");
  if (!(d->c_low >= 0.f && d->c_low <= d->c_high && d->c_high <= 1.f))
    return fail(FFSVA_EINVAL, "need 0 <= c_low <= c_high <= 1");
  if (!(d->filter_degree >= 0.f && d->filter_degree <= 1.f))
    return fail(FFSVA_EINVAL, "filter_degree must lie in [0, 1] (PAPER.md L193)");
  if (d->snm_batch < 1) return fail(FFSVA_EINVAL, "snm_batch < 1");
  if (d->q_sdd < 0 || d->q_snm < 0) return fail(FFSVA_EINVAL, "negative queue threshold");
  if (d->distance < FFSVA_DIST_MSE || d->distance > FFSVA_DIST_NRMSE)
    return fail(FFSVA_EINVAL, "distance must be FFSVA_DIST_MSE, _SAD or _NRMSE");
  if (d->ref_mode != FFSVA_REF_BACKGROUND && d->ref_mode != FFSVA_REF_PREVIOUS)
    return fail(FFSVA_EINVAL, "ref_mode must be FFSVA_REF_BACKGROUND or FFSVA_REF_PREVIOUS");
  if (d->number_of_objects < 0) return fail(FFSVA_EINVAL, "number_of_objects < 0");
  if (d->target_class < 0 || d->target_class >= 20) return fail(FFSVA_EINVAL, "target_class must be a VOC class 0..19");
  if (d->q_tyolo < 0) return fail(FFSVA_EINVAL, "negative queue threshold");
  if (d->ref_mode == FFSVA_REF_PREVIOUS && d->distance == FFSVA_DIST_NRMSE)
    return fail(FFSVA_EINVAL, "NRMSE needs a fixed reference (its normaliser is sum R^2)");
  return FFSVA_OK;
}

// Shared validation of a frame list: streams present, one device, state loaded.
ffsva_status validate_frames(const ffsva_frame* frames, int32_t n, bool need_snm, DeviceCtx** ctx_out) {
  if (n < 0) return fail(FFSVA_EINVAL, "n < 0");
  if (n > 0 && !frames) return fail(FFSVA_EINVAL, "frames is NULL");
  DeviceCtx* ctx = nullptr;
  for (int32_t i = 0; i < n; ++i) {
    const ffsva_stream* s = frames[i].stream;
    if (!s) return fail(FFSVA_EINVAL, "frame without stream");
    if (!frames[i].pixels) return fail(FFSVA_EINVAL, "frame without pixels");
    if (!ctx) ctx = s->ctx;
    if (s->ctx != ctx) return fail(FFSVA_EDEVICE, "frames of one batch live on several devices");
    if (!s->has_ref) return fail(FFSVA_ESTATE, "stream has no reference image (ffsva_set_reference)");
    if (need_snm && !s->has_snm) return fail(FFSVA_ESTATE, "stream has no SNM (ffsva_snm_load)");
  }
  if (ctx && ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  *ctx_out = ctx;
  return FFSVA_OK;
}

}  // namespace

extern "C" {

FFSVA_API const char* ffsva_version(void) { return "ffsva-b200 0.1 (sm_100a)"; }
FFSVA_API const char* ffsva_last_error(void) { return ffsva::last_error(); }
FFSVA_API uint64_t ffsva_kernel_launches(void) { return g_launches.load(); }

FFSVA_API ffsva_status ffsva_open_stream(const ffsva_stream_desc* desc, ffsva_stream** out) {
  if (!out) return fail(FFSVA_EINVAL, "out is NULL");
  ffsva_status st = validate_desc(desc);
  if (st != FFSVA_OK) return st;
  DeviceCtx* ctx = ctx_acquire(desc->device, &st);
  if (!ctx) return st;
  std::unique_ptr<ffsva_stream> s(new ffsva_stream());
  s->desc = *desc;
  s->ctx = ctx;
  {
    std::lock_guard<std::mutex> lk(ctx->mu);
    if (!ctx->free_slots.empty()) {
      s->slot = ctx->free_slots.back();
      ctx->free_slots.pop_back();
    } else if (ctx->next_slot < ctx->stats_cap) {
      s->slot = ctx->next_slot++;
    }
  }
  if (s->slot < 0) {
    ctx_release(ctx);
    return fail(FFSVA_ENOMEM, "too many open streams on this device");
  }
  const uint64_t nvals = 3ull * (uint64_t)desc->sdd_w * (uint64_t)desc->sdd_h;
  s->T = stream_threshold(*desc, 0);  // NRMSE: recomputed from sum R^2 by ffsva_set_reference
  const double tpre = ((double)desc->c_high - (double)desc->c_low) * (double)desc->filter_degree + (double)desc->c_low;
  s->L_t = logit_of(tpre);
  s->L_low = logit_of(desc->c_low);
  s->L_high = logit_of(desc->c_high);
  {
    DeviceGuard g(ctx->device);
    const size_t rbytes = ((size_t)nvals + 15) & ~(size_t)15;  // K1's band kernel bulk-copies 16-B aligned R spans
    cudaError_t e = cudaMalloc(&s->d_ref, rbytes);
    if (e == cudaSuccess) e = cudaMalloc(&s->d_snm, snm::BLOB_BYTES);
    if (e != cudaSuccess) {
      cudaFree(s->d_ref);
      cudaFree(s->d_snm);
      {
        std::lock_guard<std::mutex> lk(ctx->mu);
        ctx->free_slots.push_back(s->slot);
      }
      ctx_release(ctx);
      return cuda_fail(nullptr, e, "cudaMalloc(stream state)");
    }
    // a fresh slot starts with zero statistics
    cudaMemset(ctx->d_stats + (size_t)s->slot * NSTAT, 0, sizeof(unsigned long long) * NSTAT);
    std::lock_guard<std::mutex> lk(ctx->lat_mu);
    std::fill_n(ctx->h_lat.begin() + (std::ptrdiff_t)s->slot * NLAT, NLAT, 0);
  }
  *out = s.release();
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_close(ffsva_stream* s) {
  if (!s) return FFSVA_OK;
  DeviceCtx* ctx = s->ctx;
  {
    std::lock_guard<std::mutex> lk(ctx->mu);
    DeviceGuard g(ctx->device);
    cudaDeviceSynchronize();
    cudaFree(s->d_ref);
    cudaFree(s->d_snm);
    ctx->free_slots.push_back(s->slot);
  }
  delete s;
  ctx_release(ctx);
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_set_reference(ffsva_stream* s, const uint8_t* frames, int32_t k, int64_t frame_stride) {
  if (!s || !frames) return fail(FFSVA_EINVAL, "NULL argument");
  if (k < 1) return fail(FFSVA_EINVAL, "k < 1");
  const ffsva_stream_desc& d = s->desc;
  const int64_t fbytes = (int64_t)(d.height - 1) * d.row_pitch + 3LL * d.width;
  if (k > 1 && frame_stride < fbytes) return fail(FFSVA_EINVAL, "frame_stride smaller than a frame");
  if (k == 1 && frame_stride < 0) return fail(FFSVA_EINVAL, "frame_stride < 0");
  DeviceCtx* ctx = s->ctx;
  if (ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  std::lock_guard<std::mutex> lk(ctx->mu);
  DeviceGuard g(ctx->device);
  cudaPointerAttributes attr;
  bool on_device = false;
  if (cudaPointerGetAttributes(&attr, frames) == cudaSuccess)
    on_device = (attr.type == cudaMemoryTypeDevice || attr.type == cudaMemoryTypeManaged) && attr.device == ctx->device;
  else
    cudaGetLastError();
  const size_t total = (size_t)(k - 1) * (size_t)frame_stride + (size_t)fbytes;
  uint8_t* src = const_cast<uint8_t*>(frames);
  uint8_t* tmp = nullptr;
  cudaError_t e;
  if (!on_device) {
    if ((e = cudaMalloc(&tmp, total)) != cudaSuccess) return cuda_fail(nullptr, e, "cudaMalloc(reference staging)");
    if ((e = cudaMemcpy(tmp, frames, total, cudaMemcpyHostToDevice)) != cudaSuccess) {
      cudaFree(tmp);
      return cuda_fail(ctx, e, "cudaMemcpy(reference frames)");
    }
    src = tmp;
  }
  e = launch_reference(src, k, frame_stride, d.width, d.height, d.row_pitch, d.sdd_w, d.sdd_h, s->d_ref, nullptr);
  g_launches += 1;
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  cudaFree(tmp);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "reference kernel");
  if (d.distance == FFSVA_DIST_NRMSE) {
    // the NRMSE threshold floor(delta^2 * sum R^2) (Q24) depends on R: one 30 KB read-back per call
    std::vector<uint8_t> r(3ull * d.sdd_w * d.sdd_h);
    if ((e = cudaMemcpy(r.data(), s->d_ref, r.size(), cudaMemcpyDeviceToHost)) != cudaSuccess)
      return cuda_fail(ctx, e, "cudaMemcpy(reference sum of squares)");
    uint64_t q = 0;
    for (uint8_t v : r) q += (uint64_t)v * v;
    s->ref_sum_sq = q;
    s->T = stream_threshold(d, q);
  }
  s->has_ref = true;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_get_reference(ffsva_stream* s, uint8_t* out) {
  if (!s || !out) return fail(FFSVA_EINVAL, "NULL argument");
  if (!s->has_ref) return fail(FFSVA_ESTATE, "no reference image");
  std::lock_guard<std::mutex> lk(s->ctx->mu);
  DeviceGuard g(s->ctx->device);
  cudaError_t e = cudaMemcpy(out, s->d_ref, 3ull * s->desc.sdd_w * s->desc.sdd_h, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return cuda_fail(s->ctx, e, "cudaMemcpy(reference)");
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_snm_load(ffsva_stream* s, const ffsva_snm_desc* d, const float* params,
                                      int64_t n_params) {
  if (!s || !d || !params) return fail(FFSVA_EINVAL, "NULL argument");
  if (d->c1 != snm::C1 || d->c2 != snm::C2) return fail(FFSVA_EINVAL, "the kernels implement c1 = 16, c2 = 32");
  if (s->desc.snm_w != snm::IN || s->desc.snm_h != snm::IN)
    return fail(FFSVA_EINVAL, "the SNM kernel takes a 50x50 input (snm_w = snm_h = 50)");
  if (n_params != snm::N_PARAMS) return fail(FFSVA_EINVAL, "n_params != 9697");
  for (int64_t i = 0; i < n_params; ++i)
    if (!std::isfinite(params[i])) return fail(FFSVA_EINVAL, "non-finite SNM parameter");
  std::unique_ptr<uint8_t[]> blob(new uint8_t[snm::BLOB_BYTES]);
  pack_snm_blob(params, blob.get());
  DeviceCtx* ctx = s->ctx;
  if (ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  std::lock_guard<std::mutex> lk(ctx->mu);
  DeviceGuard g(ctx->device);
  cudaError_t e = cudaMemcpy(s->d_snm, blob.get(), snm::BLOB_BYTES, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaMemcpy(SNM weights)");
  s->has_snm = true;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_filter_batch(const ffsva_frame* frames, int32_t n, ffsva_result* results,
                                          void* cuda_stream) {
  if (n > 0 && !results) return fail(FFSVA_EINVAL, "results is NULL");
  DeviceCtx* ctx = nullptr;
  ffsva_status st = validate_frames(frames, n, true, &ctx);
  if (st != FFSVA_OK || n == 0) return st;
  std::lock_guard<std::mutex> lk(ctx->mu);
  DeviceGuard g(ctx->device);
  if (!ctx->scratch) ctx->scratch = new Batch();
  cudaStream_t cs = (cudaStream_t)cuda_stream;
  st = batch_build(ctx, ctx->scratch, frames, n, false, false, cs);
  if (st != FFSVA_OK) return st;
  st = batch_run(ctx->scratch, cs, false);
  if (st != FFSVA_OK) return st;
  return batch_fetch(ctx->scratch, results, cs);
}

FFSVA_API ffsva_status ffsva_sdd_batch(const ffsva_frame* frames, int32_t n, uint8_t* d100, uint8_t* d50,
                                       uint64_t* ssd, uint8_t* sdd_pass, void* cuda_stream) {
  DeviceCtx* ctx = nullptr;
  ffsva_status st = validate_frames(frames, n, false, &ctx);
  if (st != FFSVA_OK || n == 0) return st;
  std::lock_guard<std::mutex> lk(ctx->mu);
  DeviceGuard g(ctx->device);
  if (!ctx->scratch) ctx->scratch = new Batch();
  Batch* b = ctx->scratch;
  cudaStream_t cs = (cudaStream_t)cuda_stream;
  st = batch_build(ctx, b, frames, n, true, d100 != nullptr, cs);
  if (st != FFSVA_OK) return st;
  st = batch_run(b, cs, false);
  if (st != FFSVA_OK) return st;
  cudaError_t e = cudaSuccess;
  const size_t n100 = 3ull * b->sdd_w * b->sdd_h, n50 = n100 / 4;
  if (d100 && e == cudaSuccess) e = cudaMemcpyAsync(d100, b->d_d100, n100 * n, cudaMemcpyDeviceToHost, cs);
  if (d50 && e == cudaSuccess)
    e = cudaMemcpy2DAsync(d50, n50, b->d_d50, (size_t)b->d50_stride, n50, n, cudaMemcpyDeviceToHost, cs);
  if (ssd && e == cudaSuccess) e = cudaMemcpyAsync(ssd, b->d_ssd, 8ull * n, cudaMemcpyDeviceToHost, cs);
  if (sdd_pass && e == cudaSuccess) e = cudaMemcpyAsync(sdd_pass, b->d_pass, (size_t)n, cudaMemcpyDeviceToHost, cs);
  if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_sdd_batch copies");
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_batch_prepare(const ffsva_frame* frames, int32_t n, ffsva_batch** out) {
  if (!out) return fail(FFSVA_EINVAL, "out is NULL");
  if (n < 1) return fail(FFSVA_EINVAL, "a prepared batch needs n >= 1");
  DeviceCtx* ctx = nullptr;
  ffsva_status st = validate_frames(frames, n, true, &ctx);
  if (st != FFSVA_OK) return st;
  std::lock_guard<std::mutex> lk(ctx->mu);
  DeviceGuard g(ctx->device);
  std::unique_ptr<ffsva_batch> b(new ffsva_batch());
  cudaStream_t tmp;
  cudaError_t e = cudaStreamCreateWithFlags(&tmp, cudaStreamNonBlocking);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaStreamCreate");
  st = batch_build(ctx, b.get(), frames, n, false, false, tmp);
  cudaStreamDestroy(tmp);
  if (st != FFSVA_OK) {
    batch_free(b.get());
    return st;
  }
  *out = b.release();
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_batch_launch(ffsva_batch* b, void* cuda_stream) {
  if (!b) return fail(FFSVA_EINVAL, "batch is NULL");
  if (b->ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  std::lock_guard<std::mutex> lk(b->ctx->mu);
  DeviceGuard g(b->ctx->device);
  return batch_run(b, (cudaStream_t)cuda_stream, true);
}

FFSVA_API ffsva_status ffsva_batch_fetch(ffsva_batch* b, ffsva_result* results, void* cuda_stream) {
  if (!b) return fail(FFSVA_EINVAL, "batch is NULL");
  std::lock_guard<std::mutex> lk(b->ctx->mu);
  DeviceGuard g(b->ctx->device);
  return batch_fetch(b, results, (cudaStream_t)cuda_stream);
}

FFSVA_API ffsva_status ffsva_batch_device_outputs(ffsva_batch* b, uint64_t** ssd, uint8_t** sdd_pass,
                                                  int32_t** survivor_idx, float** logit, uint8_t** snm_pass,
                                                  uint8_t** snm_class, uint8_t** d50, int64_t* d50_stride,
                                                  int32_t** n_survivors) {
  if (!b) return fail(FFSVA_EINVAL, "batch is NULL");
  if (ssd) *ssd = b->d_ssd;
  if (sdd_pass) *sdd_pass = b->d_pass;
  if (survivor_idx) *survivor_idx = b->d_surv;
  if (logit) *logit = b->d_logit;
  if (snm_pass) *snm_pass = b->d_snm_pass;
  if (snm_class) *snm_class = b->d_snm_class;
  if (d50) *d50 = b->d_d50;
  if (d50_stride) *d50_stride = b->d50_stride;
  if (n_survivors) *n_survivors = b->d_counts;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_batch_destroy(ffsva_batch* b) {
  if (!b) return FFSVA_OK;
  {
    std::lock_guard<std::mutex> lk(b->ctx->mu);
    DeviceGuard g(b->ctx->device);
    cudaDeviceSynchronize();
    batch_free(b);
  }
  delete b;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_batch_profile(ffsva_batch* const* batches, int32_t nb, int32_t iters,
                                           float* ms_out, void* cuda_stream) {
  if (!batches || nb < 1 || iters < 1 || !ms_out) return fail(FFSVA_EINVAL, "bad argument");
  DeviceCtx* ctx = batches[0] ? batches[0]->ctx : nullptr;
  for (int32_t j = 0; j < nb; ++j)
    if (!batches[j] || batches[j]->ctx != ctx) return fail(FFSVA_EINVAL, "batches must be non-NULL, one device");
  if (ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  std::lock_guard<std::mutex> lk(ctx->mu);
  DeviceGuard g(ctx->device);
  std::vector<Batch*> bs(batches, batches + nb);
  return batch_profile(bs.data(), nb, iters, ms_out, (cudaStream_t)cuda_stream);
}

FFSVA_API ffsva_status ffsva_stream_info(ffsva_stream* s, int32_t* slot, int32_t* device) {
  if (!s) return fail(FFSVA_EINVAL, "stream is NULL");
  if (slot) *slot = s->slot;
  if (device) *device = s->ctx->device;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_stats_copy(int32_t device, uint64_t* dst, int32_t max_slots, int32_t* slots,
                                        int32_t dst_is_host, int32_t reset, void* cuda_stream) {
  if (!dst || max_slots < 0) return fail(FFSVA_EINVAL, "bad argument");
  ffsva_status st;
  DeviceCtx* ctx = ctx_acquire(device, &st);  // only used to look the context up; released below
  if (!ctx) return st;
  ffsva_status out = FFSVA_OK;
  {
    std::lock_guard<std::mutex> lk(ctx->mu);
    DeviceGuard g(ctx->device);
    const int32_t used = ctx->next_slot;
    if (slots) *slots = used;
    const int32_t ncopy = used < max_slots ? used : max_slots;
    cudaStream_t cs = (cudaStream_t)cuda_stream;
    cudaError_t e = cudaSuccess;
    // kernel counters (device table, stride NSTAT) into columns 0..7, the online runtime's latency columns (host
    // table, stride NLAT) into columns 8..23 of the FFSVA_NSTAT-wide rows. Device destinations get the latency
    // columns from a pinned snapshot, so the whole copy stays asynchronous on cs (no host synchronisation).
    const size_t row = sizeof(uint64_t) * FFSVA_NSTAT;
    std::vector<uint64_t> lat;
    uint64_t* snap = nullptr;
    if (!dst_is_host && ncopy > 0) {
      if (!ctx->h_lat_pinned) {
        e = cudaMallocHost(&ctx->h_lat_pinned, sizeof(uint64_t) * NLAT * (size_t)ctx->stats_cap);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->lat_ev, cudaEventDisableTiming);
      }
      if (e == cudaSuccess) e = cudaEventSynchronize(ctx->lat_ev);  // the previous snapshot's copy has run
      snap = ctx->h_lat_pinned;
    }
    if (e == cudaSuccess) {
      std::lock_guard<std::mutex> lk2(ctx->lat_mu);
      if (snap) std::copy(ctx->h_lat.begin(), ctx->h_lat.begin() + (std::ptrdiff_t)ncopy * NLAT, snap);
      else lat.assign(ctx->h_lat.begin(), ctx->h_lat.begin() + (std::ptrdiff_t)ncopy * NLAT);
      if (reset) std::fill(ctx->h_lat.begin(), ctx->h_lat.end(), 0);
    }
    if (e == cudaSuccess && ncopy > 0) {
      e = cudaMemcpy2DAsync(dst, row, ctx->d_stats, sizeof(uint64_t) * NSTAT, sizeof(uint64_t) * NSTAT, (size_t)ncopy,
                            dst_is_host ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice, cs);
      if (e == cudaSuccess && snap) {
        e = cudaMemcpy2DAsync(dst + NSTAT, row, snap, sizeof(uint64_t) * NLAT, sizeof(uint64_t) * NLAT,
                              (size_t)ncopy, cudaMemcpyHostToDevice, cs);
        if (e == cudaSuccess) e = cudaEventRecord(ctx->lat_ev, cs);
      }
    }
    if (e == cudaSuccess && reset) e = cudaMemsetAsync(ctx->d_stats, 0, sizeof(uint64_t) * NSTAT * ctx->stats_cap, cs);
    if (e == cudaSuccess && dst_is_host) {
      e = cudaStreamSynchronize(cs);
      for (int32_t i = 0; i < ncopy; ++i)
        std::memcpy(dst + (size_t)i * FFSVA_NSTAT + NSTAT, lat.data() + (size_t)i * NLAT, sizeof(uint64_t) * NLAT);
    }
    if (e != cudaSuccess) out = cuda_fail(ctx, e, "ffsva_stats_copy");
  }
  ctx_release(ctx);
  return out;
}

// ---------------------------------------------------------------- stream images (re-forwarding)
namespace {
constexpr uint32_t kImageMagic = 0x56534646u;  // "FFSV"
constexpr uint32_t kImageVersion = 4;  // 4: statistics row with the latency columns (FFSVA_NSTAT = 24)
constexpr int64_t kImageHeader = 256;
struct ImageHeader {
  uint32_t magic, version;
  ffsva_stream_desc desc;
  uint64_t T, ref_sum_sq;
  int64_t ref_bytes, snm_bytes, stats_bytes, total;
  uint8_t has_ref, has_snm, pad[6];
};
static_assert(sizeof(ImageHeader) <= kImageHeader, "image header");
int64_t al16(int64_t x) { return (x + 15) & ~(int64_t)15; }
int64_t image_bytes(const ffsva_stream_desc& d) {
  return kImageHeader + al16(3LL * d.sdd_w * d.sdd_h) + al16(snm::BLOB_BYTES) + 8LL * FFSVA_NSTAT;
}
}  // namespace

FFSVA_API ffsva_status ffsva_stream_image_bytes(ffsva_stream* s, int64_t* bytes) {
  if (!s || !bytes) return fail(FFSVA_EINVAL, "NULL argument");
  *bytes = image_bytes(s->desc);
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_stream_export(ffsva_stream* s, void* dst, int64_t cap, int32_t dst_is_host,
                                           void* cuda_stream) {
  if (!s || !dst) return fail(FFSVA_EINVAL, "NULL argument");
  const int64_t total = image_bytes(s->desc);
  if (cap < total) return fail(FFSVA_EINVAL, "destination smaller than ffsva_stream_image_bytes");
  DeviceCtx* ctx = s->ctx;
  if (ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  std::lock_guard<std::mutex> lk(ctx->mu);
  DeviceGuard g(ctx->device);
  if (!dst_is_host) {
    begin_ptr_checks(ctx);
    ffsva_status cs = check_device_ptr(ctx, dst, (size_t)total);
    if (cs != FFSVA_OK) return cs;
  }
  ImageHeader h{};
  h.magic = kImageMagic;
  h.version = kImageVersion;
  h.desc = s->desc;
  h.T = s->T;
  h.ref_sum_sq = s->ref_sum_sq;
  h.ref_bytes = 3LL * s->desc.sdd_w * s->desc.sdd_h;
  h.snm_bytes = snm::BLOB_BYTES;
  h.stats_bytes = 8LL * FFSVA_NSTAT;
  h.total = total;
  h.has_ref = s->has_ref;
  h.has_snm = s->has_snm;
  uint8_t* d = (uint8_t*)dst;
  const int64_t o_ref = kImageHeader, o_snm = o_ref + al16(h.ref_bytes), o_st = o_snm + al16(h.snm_bytes);
  cudaStream_t cs = (cudaStream_t)cuda_stream;
  const cudaMemcpyKind from_dev = dst_is_host ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice;
  std::vector<uint8_t> hdr(kImageHeader, 0);
  std::memcpy(hdr.data(), &h, sizeof(h));
  cudaError_t e = cudaMemcpyAsync(d, hdr.data(), kImageHeader, dst_is_host ? cudaMemcpyHostToHost : cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(d + o_ref, s->d_ref, (size_t)h.ref_bytes, from_dev, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(d + o_snm, s->d_snm, (size_t)h.snm_bytes, from_dev, cs);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(d + o_st, ctx->d_stats + (size_t)s->slot * NSTAT, 8 * NSTAT, from_dev, cs);
  std::vector<uint64_t> lat(NLAT);
  {
    std::lock_guard<std::mutex> lk2(ctx->lat_mu);
    std::copy_n(ctx->h_lat.begin() + (std::ptrdiff_t)s->slot * NLAT, NLAT, lat.begin());
  }
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(d + o_st + 8 * NSTAT, lat.data(), 8 * NLAT,
                        dst_is_host ? cudaMemcpyHostToHost : cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess) e = cudaStreamSynchronize(cs);  // hdr is a local buffer
  if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_stream_export");
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_stream_import(int32_t device, const void* src, int64_t bytes, int32_t src_is_host,
                                           ffsva_stream** out) {
  if (!src || !out || bytes < kImageHeader) return fail(FFSVA_EINVAL, "bad argument");
  ImageHeader h{};
  if (src_is_host) {
    std::memcpy(&h, src, sizeof(h));
  } else {
    DeviceGuard g(device);
    cudaError_t e = cudaMemcpy(&h, src, sizeof(h), cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(FFSVA_EINVAL, std::string("cannot read the image header: ") + cudaGetErrorString(e));
    }
  }
  if (h.magic != kImageMagic || h.version != kImageVersion) return fail(FFSVA_EINVAL, "not a stream image");
  h.desc.device = device;
  if (h.total != image_bytes(h.desc) || bytes < h.total || h.ref_bytes != 3LL * h.desc.sdd_w * h.desc.sdd_h ||
      h.snm_bytes != snm::BLOB_BYTES || h.stats_bytes != 8LL * FFSVA_NSTAT)
    return fail(FFSVA_EINVAL, "stream image sizes do not match its descriptor");
  ffsva_stream* s = nullptr;
  ffsva_status st = ffsva_open_stream(&h.desc, &s);  // validates the descriptor
  if (st != FFSVA_OK) return st;
  DeviceCtx* ctx = s->ctx;
  bool ok = true;
  {
    std::lock_guard<std::mutex> lk(ctx->mu);
    DeviceGuard g(device);
    const uint8_t* p = (const uint8_t*)src;
    const int64_t o_ref = kImageHeader, o_snm = o_ref + al16(h.ref_bytes), o_st = o_snm + al16(h.snm_bytes);
    const cudaMemcpyKind to_dev = src_is_host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
    cudaError_t e = cudaMemcpy(s->d_ref, p + o_ref, (size_t)h.ref_bytes, to_dev);
    if (e == cudaSuccess) e = cudaMemcpy(s->d_snm, p + o_snm, (size_t)h.snm_bytes, to_dev);
    if (e == cudaSuccess) e = cudaMemcpy(ctx->d_stats + (size_t)s->slot * NSTAT, p + o_st, 8 * NSTAT, to_dev);
    if (e == cudaSuccess) {
      std::vector<uint64_t> lat(NLAT);
      e = cudaMemcpy(lat.data(), p + o_st + 8 * NSTAT, 8 * NLAT, src_is_host ? cudaMemcpyHostToHost : cudaMemcpyDeviceToHost);
      std::lock_guard<std::mutex> lk2(ctx->lat_mu);
      std::copy(lat.begin(), lat.end(), ctx->h_lat.begin() + (std::ptrdiff_t)s->slot * NLAT);
    }
    if (e != cudaSuccess) {
      cuda_fail(ctx, e, "ffsva_stream_import");
      ok = false;
    }
    s->T = h.T;
    s->ref_sum_sq = h.ref_sum_sq;
    s->has_ref = h.has_ref != 0;
    s->has_snm = h.has_snm != 0;
  }
  if (!ok) {
    ffsva_close(s);
    return FFSVA_ECUDA;
  }
  *out = s;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_filter_batch_host(const ffsva_frame* frames, int32_t n, ffsva_result* results,
                                               void* cuda_stream);

}  // extern "C"
