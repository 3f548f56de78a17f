// ffsva_runtime.cpp — host runtime: device contexts, pointer validation, SNM weight packing, prepared
// batches (descriptor upload, stream-major work order, CUDA-graph capture of K1 -> K3 -> K4).
#include "ffsva_runtime.h"

#include <cuda.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>

namespace ffsva {

std::atomic<uint64_t> g_launches{0};
static thread_local std::string t_err;
static std::mutex g_mu;
static DeviceCtx* g_ctx[64] = {nullptr};
constexpr int32_t kMaxSlots = 65536;  // stats table rows per device (fixed so graphs never see a realloc)

void set_error(const std::string& msg) { t_err = msg; }
const char* last_error() { return t_err.c_str(); }

ffsva_status fail(ffsva_status st, const std::string& msg) {
  t_err = msg;
  return st;
}

ffsva_status cuda_fail(DeviceCtx* ctx, cudaError_t e, const char* what) {
  if (ctx) ctx->sticky = true;
  t_err = std::string(what) + ": " + cudaGetErrorString(e);
  return e == cudaErrorMemoryAllocation ? FFSVA_ENOMEM : FFSVA_ECUDA;
}

#define FF_CUDA(ctx, call)                                  \
  do {                                                      \
    cudaError_t _e = (call);                                \
    if (_e != cudaSuccess) return cuda_fail(ctx, _e, #call); \
  } while (0)

// ------------------------------------------------------------------ device contexts
DeviceCtx* ctx_acquire(int device, ffsva_status* st) {
  std::lock_guard<std::mutex> lk(g_mu);
  *st = FFSVA_OK;
  if (device < 0 || device >= 64) {
    *st = fail(FFSVA_EINVAL, "device ordinal out of range");
    return nullptr;
  }
  int count = 0;
  cudaError_t e = cudaGetDeviceCount(&count);
  if (e != cudaSuccess || count == 0) {
    *st = fail(FFSVA_ECUDA, std::string("no CUDA device: ") + cudaGetErrorString(e));
    return nullptr;
  }
  if (device >= count) {
    *st = fail(FFSVA_EINVAL, "device ordinal >= device count");
    return nullptr;
  }
  DeviceCtx* c = g_ctx[device];
  if (!c) {
    DeviceGuard g(device);
    cudaDeviceProp prop;
    if ((e = cudaGetDeviceProperties(&prop, device)) != cudaSuccess) {
      *st = fail(FFSVA_ECUDA, cudaGetErrorString(e));
      return nullptr;
    }
    if (prop.major != 10) {
      *st = fail(FFSVA_ECUDA, "the kernels are built for sm_100a (B200); device is sm_" +
                                  std::to_string(prop.major) + std::to_string(prop.minor));
      return nullptr;
    }
    c = new DeviceCtx();
    c->device = device;
    c->num_sms = prop.multiProcessorCount;
    c->stats_cap = kMaxSlots;
    c->h_lat.assign((size_t)kMaxSlots * NLAT, 0);
    if ((e = cudaMalloc(&c->d_stats, sizeof(unsigned long long) * NSTAT * kMaxSlots)) != cudaSuccess ||
        (e = cudaMemset(c->d_stats, 0, sizeof(unsigned long long) * NSTAT * kMaxSlots)) != cudaSuccess ||
        (e = cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = snm_configure()) != cudaSuccess) {
      *st = cuda_fail(nullptr, e, "device context init");
      delete c;
      return nullptr;
    }
    g_ctx[device] = c;
  }
  c->nstreams++;
  return c;
}

void ctx_release(DeviceCtx* c) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (--c->nstreams > 0) return;
  DeviceGuard g(c->device);
  cudaDeviceSynchronize();
  if (c->scratch) {
    batch_free(c->scratch);
    delete c->scratch;
  }
  cudaFree(c->d_stats);
  cudaFree(c->d_ring);
  cudaFreeHost(c->h_lat_pinned);
  if (c->lat_ev) cudaEventDestroy(c->lat_ev);
  cudaStreamDestroy(c->copy_stream);
  g_ctx[c->device] = nullptr;
  delete c;
}

// A device pointer must lie inside a device allocation of the context's device. Allocation ranges are cached:
// within one validation epoch (one API call) a batch of frames from one pool costs one driver query; a cached
// range is re-confirmed with the driver (same base and size) the first time a new epoch uses it.
namespace {
using GetRange = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
GetRange driver_get_range() {
  // driver entry point fetched through the runtime, so the library does not link libcuda (it must load on
  // GPU-less hosts, where every compute call then reports FFSVA_ECUDA)
  static GetRange fn = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess) f = nullptr;
    return (GetRange)f;
  }();
  return fn;
}
}  // namespace

void begin_ptr_checks(DeviceCtx* ctx) {
  std::lock_guard<std::mutex> lk(ctx->ranges_mu);
  ++ctx->range_epoch;
}

void clear_ptr_cache(DeviceCtx* ctx) {
  std::lock_guard<std::mutex> lk(ctx->ranges_mu);
  ctx->ranges.clear();
  ctx->range_mru = 0;
}

ffsva_status check_device_ptr(DeviceCtx* ctx, const void* p, size_t bytes) {
  if (!p) return fail(FFSVA_EINVAL, "NULL frame pointer");
  const uintptr_t a = (uintptr_t)p;
  GetRange get_range = driver_get_range();
  {
    std::lock_guard<std::mutex> lk(ctx->ranges_mu);
    auto& R = ctx->ranges;
    auto hit = [&](size_t i) { return a >= R[i].base && a + bytes <= R[i].base + R[i].size; };
    size_t i = ctx->range_mru < R.size() && hit(ctx->range_mru) ? ctx->range_mru : R.size();
    for (size_t j = 0; i == R.size() && j < R.size(); ++j)
      if (hit(j)) i = j;
    if (i < R.size()) {
      if (R[i].epoch == ctx->range_epoch) {
        ctx->range_mru = i;
        return FFSVA_OK;
      }
      CUdeviceptr base = 0;
      size_t size = 0;
      if (get_range && get_range(&base, &size, (CUdeviceptr)a) == CUDA_SUCCESS && (uintptr_t)base == R[i].base &&
          size == R[i].size) {
        R[i].epoch = ctx->range_epoch;
        ctx->range_mru = i;
        return FFSVA_OK;
      }
      R.erase(R.begin() + (std::ptrdiff_t)i);  // freed or re-allocated since it was cached: full check below
      ctx->range_mru = 0;
    }
  }
  cudaPointerAttributes attr;
  cudaError_t e = cudaPointerGetAttributes(&attr, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(FFSVA_EINVAL, "pixels is not a CUDA pointer");
  }
  if (attr.type != cudaMemoryTypeDevice && attr.type != cudaMemoryTypeManaged)
    return fail(FFSVA_EINVAL, "pixels must be device memory (use ffsva_filter_batch_host for host frames)");
  if (attr.device != ctx->device) return fail(FFSVA_EDEVICE, "frame pixels live on another device");
  CUdeviceptr base = 0;
  size_t size = 0;
  if (get_range && get_range(&base, &size, (CUdeviceptr)a) == CUDA_SUCCESS) {
    if (a + bytes > (uintptr_t)base + size) return fail(FFSVA_EINVAL, "frame extends past its allocation");
    std::lock_guard<std::mutex> lk(ctx->ranges_mu);
    if (ctx->ranges.size() >= 64) ctx->ranges.erase(ctx->ranges.begin());
    ctx->ranges.push_back({(uintptr_t)base, size, ctx->range_epoch});
    ctx->range_mru = ctx->ranges.size() - 1;
  }
  return FFSVA_OK;
}

int latency_bin(int64_t us) {
  if (us < 1000) return 0;
  int k = 1;
  for (int64_t ms = us / 1000; ms >= 2 && k < NLAT - 3; ms >>= 1) ++k;  // [2^(k-1), 2^k) ms -> k, capped at 13
  return k;
}

void record_latency(DeviceCtx* ctx, int32_t slot, int64_t us) {
  if (slot < 0 || slot >= ctx->stats_cap) return;
  if (us < 0) us = 0;
  std::lock_guard<std::mutex> lk(ctx->lat_mu);
  uint64_t* row = ctx->h_lat.data() + (size_t)slot * NLAT;
  row[0] += 1;
  row[1] += (uint64_t)us;
  row[2 + latency_bin(us)] += 1;
}

// ------------------------------------------------------------------ host arithmetic
// floor(delta * n) with the product taken exactly: delta = mant * 2^e2 (IEEE-754 fields).
uint64_t exact_threshold(double delta, uint64_t n) {
  uint64_t bits;
  std::memcpy(&bits, &delta, 8);
  const int expf = (int)((bits >> 52) & 0x7FF);
  const uint64_t frac = bits & ((1ull << 52) - 1);
  if ((bits >> 63) || (expf == 0 && frac == 0)) return 0;
  const uint64_t mant = expf ? (frac | (1ull << 52)) : frac;
  const int e2 = expf ? expf - 1075 : -1074;
  const unsigned __int128 prod = (unsigned __int128)mant * n;
  if (e2 >= 0) {
    if (e2 >= 64) return UINT64_MAX;
    const unsigned __int128 v = prod << e2;
    if ((v >> e2) != prod || (v >> 64) != 0) return UINT64_MAX;
    return (uint64_t)v;
  }
  if (-e2 >= 128) return 0;
  const unsigned __int128 v = prod >> (-e2);
  return (v >> 64) ? UINT64_MAX : (uint64_t)v;
}

// floor(delta^2 * q) with the product taken exactly: delta = mant * 2^e2, so delta^2 * q = mant^2 * q * 2^(2 e2)
// with mant^2 < 2^106 and q < 2^64: a 170-bit product held in three 64-bit limbs.
uint64_t exact_threshold_sq(double delta, uint64_t q) {
  uint64_t bits;
  std::memcpy(&bits, &delta, 8);
  const int expf = (int)((bits >> 52) & 0x7FF);
  const uint64_t frac = bits & ((1ull << 52) - 1);
  if ((bits >> 63) || (expf == 0 && frac == 0) || q == 0) return 0;
  const uint64_t mant = expf ? (frac | (1ull << 52)) : frac;
  const int e2 = expf ? expf - 1075 : -1074;
  const unsigned __int128 m2 = (unsigned __int128)mant * mant;  // < 2^106
  const unsigned __int128 lo = (unsigned __int128)(uint64_t)m2 * q;
  const unsigned __int128 hi = (unsigned __int128)(uint64_t)(m2 >> 64) * q;  // weight 2^64
  uint64_t w[3];  // little-endian limbs of m2 * q
  w[0] = (uint64_t)lo;
  const unsigned __int128 mid = (lo >> 64) + (uint64_t)hi;
  w[1] = (uint64_t)mid;
  w[2] = (uint64_t)(hi >> 64) + (uint64_t)(mid >> 64);
  const int sh = 2 * e2;  // value = w * 2^sh
  if (sh >= 0) {
    if (w[2] || w[1] || sh >= 64 || (sh > 0 && (w[0] >> (64 - sh)))) return UINT64_MAX;
    return w[0] << sh;
  }
  const int r = -sh;
  if (r >= 192) return 0;
  // floor(w / 2^r): shift the 192-bit value right by r and saturate to 64 bits
  uint64_t out[3] = {0, 0, 0};
  const int limb = r / 64, bit = r % 64;
  for (int k = 0; k + limb < 3; ++k) {
    out[k] = w[k + limb] >> bit;
    if (bit && k + limb + 1 < 3) out[k] |= w[k + limb + 1] << (64 - bit);
  }
  return (out[1] || out[2]) ? UINT64_MAX : out[0];
}

uint64_t stream_threshold(const ffsva_stream_desc& d, uint64_t ref_sum_sq) {
  switch (d.distance) {
    case FFSVA_DIST_SAD: return exact_threshold(d.delta_diff, 1);
    case FFSVA_DIST_NRMSE: return exact_threshold_sq(d.delta_diff, ref_sum_sq);
    default: return exact_threshold(d.delta_diff, 3ull * (uint64_t)d.sdd_w * (uint64_t)d.sdd_h);
  }
}

uint16_t bf16_bits_rne(float x) {
  uint32_t u;
  std::memcpy(&u, &x, 4);
  if ((u & 0x7F800000u) == 0x7F800000u && (u & 0x007FFFFFu)) return 0x7FC0;  // NaN
  return (uint16_t)((u + 0x7FFFu + ((u >> 16) & 1u)) >> 16);
}

[[maybe_unused]] static float bf16_value(float x) {
  uint32_t u = (uint32_t)bf16_bits_rne(x) << 16;
  float f;
  std::memcpy(&f, &u, 4);
  return f;
}

float logit_of(double t) {
  if (t <= 0.0) return -INFINITY;
  if (t >= 1.0) return INFINITY;
  return (float)std::log(t / (1.0 - t));
}

// SNM weight image (see ffsva_internal.h snm::*). params = w1[16][3][3][3], b1[16], w2[32][16][3][3], b2[32],
// wfc[4608], bfc.
void pack_snm_blob(const float* params, uint8_t* blob) {
  using namespace snm;
  std::memset(blob, 0, BLOB_BYTES);
  const float* w1 = params;
  const float* b1 = w1 + 27 * C1;
  const float* w2 = b1 + C1;
  const float* b2 = w2 + 9 * C1 * C2;
  const float* wfc = b2 + C2;
  const float* bfc = wfc + NF;
  // conv1: B matrix of patch row dy: n = 16q + oc (q = 2a + b), k = 4u + c (patch column u, channel slot c);
  // K-half h holds patch columns 2h, 2h+1. The 3x3 kernel of pool position (a, b) sits at offset (a, b) of the patch.
  uint16_t* W1 = reinterpret_cast<uint16_t*>(blob + OFF_W1);
  for (int dy = 0; dy < 4; ++dy)
    for (int q = 0; q < 4; ++q)
      for (int oc = 0; oc < C1; ++oc)
        for (int u = 0; u < 4; ++u)
          for (int c = 0; c < 3; ++c) {
            const int ky = dy - (q >> 1), kx = u - (q & 1);
            if (ky < 0 || ky > 2 || kx < 0 || kx > 2) continue;
            const int n = 16 * q + oc, h = u >> 1, kk = 4 * (u & 1) + c;
            W1[((dy * 2 + h) * 64 + n) * 8 + kk] = bf16_bits_rne(w1[((oc * 3 + c) * 3 + ky) * 3 + kx]);
          }
  // conv2: one B per MMA of conv2_mma (patch cell (Y', X')): row n = 32 * (group - g0) + oc holds the weights of pool
  // position (a, b) of that group through tap (Y' - a, X' - b); K-half h = input channels 8h..8h+7.
  for (int i = 0; i < kConv2Mmas; ++i) {
    const Conv2Mma mm = conv2_mma(i);
    uint16_t* B = reinterpret_cast<uint16_t*>(blob + OFF_W2 + mm.boff);
    const int N = 32 * mm.ng;
    for (int a = 0; a < 2; ++a)
      for (int b = 0; b < 2; ++b) {
        const int g = conv2_group(a, b) - mm.g0;
        if (g < 0 || g >= mm.ng) continue;
        const int ky = mm.cy - a, kx = mm.cx - b;
        if (ky < 0 || ky > 2 || kx < 0 || kx > 2) std::abort();  // the table only lists taps that exist
        for (int oc = 0; oc < C2; ++oc)
          for (int h = 0; h < 2; ++h)
            for (int c = 0; c < 8; ++c)
              B[(h * N + 32 * g + oc) * 8 + c] = bf16_bits_rne(w2[((oc * C1 + 8 * h + c) * 3 + ky) * 3 + kx]);
      }
  }
  std::memcpy(blob + OFF_B1, b1, C1 * 4);
  std::memcpy(blob + OFF_B2, b2, C2 * 4);
  std::memcpy(blob + OFF_BFC, bfc, 4);
  // FC weights: bf16 values (Q15) held as fp32, [channel quad][pooled pixel][4] so a lane reads its pixel's 32 weights
  // with eight 16-byte loads, consecutive lanes at consecutive addresses
  float* F = reinterpret_cast<float*>(blob + OFF_WFC);
  for (int c = 0; c < C2; ++c)
    for (int p = 0; p < P2 * P2; ++p) {
      const uint32_t bits = (uint32_t)bf16_bits_rne(wfc[c * P2 * P2 + p]) << 16;
      std::memcpy(&F[((c >> 2) * P2 * P2 + p) * 4 + (c & 3)], &bits, 4);
    }
}

// ------------------------------------------------------------------ batches
static size_t al(size_t x) { return (x + 255) & ~(size_t)255; }

void batch_free(Batch* b) {
  if (b->graph) cudaGraphExecDestroy(b->graph);
  b->graph = nullptr;
  cudaFree(b->d_mem);
  cudaFreeHost(b->h_in);
  cudaFreeHost(b->h_out);
  b->d_mem = nullptr;
  b->h_in = b->h_out = nullptr;
  b->cap = 0;
}

static ffsva_status batch_alloc(DeviceCtx* ctx, Batch* b, int32_t cap, int32_t sdd_w, int32_t sdd_h, bool d100) {
  batch_free(b);
  const size_t n = (size_t)cap;
  b->d50_stride = (int64_t)((3 * (sdd_w / 2) * (sdd_h / 2) + 15) & ~15);
  // input block (mirrors h_in)
  size_t off = 0;
  const size_t o_desc = off; off += al(64 * n);
  const size_t o_perm = off; off += al(4 * n);
  const size_t o_seg = off; off += al(4 * (n + 1));
  const size_t o_segb = off; off += al(8 * n);  // seg_batch[cap] then seg_slot[cap]
  const size_t o_xb = off; off += al(4 * (size_t)(sdd_w + 1));
  const size_t o_yb = off; off += al(4 * (size_t)(sdd_h + 1));
  const size_t o_pm = off; off += al(8 * n);    // PREVIOUS-mode (frame, prev) pairs
  const size_t o_last = off; off += al(4 * n);  // PREVIOUS-mode streams' last frames
  b->in_bytes = off;
  const size_t o_d50 = off; off += al((size_t)b->d50_stride * n);
  const size_t o_d100 = off; off += d100 ? al((size_t)3 * sdd_w * sdd_h * n) : 0;
  const size_t o_acc = off; off += al(8 * n);
  const size_t o_work = off; off += al(4 * n);
  const size_t o_posw = off; off += al(4 * (n + 1));
  const size_t o_chunks = off; off += al(4 * (n + 1));
  const size_t o_counts = off; off += al(16);
  const size_t o_out = off;
  const size_t out_bytes = 8 * n + 4 * n + 4 * n + 3 * n;
  off += al(out_bytes);
  b->d_bytes = off;
  cudaError_t e = cudaMalloc(&b->d_mem, off);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "cudaMalloc(batch)");
  uint8_t* base = (uint8_t*)b->d_mem;
  b->d_desc = (FrameDesc*)(base + o_desc);
  b->d_perm = (int32_t*)(base + o_perm);
  b->d_seg_lo = (int32_t*)(base + o_seg);
  b->d_seg_batch = (int32_t*)(base + o_segb);
  b->d_xb = (int32_t*)(base + o_xb);
  b->d_yb = (int32_t*)(base + o_yb);
  b->d_pm = (int32_t*)(base + o_pm);
  b->d_last = (int32_t*)(base + o_last);
  b->d_d50 = base + o_d50;
  b->d_d100 = d100 ? base + o_d100 : nullptr;
  b->d_acc = (unsigned long long*)(base + o_acc);
  b->d_work = (int32_t*)(base + o_work);
  b->d_posw = (int32_t*)(base + o_posw);
  b->d_chunks = (int32_t*)(base + o_chunks);
  b->d_counts = (int32_t*)(base + o_counts);
  b->d_out = base + o_out;
  b->d_ssd = (uint64_t*)(b->d_out);
  b->d_logit = (float*)(b->d_out + 8 * n);
  b->d_surv = (int32_t*)(b->d_out + 12 * n);
  b->d_pass = b->d_out + 16 * n;
  b->d_snm_pass = b->d_out + 17 * n;
  b->d_snm_class = b->d_out + 18 * n;
  b->out_bytes = out_bytes;
  if ((e = cudaMemset(b->d_acc, 0, 8 * n)) != cudaSuccess) return cuda_fail(ctx, e, "cudaMemset(acc_ssd)");
  if ((e = cudaMemset(b->d_counts, 0, 16)) != cudaSuccess) return cuda_fail(ctx, e, "cudaMemset(counts)");
  if ((e = cudaMallocHost(&b->h_in, b->in_bytes)) != cudaSuccess) return cuda_fail(nullptr, e, "cudaMallocHost");
  if ((e = cudaMallocHost(&b->h_out, out_bytes)) != cudaSuccess) return cuda_fail(nullptr, e, "cudaMallocHost");
  b->cap = cap;
  b->sdd_w = sdd_w;
  b->sdd_h = sdd_h;
  b->want_d100 = d100;
  b->ctx = ctx;
  return FFSVA_OK;
}

ffsva_status batch_build(DeviceCtx* ctx, Batch* b, const ffsva_frame* frames, int32_t n, bool sdd_only,
                         bool want_d100, cudaStream_t st) {
  NvtxRange r("ffsva batch: build (validate, plan, upload descriptors)");
  const StreamState* s0 = frames[0].stream;
  const int32_t sdd_w = s0->desc.sdd_w, sdd_h = s0->desc.sdd_h;
  SddPlan plan;
  begin_ptr_checks(ctx);
  for (int32_t i = 0; i < n; ++i) {
    const StreamState* s = frames[i].stream;
    if (s->desc.sdd_w != sdd_w || s->desc.sdd_h != sdd_h)
      return fail(FFSVA_EINVAL, "all frames of a batch must share the SDD grid");
    const int64_t bytes = (int64_t)(s->desc.height - 1) * s->desc.row_pitch + 3 * s->desc.width;
    ffsva_status cs = check_device_ptr(ctx, frames[i].pixels, (size_t)bytes);
    if (cs != FFSVA_OK) return cs;
    sdd_plan_add(plan, s->desc.width, s->desc.height, s->desc.row_pitch, frames[i].pixels, sdd_h);
    if (s->desc.ref_mode == FFSVA_REF_PREVIOUS) want_d100 = true;  // K2 reads every frame's D100
  }
  // K1 variant (band / CTA-pair cluster / register streaming) and its shared-memory layout
  sdd_plan_finish(plan, sdd_w, sdd_h);
  if (b->cap < n || b->sdd_w != sdd_w || b->sdd_h != sdd_h || (want_d100 && !b->want_d100)) {
    ffsva_status as = batch_alloc(ctx, b, std::max(n, b->cap), sdd_w, sdd_h, want_d100 || b->want_d100);
    if (as != FFSVA_OK) return as;
  }
  if (b->graph) {
    cudaGraphExecDestroy(b->graph);
    b->graph = nullptr;
  }
  cudaError_t e = sdd_configure(plan.smem);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "sdd_configure");
  b->n = n;
  b->plan = plan;
  b->sdd_only = sdd_only;
  // ---- host staging: descriptors, stream-major permutation, segments
  const size_t cap = (size_t)b->cap;
  FrameDesc* hd = (FrameDesc*)b->h_in;
  int32_t* hperm = (int32_t*)(b->h_in + al(64 * cap));
  int32_t* hseg = (int32_t*)(b->h_in + al(64 * cap) + al(4 * cap));
  int32_t* hsegb = (int32_t*)(b->h_in + al(64 * cap) + al(4 * cap) + al(4 * (cap + 1)));
  bool sorted = true;
  for (int32_t i = 0; i < n; ++i) {
    const StreamState* s = frames[i].stream;
    FrameDesc& d = hd[i];
    d.pixels = frames[i].pixels;
    d.ref = s->d_ref;
    d.snm = s->d_snm;
    d.pitch = s->desc.row_pitch;
    d.T = s->T;
    d.W = s->desc.width;
    d.H = s->desc.height;
    d.L_t = s->L_t;
    d.L_low = s->L_low;
    d.L_high = s->L_high;
    d.slot = (uint16_t)s->slot;
    d.metric = (uint8_t)s->desc.distance;
    d.mode = (uint8_t)s->desc.ref_mode;
    hperm[i] = i;
    if (i && s->slot < frames[i - 1].stream->slot) sorted = false;
  }
  if (!sorted)
    std::stable_sort(hperm, hperm + n, [&](int32_t x, int32_t y) { return hd[x].slot < hd[y].slot; });
  int32_t nseg = 0;
  for (int32_t k = 0; k < n; ++k)
    if (k == 0 || hd[hperm[k]].slot != hd[hperm[k - 1]].slot) {
      hseg[nseg] = k;
      hsegb[nseg] = frames[hperm[k]].stream->desc.snm_batch;
      hsegb[cap + nseg] = frames[hperm[k]].stream->slot;
      ++nseg;
    }
  hseg[nseg] = n;
  b->n_seg = nseg;
  // PREVIOUS-mode plan (Q25): each such frame's previous frame of its stream in input order (-1: the
  // stream's R), and each such stream's last frame (its D100 becomes the stream's R after the batch)
  {
    int32_t* hpm = (int32_t*)(b->h_in + ((uint8_t*)b->d_pm - (uint8_t*)b->d_mem));
    int32_t* hlast = (int32_t*)(b->h_in + ((uint8_t*)b->d_last - (uint8_t*)b->d_mem));
    std::vector<std::pair<int32_t, int32_t>> last;  // (slot, latest frame) per PREVIOUS-mode stream
    int32_t npm = 0;
    for (int32_t i = 0; i < n; ++i) {
      if (hd[i].mode != kRefPrevious) continue;
      auto it = std::find_if(last.begin(), last.end(),
                             [&](const std::pair<int32_t, int32_t>& p) { return p.first == hd[i].slot; });
      int32_t prev = -1;
      if (it != last.end()) {
        prev = it->second;
        it->second = i;
      } else {
        last.emplace_back(hd[i].slot, i);
      }
      hpm[2 * npm] = i;
      hpm[2 * npm + 1] = prev;
      ++npm;
    }
    for (size_t k = 0; k < last.size(); ++k) hlast[k] = last[k].second;
    b->n_pm = npm;
    b->n_last = (int32_t)last.size();
  }
  // cell boundary tables (C1: cell i covers [floor(i*S/D), floor((i+1)*S/D))) when the batch shares W / H
  int32_t* hxb = (int32_t*)((uint8_t*)b->h_in + ((uint8_t*)b->d_xb - (uint8_t*)b->d_mem));
  int32_t* hyb = (int32_t*)((uint8_t*)b->h_in + ((uint8_t*)b->d_yb - (uint8_t*)b->d_mem));
  b->uni_W = hd[0].W;
  b->uni_H = hd[0].H;
  for (int32_t i = 1; i < n; ++i) {
    if (hd[i].W != b->uni_W) b->uni_W = -1;
    if (hd[i].H != b->uni_H) b->uni_H = -1;
  }
  if (b->uni_W > 0)
    for (int32_t i = 0; i <= sdd_w; ++i) hxb[i] = (int32_t)(((int64_t)i * b->uni_W) / sdd_w);
  if (b->uni_H > 0)
    for (int32_t i = 0; i <= sdd_h; ++i) hyb[i] = (int32_t)(((int64_t)i * b->uni_H) / sdd_h);
  e = cudaMemcpyAsync(b->d_mem, b->h_in, b->in_bytes, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaMemcpyAsync(descriptors)");
  // the staging buffer is reused by the next build: make sure this copy has consumed it
  e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaStreamSynchronize(descriptors)");
  return FFSVA_OK;
}

// SNM grid: one persistent CTA per SM (the kernel holds all 512 TMEM columns), no more CTAs than frames.
int snm_grid(const Batch* b) { return std::max(1, std::min(b->n, kSnmCtasPerSm * b->ctx->num_sms)); }

SddArgs make_sdd_args(Batch* b, int32_t i0, int32_t cnt) {
  SddArgs sa{};
  sa.frames = b->d_desc + i0;
  sa.n = cnt;
  sa.sdd_w = b->sdd_w;
  sa.sdd_h = b->sdd_h;
  sa.d50 = b->d_d50 + (size_t)i0 * b->d50_stride;
  sa.d50_stride = b->d50_stride;
  sa.d100 = b->want_d100 ? b->d_d100 + (size_t)i0 * 3 * b->sdd_w * b->sdd_h : nullptr;
  sa.acc_ssd = b->d_acc + i0;
  sa.stats = b->ctx->d_stats;
  sdd_plan_apply(b->plan, sa);
  sa.uni_W = b->uni_W;
  sa.uni_H = b->uni_H;
  sa.cellw = b->uni_W > 0 ? (b->uni_W + b->sdd_w - 1) / b->sdd_w : 0;
  sa.xbounds = b->uni_W > 0 ? b->d_xb : nullptr;
  sa.ybounds = b->uni_H > 0 ? b->d_yb : nullptr;
  return sa;
}

CompactArgs make_compact_args(Batch* b) {
  DeviceCtx* ctx = b->ctx;
  CompactArgs ca{};
  ca.frames = b->d_desc;
  ca.acc_ssd = b->d_acc;
  ca.ssd = b->d_ssd;
  ca.pass = b->d_pass;
  ca.n = b->n;
  ca.perm = b->d_perm;
  ca.seg_lo = b->d_seg_lo;
  ca.n_seg = b->n_seg;
  ca.seg_batch = b->d_seg_batch;
  ca.seg_slot = b->d_seg_batch + b->cap;
  ca.stats = ctx->d_stats;
  ca.snm_ctas = b->sdd_only ? 0 : snm_grid(b);
  ca.survivor_idx = b->d_surv;
  ca.work = b->d_work;
  ca.posw = b->d_posw;
  ca.chunks = b->d_chunks;
  ca.counts = b->d_counts;
  ca.logit = b->d_logit;
  ca.snm_pass = b->d_snm_pass;
  ca.snm_class = b->d_snm_class;
  return ca;
}

SnmArgs make_snm_args(Batch* b) {
  SnmArgs na{};
  na.frames = b->d_desc;
  na.d50 = b->d_d50;
  na.d50_stride = b->d50_stride;
  na.work = b->d_work;
  na.chunks = b->d_chunks;
  na.counts = b->d_counts;
  na.logit = b->d_logit;
  na.snm_pass = b->d_snm_pass;
  na.snm_class = b->d_snm_class;
  na.stats = b->ctx->d_stats;
  na.grid = snm_grid(b);
  return na;
}

PrevArgs make_prev_args(Batch* b) {
  PrevArgs pa{};
  pa.frames = b->d_desc;
  pa.d100 = b->d_d100;
  pa.n_values = 3 * b->sdd_w * b->sdd_h;
  pa.pairs = b->d_pm;
  pa.n_pm = b->n_pm;
  pa.last = b->d_last;
  pa.n_last = b->n_last;
  pa.acc_ssd = b->d_acc;
  pa.stats = b->ctx->d_stats;
  return pa;
}

int prev_launches(const Batch* b) { return b->n_pm > 0 ? (b->n_last > 0 ? 2 : 1) : 0; }

static ffsva_status batch_launch_kernels(Batch* b, cudaStream_t st, int* nk, cudaEvent_t* ev = nullptr) {
  DeviceCtx* ctx = b->ctx;
  if (ev) cudaEventRecord(ev[0], st);
  FF_CUDA(ctx, launch_sdd(make_sdd_args(b, 0, b->n), st));
  FF_CUDA(ctx, launch_prev(make_prev_args(b), st));
  if (ev) cudaEventRecord(ev[1], st);
  FF_CUDA(ctx, launch_compact(make_compact_args(b), st));
  if (ev) cudaEventRecord(ev[2], st);
  *nk = 2 + prev_launches(b);
  if (!b->sdd_only) {
    FF_CUDA(ctx, launch_snm(make_snm_args(b), st));
    *nk += 1;
  }
  if (ev) cudaEventRecord(ev[3], st);
  return FFSVA_OK;
}

ffsva_status batch_profile(Batch* const* batches, int32_t nb, int32_t iters, float* ms_out, cudaStream_t st) {
  DeviceCtx* ctx = batches[0]->ctx;
  cudaEvent_t ev[4];
  for (auto& e : ev) FF_CUDA(ctx, cudaEventCreate(&e));
  double acc[3] = {0, 0, 0};
  int count = 0;
  ffsva_status s = FFSVA_OK;
  for (int it = 0; it < iters && s == FFSVA_OK; ++it)
    for (int32_t j = 0; j < nb && s == FFSVA_OK; ++j) {
      int nk = 0;
      s = batch_launch_kernels(batches[j], st, &nk, ev);
      g_launches += nk;
      if (s != FFSVA_OK) break;
      cudaError_t e = cudaEventSynchronize(ev[3]);
      if (e != cudaSuccess) {
        s = cuda_fail(ctx, e, "cudaEventSynchronize(profile)");
        break;
      }
      float t[3];
      cudaEventElapsedTime(&t[0], ev[0], ev[1]);
      cudaEventElapsedTime(&t[1], ev[1], ev[2]);
      cudaEventElapsedTime(&t[2], ev[2], ev[3]);
      for (int k = 0; k < 3; ++k) acc[k] += t[k];
      ++count;
    }
  for (auto& e : ev) cudaEventDestroy(e);
  if (s != FFSVA_OK) return s;
  for (int k = 0; k < 3; ++k) ms_out[k] = count ? (float)(acc[k] / count) : 0.f;
  return FFSVA_OK;
}

ffsva_status batch_run(Batch* b, cudaStream_t st, bool use_graph) {
  NvtxRange r("ffsva batch: K1 -> K3 -> K4");
  DeviceCtx* ctx = b->ctx;
  if (b->n == 0) return FFSVA_OK;
  if (!use_graph || st == nullptr) {
    int nk = 0;
    ffsva_status s = batch_launch_kernels(b, st, &nk);
    g_launches += nk;
    return s;
  }
  if (!b->graph) {
    cudaGraph_t g = nullptr;
    FF_CUDA(ctx, cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
    int nk = 0;
    ffsva_status s = batch_launch_kernels(b, st, &nk);
    cudaError_t e = cudaStreamEndCapture(st, &g);
    if (s != FFSVA_OK) return s;
    if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaStreamEndCapture");
    e = cudaGraphInstantiate(&b->graph, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaGraphInstantiate");
    b->graph_kernels = nk;
  }
  FF_CUDA(ctx, cudaGraphLaunch(b->graph, st));
  g_launches += b->graph_kernels;
  return FFSVA_OK;
}

ffsva_status batch_fetch(Batch* b, ffsva_result* results, cudaStream_t st) {
  DeviceCtx* ctx = b->ctx;
  const int32_t n = b->n;
  if (n == 0) return FFSVA_OK;
  if (results) {
    FF_CUDA(ctx, cudaMemcpyAsync(b->h_out, b->d_out, b->out_bytes, cudaMemcpyDeviceToHost, st));
  }
  FF_CUDA(ctx, cudaStreamSynchronize(st));
  if (!results) return FFSVA_OK;
  const size_t cap = (size_t)b->cap;
  const uint64_t* ssd = (const uint64_t*)b->h_out;
  const float* lg = (const float*)(b->h_out + 8 * cap);
  const int32_t* sv = (const int32_t*)(b->h_out + 12 * cap);
  const uint8_t* ps = b->h_out + 16 * cap;
  const uint8_t* sp = b->h_out + 17 * cap;
  const uint8_t* sc = b->h_out + 18 * cap;
  for (int32_t i = 0; i < n; ++i) {
    ffsva_result& r = results[i];
    r.ssd = ssd[i];
    r.sdd_pass = ps[i];
    r.snm_pass = sp[i];
    r.snm_class = sc[i];
    r.tyolo_pass = 0;
    r.tyolo_count = -1;  // the batch API stops after the SNM (T-YOLO: ffsva_tyolo_run / the online runtime)
    r.reserved = 0;
    r.logit = lg[i];
    r.survivor_idx = sv[i];
  }
  return FFSVA_OK;
}

}  // namespace ffsva
