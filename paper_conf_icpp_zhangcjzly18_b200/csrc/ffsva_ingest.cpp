// ffsva_ingest.cpp — ffsva_filter_batch_host: the cascade for frames resident in HOST memory.
//
// The paper's SNM stage pays for "image data must be loaded from CPU to GPU memory"; here the
// raw frames cross PCIe once and the copy is overlapped with the SDD kernel: frames are staged through a
// two-slot device ring of C-frame chunks on a dedicated copy stream, K1 runs on chunk c while chunk c+1 is in
// flight, and K3/K4 (which only touch the 7.5 KB D50 images) run once over the whole batch.
#include <algorithm>
#include <memory>
#include <vector>

#include "ffsva_runtime.h"

using namespace ffsva;

namespace {
constexpr int kChunk = 32;  // frames per staging chunk
}

extern "C" FFSVA_API ffsva_status ffsva_filter_batch_host(const ffsva_frame* frames, int32_t n,
                                                          ffsva_result* results, void* cuda_stream) {
  if (n < 0) return fail(FFSVA_EINVAL, "n < 0");
  if (n == 0) return FFSVA_OK;
  if (!frames || !results) return fail(FFSVA_EINVAL, "NULL argument");
  DeviceCtx* ctx = nullptr;
  for (int32_t i = 0; i < n; ++i) {
    const ffsva_stream* s = frames[i].stream;
    if (!s || !frames[i].pixels) return fail(FFSVA_EINVAL, "frame without stream or pixels");
    if (!ctx) ctx = s->ctx;
    if (s->ctx != ctx) return fail(FFSVA_EDEVICE, "frames of one batch live on several devices");
    if (!s->has_ref || !s->has_snm) return fail(FFSVA_ESTATE, "stream has no reference image or no SNM");
  }
  if (ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  std::lock_guard<std::mutex> lk(ctx->mu);
  DeviceGuard g(ctx->device);
  cudaStream_t cs = (cudaStream_t)cuda_stream;

  // ---- staging ring: 2 chunks x kChunk slots of the largest frame
  size_t slot = 0;
  for (int32_t i = 0; i < n; ++i) {
    const ffsva_stream_desc& d = frames[i].stream->desc;
    slot = std::max(slot, (size_t)d.height * (size_t)d.row_pitch);
  }
  slot = (slot + 255) & ~(size_t)255;
  const size_t need = 2 * kChunk * slot;
  cudaError_t e;
  if (ctx->ring_bytes < need) {
    cudaFree(ctx->d_ring);
    ctx->d_ring = nullptr;
    ctx->ring_bytes = 0;
    if ((e = cudaMalloc(&ctx->d_ring, need)) != cudaSuccess) return cuda_fail(nullptr, e, "cudaMalloc(ring)");
    ctx->ring_bytes = need;
    ctx->ranges.clear();
  }
  // descriptors point into the ring (slot reuse is ordered by events below)
  std::vector<ffsva_frame> staged(frames, frames + n);
  for (int32_t i = 0; i < n; ++i) {
    const int c = i / kChunk, j = i % kChunk;
    staged[i].pixels = ctx->d_ring + ((size_t)(c & 1) * kChunk + j) * slot;
  }
  if (!ctx->scratch) ctx->scratch = new Batch();
  Batch* b = ctx->scratch;
  ffsva_status st = batch_build(ctx, b, staged.data(), n, false, false, cs);
  if (st != FFSVA_OK) return st;

  cudaEvent_t ev_copy[2], ev_done[2];
  for (int k = 0; k < 2; ++k) {
    cudaEventCreateWithFlags(&ev_copy[k], cudaEventDisableTiming);
    cudaEventCreateWithFlags(&ev_done[k], cudaEventDisableTiming);
  }
  // the copy stream must not overwrite ring slots still read by an earlier call on cs
  cudaEventRecord(ev_done[0], cs);
  cudaEventRecord(ev_done[1], cs);
  const int nchunks = (n + kChunk - 1) / kChunk;
  const int nb = b->sdd_h / 2;
  st = FFSVA_OK;
  for (int c = 0; c < nchunks && st == FFSVA_OK; ++c) {
    const int k = c & 1, i0 = c * kChunk, cnt = std::min(kChunk, n - i0);
    cudaStreamWaitEvent(ctx->copy_stream, ev_done[k], 0);
    for (int j = 0; j < cnt; ++j) {
      const ffsva_stream_desc& d = frames[i0 + j].stream->desc;
      e = cudaMemcpyAsync(const_cast<uint8_t*>(staged[i0 + j].pixels), frames[i0 + j].pixels,
                          (size_t)(d.height - 1) * d.row_pitch + 3 * (size_t)d.width, cudaMemcpyHostToDevice,
                          ctx->copy_stream);
      if (e != cudaSuccess) {
        st = cuda_fail(ctx, e, "cudaMemcpyAsync(frame H2D)");
        break;
      }
    }
    if (st != FFSVA_OK) break;
    cudaEventRecord(ev_copy[k], ctx->copy_stream);
    cudaStreamWaitEvent(cs, ev_copy[k], 0);
    SddArgs sa{};
    sa.frames = b->d_desc + i0;
    sa.n = cnt;
    sa.sdd_w = b->sdd_w;
    sa.sdd_h = b->sdd_h;
    sa.d50 = b->d_d50 + (size_t)i0 * b->d50_stride;
    sa.d50_stride = b->d50_stride;
    sa.d100 = nullptr;
    sa.partial = b->d_partial + (size_t)i0 * 2 * nb;
    sa.counter = b->d_counter + i0;
    sa.ssd = b->d_ssd + i0;
    sa.pass = b->d_pass + i0;
    sa.stats = ctx->d_stats;
    sa.max_chunks = b->max_chunks;
    sa.vec16 = b->vec16;
    sa.bulk = b->bulk;
    sa.stage_bytes = b->stage_bytes;
    if ((e = launch_sdd(sa, cs)) != cudaSuccess) st = cuda_fail(ctx, e, "launch_sdd");
    g_launches += 1;
    cudaEventRecord(ev_done[k], cs);
  }
  if (st == FFSVA_OK) {
    // K3 + K4 over the whole batch (run the prepared batch minus its SDD stage)
    CompactArgs ca{};
    ca.pass = b->d_pass;
    ca.n = n;
    ca.perm = b->d_perm;
    ca.seg_lo = b->d_seg_lo;
    ca.n_seg = b->n_seg;
    ca.seg_batch = b->d_seg_batch;
    ca.seg_slot = b->d_seg_batch + b->cap;
    ca.stats = ctx->d_stats;
    ca.snm_ctas = std::max(1, std::min(n, 2 * ctx->num_sms));
    ca.survivor_idx = b->d_surv;
    ca.work = b->d_work;
    ca.posw = b->d_posw;
    ca.chunks = b->d_chunks;
    ca.counts = b->d_counts;
    ca.logit = b->d_logit;
    ca.snm_pass = b->d_snm_pass;
    ca.snm_class = b->d_snm_class;
    if ((e = launch_compact(ca, cs)) != cudaSuccess) st = cuda_fail(ctx, e, "launch_compact");
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
    na.stats = ctx->d_stats;
    na.grid = std::max(1, std::min(n, 2 * ctx->num_sms));
    if (st == FFSVA_OK && (e = launch_snm(na, cs)) != cudaSuccess) st = cuda_fail(ctx, e, "launch_snm");
    g_launches += 2;
  }
  if (st == FFSVA_OK) st = batch_fetch(b, results, cs);
  cudaStreamSynchronize(ctx->copy_stream);
  for (int k = 0; k < 2; ++k) {
    cudaEventDestroy(ev_copy[k]);
    cudaEventDestroy(ev_done[k]);
  }
  return st;
}
