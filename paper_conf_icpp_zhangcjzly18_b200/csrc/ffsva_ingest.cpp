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
    clear_ptr_cache(ctx);
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
    if ((e = launch_sdd(make_sdd_args(b, i0, cnt), cs)) != cudaSuccess) st = cuda_fail(ctx, e, "launch_sdd");
    g_launches += 1;
    cudaEventRecord(ev_done[k], cs);
  }
  if (st == FFSVA_OK) {
    // K2 (PREVIOUS-mode streams) + K3 + K4 over the whole batch (they only touch D100 / D50, not the staged frames)
    if ((e = launch_prev(make_prev_args(b), cs)) != cudaSuccess) st = cuda_fail(ctx, e, "launch_prev");
    g_launches += prev_launches(b);
    if (st == FFSVA_OK && (e = launch_compact(make_compact_args(b), cs)) != cudaSuccess)
      st = cuda_fail(ctx, e, "launch_compact");
    if (st == FFSVA_OK && (e = launch_snm(make_snm_args(b), cs)) != cudaSuccess) st = cuda_fail(ctx, e, "launch_snm");
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
