/*
 * synth_cuda.cu — device twin of the synthetic video generator (workload
 * generation only; see ffsva_synth.h). Fills large HBM frame pools for the
 * benchmark without a PCIe round trip. Built into synth/libffsva_synth_cuda.so.
 * Byte-identical to synth_host.c because both evaluate the same inline
 * functions of ffsva_synth.h (checked by tests/test_synth.py on the GPU).
 */
#include <cuda_runtime.h>
#include "ffsva_synth.h"

namespace {

__global__ void synth_ctx_kernel(ffsva_synth_params p, const int32_t* __restrict__ streams,
                                 const int64_t* __restrict__ frames, int32_t n, int32_t ref,
                                 ffsva_synth_ctx* __restrict__ ctx) {
  int32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) ffsva_synth_frame_ctx(&p, streams[i], frames[i], ref, &ctx[i]);
}

/* One thread per pixel; blockIdx.y walks frames. */
__global__ void synth_pixel_kernel(const ffsva_synth_ctx* __restrict__ ctx, int32_t W, int32_t H,
                                   uint8_t* __restrict__ out, int64_t frame_stride, int64_t pitch) {
  const ffsva_synth_ctx c = ctx[blockIdx.y];
  uint8_t* base = out + (int64_t)blockIdx.y * frame_stride;
  int64_t npix = (int64_t)W * H;
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < npix; q += (int64_t)gridDim.x * blockDim.x) {
    int32_t y = (int32_t)(q / W), x = (int32_t)(q % W);
    uint8_t* px = base + (int64_t)y * pitch + 3 * x;
    px[0] = ffsva_synth_pixel(&c, y, x, 0);
    px[1] = ffsva_synth_pixel(&c, y, x, 1);
    px[2] = ffsva_synth_pixel(&c, y, x, 2);
  }
}

}  // namespace

extern "C" int ffsva_synth_frames_cuda(const ffsva_synth_params* p, const int32_t* d_streams, const int64_t* d_frames,
                                       int32_t n, int32_t ref, uint8_t* d_out, int64_t frame_stride, int64_t pitch,
                                       void* stream) {
  if (n <= 0) return 0;
  cudaStream_t st = (cudaStream_t)stream;
  ffsva_synth_ctx* ctx = nullptr;
  if (cudaMallocAsync((void**)&ctx, sizeof(ffsva_synth_ctx) * n, st) != cudaSuccess) return -1;
  synth_ctx_kernel<<<(n + 127) / 128, 128, 0, st>>>(*p, d_streams, d_frames, n, ref, ctx);
  for (int32_t f0 = 0; f0 < n; f0 += 65535) {
    int32_t nf = n - f0 < 65535 ? n - f0 : 65535;
    dim3 grid(128, nf);
    synth_pixel_kernel<<<grid, 256, 0, st>>>(ctx + f0, p->width, p->height, d_out + (int64_t)f0 * frame_stride,
                                             frame_stride, pitch);
  }
  cudaFreeAsync(ctx, st);
  return cudaGetLastError() == cudaSuccess ? 0 : -3;
}
