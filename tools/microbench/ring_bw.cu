// Read bandwidth of the K1 narrow-row access pattern without its arithmetic: persistent CTAs, one producer thread
// bulk-copying consecutive chunks (cp.async.bulk, L2 evict-first) into a ring of NS shared-memory stages, consumer
// warps that only wait for each stage and release it. Prints GB/s per (chunk bytes, stages, consumer warps, CTAs
// per SM) over a buffer of `MB` megabytes (default 207: config M1's 300 frames of 640x360).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ring_bw ring_bw.cu && ./ring_bw [MB]
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>

__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done = 0;
  while (!done)
    asm volatile("{\n.reg .pred q;\nmbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2;\nselp.u32 %0,1,0,q;\n}"
                 : "=r"(done)
                 : "r"(bar), "r"(parity)
                 : "memory");
}

__global__ void ring(const uint8_t* __restrict__ p, int64_t chunks, int chunk_bytes, int ns, int touch,
                     unsigned long long* out) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t full[16], empty[16];
  const int cons = blockDim.x / 32 - 1;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t c0 = blockIdx.x * chunks / gridDim.x, c1 = (blockIdx.x + 1) * chunks / gridDim.x;
  const int n = (int)(c1 - c0);
  if (threadIdx.x == 0) {
    for (int s = 0; s < ns; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&full[s])));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(&empty[s])),
                   "r"(cons));
    }
  }
  __syncthreads();
  if (warp == cons) {
    if (lane == 0) {
      uint64_t pol;
      asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
      for (int i = 0; i < n; ++i) {
        const int s = i % ns;
        if (i >= ns) mbar_wait((uint32_t)__cvta_generic_to_shared(&empty[s]), (uint32_t)((i / ns - 1) & 1));
        const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&full[s]);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(chunk_bytes) : "memory");
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::
                "r"((uint32_t)__cvta_generic_to_shared(sm + (size_t)s * chunk_bytes)),
            "l"(p + (c0 + i) * chunk_bytes), "r"(chunk_bytes), "r"(bar), "l"(pol)
            : "memory");
      }
    }
    return;
  }
  uint32_t acc = 0;
  for (int i = 0; i < n; ++i) {
    const int s = i % ns;
    mbar_wait((uint32_t)__cvta_generic_to_shared(&full[s]), (uint32_t)((i / ns) & 1));
    if (touch) {  // each consumer warp reads its share of the stage once (LDS.128)
      const uint4* q = reinterpret_cast<const uint4*>(sm + (size_t)s * chunk_bytes);
      for (int k = warp * 32 + lane; k < chunk_bytes / 16; k += cons * 32) acc += q[k].x ^ q[k].w;
    }
    __syncwarp();
    if (lane == 0)
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(&empty[s]))
                   : "memory");
  }
  if (acc == 0x12345678u) atomicAdd(out, 1ull);
}

int main(int argc, char** argv) {
  const size_t mb = argc > 1 ? (size_t)atoi(argv[1]) : 207;
  const size_t bytes = mb << 20;
  uint8_t* d;
  unsigned long long* o;
  cudaMalloc(&d, bytes + (1 << 20));
  cudaMalloc(&o, 8);
  cudaMemset(d, 1, bytes);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaFuncSetAttribute(ring, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int chunk_sizes[] = {7680, 15360, 28800, 57600};
  const int stages[] = {2, 4, 6, 8, 12};
  const int warps[] = {1, 4, 10};
  for (int touch = 0; touch < 2; ++touch)
    for (int cb : chunk_sizes)
      for (int ns : stages)
        for (int cw : warps) {
          const size_t smem = (size_t)ns * cb;
          if (smem > 220 * 1024) continue;
          int per_sm = 0;
          cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, ring, 32 * (cw + 1), smem);
          if (per_sm < 1) continue;
          const int64_t chunks = (int64_t)(bytes / cb);
          const int grid = sms * per_sm;
          ring<<<grid, 32 * (cw + 1), smem>>>(d, chunks, cb, ns, touch, o);
          cudaEventRecord(e0);
          const int reps = 5;
          for (int r = 0; r < reps; ++r) ring<<<grid, 32 * (cw + 1), smem>>>(d, chunks, cb, ns, touch, o);
          cudaEventRecord(e1);
          cudaEventSynchronize(e1);
          float ms;
          cudaEventElapsedTime(&ms, e0, e1);
          printf("touch %d chunk %6d stages %2d cons_warps %2d ctas/sm %d: %7.1f GB/s (%.1f us)\n", touch, cb, ns, cw,
                 per_sm, (double)chunks * cb * reps / (ms / 1e3) / 1e9, ms * 1e3 / reps);
        }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
  return 0;
}
