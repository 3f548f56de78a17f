// tcgen05.mma issue rate for the small shapes K4 (the SNM) uses: M128 x N{16..256} x K16 bf16 -> fp32 TMEM,
// one CTA per SM, one elected thread issuing `reps` MMAs round-robin over CH accumulators (no dependence between
// chains), then one commit. All operands are warp-uniform and the issue loop is unrolled 8x, so the loop adds no
// more than a counter. Prints clocks per MMA and the implied fraction of the SM's dense-bf16 rate
// (M128 N256 K16 = 1,048,576 FLOP = 128 clk at 8,192 FLOP/clk).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mma_rate mma_rate.cu && ./mma_rate
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>

__device__ __forceinline__ uint32_t saddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((a >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}

template <int CH, int M>
__global__ void mma_rate(int N, int reps, unsigned long long* clk) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t s_tmem;
  for (int i = threadIdx.x; i < 65536 / 16; i += blockDim.x) reinterpret_cast<uint4*>(sm)[i] = make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(saddr(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(saddr(&s_tmem)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = s_tmem;
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
  const uint32_t a = saddr(sm), b = saddr(sm + 32768);
  if (threadIdx.x < 32) {
    const uint64_t bd = desc(b, 4096, 128);
    const uint64_t a0 = desc(a, 2048, 128);
    long long t0 = clock64();
    for (int r = 0; r < reps; r += 8) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const uint32_t d = tmem + (uint32_t)((i % CH) * (512 / CH));
        asm volatile(
            "{\n\t.reg .pred e, p;\n\telect.sync _|e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(d),
            "l"(a0 + (uint64_t)i), "l"(bd), "r"(idesc), "n"(1));
      }
    }
    asm volatile(
        "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}\n" ::"r"(saddr(&bar))
        : "memory");
    uint32_t done = 0;
    while (!done)
      asm volatile("{\n.reg .pred q;\nmbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0;\nselp.u32 %0,1,0,q;\n}"
                   : "=r"(done)
                   : "r"(saddr(&bar))
                   : "memory");
    long long t1 = clock64();
    if (threadIdx.x == 0) clk[blockIdx.x] = (unsigned long long)(t1 - t0);
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}

template <int CH, int M>
void run(int sms, int N, unsigned long long* d) {
  cudaFuncSetAttribute(mma_rate<CH, M>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
  unsigned long long h[256];
  const int reps = 4096;
  for (int it = 0; it < 2; ++it) mma_rate<CH, M><<<sms, 128, 65536>>>(N, reps, d);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    printf("error %s\n", cudaGetErrorString(e));
    exit(1);
  }
  cudaMemcpy(h, d, sms * 8, cudaMemcpyDeviceToHost);
  double mean = 0;
  for (int i = 0; i < sms; ++i) mean += (double)h[i] / sms;
  const double per = mean / reps;
  const double ideal = (double)M * N / 256.0;
  printf("M%d N%-3d K16 chains %d: %6.2f clk/MMA (peak-rate %5.1f clk) -> %.2f of the SM's bf16 peak\n", M, N, CH, per,
         ideal, ideal / per);
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long* d;
  cudaMalloc(&d, sms * 8);
  for (int N : {16, 32, 48, 64, 96, 128, 192, 256}) {
    run<1, 128>(sms, N, d);
    run<2, 128>(sms, N, d);
    if (N <= 128) run<4, 128>(sms, N, d);
  }
  for (int N : {64, 128, 256}) run<2, 64>(sms, N, d);
  return 0;
}
