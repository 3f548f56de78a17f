// Achievable HBM read bandwidth on B200 for K1-like streaming (ceiling for the SDD kernel's roofline):
//  (a) LDG.128 non-allocating streaming reduce, grid = 148 x k CTAs, grid-stride;
//  (b) cp.async.bulk into shared memory (TMA engine) per CTA chunk + trivial reduce.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o read_bw read_bw.cu && ./read_bw
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void ldg_reduce(const uint4* __restrict__ p, size_t n16, unsigned long long* out) {
  uint32_t acc = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p + i));
    acc += v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x12345678u) atomicAdd(out, 1ull);
}

__global__ void ldg_reduce_unroll(const uint4* __restrict__ p, size_t n16, unsigned long long* out) {
  uint32_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  for (; i + 7 * stride < n16; i += 8 * stride) {
    uint4 v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k)
      asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[k].x), "=r"(v[k].y), "=r"(v[k].z), "=r"(v[k].w) : "l"(p + i + k * stride));
#pragma unroll
    for (int k = 0; k < 8; ++k) acc += v[k].x ^ v[k].y ^ v[k].z ^ v[k].w;
  }
  for (; i < n16; i += stride) acc += p[i].x;
  if (acc == 0x12345678u) atomicAdd(out, 1ull);
}

__global__ void bulk_reduce(const uint8_t* __restrict__ p, size_t chunks, int chunk_bytes, unsigned long long* out) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar;
  const uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar);
  uint32_t acc = 0, phase = 0;
  if (threadIdx.x == 0) { asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b)); }
  __syncthreads();
  for (size_t c = blockIdx.x; c < chunks; c += gridDim.x) {
    if (threadIdx.x == 0) {
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(chunk_bytes));
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"((uint32_t)__cvta_generic_to_shared(sm)), "l"(p + c * chunk_bytes), "r"(chunk_bytes), "r"(b) : "memory");
    }
    uint32_t done = 0;
    while (!done) asm volatile("{\n.reg .pred q;\nmbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2;\nselp.u32 %0,1,0,q;\n}" : "=r"(done) : "r"(b), "r"(phase) : "memory");
    phase ^= 1;
    for (int i = threadIdx.x; i < chunk_bytes / 16; i += blockDim.x) { uint4 v = ((uint4*)sm)[i]; acc += v.x ^ v.w; }
    __syncthreads();
  }
  if (acc == 0x12345678u) atomicAdd(out, 1ull);
}

int main() {
  const size_t bytes = 2488320000ull;  // one M2 step: 900 frames of 1280x720 RGB8
  uint8_t* d; unsigned long long* o;
  cudaMalloc(&d, bytes * 2); cudaMalloc(&o, 8); cudaMemset(d, 1, bytes * 2);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  auto run = [&](const char* name, auto fn) {
    for (int w = 0; w < 3; ++w) fn(w & 1);
    float best = 1e9;
    for (int it = 0; it < 10; ++it) {
      cudaEventRecord(e0); fn(it & 1); cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
    }
    printf("%-40s %8.3f ms  %7.1f GB/s\n", name, best, bytes / (best / 1e3) / 1e9);
  };
  for (int k : {4, 8, 16, 32}) {
    char nm[64]; snprintf(nm, 64, "ldg128 nc grid=%dx%d thr=512", sms, k);
    run(nm, [&](int h) { ldg_reduce<<<sms * k / 2, 512>>>((const uint4*)(d + h * bytes), bytes / 16, o); });
  }
  for (int k : {2, 4, 8}) {
    char nm[64]; snprintf(nm, 64, "ldg128 nc unroll8 grid=%dx%d thr=256", sms, k);
    run(nm, [&](int h) { ldg_reduce_unroll<<<sms * k, 256>>>((const uint4*)(d + h * bytes), bytes / 16, o); });
  }
  for (int cb : {16384, 32768, 65536}) {
    cudaFuncSetAttribute(bulk_reduce, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    for (int k : {2, 4, 6}) {
      if (cb * k > 200 * 1024) continue;
      char nm[64]; snprintf(nm, 64, "bulk %d B chunks, %d CTAs/SM", cb, k);
      run(nm, [&](int h) { bulk_reduce<<<sms * k, 256, cb>>>(d + h * bytes, bytes / cb, cb, o); });
    }
  }
  return 0;
}
