// ffsva_snm.cu — K4: the stream-specialised network model (SNM) on tcgen05 tensor cores.
//
// Method: "SNM is a three-layer CNN (CONV, CONV, and FC)" that outputs the probability c of the
// target (L159) on 50x50 images (L167); frames with c >= t_pre go on (L165), t_pre from Eq. (2) (L193); SNM
// scores frames in dynamic batches so a stream's model is loaded once per batch (L219-L223).
// Readings: conv1 3->16 and conv2 16->32, 3x3, zero pad 1, ReLU, 2x2 max-pool (floor), FC
// 4608->1 logit (Q9, Q11); input (v-128)/128 (Q10); bf16 operands, fp32 accumulation, pooled conv1 rounded
// to bf16, conv2 output and FC in fp32 (Q15).
//
// B200 mapping — implicit GEMM with no im2col: every 3x3 tap is a shifted view of one shared-memory image.
//   * Activations are stored pixel-major with 8 channels per 16-byte row, which is exactly a row of a tcgen05
//     K-major no-swizzle core matrix. An M=128 tile is a 16-row x 8-column patch of output pixels: core
//     matrix j (8 rows of the MMA) = image row y0+j, so SBO = one padded image row; a tap (dy, dx) is the
//     same descriptor shifted by (dy*Wp + dx)*16 bytes.
//   * conv1 (K = 9 taps x 3 channels): each K=16 MMA carries two taps (one per 8-channel K-half, LBO = the
//     byte distance between them) -> 5 MMAs of N=16 per tile, 28 tiles per frame (4 row strips x 7 column
//     strips, the last strip of each overlapping so the 50x50 output is covered exactly).
//   * conv2 (K = 9 taps x 16 channels): the two K-halves are two 8-channel planes (LBO = plane size) ->
//     9 MMAs of N=32 per tile, 6 tiles (24x24 outputs survive the floor pooling; row/col 24 are skipped).
//   * Accumulators live in TMEM (M=128 lanes x N fp32 columns per tile). The tile shape puts each 2x2
//     pooling quad in lanes {l, l^1, l^8, l^9} of one warp, so max-pooling is two shuffles per value right
//     after tcgen05.ld; bias and ReLU commute with max and are applied after pooling.
//   * conv1's epilogue writes bf16 pooled activations straight into conv2's operand image; conv2's epilogue
//     multiplies the pooled features by the FC weights in fp32 and reduces to one logit per frame.
// One CTA (128 threads, 4 warps = the 4 TMEM lane quadrants) per SM-half, persistent over dynamic batches
// (chunks of <= BatchSize survivors of one stream): the stream's 30 KB weight image is copied into shared
// memory once per chunk. Thread 0 issues all MMAs and commits them to one mbarrier.
#include <cuda_bf16.h>

#include "ffsva_internal.h"

namespace ffsva {
namespace {

using namespace snm;

constexpr int kThreads = 128;
constexpr int X1W = 52, X1H = 52;                    // conv1 operand image: 50x50 + zero border, 8 ch (3 used)
constexpr int X1_BYTES = X1W * X1H * 16;             // 43264
constexpr int X2W = 26, X2H = 26;                    // conv2 operand image: 25x25 + zero border, 2 planes x 8 ch
constexpr int X2_PLANE = X2W * X2H * 16;             // 10816
constexpr int X2_BYTES = 2 * X2_PLANE;               // 21632
constexpr int OFF_X1 = 0;
constexpr int OFF_X2 = OFF_X1 + X1_BYTES;            // 43264
constexpr int OFF_WB = OFF_X2 + X2_BYTES;            // 64896
constexpr int OFF_RED = OFF_WB + BLOB_BYTES;         // 95312
constexpr int OFF_BAR = OFF_RED + 64;                // 95376
constexpr int OFF_TMEM = OFF_BAR + 8;                // 95384
constexpr int SMEM_BYTES = OFF_TMEM + 8;             // 95392
constexpr uint32_t kTmemCols = 256;

constexpr int kConv1Tiles = 28;
constexpr int kConv1Half = 14;
__constant__ int8_t c1_y0[4] = {0, 16, 32, 34};
__constant__ int8_t c1_x0[7] = {0, 8, 16, 24, 32, 40, 42};
// conv1 MMA j: A starts at tap (dy, dx); the second K-half is LBO bytes further.
__constant__ int8_t c1_dy[5] = {0, 1, 2, 0, 2};
__constant__ int8_t c1_dx[5] = {0, 0, 0, 2, 1};
__constant__ int16_t c1_lbo[5] = {16, 16, 16, X1W * 16, 16};

// ---------------------------------------------------------------- PTX wrappers (sm_100a)
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// UMMA shared-memory descriptor, K-major, SWIZZLE_NONE: start, leading (K) byte offset, stride (M/N) byte
// offset, all >> 4; version 1 (bits 46-47) for sm_100.
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}

// Instruction descriptor kind::f16: D fp32 (bits 4-5 = 1), A bf16 (7-9 = 1), B bf16 (10-12 = 1), both
// K-major, N >> 3 at bits 17-22, M >> 4 at bits 24-28.
__host__ __device__ constexpr uint32_t idesc_bf16(int M, int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void mma_bf16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar)
               : "memory");
}

__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
  }
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float (&v)[16]) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}

// 2x2 max over the pooling quad {l, l^1, l^8, l^9}.
__device__ __forceinline__ float quad_max(float x) {
  x = fmaxf(x, __shfl_xor_sync(0xffffffffu, x, 1));
  return fmaxf(x, __shfl_xor_sync(0xffffffffu, x, 8));
}

__device__ __forceinline__ uint32_t pack_bf16(float lo, float hi) {
  __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&h);
}

__device__ __forceinline__ uint32_t u8_to_bf16(uint32_t v) {  // (v - 128) / 128 is exact in bf16
  return (uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(((float)v - 128.0f) * 0.0078125f));
}

// ---------------------------------------------------------------- per-tile epilogues
// conv1 tile: TMEM columns [col, col+16) hold the 128x16 fp32 accumulator of the 16x8 output patch at
// (y0, x0). Pool, add bias, ReLU, round to bf16, store into conv2's operand image X2.
__device__ __forceinline__ void conv1_epilogue(uint32_t tmem, int col, int y0, int x0, uint8_t* X2,
                                               const float* b1, uint16_t* dbg) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float v[16];
  tmem_ld16(tmem + ((uint32_t)(32 * warp) << 16) + (uint32_t)col, v);
#pragma unroll
  for (int c = 0; c < 16; ++c) v[c] = quad_max(v[c]);
  const int q = (lane & 1) | ((lane >> 2) & 2);  // which 4 channels this quad lane writes
  const int y = y0 + 4 * warp + (lane >> 3), x = x0 + (lane & 7);
  const int py = y >> 1, px = x >> 1;
  float o[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const float s = q == 0 ? v[i] : q == 1 ? v[4 + i] : q == 2 ? v[8 + i] : v[12 + i];
    o[i] = fmaxf(s + b1[4 * q + i], 0.0f);
  }
  uint2 w;
  w.x = pack_bf16(o[0], o[1]);
  w.y = pack_bf16(o[2], o[3]);
  *reinterpret_cast<uint2*>(X2 + (q >> 1) * X2_PLANE + ((py + 1) * X2W + (px + 1)) * 16 + (q & 1) * 8) = w;
  if (dbg) *reinterpret_cast<uint2*>(dbg + (py * P1 + px) * 16 + 4 * q) = w;
}

// conv2 tile: 128x32 fp32 accumulator of the 16x8 patch at (y0, x0); returns this thread's FC partial sum.
__device__ __forceinline__ float conv2_epilogue(uint32_t tmem, int col, int y0, int x0, const float* b2,
                                                const float* wfc, float* dbg) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int q = (lane & 1) | ((lane >> 2) & 2);
  const int y = y0 + 4 * warp + (lane >> 3), x = x0 + (lane & 7);
  const int py = y >> 1, px = x >> 1;
  const bool own = (y0 == 0) || (py >= 8);  // pooled rows 4..7 belong to the y0 = 0 tile
  float acc = 0.0f;
#pragma unroll
  for (int h = 0; h < 2; ++h) {  // channels 16h .. 16h+15
    float v[16];
    tmem_ld16(tmem + ((uint32_t)(32 * warp) << 16) + (uint32_t)(col + 16 * h), v);
#pragma unroll
    for (int c = 0; c < 16; ++c) v[c] = quad_max(v[c]);
    // this lane handles channels 16h + 4q .. 16h + 4q + 3
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float s = q == 0 ? v[i] : q == 1 ? v[4 + i] : q == 2 ? v[8 + i] : v[12 + i];
      const int c = 16 * h + 4 * q + i;
      const float r = fmaxf(s + b2[c], 0.0f);
      if (own) {
        acc = fmaf(r, wfc[c * (P2 * P2) + py * P2 + px], acc);
        if (dbg) dbg[c * (P2 * P2) + py * P2 + px] = r;
      }
    }
  }
  return acc;
}

__global__ void __launch_bounds__(kThreads, 2) snm_kernel(SnmArgs a) {
  extern __shared__ __align__(128) uint8_t sm[];
  uint8_t* X1 = sm + OFF_X1;
  uint8_t* X2 = sm + OFF_X2;
  uint8_t* WB = sm + OFF_WB;
  float* red = reinterpret_cast<float*>(sm + OFF_RED);
  uint32_t* s_tmem = reinterpret_cast<uint32_t*>(sm + OFF_TMEM);
  __shared__ int s_chunk;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const uint32_t bar = smem_addr(sm + OFF_BAR);

  if (a.counts[1] == 0) return;  // no survivors in this batch

  // zero both operand images once: borders and unused channel slots stay zero for the whole kernel
  for (int i = tid; i < (X1_BYTES + X2_BYTES) / 16; i += kThreads)
    reinterpret_cast<uint4*>(sm)[i] = make_uint4(0u, 0u, 0u, 0u);
  if (tid == 0) {
    mbar_init(bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_addr(s_tmem)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *s_tmem;
  uint32_t phase = 0;

  const uint32_t x1a = smem_addr(X1), x2a = smem_addr(X2);
  const uint32_t w1a = smem_addr(WB + OFF_W1), w2a = smem_addr(WB + OFF_W2);
  const float* b1 = reinterpret_cast<const float*>(WB + OFF_B1);
  const float* b2 = reinterpret_cast<const float*>(WB + OFF_B2);
  const float* wfc = reinterpret_cast<const float*>(WB + OFF_WFC);
  const float bfc = 0.0f;  // read per chunk below
  (void)bfc;
  const int n_chunks = a.counts[1];

  for (;;) {
    if (tid == 0) s_chunk = atomicAdd(a.counts + 2, 1);
    __syncthreads();
    const int k = s_chunk;
    if (k >= n_chunks) break;
    const int start = a.chunks[k], end = a.chunks[k + 1];
    const FrameDesc fd0 = a.frames[a.work[start]];
    // dynamic batch: this stream's SNM weight image is loaded once for the whole chunk (L219)
    {
      const uint4* src = reinterpret_cast<const uint4*>(fd0.snm);
      uint4* dst = reinterpret_cast<uint4*>(WB);
      for (int i = tid; i < BLOB_BYTES / 16; i += kThreads) dst[i] = __ldg(src + i);
    }
    const float fc_bias = __ldg(reinterpret_cast<const float*>(fd0.snm + OFF_BFC));
    uint32_t cnt_pass = 0, cnt_c0 = 0, cnt_c1 = 0, cnt_c2 = 0;

    for (int j = start; j < end; ++j) {
      const int f = a.work[j];
      // ---- input: D50 u8 -> (v-128)/128 bf16 into X1 interior (pixel = 16 B: 3 channels + 5 zeros)
      const uint8_t* d = a.d50 + (int64_t)f * a.d50_stride;
      for (int p = tid; p < IN * IN; p += kThreads) {
        const int y = p / IN, x = p - y * IN;
        const uint32_t c0 = d[3 * p], c1 = d[3 * p + 1], c2 = d[3 * p + 2];
        uint4 w;
        w.x = u8_to_bf16(c0) | (u8_to_bf16(c1) << 16);
        w.y = u8_to_bf16(c2);
        w.z = 0u;
        w.w = 0u;
        *reinterpret_cast<uint4*>(X1 + ((y + 1) * X1W + (x + 1)) * 16) = w;
      }
      fence_proxy_async();
      fence_before();
      __syncthreads();

      // ---- conv1, two halves of 14 tiles (224 TMEM columns each)
      uint16_t* dbg1 = a.dbg_p1 ? a.dbg_p1 + (int64_t)j * (P1 * P1 * 16) : nullptr;
      for (int half = 0; half < 2; ++half) {
        if (tid == 0) {
          fence_after();
          for (int t = half * kConv1Half; t < (half + 1) * kConv1Half; ++t) {
            const int y0 = c1_y0[t / 7], x0 = c1_x0[t % 7];
            const uint32_t dcol = tmem + (uint32_t)((t - half * kConv1Half) * 16);
#pragma unroll
            for (int m = 0; m < CONV1_MMAS; ++m) {
              const uint32_t aaddr = x1a + (uint32_t)(((y0 + c1_dy[m]) * X1W + (x0 + c1_dx[m])) * 16);
              mma_bf16(dcol, umma_desc(aaddr, (uint32_t)c1_lbo[m], X1W * 16),
                       umma_desc(w1a + (uint32_t)(m * 2 * C1 * 16), C1 * 16, 128), idesc_bf16(128, 16),
                       m > 0 ? 1u : 0u);
            }
          }
          mma_commit(bar);
        }
        __syncwarp();
        mbar_wait(bar, phase);
        phase ^= 1u;
        fence_after();
        for (int t = half * kConv1Half; t < (half + 1) * kConv1Half; ++t)
          conv1_epilogue(tmem, (t - half * kConv1Half) * 16, c1_y0[t / 7], c1_x0[t % 7], X2, b1, dbg1);
        fence_before();
        __syncthreads();
      }

      // ---- conv2: 6 tiles x 9 taps, N = 32
      fence_proxy_async();
      __syncthreads();
      if (tid == 0) {
        fence_after();
        for (int t = 0; t < 6; ++t) {
          const int y0 = (t / 3) * 8, x0 = (t % 3) * 8;
          const uint32_t dcol = tmem + (uint32_t)(t * 32);
#pragma unroll
          for (int tap = 0; tap < 9; ++tap) {
            const int dy = tap / 3, dx = tap % 3;
            const uint32_t aaddr = x2a + (uint32_t)(((y0 + dy) * X2W + (x0 + dx)) * 16);
            mma_bf16(dcol, umma_desc(aaddr, X2_PLANE, X2W * 16), umma_desc(w2a + (uint32_t)(tap * 2 * C2 * 16), C2 * 16, 128),
                     idesc_bf16(128, 32), tap > 0 ? 1u : 0u);
          }
        }
        mma_commit(bar);
      }
      __syncwarp();
      mbar_wait(bar, phase);
      phase ^= 1u;
      fence_after();
      float* dbg2 = a.dbg_p2 ? a.dbg_p2 + (int64_t)j * NF : nullptr;
      float acc = 0.0f;
      for (int t = 0; t < 6; ++t) acc += conv2_epilogue(tmem, t * 32, (t / 3) * 8, (t % 3) * 8, b2, wfc, dbg2);
      // ---- FC reduction -> logit -> Eq. (2) decision
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
      if (lane == 0) red[warp] = acc;
      fence_before();
      __syncthreads();
      if (tid == 0) {
        const float logit = fc_bias + ((red[0] + red[1]) + (red[2] + red[3]));
        const FrameDesc fd = a.frames[f];
        const uint8_t p = logit >= fd.L_t ? 1 : 0;
        const uint8_t cls = logit < fd.L_low ? 0 : (logit > fd.L_high ? 2 : 1);
        a.logit[f] = logit;
        a.snm_pass[f] = p;
        a.snm_class[f] = cls;
        cnt_pass += p;
        cnt_c0 += cls == 0;
        cnt_c1 += cls == 1;
        cnt_c2 += cls == 2;
      }
    }
    if (tid == 0 && a.stats) {
      unsigned long long* st = a.stats + (int64_t)fd0.slot * NSTAT;
      atomicAdd(st + 2, (unsigned long long)cnt_pass);
      atomicAdd(st + 4, (unsigned long long)cnt_c0);
      atomicAdd(st + 5, (unsigned long long)cnt_c1);
      atomicAdd(st + 6, (unsigned long long)cnt_c2);
    }
    __syncthreads();
  }

  fence_before();
  __syncthreads();
  if (warp == 0) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
  }
}

}  // namespace

int snm_smem_bytes() { return SMEM_BYTES; }

cudaError_t snm_configure() {
  static bool done = false;
  if (done) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(snm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
  if (e == cudaSuccess) done = true;
  return e;
}

cudaError_t launch_snm(const SnmArgs& a, cudaStream_t st) {
  snm_kernel<<<a.grid, kThreads, SMEM_BYTES, st>>>(a);
  return cudaGetLastError();
}

}  // namespace ffsva
