// ffsva_snm.cu — K4: the stream-specialised network model (SNM) on tcgen05 tensor cores.
//
// Method: "SNM is a three-layer CNN (CONV, CONV, and FC)" that outputs the probability c of the
// target (L159) on 50x50 images (L167); frames with c >= t_pre go on (L165), t_pre from Eq. (2) (L193); SNM
// scores frames in dynamic batches so a stream's model is loaded once per batch (L219-L223).
// Readings: conv1 3->16 and conv2 16->32, 3x3, zero pad 1, ReLU, 2x2 max-pool (floor), FC
// 4608->1 logit (Q9, Q11); input (v-128)/128 (Q10); bf16 operands, fp32 accumulation, pooled conv1 rounded
// to bf16, conv2 output and FC in fp32 (Q15).
//
// B200 mapping — implicit GEMMs, no im2col, pooling folded into the N dimension:
//   * GEMM rows are POOLED output pixels; a 2x2-pool's four conv outputs are four accumulator column groups of the
//     same TMEM lane, so the max-pool is an in-register max over four column groups; bias and ReLU commute with max
//     and are applied once after it (max(v0..v3, -b) + b).
//   * Cost model (tools/microbench/mma_rate.cu, one B200): an M128 K16 bf16 MMA costs 32 + N/4 clocks up to N = 128
//     (shared-memory operand reads: the 4 KB A tile plus N x 32 B of B at 128 B/clk) and N/2 clocks beyond, so an MMA
//     should read each A tile for as many output columns as possible.
//   * conv1: the A row of pooled pixel (py, px) is its 4x4 input patch row dy (padded input row 2py + dy, columns
//     2px..2px+3) x 4 channel slots (3 used); the four pool positions differ only in where their 3x3 kernel sits in
//     the patch, so ONE A operand feeds N = 4 positions x 16 channels: per 128-row tile two N = 64 MMAs (patch rows
//     1, 2) and two N = 32 MMAs (row 0 reaches only positions a = 0, row 3 only a = 1). The input lives in two
//     row-parity planes of 26 two-pixel entries per row, so GEMM row r = plane entry r: pooled pixel (r / 26, r % 26)
//     and every patch row is a constant-stride view (rows 16 B apart, K-halves 16 B apart, 8-row groups 128 B apart):
//     6 tiles cover the 25 x 25 pooled outputs (650 of 768 rows useful).
//   * conv2: the 4x4 patch of a pooled output pixel has 16 cells; a cell's A view (16 channels = two 8-channel
//     parity planes, rows = plane entries r, pooled pixel (r / 14, r % 14)) serves every pool position whose 3x3
//     window holds it, so the 36 (position, tap) products of a tile take 18 MMAs (4 x N128, 6 x N64, 8 x N32,
//     snm::conv2_mma) instead of 36 x N32; 2 tiles cover the 12 x 12 pooled outputs.
//   * conv1's epilogue writes bf16 pooled activations straight into conv2's parity planes; conv2's epilogue
//     multiplies the pooled features by the FC weights (bf16 values) in fp32 and reduces to one logit per frame.
// One warp-specialised persistent CTA per SM (512 threads, all 512 TMEM columns), frames pipelined through
// mbarrier rings: warp 0 stages each frame's D50 image (bulk copy) and the stream's weight image when the stream
// changes; warps 2-3 convert D50 to conv1's bf16 operand (two buffers); warp 1 issues the MMAs (conv1 tiles into a
// ring of four 64-column TMEM slots, conv2 tiles into two 128-column slots, frame j+1's conv1 interleaved with frame
// j's conv2); warps 4-7 and 8-11 drain the even and the odd conv1 tiles into conv2's operand (two buffers); warps
// 12-15 drain conv2 tiles, apply the FC and decide. CTA c scores the survivors [c*m/G, (c+1)*m/G) of the stream-major work order, so a stream's
// weights are loaded once per CTA and per stream (a dynamic batch's frames are consecutive, L219).
#include <cuda_bf16.h>

#include "ffsva_internal.h"
#include "ffsva_ptx.h"

namespace ffsva {
namespace {

using namespace snm;
using namespace ptx;

#ifndef FFSVA_K4_ABL
#define FFSVA_K4_ABL 0  // A/B only (wrong results): 1 no conversion, 2 no conv1 epilogue, 4 no conv2 epilogue, 8 no MMAs
#endif
#ifndef FFSVA_K4_PROF
#define FFSVA_K4_PROF 0  // A/B only: per-wait clock totals of CTA 0, printed at exit
#endif
#if FFSVA_K4_PROF
}  // namespace
}  // namespace ffsva
#include <cstdio>
namespace ffsva {
namespace {
__shared__ unsigned long long s_prof[16];
#define KW(id, call)                                                        \
  do {                                                                      \
    const long long _t0 = clock64();                                        \
    call;                                                                   \
    if ((threadIdx.x & 31) == 0) atomicAdd(&s_prof[id], (unsigned long long)(clock64() - _t0)); \
  } while (0)
#else
#define KW(id, call) call
#endif
constexpr int kThreads = 512;
constexpr int NIN = 3;   // D50 staging ring
constexpr int NA1 = 2;   // conv1 operand buffers
constexpr int NA2 = 3;   // conv2 operand buffers (frames j-2 .. j: conv2 runs two frames behind conv1)
constexpr int kConvWarps = 6;  // warps 2-7 convert
constexpr int NI = 16;   // per-frame info ring (frames in flight between the producer and the conv2 epilogue)
// conv1 operand: 2 row-parity planes x 26 rows x 26 entries (two padded pixels x 4 channel slots, 16 B)
constexpr int A1_ROW = 26;                                  // entries per plane row
constexpr int A1_PLANE = 26 * A1_ROW * 16;                  // 10816 B
constexpr int A1_BYTES = 23552;                             // + tail read by junk rows of tile 5 (entry 1470 max)
static_assert(A1_BYTES >= (A1_PLANE / 16 + 26 + 767 + 1 + 1) * 16, "conv1 operand tail");
constexpr int kTiles1 = 6;
// conv2 operand: 8 planes [ypar][xpar][chalf] x 14 rows x 14 entries of 8 channels (padded pooled conv1 27x27)
constexpr int A2_COLS = 14;
constexpr int A2_PLANE = 14 * A2_COLS * 16 + 32;            // 3168 B: the two column-parity planes of a channel half
                                                            // are 2 * 3168 = 64 (mod 128) B apart, so the conv1
                                                            // epilogue's stores of both parities do not share banks
constexpr int A2_BYTES = 26512;                             // + tail read by junk rows of tile 1 (entry 1656 max)
static_assert(A2_BYTES >= (7 * A2_PLANE / 16 + 255 + A2_COLS + 1 + 1) * 16, "conv2 operand tail");
constexpr int D50_BYTES = 7504;                             // staged D50 image (one frame)

constexpr int OFF_WB = 0;                                   // the stream's weight image (snm::BLOB_BYTES)
constexpr int OFF_A1 = 63744;                               // NA1 buffers
constexpr int OFF_A2 = OFF_A1 + NA1 * A1_BYTES;             // 110848, NA2 buffers
constexpr int OFF_IN = OFF_A2 + NA2 * A2_BYTES;             // 190384, NIN stages
constexpr int OFF_INFO = OFF_IN + NIN * D50_BYTES;          // 212896: int2 [NI] (frame, flags)
constexpr int OFF_RED = OFF_INFO + NI * 8;                  // float [2][4]
constexpr int OFF_BAR = OFF_RED + 32;
// mbarriers (8 B each)
constexpr int B_IN_FULL = 0, B_IN_EMPTY = B_IN_FULL + NIN, B_W_FULL = B_IN_EMPTY + NIN, B_W_EMPTY = B_W_FULL + 1,
              B_INFO_EMPTY = B_W_EMPTY + 1, B_A1_FULL = B_INFO_EMPTY + NI, B_A1_EMPTY = B_A1_FULL + NA1,
              B_C1_FULL = B_A1_EMPTY + NA1, B_C1_EMPTY = B_C1_FULL + 4, B_A2_FULL = B_C1_EMPTY + 4,
              B_A2_EMPTY = B_A2_FULL + NA2, B_C2_FULL = B_A2_EMPTY + NA2, B_C2_EMPTY = B_C2_FULL + 2,
              N_BARS = B_C2_EMPTY + 2;
constexpr int OFF_TMEM = OFF_BAR + N_BARS * 8;
constexpr int SMEM_BYTES = OFF_TMEM + 16;
static_assert(OFF_A1 >= BLOB_BYTES && OFF_A1 % 128 == 0, "weight image fits");
static_assert(OFF_A2 % 16 == 0 && OFF_IN % 16 == 0 && OFF_INFO % 16 == 0 && OFF_BAR % 8 == 0, "alignment");
static_assert(SMEM_BYTES <= 227 * 1024, "one CTA per SM");
constexpr uint32_t kTmemCols = 512;                         // conv1: 4 x 64 columns; conv2: 256 + 2 x 128
constexpr uint32_t kC2Col = 256;

// per-frame flags in the info ring
constexpr int F_SEG_FIRST = 1, F_SEG_LAST = 2, F_POP_OPEN = 4;

__device__ __forceinline__ float max3(float a, float b, float c) {
  float d;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
  return d;
}
// max over the four pool positions (16 consecutive channels from column col of each group), then bias and ReLU:
// max_q(v_q + b) clamped at 0 == max(v_0, v_1, v_2, v_3, -b) + b (fp addition is monotone)
__device__ __forceinline__ void pool_bias_relu16(uint32_t taddr, int col, int group_cols, const float* bias,
                                                 float (&v)[16]) {
  uint32_t r0[16], r1[16], r2[16], r3[16];
  tmem_ld16(taddr + (uint32_t)col, r0);
  tmem_ld16(taddr + (uint32_t)(col + group_cols), r1);
  tmem_ld16(taddr + (uint32_t)(col + 2 * group_cols), r2);
  tmem_ld16(taddr + (uint32_t)(col + 3 * group_cols), r3);
  tmem_wait_ld2(r0, r1);
  reg_fence2(r2, r3);
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    const float b = bias[i];
    v[i] = max3(max3(__uint_as_float(r0[i]), __uint_as_float(r1[i]), __uint_as_float(r2[i])), __uint_as_float(r3[i]),
                -b) + b;
  }
}

__device__ __forceinline__ const uint8_t* d50_of(const SnmArgs& a, int f) {
  return a.d50 + (a.d50_index ? (int64_t)__ldg(a.d50_index + f) : (int64_t)f) * a.d50_stride;
}

// ---------------------------------------------------------------- MMA issue (warp 1, one elected lane)
// conv1 tile t of the frame in A1 buffer a1 into TMEM columns d..d+63 ([a][b][16 channels]).
__device__ __forceinline__ void issue_conv1_tile(uint32_t d, uint32_t a1, int t, uint32_t w1) {
  const uint32_t id64 = idesc_bf16(128, 64), id32 = idesc_bf16(128, 32);
  const uint32_t r0 = a1 + (uint32_t)(128 * t * 16);
  // patch row dy: plane dy & 1, plane row offset dy >> 1 (26 entries)
  const uint32_t row0 = r0, row1 = r0 + A1_PLANE, row2 = r0 + A1_ROW * 16, row3 = r0 + A1_PLANE + A1_ROW * 16;
  mma_bf16(d, umma_desc(row1, 16, 128), umma_desc(w1 + 1 * 2048, 1024, 128), id64, 0u);
  mma_bf16(d, umma_desc(row2, 16, 128), umma_desc(w1 + 2 * 2048, 1024, 128), id64, 1u);
  mma_bf16(d, umma_desc(row0, 16, 128), umma_desc(w1 + 0 * 2048, 1024, 128), id32, 1u);
  mma_bf16(d + 32, umma_desc(row3, 16, 128), umma_desc(w1 + 3 * 2048 + 512, 1024, 128), id32, 1u);
}

// conv2 tile u of the frame in A2 buffer a2 into TMEM columns d..d+127 ([group][32 channels]).
__device__ __forceinline__ void issue_conv2_tile(uint32_t d, uint32_t a2, int u, uint32_t w2) {
#pragma unroll
  for (int i = 0; i < kConv2Mmas; ++i) {
    const Conv2Mma mm = conv2_mma(i);
    const uint32_t plane = (uint32_t)((((mm.cy & 1) * 2 + (mm.cx & 1)) * 2) * A2_PLANE);
    const uint32_t start = (uint32_t)((128 * u + (mm.cy >> 1) * A2_COLS + (mm.cx >> 1)) * 16);
    const int N = 32 * mm.ng;
    mma_bf16(d + (uint32_t)(32 * mm.g0), umma_desc(a2 + plane + start, A2_PLANE, 128),
             umma_desc(w2 + (uint32_t)mm.boff, (uint32_t)(N * 16), 128), idesc_bf16(128, N), i > 0 ? 1u : 0u);
  }
}

// ---------------------------------------------------------------- input conversion (warps 2-3)
// D50 (50x50x3 u8, row-major) -> (v-128)/128 bf16 (C5, exact) into conv1's row-parity planes. A thread writes one
// 16-byte entry = padded columns (2e, 2e+1) = image columns (2e-1, 2e) of one row, 4 channel slots each (3 used);
// its 6 source bytes are funnel-shifted out of two aligned words (lanes ~6 B apart: conflict-free loads, contiguous
// 16-byte stores). bf16 of (v-128)/128 = high half of fma(2^23 + v, 1/128, -65537), 2^23 + v by one PRMT.
__device__ __forceinline__ uint32_t bf16_hi_of_byte(uint32_t w, uint32_t k) {
  return __float_as_uint(fmaf(__uint_as_float(__byte_perm(w, 0x4B000000u, 0x7440u | k)), 0.0078125f, -65537.0f));
}
__device__ __forceinline__ void convert_input(const uint8_t* d, uint8_t* A1, int t) {
  constexpr int kEntries = IN * A1_ROW;  // 50 rows x 26 entries
  constexpr int kStride = 32 * kConvWarps;
#pragma unroll
  for (int i = 0; i < (kEntries + kStride - 1) / kStride; ++i) {
    const int q = t + i * kStride;
    if (q >= kEntries) break;
    const int y = q / A1_ROW, e = q - y * A1_ROW;
    // bytes [o, o + 6) of the image: columns 2e-1 and 2e (column -1 / 50 are the zero border)
    const int o = y * 3 * IN + 6 * e - 3;
    const int ob = o < 0 ? 0 : o & ~3;  // aligned base word (the first entry of row 0 starts before the image)
    const uint32_t* w = reinterpret_cast<const uint32_t*>(d + ob);
    const uint32_t w0 = w[0], w1 = w[1], w2 = w[2];
    const uint32_t sh = (uint32_t)(o - ob) * 8u;  // 0..24 bits (o >= ob except row 0, entry 0: handled below)
    const uint32_t lo = __funnelshift_r(w0, w1, sh), hi = __funnelshift_r(w1, w2, sh);  // bytes o .. o+7
    uint32_t c[6];
    c[0] = bf16_hi_of_byte(lo, 0);
    c[1] = bf16_hi_of_byte(lo, 1);
    c[2] = bf16_hi_of_byte(lo, 2);
    c[3] = bf16_hi_of_byte(lo, 3);
    c[4] = bf16_hi_of_byte(hi, 0);
    c[5] = bf16_hi_of_byte(hi, 1);
    uint4 v = make_uint4(__byte_perm(c[0], c[1], 0x7632), c[2] >> 16, __byte_perm(c[3], c[4], 0x7632), c[5] >> 16);
    if (e == 0) v.x = v.y = 0u;                   // column -1: left border
    if (e == A1_ROW - 1) v.z = v.w = 0u;          // column 50: right border
    if (o < 0) {                                  // row 0, entry 0: column 0 is bytes 0..2
      v.z = __byte_perm(bf16_hi_of_byte(w0, 0), bf16_hi_of_byte(w0, 1), 0x7632);
      v.w = bf16_hi_of_byte(w0, 2) >> 16;
    }
    const int Y = y + 1;
    *reinterpret_cast<uint4*>(A1 + (Y & 1) * A1_PLANE + ((Y >> 1) * A1_ROW + e) * 16) = v;
  }
}

// ---------------------------------------------------------------- epilogues
// conv1 tile t, TMEM slot columns col: lane (quadrant qd, l) = GEMM row r = 128t + 32qd + l = pooled pixel
// (r / 26, r % 26); bias, ReLU, bf16 into conv2's parity planes (border entries stay zero).
__device__ __forceinline__ void conv1_epilogue(uint32_t tmem, uint32_t col, int t, uint8_t* A2, const float* b1) {
  const int qd = (threadIdx.x >> 5) & 3, l = threadIdx.x & 31;
  float v[16];
  pool_bias_relu16(tmem + ((uint32_t)(32 * qd) << 16), (int)col, 16, b1, v);
  const int r = 128 * t + 32 * qd + l;
  const int py = r / A1_ROW, px = r - py * A1_ROW;
  if (py < P1 && px < P1) {
    uint32_t w[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) w[i] = pack_bf16(v[2 * i], v[2 * i + 1]);
    const int Y = py + 1, X = px + 1;
    uint8_t* p = A2 + ((((Y & 1) * 2 + (X & 1)) * 2) * A2_PLANE + ((Y >> 1) * A2_COLS + (X >> 1)) * 16);
    *reinterpret_cast<uint4*>(p) = make_uint4(w[0], w[1], w[2], w[3]);
    *reinterpret_cast<uint4*>(p + A2_PLANE) = make_uint4(w[4], w[5], w[6], w[7]);
  }
}

// conv2 tile u: lane (qd, l) = GEMM row r = 128u + 32qd + l = pooled pixel (r / 14, r % 14); returns the FC partial
// sum over its 32 channels (0 for rows outside the 12 x 12 floor-pooled output).
__device__ __forceinline__ float conv2_epilogue(uint32_t tmem, int u, const float* b2, const float* wfc) {
  const int qd = (threadIdx.x >> 5) & 3, l = threadIdx.x & 31;
  const int r = 128 * u + 32 * qd + l;
  const int py = r / A2_COLS, px = r - py * A2_COLS;
  const bool own = py < P2 && px < P2;
  const float4* wq = reinterpret_cast<const float4*>(wfc) + py * P2 + min(px, P2 - 1);  // in smem for every lane
  float acc = 0.f;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    float v[16];
    pool_bias_relu16(tmem + ((uint32_t)(32 * qd) << 16), (int)kC2Col + 128 * u + 16 * h, 32, b2 + 16 * h, v);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const float4 w = wq[(4 * h + q) * (P2 * P2)];
      acc = fmaf(v[4 * q], w.x, acc);
      acc = fmaf(v[4 * q + 1], w.y, acc);
      acc = fmaf(v[4 * q + 2], w.z, acc);
      acc = fmaf(v[4 * q + 3], w.w, acc);
    }
  }
  return own ? acc : 0.f;
}

__global__ void __launch_bounds__(kThreads, 1) snm_kernel(SnmArgs a) {
  extern __shared__ __align__(1024) uint8_t sm[];
#if FFSVA_K4_PROF
  const long long t_start = clock64();
  if (threadIdx.x < 16) s_prof[threadIdx.x] = 0;
#endif
  const int m = a.counts[0];
  const int j0 = (int)((int64_t)blockIdx.x * m / gridDim.x), j1 = (int)((int64_t)(blockIdx.x + 1) * m / gridDim.x);
  const int S = j1 - j0;  // frames of this CTA (every role walks the same sequence)
  if (S <= 0) return;
  const int tid = threadIdx.x, lane = tid & 31;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);  // warp-uniform (uniform registers)
  uint8_t* WB = sm + OFF_WB;
  int2* info = reinterpret_cast<int2*>(sm + OFF_INFO);
  float* red = reinterpret_cast<float*>(sm + OFF_RED);
  uint32_t* s_tmem = reinterpret_cast<uint32_t*>(sm + OFF_TMEM);
  const uint32_t bars = smem_addr(sm + OFF_BAR);
  auto bar = [&](int i) { return bars + 8u * (uint32_t)i; };

  // zero both operand buffers of each GEMM (padding borders, the unused 4th channel slot, the junk-row tails)
  for (int i = tid; i < (NA1 * A1_BYTES + NA2 * A2_BYTES) / 16; i += kThreads)
    reinterpret_cast<uint4*>(sm + OFF_A1)[i] = make_uint4(0, 0, 0, 0);
  if (tid == 0) {
    for (int i = 0; i < NIN; ++i) {
      mbar_init(bar(B_IN_FULL + i), 1);
      mbar_init(bar(B_IN_EMPTY + i), kConvWarps);
    }
    mbar_init(bar(B_W_FULL), 1);
    mbar_init(bar(B_W_EMPTY), 1);
    for (int i = 0; i < NI; ++i) mbar_init(bar(B_INFO_EMPTY + i), 1);
    for (int i = 0; i < NA1; ++i) {
      mbar_init(bar(B_A1_FULL + i), kConvWarps);
      mbar_init(bar(B_A1_EMPTY + i), 1);
    }
    for (int i = 0; i < NA2; ++i) {
      mbar_init(bar(B_A2_FULL + i), 4);
      mbar_init(bar(B_A2_EMPTY + i), 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(bar(B_C2_FULL + i), 2);
      mbar_init(bar(B_C2_EMPTY + i), 4);
    }
    for (int i = 0; i < 4; ++i) {
      mbar_init(bar(B_C1_FULL + i), 2);
      mbar_init(bar(B_C1_EMPTY + i), 4);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) tmem_alloc(smem_addr(s_tmem), kTmemCols);
  fence_proxy_async();  // the zeroed operand buffers are read by the tensor cores
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *s_tmem;

  if (warp == 0) {
    // ---------------- producer: per-frame info, D50 staging, the stream's weight image per segment
    if (lane == 0) {
      const uint32_t in0 = smem_addr(sm + OFF_IN);
      int k = 0, nch = 0;  // chunk containing frame j (pop_start counting, online mode)
      if (a.pop_start) {
        nch = a.counts[1];
        int lo = 0, hi = nch - 1;  // last k with chunks[k] <= j0
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (__ldg(a.chunks + mid) <= j0) lo = mid;
          else hi = mid - 1;
        }
        k = lo;
      }
      int f = __ldg(a.work + j0);
      const uint8_t* snm = a.frames[f].snm;
      const uint8_t* src = d50_of(a, f);
      const uint8_t* prev = nullptr;
      int g = -1;
      for (int s = 0; s < S; ++s) {
        const int j = j0 + s;
        int fn = -1;
        const uint8_t *snm_n = nullptr, *src_n = nullptr;
        if (s + 1 < S) {  // one frame of lookahead: the next frame's stream decides this frame's segment end
          fn = __ldg(a.work + j + 1);
          snm_n = a.frames[fn].snm;
          src_n = d50_of(a, fn);
        }
        const bool first = snm != prev, last = s + 1 == S || snm_n != snm;
        int flags = (first ? F_SEG_FIRST : 0) | (last ? F_SEG_LAST : 0);
        if (a.pop_start) {
          while (k + 1 < nch && __ldg(a.chunks + k + 1) <= j) ++k;
          if (__ldg(a.chunks + k) == j && a.pop_start[k]) flags |= F_POP_OPEN;
        }
        if (first) ++g;
        if (s >= NI) KW(0, mbar_wait_sleep(bar(B_INFO_EMPTY + s % NI), (uint32_t)((s / NI - 1) & 1)));
        info[s % NI] = make_int2(f, flags);
        if (s >= NIN) KW(1, mbar_wait_sleep(bar(B_IN_EMPTY + s % NIN), (uint32_t)((s / NIN - 1) & 1)));
        mbar_expect_tx(bar(B_IN_FULL + s % NIN), D50_BYTES);
        bulk_g2s(in0 + (uint32_t)((s % NIN) * D50_BYTES), src, D50_BYTES, bar(B_IN_FULL + s % NIN));
        if (first) {  // dynamic batch: one weight load per run of one stream's frames (L219)
          if (g >= 1) KW(2, mbar_wait_sleep(bar(B_W_EMPTY), (uint32_t)((g - 1) & 1)));
          mbar_expect_tx(bar(B_W_FULL), BLOB_BYTES);
          constexpr int kPiece = 16384;
          for (int o = 0; o < BLOB_BYTES; o += kPiece)
            bulk_g2s(smem_addr(WB) + (uint32_t)o, snm + o, (uint32_t)min(kPiece, BLOB_BYTES - o), bar(B_W_FULL));
        }
        prev = snm;
        f = fn;
        snm = snm_n;
        src = src_n;
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issue: conv2 lags conv1 by two frames (frame s's conv1 tiles interleaved with frame s-2's
    // conv2 tiles), so that every MMA's inputs were produced at least one conv2 tile earlier
    const uint32_t a1b = smem_addr(sm + OFF_A1), a2b = smem_addr(sm + OFF_A2);
    const uint32_t w1 = smem_addr(WB + OFF_W1), w2 = smem_addr(WB + OFF_W2);
    int g = -1;
    auto c1 = [&](int s, int t) {
      const int T = kTiles1 * s + t, slot = T & 3;
      if (T >= 4) KW(3, mbar_wait(bar(B_C1_EMPTY + slot), (uint32_t)(((T >> 2) - 1) & 1)));
      fence_after();
      if (!(FFSVA_K4_ABL & 8))
        issue_conv1_tile(tmem + (uint32_t)(64 * slot), a1b + (uint32_t)((s % NA1) * A1_BYTES), t, w1);
      mma_commit(bar(B_C1_FULL + slot));
      mbar_arrive_elect(bar(B_C1_FULL + slot));  // release: the epilogue warps may read this frame's info
    };
    auto c2 = [&](int s, int u) {
      if (u == 0) {
        KW(4, mbar_wait(bar(B_A2_FULL + s % NA2), (uint32_t)((s / NA2) & 1)));
        fence_after();
      }
      if (s >= 1) KW(5, mbar_wait(bar(B_C2_EMPTY + u), (uint32_t)((s - 1) & 1)));
      fence_after();
      if (!(FFSVA_K4_ABL & 8))
        issue_conv2_tile(tmem + kC2Col + (uint32_t)(128 * u), a2b + (uint32_t)((s % NA2) * A2_BYTES), u, w2);
      mma_commit(bar(B_C2_FULL + u));
      mbar_arrive_elect(bar(B_C2_FULL + u));
      if (u == 1) mma_commit(bar(B_A2_EMPTY + s % NA2));
    };
    int nc2 = 0;  // next frame whose conv2 is not issued yet
    for (int s = 0;; ++s) {
      const bool have = s < S;
      bool first = false;
      if (have) {
        KW(6, mbar_wait(bar(B_A1_FULL + s % NA1), (uint32_t)((s / NA1) & 1)));
        first = (info[s % NI].y & F_SEG_FIRST) != 0;
      }
      // a new stream's weight image replaces the old one only after every earlier frame's conv2 has been issued
      // (and drained by the conv2 epilogue, which releases the image): drain the lag at a stream change and at the end
      if (!have || (first && s > 0)) {
        for (; nc2 < s; ++nc2) {
          c2(nc2, 0);
          c2(nc2, 1);
        }
        if (!have) break;
      }
      if (first) {
        ++g;
        KW(7, mbar_wait(bar(B_W_FULL), (uint32_t)(g & 1)));
      }
      const bool lag = nc2 <= s - 2;
      c1(s, 0);
      c1(s, 1);
      c1(s, 2);
      c1(s, 3);
      if (lag) c2(nc2, 0);
      c1(s, 4);
      c1(s, 5);
      mma_commit(bar(B_A1_EMPTY + s % NA1));
      if (lag) c2(nc2++, 1);
    }
  } else if (warp >= 2 && warp < 2 + kConvWarps) {
    // ---------------- D50 -> conv1 operand
    const int t = tid - 64;
    for (int s = 0; s < S; ++s) {
      KW(8, mbar_wait(bar(B_IN_FULL + s % NIN), (uint32_t)((s / NIN) & 1)));
      if (s >= NA1) KW(9, mbar_wait(bar(B_A1_EMPTY + s % NA1), (uint32_t)((s / NA1 - 1) & 1)));
      if (!(FFSVA_K4_ABL & 1)) convert_input(sm + OFF_IN + (s % NIN) * D50_BYTES, sm + OFF_A1 + (s % NA1) * A1_BYTES, t);
      fence_proxy_async();
      __syncwarp();
      mbar_arrive_elect(bar(B_A1_FULL + s % NA1));
      mbar_arrive_elect(bar(B_IN_EMPTY + s % NIN));
    }
  } else if (warp >= 8 && warp < 12) {
    // ---------------- conv1 epilogue -> conv2 operand
    for (int s = 0; s < S; ++s) {
      uint8_t* A2 = sm + OFF_A2 + (s % NA2) * A2_BYTES;
      if (s >= NA2) KW(10, mbar_wait(bar(B_A2_EMPTY + s % NA2), (uint32_t)((s / NA2 - 1) & 1)));
      float b1[16];
      for (int t = 0; t < kTiles1; ++t) {
        const int T = kTiles1 * s + t, slot = T & 3;
        KW(11, mbar_wait(bar(B_C1_FULL + slot), (uint32_t)((T >> 2) & 1)));
        fence_after();
        if (t == 0) {
#pragma unroll
          for (int i = 0; i < 16; ++i) b1[i] = reinterpret_cast<const float*>(WB + OFF_B1)[i];
        }
        if (!(FFSVA_K4_ABL & 2)) conv1_epilogue(tmem, (uint32_t)(64 * slot), t, A2, b1);
        fence_before();
        __syncwarp();
        mbar_arrive_elect(bar(B_C1_EMPTY + slot));
      }
      fence_proxy_async();  // conv2's operand was written through the generic proxy
      __syncwarp();
      mbar_arrive_elect(bar(B_A2_FULL + s % NA2));
    }
  } else if (warp >= 12) {
    // ---------------- conv2 epilogue, FC, decision
    const float* b2 = reinterpret_cast<const float*>(WB + OFF_B2);
    const float* wfc = reinterpret_cast<const float*>(WB + OFF_WFC);
    const int qd = warp & 3;
    uint32_t cnt_pass = 0, cnt_c0 = 0, cnt_c1 = 0, cnt_c2 = 0, cnt_pop = 0;
    for (int s = 0; s < S; ++s) {
      float acc = 0.f;
      for (int u = 0; u < 2; ++u) {
        KW(12, mbar_wait(bar(B_C2_FULL + u), (uint32_t)(s & 1)));
        fence_after();
        if (!(FFSVA_K4_ABL & 4)) acc += conv2_epilogue(tmem, u, b2, wfc);
        fence_before();
        __syncwarp();
        mbar_arrive_elect(bar(B_C2_EMPTY + u));
      }
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
      if (elect_one()) red[(s & 1) * 4 + qd] = acc;
      KW(13, asm volatile("bar.sync 1, 128;" ::: "memory"));
      if (warp == 12 && elect_one()) {
        const int2 in = info[s % NI];
        const int f = in.x;
        const float* r = red + (s & 1) * 4;
        const float logit = *reinterpret_cast<const float*>(WB + OFF_BFC) + ((r[0] + r[1]) + (r[2] + r[3]));
        const FrameDesc& fd = a.frames[f];
        const uint8_t p = logit >= fd.L_t ? 1 : 0;
        const uint8_t cls = logit < fd.L_low ? 0 : (logit > fd.L_high ? 2 : 1);
        a.logit[f] = logit;
        a.snm_pass[f] = p;
        a.snm_class[f] = cls;
        cnt_pass += p;
        cnt_c0 += cls == 0;
        cnt_c1 += cls == 1;
        cnt_c2 += cls == 2;
        cnt_pop += (in.y & F_POP_OPEN) ? 1 : 0;
        if (in.y & F_SEG_LAST) {
          if (a.stats) {
            unsigned long long* st = a.stats + (int64_t)fd.slot * NSTAT;
            atomicAdd(st + 2, (unsigned long long)cnt_pass);
            atomicAdd(st + 4, (unsigned long long)cnt_c0);
            atomicAdd(st + 5, (unsigned long long)cnt_c1);
            atomicAdd(st + 6, (unsigned long long)cnt_c2);
            if (cnt_pop) atomicAdd(st + 7, (unsigned long long)cnt_pop);
          }
          cnt_pass = cnt_c0 = cnt_c1 = cnt_c2 = cnt_pop = 0;
          mbar_arrive(bar(B_W_EMPTY));  // this stream's weights are no longer read
        }
        mbar_arrive(bar(B_INFO_EMPTY + s % NI));
      }
    }
  }

  fence_before();
  __syncthreads();
#if FFSVA_K4_PROF
  if (blockIdx.x == 0 && tid == 0) {
    printf("K4PROF S=%d total=%lld", S, clock64() - t_start);
    for (int i = 0; i < 14; ++i) printf(" w%d=%llu", i, s_prof[i]);
    printf("\n");
  }
#endif
  if (warp == 1) {
    fence_after();
    tmem_dealloc(tmem, kTmemCols);
  }
}

}  // namespace

int snm_smem_bytes() { return SMEM_BYTES; }

cudaError_t snm_configure() {
  // the attribute is per device: called by every device context's creation (on that device), never cached
  return cudaFuncSetAttribute(snm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
}

cudaError_t launch_snm(const SnmArgs& a, cudaStream_t st) {
  snm_kernel<<<a.grid, kThreads, SMEM_BYTES, st>>>(a);
  return cudaGetLastError();
}

}  // namespace ffsva
