// ffsva_snm.cu — K4: the stream-specialised network model (SNM) on tcgen05 tensor cores.
//
// Method: "SNM is a three-layer CNN (CONV, CONV, and FC)" that outputs the probability c of the
// target (L159) on 50x50 images (L167); frames with c >= t_pre go on (L165), t_pre from Eq. (2) (L193); SNM
// scores frames in dynamic batches so a stream's model is loaded once per batch (L219-L223).
// Readings: conv1 3->16 and conv2 16->32, 3x3, zero pad 1, ReLU, 2x2 max-pool (floor), FC
// 4608->1 logit (Q9, Q11); input (v-128)/128 (Q10); bf16 operands, fp32 accumulation, pooled conv1 rounded
// to bf16, conv2 output and FC in fp32 (Q15).
//
// B200 mapping — implicit GEMM, no im2col, pooling folded into the N dimension:
//   * GEMM rows are POOLED output pixels; a 2x2-pool's four conv outputs are four accumulator column groups of the
//     same TMEM lane, so the max-pool is an in-register max over four column groups (no cross-lane shuffles); bias
//     and ReLU commute with max and are applied once after it.
//   * conv1: the A row of pooled pixel (py, px) is its 4x4 input patch (padded rows 2py..2py+3, columns
//     2px..2px+3) x 4 channel slots (3 used); the four pool positions differ only in where their 3x3 kernel sits in
//     the patch, so ONE A operand feeds N = 64 = 4 positions x 16 channels with per-position (zero-padded) weights:
//     4 MMAs (M128 N64 K16, one per patch row) per tile of 4 pooled rows x 32 px instead of 24 narrow ones. The
//     input lives in two row-parity planes of 64-px rows, 8 bytes per pixel, so a patch row of consecutive pooled
//     pixels is a constant-stride view (rows 16 B apart, K-halves 16 B apart, 8-row groups 128 B apart): each
//     patch row is the same UMMA descriptor moved by one plane row.
//   * conv2 (16 channels = two 8-channel planes, LBO = plane distance): per pool position and tap one MMA
//     (M128, N32) per tile x 2 tiles of 8 pooled rows x 16 px, A from four parity planes like conv1's patch rows.
//   * conv1's epilogue writes bf16 pooled activations straight into conv2's parity planes; conv2's epilogue
//     multiplies the pooled features by the FC weights (bf16 values) in fp32 and reduces to one logit per frame.
// Two persistent CTAs per SM (8 warps and 256 TMEM columns each: conv1 runs as two waves of <= 4 tiles, conv2's two
// tiles reuse the columns), so one CTA's epilogues overlap the other's MMAs. MMAs are issued by a whole warp (one
// elected lane) per warp group and committed per tile to its own mbarrier so epilogues start as soon as a tile lands.
// Work = dynamic-batch units (<= BatchSize survivors of one stream, split further when the batch is small); the
// stream's 26 KB weight image is copied into shared memory once per unit (skipped when the previous unit was the
// same stream), and the next frame's D50 image is prefetched with a bulk copy.
#include <cuda_bf16.h>

#include "ffsva_internal.h"
#include "ffsva_ptx.h"

namespace ffsva {
namespace {

using namespace snm;

constexpr int kThreads = 256;
// conv1 operand: 2 row-parity planes x 27 rows x 64 px x 8 B (padded input 52x52, 4 channel slots, 3 used)
constexpr int A1_COLS = 64, A1_ROWS = 27;
constexpr int A1_ROWB = A1_COLS * 8;                        // 512: pooled row -> next plane row = four 8-row groups
constexpr int A1_PLANE = A1_ROWS * A1_ROWB;                 // 13824
constexpr int A1_BYTES = 2 * A1_PLANE + 512;                // + tail read by junk columns of the last plane row
// conv2 operand: 8 planes [ypar][xpar][chalf] x 14 rows x 16 px x 16 B (padded pooled conv1 27x27, 16 ch)
constexpr int A2_COLS = 16, A2_ROWS = 14;
constexpr int A2_PLANE = A2_ROWS * A2_COLS * 16;            // 3584
constexpr int A2_BYTES = 8 * A2_PLANE + 512;                // + zero tail read by junk rows of the last tile
constexpr int D50_BYTES = 7504;                             // staged D50 image (one frame)
constexpr int OFF_A1 = 0;
constexpr int OFF_A2 = OFF_A1 + A1_BYTES;                   // 28160
constexpr int OFF_WB = OFF_A2 + A2_BYTES;                   // 57344
constexpr int OFF_IN = OFF_WB + BLOB_BYTES;                 // 2 staging buffers
constexpr int OFF_LUT = OFF_IN + 2 * D50_BYTES;             // u16[256]: bf16 bits of (v - 128) / 128
constexpr int OFF_RED = OFF_LUT + 512;
constexpr int OFF_BAR = OFF_RED + 64;                       // 7 conv1 + 2 conv2 + 2 input mbarriers
constexpr int OFF_TMEM = OFF_BAR + 16 * 8;
constexpr int SMEM_BYTES = OFF_TMEM + 16;
static_assert(SMEM_BYTES <= 113 * 1024, "two CTAs per SM");
static_assert(OFF_A2 % 16 == 0 && OFF_WB % 16 == 0 && OFF_IN % 16 == 0, "16-byte alignment");
constexpr uint32_t kTmemCols = 256;

constexpr int kTiles1 = 7;
__constant__ int8_t c1_py0[kTiles1] = {0, 4, 8, 12, 16, 20, 21};  // last tile overlaps (idempotent writes)

// PTX wrappers (tcgen05 MMA / TMEM, mbarriers, bulk copies): ffsva_ptx.h
using namespace ptx;

// max over the four pool positions: 16 consecutive channels starting at column col of each position group
__device__ __forceinline__ void pooled16(uint32_t taddr, int col, int group_cols, float (&v)[16]) {
  uint32_t r0[16], r1[16], r2[16], r3[16];
  tmem_ld16(taddr + (uint32_t)col, r0);
  tmem_ld16(taddr + (uint32_t)(col + group_cols), r1);
  tmem_ld16(taddr + (uint32_t)(col + 2 * group_cols), r2);
  tmem_ld16(taddr + (uint32_t)(col + 3 * group_cols), r3);
  tmem_wait_ld2(r0, r1);
  tmem_wait_ld2(r2, r3);
#pragma unroll
  for (int i = 0; i < 16; ++i)
    v[i] = fmaxf(fmaxf(__uint_as_float(r0[i]), __uint_as_float(r1[i])),
                 fmaxf(__uint_as_float(r2[i]), __uint_as_float(r3[i])));
}

__device__ __forceinline__ uint32_t u8_to_bf16(uint32_t v) {  // (v - 128) / 128 is exact in bf16
  return (uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(((float)v - 128.0f) * 0.0078125f));
}

__device__ __forceinline__ const uint8_t* d50_of(const SnmArgs& a, int f) {
  return a.d50 + (a.d50_index ? (int64_t)__ldg(a.d50_index + f) : (int64_t)f) * a.d50_stride;
}

// ---------------------------------------------------------------- input staging
// D50 (50x50x3 u8, row-major) -> (v-128)/128 bf16 (C5, exact) into conv1's row-parity planes, one 8-byte pixel
// (3 channels + a zero slot) per store. Groups of 4 pixels = 12 bytes = three aligned 32-bit shared loads; each
// channel through a 256-entry bf16 table.
__device__ __forceinline__ void convert_input(const uint8_t* d, uint8_t* A1, const uint16_t* lut) {
  constexpr int kGroups = snm::IN * snm::IN / 4;  // 625
  for (int g = threadIdx.x; g < kGroups; g += kThreads) {
    const uint32_t* w = reinterpret_cast<const uint32_t*>(d + 12 * g);
    const uint32_t w0 = w[0], w1 = w[1], w2 = w[2];
    const uint32_t b[12] = {w0 & 255u, (w0 >> 8) & 255u, (w0 >> 16) & 255u, w0 >> 24,
                            w1 & 255u, (w1 >> 8) & 255u, (w1 >> 16) & 255u, w1 >> 24,
                            w2 & 255u, (w2 >> 8) & 255u, (w2 >> 16) & 255u, w2 >> 24};
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int p = 4 * g + q;
      const int y = p / snm::IN, x = p - y * snm::IN;
      const int Y = y + 1, X = x + 1;
      const uint2 v = make_uint2((uint32_t)lut[b[3 * q]] | ((uint32_t)lut[b[3 * q + 1]] << 16), (uint32_t)lut[b[3 * q + 2]]);
      *reinterpret_cast<uint2*>(A1 + (Y & 1) * A1_PLANE + (Y >> 1) * A1_ROWB + X * 8) = v;
    }
  }
}

// ---------------------------------------------------------------- MMA issue (one thread per warp group)
// conv1 tile t (pooled rows py0..py0+3 x 32 px) into TMEM columns col..col+63 ([pool position][16 channels]):
// patch row dy of pooled row py is padded input row 2py + dy = plane (dy & 1), plane row py + (dy >> 1).
__device__ __forceinline__ void issue_conv1_tile(uint32_t tmem, uint32_t col, int t, uint32_t a1, uint32_t w1) {
  const int py0 = c1_py0[t];
  const uint32_t idesc = idesc_bf16(128, 64);
#pragma unroll
  for (int dy = 0; dy < 4; ++dy) {
    const uint32_t arow = a1 + (uint32_t)((dy & 1) * A1_PLANE + (py0 + (dy >> 1)) * A1_ROWB);
    // K-halves = patch columns (0,1) and (2,1+2): 16 B apart; 8-row groups (8 pooled px) 128 B apart
    mma_bf16(tmem + col, umma_desc(arow, 16, 128), umma_desc(w1 + (uint32_t)(dy * 2 * 64 * 16), 64 * 16, 128), idesc,
             dy > 0 ? 1u : 0u);
  }
}

__device__ __forceinline__ void issue_conv2_tile(uint32_t tmem, int u, uint32_t a2, uint32_t w2) {
  const int py0 = 4 * u;
  const uint32_t idesc = idesc_bf16(128, 32);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const int a = q >> 1, b = q & 1;
    const uint32_t d = tmem + (uint32_t)(u * 128 + q * 32);
#pragma unroll
    for (int tap = 0; tap < 9; ++tap) {
      const int dy = tap / 3, dx = tap % 3;
      const int ypar = (a + dy) & 1, roff = (a + dy) >> 1, xpar = (b + dx) & 1, coff = (b + dx) >> 1;
      const uint32_t addr = a2 + (uint32_t)(((ypar * 2 + xpar) * 2) * A2_PLANE + ((py0 + roff) * A2_COLS + coff) * 16);
      mma_bf16(d, umma_desc(addr, A2_PLANE, 128), umma_desc(w2 + (uint32_t)(tap * 2 * C2 * 16), C2 * 16, 128), idesc,
               tap > 0 ? 1u : 0u);
    }
  }
}

// ---------------------------------------------------------------- epilogues
// conv1 tile t: lane (quadrant qd, l) = pooled pixel (py0 + qd, l); bias, ReLU, bf16 into conv2's planes.
__device__ __forceinline__ void conv1_epilogue(uint32_t tmem, uint32_t col, int t, uint8_t* A2, const float* b1,
                                               uint16_t* dbg) {
  const int qd = (threadIdx.x >> 5) & 3, l = threadIdx.x & 31;
  float v[16];
  pooled16(tmem + ((uint32_t)(32 * qd) << 16), (int)col, 16, v);
  const int py = c1_py0[t] + qd, px = l;
  if (px < P1) {
    uint32_t w[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) w[i] = pack_bf16(fmaxf(v[2 * i] + b1[2 * i], 0.f), fmaxf(v[2 * i + 1] + b1[2 * i + 1], 0.f));
    const int Y = py + 1, X = px + 1;
    uint8_t* p = A2 + ((((Y & 1) * 2 + (X & 1)) * 2) * A2_PLANE + ((Y >> 1) * A2_COLS + (X >> 1)) * 16);
    *reinterpret_cast<uint4*>(p) = make_uint4(w[0], w[1], w[2], w[3]);
    *reinterpret_cast<uint4*>(p + A2_PLANE) = make_uint4(w[4], w[5], w[6], w[7]);
    if (dbg) {
      uint4* d = reinterpret_cast<uint4*>(dbg + (py * P1 + px) * 16);
      d[0] = make_uint4(w[0], w[1], w[2], w[3]);
      d[1] = make_uint4(w[4], w[5], w[6], w[7]);
    }
  }
}

// conv2 tile u: lane (qd, l) = pooled pixel (4u + 2qd + (l >> 4), l & 15); returns the FC partial sum.
__device__ __forceinline__ float conv2_epilogue(uint32_t tmem, int u, const float* b2, const uint16_t* wfc, float* dbg) {
  const int qd = (threadIdx.x >> 5) & 3, l = threadIdx.x & 31;
  const int py = 4 * u + 2 * qd + (l >> 4), px = l & 15;
  const bool own = px < P2 && (u == 0 ? py < 8 : py >= 8);
  float acc = 0.f;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    float v[16];
    pooled16(tmem + ((uint32_t)(32 * qd) << 16), u * 128 + 16 * h, 32, v);
    if (own) {
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        const int c = 16 * h + i;
        const float r = fmaxf(v[i] + b2[c], 0.f);
        acc = fmaf(r, __uint_as_float((uint32_t)wfc[c * (P2 * P2) + py * P2 + px] << 16), acc);
        if (dbg) dbg[c * (P2 * P2) + py * P2 + px] = r;
      }
    }
  }
  return acc;
}

__global__ void __launch_bounds__(kThreads, kSnmCtasPerSm) snm_kernel(SnmArgs a) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* A1 = sm + OFF_A1;
  uint8_t* A2 = sm + OFF_A2;
  uint8_t* WB = sm + OFF_WB;
  uint8_t* stage = sm + OFF_IN;
  float* red = reinterpret_cast<float*>(sm + OFF_RED);
  uint32_t* s_tmem = reinterpret_cast<uint32_t*>(sm + OFF_TMEM);
  __shared__ int s_chunk;
  const int tid = threadIdx.x, lane = tid & 31;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0), grp = warp >> 2;  // warp-uniform (uniform registers)
  const uint32_t bar0 = smem_addr(sm + OFF_BAR);  // bar0 + 8*i: i < 7 conv1 tiles, 7..8 conv2 tiles, 9..10 input
  const int n_chunks = a.counts[1];
  if (n_chunks == 0) return;  // no survivors in this batch

  for (int i = tid; i < (A1_BYTES + A2_BYTES) / 16; i += kThreads) reinterpret_cast<uint4*>(sm)[i] = make_uint4(0, 0, 0, 0);
  uint16_t* lut = reinterpret_cast<uint16_t*>(sm + OFF_LUT);
  lut[tid] = (uint16_t)u8_to_bf16((uint32_t)tid);  // kThreads == 256 entries
  if (tid == 0) {
    for (int i = 0; i < 11; ++i) mbar_init(bar0 + 8 * i, 1);
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
  const uint32_t a1 = smem_addr(A1), a2 = smem_addr(A2);
  const uint32_t w1 = smem_addr(WB + OFF_W1), w2 = smem_addr(WB + OFF_W2);
  const float* b1 = reinterpret_cast<const float*>(WB + OFF_B1);
  const float* b2 = reinterpret_cast<const float*>(WB + OFF_B2);
  const uint16_t* wfc = reinterpret_cast<const uint16_t*>(WB + OFF_WFC);
  uint32_t ph = 0;           // parity of the per-frame mbarriers (one phase per frame)
  uint32_t in_ph = 0;        // bit i: parity of input staging buffer i
  const uint8_t* loaded = nullptr;  // weight image currently in shared memory

  for (;;) {
    if (tid == 0) s_chunk = atomicAdd(a.counts + 2, 1);
    __syncthreads();
    const int k = s_chunk;
    if (k >= n_chunks) break;
    const int start = a.chunks[k], end = a.chunks[k + 1];
    const FrameDesc fd0 = a.frames[a.work[start]];
    if (fd0.snm != loaded) {  // dynamic batch: one weight load per batch of this stream (L219)
      const uint4* src = reinterpret_cast<const uint4*>(fd0.snm);
      uint4* dst = reinterpret_cast<uint4*>(WB);
      for (int i = tid; i < BLOB_BYTES / 16; i += kThreads) dst[i] = __ldg(src + i);
      loaded = fd0.snm;
    }
    const float fc_bias = __ldg(reinterpret_cast<const float*>(fd0.snm + OFF_BFC));
    uint32_t cnt_pass = 0, cnt_c0 = 0, cnt_c1 = 0, cnt_c2 = 0;
    if (tid == 0) {  // stage the unit's first two D50 images
      mbar_expect_tx(bar0 + 8 * 9, D50_BYTES);
      bulk_g2s(smem_addr(stage), d50_of(a, a.work[start]), D50_BYTES, bar0 + 8 * 9);
      if (start + 1 < end) {
        mbar_expect_tx(bar0 + 8 * 10, D50_BYTES);
        bulk_g2s(smem_addr(stage + D50_BYTES), d50_of(a, a.work[start + 1]), D50_BYTES, bar0 + 8 * 10);
      }
    }
    mbar_wait(bar0 + 8 * 9, in_ph & 1u);
    in_ph ^= 1u;
    convert_input(stage, A1, lut);
    fence_proxy_async();
    const bool issuer = (warp & 3) == 0;  // warp 0 issues group 0's tiles, warp 4 group 1's (one elected lane)
    for (int j = start; j < end; ++j) {
      const int f = a.work[j];
      const int buf = (j - start) & 1;
      fence_before();
      __syncthreads();  // frame j's conv1 operand (and the unit's weights) are in shared memory

      // ---- conv1: 7 tiles in two waves of TMEM columns (tile t -> columns (t % 4) * 64); each warp group issues
      // and drains its own tiles (0, 2 | 4, 6 and 1, 3 | 5), one commit per tile. Wave B reuses wave A's columns of
      // the same group once the whole group has read them (named barrier 1 + grp over its 128 threads).
      uint16_t* dbg1 = a.dbg_p1 ? a.dbg_p1 + (int64_t)j * (P1 * P1 * 16) : nullptr;
#pragma unroll
      for (int wave = 0; wave < 2; ++wave) {
        if (issuer) {
          fence_after();
          for (int t = grp + 4 * wave; t < min(kTiles1, 4 * wave + 4); t += 2) {
            issue_conv1_tile(tmem, (uint32_t)((t & 3) * 64), t, a1, w1);
            mma_commit(bar0 + 8 * t);
          }
        }
        __syncwarp();
        for (int t = grp + 4 * wave; t < min(kTiles1, 4 * wave + 4); t += 2) {
          mbar_wait(bar0 + 8 * t, ph);
          fence_after();
          conv1_epilogue(tmem, (uint32_t)((t & 3) * 64), t, A2, b1, dbg1);
        }
        if (wave == 0) {  // the group's wave-A columns are drained before its wave-B MMAs overwrite them
          fence_before();
          if (grp == 0) asm volatile("bar.sync 1, 128;" ::: "memory");
          else asm volatile("bar.sync 2, 128;" ::: "memory");
        }
      }
      fence_proxy_async();  // conv1's epilogue wrote conv2's operand through the generic proxy
      fence_before();
      __syncthreads();  // every conv1 tile has landed: conv1's operand is free again

      // ---- conv2: one tile per warp group; while its MMAs run, stage frame j+1's conv1 operand
      if (issuer) {
        fence_after();
        issue_conv2_tile(tmem, grp, a2, w2);
        mma_commit(bar0 + 8 * (7 + grp));
      }
      __syncwarp();
      if (j + 1 < end) {
        const int nb = buf ^ 1;
        mbar_wait(bar0 + 8 * (9 + nb), (in_ph >> nb) & 1u);
        in_ph ^= 1u << nb;
        convert_input(stage + nb * D50_BYTES, A1, lut);
        fence_proxy_async();
      }
      if (tid == 0 && j + 2 < end) {  // frame j's staging buffer is consumed: prefetch frame j+2 into it
        mbar_expect_tx(bar0 + 8 * (9 + buf), D50_BYTES);
        bulk_g2s(smem_addr(stage + buf * D50_BYTES), d50_of(a, a.work[j + 2]), D50_BYTES, bar0 + 8 * (9 + buf));
      }
      mbar_wait(bar0 + 8 * (7 + grp), ph);
      fence_after();
      float* dbg2 = a.dbg_p2 ? a.dbg_p2 + (int64_t)j * NF : nullptr;
      float acc = conv2_epilogue(tmem, grp, b2, wfc, dbg2);
      ph ^= 1u;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
      if (lane == 0) red[warp] = acc;
      fence_before();
      __syncthreads();
      if (tid == 0) {
        float logit = fc_bias;
#pragma unroll
        for (int w = 0; w < kThreads / 32; ++w) logit += red[w];
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
      if (a.pop_start && a.pop_start[k]) atomicAdd(st + 7, 1ull);
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
  // the attribute is per device: called by every device context's creation (on that device), never cached
  return cudaFuncSetAttribute(snm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
}

cudaError_t launch_snm(const SnmArgs& a, cudaStream_t st) {
  snm_kernel<<<a.grid, kThreads, SMEM_BYTES, st>>>(a);
  return cudaGetLastError();
}

}  // namespace ffsva
