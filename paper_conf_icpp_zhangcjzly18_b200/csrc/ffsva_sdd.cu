// ffsva_sdd.cu — K1: frame ingest + integer box downsample (D100 and D50 in one pass) + SDD distance, for many
// frames of many streams in one launch. (The threshold of the summed distance happens in K3, after the kernel
// boundary has made every partial sum visible — no grid-scope fences here.)
//
// Method: raw frames are resized to each filter's feature size before the filter runs (L187;
// SDD 100x100 L155, SNM 50x50 L167); SDD computes the distance of the 100x100 image to the stream's
// reference image by MSE and keeps the frame iff MSE > delta_diff (L151). Readings: integer
// box filter with round-half-up (Q1, Q2), RGB kept (Q3), SSD in integers with an exact threshold (Q4, Q5),
// D50 from the raw frame = union of 2x2 D100 cells (Q8).
//
// Two variants, chosen per batch by the host:
//  * sdd_bulk_kernel (rows 16-B aligned, one 100-grid row fits in shared memory — every workload of the
//    benchmark): one CTA per (frame, 100-grid row), CTA pairs form thread-block clusters. One thread issues
//    cp.async.bulk copies (TMA engine, L2 evict-first) of the row's source rows into shared memory against an
//    mbarrier, so the SM's whole share of the frame is in flight without tying up registers (the row of R is
//    copied into shared memory by the other threads meanwhile, off the cell phase's critical path); column sums are
//    packed 2x16-bit SIMD adds of 16-byte shared loads; the odd CTA of a pair pushes its horizontal 2-cell sums
//    into the even CTA's shared memory with st.async (DSMEM, mbarrier transaction completion, no fence) and
//    the even CTA emits the D50 row from the four 100-cell sums.
//  * sdd_kernel (any alignment / very wide rows): one CTA per (frame, 50-grid row), rows streamed straight to
//    registers with 16-byte non-allocating loads (or byte loads for unaligned rows), 8 rows in flight.
// Both add their row's squared-difference sum to a per-frame u64 accumulator (relaxed atomic) and count the
// frame in the per-stream statistics.
#include <cooperative_groups.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "ffsva_internal.h"
#include "ffsva_ptx.h"

namespace cg = cooperative_groups;

namespace ffsva {
namespace {

__device__ __forceinline__ uint4 ld_stream16(const uint8_t* p) {
  uint4 r;
  asm("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p));
  return r;
}

// Bytes 0..15 of a 16-byte chunk -> 8 accumulators of two 16-bit lanes:
// a[2k] holds bytes (4k, 4k+2), a[2k+1] holds bytes (4k+1, 4k+3).
__device__ __forceinline__ void acc16(uint32_t (&a)[8], const uint4& v) {
  a[0] += v.x & 0x00FF00FFu; a[1] += (v.x >> 8) & 0x00FF00FFu;
  a[2] += v.y & 0x00FF00FFu; a[3] += (v.y >> 8) & 0x00FF00FFu;
  a[4] += v.z & 0x00FF00FFu; a[5] += (v.z >> 8) & 0x00FF00FFu;
  a[6] += v.w & 0x00FF00FFu; a[7] += (v.w >> 8) & 0x00FF00FFu;
}

__device__ __forceinline__ uint4 load_chunk(const uint8_t* row, int c, int rowbytes, bool vec16) {
  if (vec16) return ld_stream16(row + 16 * c);
  uint32_t w[4] = {0u, 0u, 0u, 0u};
#pragma unroll
  for (int j = 0; j < 16; ++j) {
    int b = 16 * c + j;
    uint32_t v = b < rowbytes ? (uint32_t)__ldg(row + b) : 0u;
    w[j >> 2] |= v << (8 * (j & 3));
  }
  return make_uint4(w[0], w[1], w[2], w[3]);
}

// Two rows of one 16-byte chunk at once: even bytes by AND, odd bytes by PRMT into 16-bit lanes, and one
// 3-input add per accumulator (3 integer ops per 4 bytes per row instead of 5).
__device__ __forceinline__ void acc16x2(uint32_t (&a)[8], const uint4& v, const uint4& w) {
  a[0] += (v.x & 0x00FF00FFu) + (w.x & 0x00FF00FFu);
  a[1] += __byte_perm(v.x, 0u, 0x4341) + __byte_perm(w.x, 0u, 0x4341);
  a[2] += (v.y & 0x00FF00FFu) + (w.y & 0x00FF00FFu);
  a[3] += __byte_perm(v.y, 0u, 0x4341) + __byte_perm(w.y, 0u, 0x4341);
  a[4] += (v.z & 0x00FF00FFu) + (w.z & 0x00FF00FFu);
  a[5] += __byte_perm(v.z, 0u, 0x4341) + __byte_perm(w.z, 0u, 0x4341);
  a[6] += (v.w & 0x00FF00FFu) + (w.w & 0x00FF00FFu);
  a[7] += __byte_perm(v.w, 0u, 0x4341) + __byte_perm(w.w, 0u, 0x4341);
}

// Sum of colsum[3x] for x in [x0, x1): the common cell widths (<= 24 pixels: frames up to 2400 px wide on a
// 100-cell grid) run a fully unrolled predicated loop.
__device__ __forceinline__ uint32_t cell_sum(const uint16_t* col, int x0, int x1) {
  uint32_t s = 0;
  if (x1 - x0 <= 24) {
#pragma unroll
    for (int k = 0; k < 24; ++k)
      if (x0 + k < x1) s += col[3 * (x0 + k)];
  } else {
    for (int x = x0; x < x1; ++x) s += col[3 * x];
  }
  return s;
}

// Sum of col[3x], x in [x0, x1) with x1 - x0 <= N: fully unrolled, predicated.
template <int N>
__device__ __forceinline__ uint32_t cell_sum_n(const uint16_t* col, int x0, int x1) {
  uint32_t s = 0;
  const uint16_t* p = col + 3 * x0;
  const int w = x1 - x0;
#pragma unroll
  for (int k = 0; k < N; ++k)
    if (k < w) s += p[3 * k];
  return s;
}

// floor(a / n) for a < 2^31 and a quotient below 2^16 (box means: <= 255), without the ~20-instruction integer
// division: the float estimate (relative error < 2^-21, so off by at most one) and one remainder correction.
__device__ __forceinline__ uint32_t udiv_small(uint32_t a, uint32_t n) {
  uint32_t q = __float2uint_rz(__uint2float_rn(a) * __frcp_rn(__uint2float_rn(n)));
  const int r = (int)(a - q * n);
  if (r < 0) --q;
  else if (r >= (int)n) ++q;
  return q;
}

// Round-half-up mean (s + n/2) / n of a box (C1).
__device__ __forceinline__ uint32_t box_mean(uint32_t s, uint32_t n) { return udiv_small(s + (n >> 1), n); }

// Cell sum of one channel with the unroll matched to the frame's widest cell (cellw).
__device__ __forceinline__ uint32_t cell_sum_w(const uint16_t* col, int x0, int x1, int cellw) {
  if (cellw <= 8) return cell_sum_n<8>(col, x0, x1);
  if (cellw <= 13) return cell_sum_n<13>(col, x0, x1);
  if (cellw <= 16) return cell_sum_n<16>(col, x0, x1);
  if (cellw <= 20) return cell_sum_n<20>(col, x0, x1);
  return cell_sum(col, x0, x1);
}

// Store the 16 column sums of chunk c (u16 each) for one 100-grid row.
__device__ __forceinline__ void store_colsum(uint32_t* colw, int c, const uint32_t (&a)[8]) {
  uint4 lo, hi;
  lo.x = __byte_perm(a[0], a[1], 0x5410); lo.y = __byte_perm(a[0], a[1], 0x7632);
  lo.z = __byte_perm(a[2], a[3], 0x5410); lo.w = __byte_perm(a[2], a[3], 0x7632);
  hi.x = __byte_perm(a[4], a[5], 0x5410); hi.y = __byte_perm(a[4], a[5], 0x7632);
  hi.z = __byte_perm(a[6], a[7], 0x5410); hi.w = __byte_perm(a[6], a[7], 0x7632);
  reinterpret_cast<uint4*>(colw)[2 * c] = lo;
  reinterpret_cast<uint4*>(colw)[2 * c + 1] = hi;
}

// x boundaries of the 100-grid cells of a W-pixel row: xb[i] = floor(i*W/sdd_w), i = 0..sdd_w.
__device__ __forceinline__ void fill_xbounds(int* xb, int W, int sdd_w) {
  for (int i = threadIdx.x; i <= sdd_w; i += blockDim.x) xb[i] = (int)(((uint32_t)i * (uint32_t)W) / (uint32_t)sdd_w);
}

// One value's share of the SDD distance: (D - R)^2 for MSE and NRMSE, |D - R| for SAD.
__device__ __forceinline__ uint32_t dist_term(int diff, uint8_t metric) {
  return metric == kDistSad ? (uint32_t)abs(diff) : (uint32_t)(diff * diff);
}

// Block-reduce this thread's SSD share; thread 0 adds it to the frame's accumulator and the stream's stats.
__device__ __forceinline__ void ssd_commit(uint32_t v, uint32_t* red, const SddArgs& a, int f, int slot,
                                           bool count_frame) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += red[w];
    atomicAdd(a.acc_ssd + f, t);
    if (a.stats) {
      unsigned long long* st = a.stats + (int64_t)slot * NSTAT;
      atomicAdd(st + 3, t);
      if (count_frame) atomicAdd(st + 0, 1ull);
    }
  }
}

// ------------------------------------------------------------------ register-streaming variant
template <bool kD100>
__global__ void __launch_bounds__(512) sdd_kernel(SddArgs a) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int nb = a.sdd_h >> 1;  // bands per frame
  const int f = blockIdx.x / nb;
  const int band = blockIdx.x - f * nb;
  const FrameDesc fd = a.frames[f];
  const int W = fd.W, H = fd.H, sdd_w = a.sdd_w, sdd_h = a.sdd_h;
  const int rowbytes = 3 * W;
  const int nchunk = (rowbytes + 15) >> 4;
  const int cs = nchunk * 16;  // u16 column sums per 100-grid row
  uint16_t* colsum = reinterpret_cast<uint16_t*>(smem);                  // [2][cs]
  uint32_t* cell = reinterpret_cast<uint32_t*>(smem + 4 * (size_t)cs);   // [2][3*sdd_w]
  int* xb = reinterpret_cast<int*>(cell + 6 * sdd_w);                    // [sdd_w + 1]
  __shared__ uint32_t red[16];

  // Source rows of the two 100-grid rows of this band: [ya0, ya1) and [ya1, yb1).
  const int ya0 = (int)(((uint32_t)(2 * band) * (uint32_t)H) / (uint32_t)sdd_h);
  const int ya1 = (int)(((uint32_t)(2 * band + 1) * (uint32_t)H) / (uint32_t)sdd_h);
  const int yb1 = (int)(((uint32_t)(2 * band + 2) * (uint32_t)H) / (uint32_t)sdd_h);
  const int rows = yb1 - ya0, split = ya1 - ya0;
  fill_xbounds(xb, W, sdd_w);

  // ---- phase 1: stream the band's rows, vertical column sums in registers
  for (int c = threadIdx.x; c < nchunk; c += blockDim.x) {
    uint32_t accA[8] = {0, 0, 0, 0, 0, 0, 0, 0}, accB[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    const uint8_t* base = fd.pixels + (int64_t)ya0 * fd.pitch;
    for (int r0 = 0; r0 < rows; r0 += 8) {
      uint4 v[8];
#pragma unroll
      for (int i = 0; i < 8; ++i)
        v[i] = (r0 + i < rows) ? load_chunk(base + (int64_t)(r0 + i) * fd.pitch, c, rowbytes, a.vec16)
                               : make_uint4(0u, 0u, 0u, 0u);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        if (r0 + i < split) acc16(accA, v[i]);
        else acc16(accB, v[i]);
      }
    }
    store_colsum(reinterpret_cast<uint32_t*>(colsum), c, accA);
    store_colsum(reinterpret_cast<uint32_t*>(colsum + cs), c, accB);
  }
  __syncthreads();

  // ---- phase 2: 100-grid cell sums, D100, SSD against R
  const int row3 = 3 * sdd_w;
  uint32_t ssd_local = 0;
  for (int o = threadIdx.x; o < 2 * row3; o += blockDim.x) {
    const int sub = o >= row3;
    const int r = o - sub * row3;
    const int cx = r / 3, ch = r - 3 * cx;
    const int x0 = xb[cx], x1 = xb[cx + 1];
    const uint16_t* col = colsum + sub * cs + ch;
    uint32_t s = 0;
    for (int x = x0; x < x1; ++x) s += col[3 * x];
    cell[o] = s;
    const uint32_t n = (uint32_t)(x1 - x0) * (uint32_t)(sub ? rows - split : split);
    const uint32_t d = box_mean(s, n);
    const int yrow = 2 * band + sub;
    if (kD100) a.d100[(int64_t)f * sdd_h * row3 + (int64_t)yrow * row3 + r] = (uint8_t)d;
    const int diff = (int)d - (int)__ldg(fd.ref + (int64_t)yrow * row3 + r);
    ssd_local += dist_term(diff, fd.metric);
  }
  if (fd.mode == kRefPrevious) ssd_local = 0;  // K2 measures against the previous frame's D100
  __syncthreads();

  // ---- phase 3: D50 row from the four 100-cell sums of each 50-cell
  const int half3 = 3 * (sdd_w >> 1);
  for (int o = threadIdx.x; o < half3; o += blockDim.x) {
    const int cx = o / 3, ch = o - 3 * cx;
    const uint32_t s = cell[6 * cx + ch] + cell[6 * cx + 3 + ch] + cell[row3 + 6 * cx + ch] +
                       cell[row3 + 6 * cx + 3 + ch];
    const uint32_t n = (uint32_t)(xb[2 * cx + 2] - xb[2 * cx]) * (uint32_t)rows;
    const int64_t slot = a.d50_index ? (int64_t)__ldg(a.d50_index + f) : (int64_t)f;
    a.d50[slot * a.d50_stride + (int64_t)band * half3 + o] = (uint8_t)box_mean(s, n);
  }
  ssd_commit(ssd_local, red, a, f, fd.slot, band == 0);
}

// ------------------------------------------------------------------ bulk-async (TMA engine) + cluster variant
// PTX wrappers: ffsva_ptx.h
using ptx::map_to_rank;
using ptx::mbar_expect_tx;
using ptx::st_async_u32;

constexpr int kBulkThreads = 256;  // block size for rows of > 128 16-byte chunks; 128 threads for narrower rows
                                   // (360p: twice the resident CTAs per SM for small per-CTA byte counts)
constexpr int kBulkMaxStage = 160 * 1024;  // larger rows (e.g. 4K) take the register-streaming kernel

#ifndef FFSVA_K1_MINBLOCKS
#define FFSVA_K1_MINBLOCKS 6  // 6 CTAs/SM: caps registers at 40 (A/B knob)
#endif
#ifndef FFSVA_K1_REFPRE
#define FFSVA_K1_REFPRE 1     // R row staged in shared memory during the bulk copy (A/B knob)
#endif
#ifndef FFSVA_K1_EARLYBAR
#define FFSVA_K1_EARLYBAR 1   // CTA barrier right after the mbarrier init, not after the x-bounds / R-row loads (A/B knob)
#endif
#ifndef FFSVA_K1_CELL16
#define FFSVA_K1_CELL16 1     // cell sums unrolled to 16 (cells <= 16 px) instead of 24 (A/B knob)
#endif
#ifndef FFSVA_K1_MINB128
#define FFSVA_K1_MINB128 16   // 128-thread CTAs (rows of <= 128 chunks, e.g. 360p): 16 CTAs/SM, 32 registers (A/B knob)
#endif
// kNT threads per CTA, each owning up to kCh 16-byte chunks of the row; kMinB resident CTAs per SM (register cap).
// Variants (k1_threads): 128/1/16 for rows of <= 128 chunks (360p); 256/1/7 for <= 256 chunks (720p: 32 registers
// and a 33 KB footprint, so seven CTAs fit an SM); 384/1/3 for 1080p rows (one chunk and one 100-grid value per
// thread); 256/2/6 for everything else up to 512 chunks.
template <bool kD100, int kNT, int kCh, int kMinB>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kNT, kMinB)
    sdd_bulk_kernel(SddArgs a) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t bar_data;   // this row's source bytes have landed
  __shared__ __align__(8) uint64_t bar_pair;   // (even CTA) the odd CTA's 2-cell sums have landed
  __shared__ uint32_t red[kNT / 32];
  const int sdd_w = a.sdd_w, sdd_h = a.sdd_h;
  const int f = blockIdx.y;              // frame (launches of > 65535 frames are split on the host)
  const int r = blockIdx.x;              // 100-grid row; the cluster pairs rows 2b and 2b+1
  const uint32_t rank = (uint32_t)r & 1u;
  const FrameDesc fd = a.frames[f];
  const int W = fd.W, H = fd.H;
  const int rb16 = (3 * W + 15) & ~15;
  const int nchunk = rb16 >> 4;
  // row boundaries: the host table (set only when every frame of the batch has height uni_H, so its loads do not
  // wait for the frame descriptor), else 32-bit division (H <= 65535, sdd_h <= 4096 are validated: r*H < 2^28)
  const bool ytab = a.ybounds != nullptr;
  const int y0 = ytab ? __ldg(a.ybounds + r) : (int)(((uint32_t)r * (uint32_t)H) / (uint32_t)sdd_h);
  const int y1 = ytab ? __ldg(a.ybounds + r + 1) : (int)(((uint32_t)(r + 1) * (uint32_t)H) / (uint32_t)sdd_h);
  const int rows = y1 - y0;
  const int half3 = 3 * (sdd_w >> 1);
  // cell sums live in the stage behind the column sums (written only after the stage is consumed; the host sizes the
  // stage >= 2*rb16 + 12*sdd_w), which keeps a 720p CTA at 33 KB
  uint32_t* cell = reinterpret_cast<uint32_t*>(smem + 2 * rb16);        // [3*sdd_w]
  uint32_t* pair_in = reinterpret_cast<uint32_t*>(smem + a.stage_bytes);  // [half3]
  int* xb = reinterpret_cast<int*>(pair_in + half3);                   // [sdd_w + 1]
  uint8_t* ref_s = reinterpret_cast<uint8_t*>(xb + sdd_w + 1);         // [3*sdd_w] this row of R
  const uint32_t bar_d = (uint32_t)__cvta_generic_to_shared(&bar_data);
  const uint32_t bar_p = (uint32_t)__cvta_generic_to_shared(&bar_pair);

  if (threadIdx.x == 0) {
    ptx::mbar_init(bar_d, 1);
    ptx::mbar_init(bar_p, 1);
    if (rank == 0) mbar_expect_tx(bar_p, (uint32_t)(4 * half3));  // our own arrival + the peer's bytes
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    mbar_expect_tx(bar_d, (uint32_t)(rows * rb16));
    const uint32_t dst = (uint32_t)__cvta_generic_to_shared(smem);
    const uint8_t* src = fd.pixels + (int64_t)y0 * fd.pitch;
    if (fd.pitch == rb16) {
      ptx::bulk_g2s_hint(dst, src, (uint32_t)(rows * rb16), bar_d, pol);
    } else {
      for (int y = 0; y < rows; ++y) ptx::bulk_g2s_hint(dst + y * rb16, src + (int64_t)y * fd.pitch, (uint32_t)rb16, bar_d, pol);
    }
  }
  // publish the peer's mbarrier before any remote st.async (relaxed: no memory fence needed beyond
  // fence.mbarrier_init); the matching wait comes right before the DSMEM exchange
#if FFSVA_K1_EARLYBAR
  __syncthreads();  // publishes the mbarrier init only; the xb / R-row writes below are ordered by later barriers
#endif
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
  if (a.xbounds) {  // set only for uniform-width batches
    for (int i = threadIdx.x; i <= sdd_w; i += blockDim.x) xb[i] = __ldg(a.xbounds + i);
  } else {
    fill_xbounds(xb, W, sdd_w);
  }
#if FFSVA_K1_REFPRE
  // this row of R into shared memory while the bulk copy is in flight: the cell phase then reads it at shared
  // latency instead of one dependent L2 round trip per loop iteration (which kept the stage occupied)
  {
    const uint8_t* rrow = fd.ref + (int64_t)r * (3 * sdd_w);
    const int n3 = 3 * sdd_w;
    if ((((uintptr_t)rrow) & 3) == 0 && (n3 & 3) == 0) {
      for (int i = threadIdx.x; i < (n3 >> 2); i += blockDim.x)
        reinterpret_cast<uint32_t*>(ref_s)[i] = __ldg(reinterpret_cast<const uint32_t*>(rrow) + i);
    } else {
      for (int i = threadIdx.x; i < n3; i += blockDim.x) ref_s[i] = __ldg(rrow + i);
    }
  }
#endif
#if !FFSVA_K1_EARLYBAR
  __syncthreads();
#endif
  ptx::mbar_wait(bar_d, 0);

  // ---- column sums of the row's source rows (<= 2 16-byte chunks per thread)
  uint32_t acc[kCh][8];
#pragma unroll
  for (int k = 0; k < kCh; ++k) {
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[k][j] = 0u;
    const int c = threadIdx.x + k * kNT;
    if (c < nchunk) {
      const uint8_t* p = smem + 16 * c;
      int y = 0;
      for (; y + 1 < rows; y += 2)
        acc16x2(acc[k], *reinterpret_cast<const uint4*>(p + y * rb16), *reinterpret_cast<const uint4*>(p + (y + 1) * rb16));
      if (y < rows) acc16(acc[k], *reinterpret_cast<const uint4*>(p + y * rb16));
    }
  }
  __syncthreads();  // the stage is consumed; its first 2*rb16 bytes now hold the u16 column sums
  uint16_t* colsum = reinterpret_cast<uint16_t*>(smem);
#pragma unroll
  for (int k = 0; k < kCh; ++k) {
    const int c = threadIdx.x + k * kNT;
    if (c < nchunk) store_colsum(reinterpret_cast<uint32_t*>(colsum), c, acc[k]);
  }
  __syncthreads();

  // ---- 100-grid cells of this row (one thread per cell and channel): D100, SSD vs R
  const int row3 = 3 * sdd_w;
  const int cellw = a.xbounds ? a.cellw : (W + sdd_w - 1) / sdd_w;  // widest cell (uniform over the CTA)
  uint32_t ssd_local = 0;
  for (int o = threadIdx.x; o < row3; o += blockDim.x) {
    const int cx = o / 3, ch = o - 3 * cx;
    const int x0 = xb[cx], x1 = xb[cx + 1];
    const uint16_t* col = colsum + ch;
    const uint32_t s = cell_sum_w(col, x0, x1, cellw);
    cell[o] = s;
    const uint32_t n = (uint32_t)(x1 - x0) * (uint32_t)rows;
    const uint32_t d = box_mean(s, n);
    if (kD100) a.d100[(int64_t)f * sdd_h * row3 + (int64_t)r * row3 + o] = (uint8_t)d;
#if FFSVA_K1_REFPRE
    const int diff = (int)d - (int)ref_s[o];
#else
    const int diff = (int)d - (int)__ldg(fd.ref + (int64_t)r * row3 + o);
#endif
    ssd_local += dist_term(diff, fd.metric);
  }
  if (fd.mode == kRefPrevious) ssd_local = 0;  // K2 measures against the previous frame's D100
  __syncthreads();

  // ---- D50 row: odd CTA -> even CTA (st.async into the peer's shared memory), even CTA combines 2x2 cells.
  // Only the odd CTA touches its peer's memory, so only it waits on the cluster barrier (for the peer's
  // mbarrier init); the even CTA stays alive until the peer's bytes land on its mbarrier.
  if (rank == 1) {
    asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
    const uint32_t rbase = map_to_rank((uint32_t)__cvta_generic_to_shared(pair_in), 0);
    const uint32_t rbar = map_to_rank(bar_p, 0);
    for (int o = threadIdx.x; o < half3; o += blockDim.x) {
      const int cx = o / 3, ch = o - 3 * cx;
      st_async_u32(rbase + 4u * (uint32_t)o, cell[6 * cx + ch] + cell[6 * cx + 3 + ch], rbar);
    }
  } else {
    const int yb = ytab ? __ldg(a.ybounds + r + 2) : (int)(((uint32_t)(r + 2) * (uint32_t)H) / (uint32_t)sdd_h);
    const int64_t slot = a.d50_index ? (int64_t)__ldg(a.d50_index + f) : (int64_t)f;
    uint8_t* d50row = a.d50 + slot * a.d50_stride + (int64_t)(r >> 1) * half3;
    ptx::mbar_wait(bar_p, 0);
    for (int o = threadIdx.x; o < half3; o += blockDim.x) {
      const int cx = o / 3, ch = o - 3 * cx;
      const uint32_t s = cell[6 * cx + ch] + cell[6 * cx + 3 + ch] + pair_in[o];
      const uint32_t n = (uint32_t)(xb[2 * cx + 2] - xb[2 * cx]) * (uint32_t)(yb - y0);
      d50row[o] = (uint8_t)box_mean(s, n);
    }
  }
  ssd_commit(ssd_local, red, a, f, fd.slot, r == 0);
}

// ------------------------------------------------------------------ narrow rows: both rows of a pair in one CTA
// For rows of <= 128 16-byte chunks (360p) the CTA-pair kernel's CTAs are short-lived enough that cluster dispatch
// limits residency (ncu, M1: 38 % of warps active against 100 % possible). This variant gives one 256-thread CTA
// both 100-grid rows 2b, 2b+1 of a 50-grid row: one bulk copy of their contiguous source rows, threads 0-127 take
// row 2b and 128-255 row 2b+1 through the column and cell phases, and the D50 row is formed in shared memory (no
// cluster, no DSMEM). Shared memory: stage (>= 4*rb16 + 24*sdd_w: the two u16 column-sum rows, then the u32 cell
// sums of both rows once the stage is consumed) | xb[sdd_w + 1] | both rows of R.
__global__ void __launch_bounds__(256, 8) sdd_band2_kernel_impl(SddArgs a, bool d100) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t bar_data;
  __shared__ uint32_t red[8];
  const int sdd_w = a.sdd_w, sdd_h = a.sdd_h;
  const int f = blockIdx.y;
  const int b = blockIdx.x;  // 50-grid row: 100-grid rows 2b, 2b+1
  const FrameDesc fd = a.frames[f];
  const int W = fd.W, H = fd.H;
  const int rb16 = (3 * W + 15) & ~15;
  const int nchunk = rb16 >> 4;
  const bool ytab = a.ybounds != nullptr;
  const int r0 = 2 * b;
  const int y0 = ytab ? __ldg(a.ybounds + r0) : (int)(((uint32_t)r0 * (uint32_t)H) / (uint32_t)sdd_h);
  const int ym = ytab ? __ldg(a.ybounds + r0 + 1) : (int)(((uint32_t)(r0 + 1) * (uint32_t)H) / (uint32_t)sdd_h);
  const int y1 = ytab ? __ldg(a.ybounds + r0 + 2) : (int)(((uint32_t)(r0 + 2) * (uint32_t)H) / (uint32_t)sdd_h);
  const int rows = y1 - y0;
  const int row3 = 3 * sdd_w, half3 = 3 * (sdd_w >> 1);
  uint32_t* cell = reinterpret_cast<uint32_t*>(smem + 4 * rb16);          // [2][row3], in the consumed stage
  int* xb = reinterpret_cast<int*>(smem + a.stage_bytes);                 // [sdd_w + 1]
  uint8_t* ref_s = reinterpret_cast<uint8_t*>(xb + sdd_w + 1);            // [2][row3]
  const uint32_t bar_d = (uint32_t)__cvta_generic_to_shared(&bar_data);

  if (threadIdx.x == 0) {
    ptx::mbar_init(bar_d, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    mbar_expect_tx(bar_d, (uint32_t)(rows * rb16));
    const uint32_t dst = (uint32_t)__cvta_generic_to_shared(smem);
    const uint8_t* src = fd.pixels + (int64_t)y0 * fd.pitch;
    if (fd.pitch == rb16) {
      ptx::bulk_g2s_hint(dst, src, (uint32_t)(rows * rb16), bar_d, pol);
    } else {
      for (int y = 0; y < rows; ++y) ptx::bulk_g2s_hint(dst + y * rb16, src + (int64_t)y * fd.pitch, (uint32_t)rb16, bar_d, pol);
    }
  }
#if FFSVA_K1_EARLYBAR
  __syncthreads();  // publishes the mbarrier init only; the xb / R-row writes below are ordered by later barriers
#endif
  if (a.xbounds) {
    for (int i = threadIdx.x; i <= sdd_w; i += blockDim.x) xb[i] = __ldg(a.xbounds + i);
  } else {
    fill_xbounds(xb, W, sdd_w);
  }
  {  // both rows of R (contiguous) while the copy is in flight
    const uint8_t* rrow = fd.ref + (int64_t)r0 * row3;
    const int n6 = 2 * row3;
    if ((((uintptr_t)rrow) & 3) == 0 && (n6 & 3) == 0) {
      for (int i = threadIdx.x; i < (n6 >> 2); i += blockDim.x)
        reinterpret_cast<uint32_t*>(ref_s)[i] = __ldg(reinterpret_cast<const uint32_t*>(rrow) + i);
    } else {
      for (int i = threadIdx.x; i < n6; i += blockDim.x) ref_s[i] = __ldg(rrow + i);
    }
  }
#if !FFSVA_K1_EARLYBAR
  __syncthreads();
#endif
  ptx::mbar_wait(bar_d, 0);

  // ---- column sums: threads 0-127 over row 2b's source rows, 128-255 over row 2b+1's
  const int h = threadIdx.x >> 7, c = threadIdx.x & 127;
  const int ylo = h ? ym - y0 : 0, yhi = h ? rows : ym - y0;
  uint32_t acc[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) acc[j] = 0u;
  if (c < nchunk) {
    const uint8_t* p = smem + 16 * c;
    int y = ylo;
    for (; y + 1 < yhi; y += 2)
      acc16x2(acc, *reinterpret_cast<const uint4*>(p + y * rb16), *reinterpret_cast<const uint4*>(p + (y + 1) * rb16));
    if (y < yhi) acc16(acc, *reinterpret_cast<const uint4*>(p + y * rb16));
  }
  __syncthreads();  // the stage is consumed: [h * 2*rb16, (h+1) * 2*rb16) now holds row h's u16 column sums
  if (c < nchunk) store_colsum(reinterpret_cast<uint32_t*>(smem + h * 2 * rb16), c, acc);
  __syncthreads();

  // ---- 100-grid cells of both rows: D100, distance vs R
  const int cellw = a.xbounds ? a.cellw : (W + sdd_w - 1) / sdd_w;
  uint32_t ssd_local = 0;
  for (int o = threadIdx.x; o < 2 * row3; o += blockDim.x) {
    const int sub = o >= row3;
    const int rr = o - sub * row3;
    const int cx = rr / 3, ch = rr - 3 * cx;
    const int x0 = xb[cx], x1 = xb[cx + 1];
    const uint16_t* col = reinterpret_cast<const uint16_t*>(smem + sub * 2 * rb16) + ch;
    const uint32_t sum = cell_sum_w(col, x0, x1, cellw);
    cell[o] = sum;
    const uint32_t n = (uint32_t)(x1 - x0) * (uint32_t)(sub ? y1 - ym : ym - y0);
    const uint32_t d = box_mean(sum, n);
    if (d100) a.d100[(int64_t)f * sdd_h * row3 + (int64_t)(r0 + sub) * row3 + rr] = (uint8_t)d;
    ssd_local += dist_term((int)d - (int)ref_s[o], fd.metric);
  }
  if (fd.mode == kRefPrevious) ssd_local = 0;  // K2 measures against the previous frame's D100
  __syncthreads();

  // ---- D50 row from the four 100-cell sums of each 50-cell
  {
    const int64_t slot = a.d50_index ? (int64_t)__ldg(a.d50_index + f) : (int64_t)f;
    uint8_t* d50row = a.d50 + slot * a.d50_stride + (int64_t)b * half3;
    for (int o = threadIdx.x; o < half3; o += blockDim.x) {
      const int cx = o / 3, ch = o - 3 * cx;
      const uint32_t sum = cell[6 * cx + ch] + cell[6 * cx + 3 + ch] + cell[row3 + 6 * cx + ch] +
                           cell[row3 + 6 * cx + 3 + ch];
      const uint32_t n = (uint32_t)(xb[2 * cx + 2] - xb[2 * cx]) * (uint32_t)rows;
      d50row[o] = (uint8_t)box_mean(sum, n);
    }
  }
  ssd_commit(ssd_local, red, a, f, fd.slot, b == 0);
}

// ------------------------------------------------------------------ narrow rows: warp-segment pipeline
// K1 for rows of <= 128 16-byte chunks (360p) without CTA barriers. A persistent CTA = one producer warp + kG
// groups of kSegWarps consumer warps; the producer bulk-copies the CTA's units (frame, 50-grid row = two 100-grid rows)
// into a kNS-stage ring (full / empty mbarriers), group g consumes units g, g + kG, ... Within a group, warp w owns
// a horizontal segment of the 50-grid row (50-cells [k0, k1), at most 10) and does all of its work alone:
//   column phase — lane = 16-byte chunk of the segment's window (<= 32 chunks), packed 2 x 16-bit vertical sums of
//                  each 100-grid row's source rows into a warp-private u16 column-sum row;
//   cell phase   — lane = 100-grid cell of the segment, all three channels at once from u32 pairs of column sums
//                  (absolute word w holds columns 2w, 2w+1, so w mod 3 fixes its channels: residue 0 = (c0, c1),
//                  1 = (c2, c0), 2 = (c1, c2); a lone edge column is added alone), box means by multiply-high
//                  (magic table: floor(2^32 / n) + 1, exact while sum * n < 2^32), D100 (optional), distance to R;
//   D50          — each lane sums its cell over the two rows, the horizontal pair is one shuffle, even lanes emit
//                  the 50-cell (Q8);
// then lane 0 releases the stage (empty mbarrier, one arrival per warp). Warps only ever wait for data, never for
// each other. The distance accumulates per lane over a warp's consecutive units of one frame and is reduced with one
// atomic per warp and frame.
constexpr int kSegWarps = 5;   // consumer warps per unit (half_w <= 50: at most 10 50-cells per warp)

// kMinB CTAs per SM (register cap); a cell spans between kW0 and kW1 u32 words of column sums (kW0 loads need no
// predicate); a 100-grid row has at most kMaxRows source rows. Boxes of one pixel are excluded by the host (the
// magic table's n = 1 entry is not used).
template <int kG, int kNS, int kMinB, int kW0, int kW1, int kMaxRows>
__global__ void __launch_bounds__(32 * (kG * kSegWarps + 1), kMinB) sdd_seg_kernel(SddArgs a) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t full[kNS], empty[kNS];
  __shared__ int ybnd[kNS][3];  // source-row bounds of the unit's two 100-grid rows (frame rows)
  __shared__ int unit_f[kNS], unit_b[kNS], unit_roff[kNS];
  const int sdd_w = a.sdd_w, sdd_h = a.sdd_h, half_w = sdd_w >> 1;
  constexpr int kCons = kG * kSegWarps;
  // a stage = the unit's source rows, then (at r_base) the 16-byte aligned span holding its two rows of R
  const int r_base = a.stage_bytes - ((6 * sdd_w + 31) & ~15);
  uint8_t* stage = smem;                                                                    // [kNS][stage_bytes]
  uint16_t* colsum = reinterpret_cast<uint16_t*>(smem + (size_t)kNS * a.stage_bytes);       // [kCons][2][512]
  uint32_t* magic = reinterpret_cast<uint32_t*>(colsum + kCons * 2 * 512);                  // [magic_n]
  const int nb = sdd_h >> 1;  // units per frame
  const int64_t U = (int64_t)a.n * nb;
  const int64_t u_begin = (int64_t)blockIdx.x * U / gridDim.x;
  const int n_units = (int)((int64_t)(blockIdx.x + 1) * U / gridDim.x - u_begin);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int st = 0; st < kNS; ++st) {
      ptx::mbar_init((uint32_t)__cvta_generic_to_shared(&full[st]), 1);
      ptx::mbar_init((uint32_t)__cvta_generic_to_shared(&empty[st]), kSegWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (int n = threadIdx.x; n < a.magic_n; n += blockDim.x)
    magic[n] = n > 1 ? 0xFFFFFFFFu / (uint32_t)n + 1u : (uint32_t)n;
  __syncthreads();  // the only CTA barrier: mbarrier init + magic table

  if (warp == kCons) {
    // ---------------- producer warp (lane 0): the CTA's units in order through the stage ring
    if (lane == 0) {
      int fi = (int)(u_begin / nb), bi = (int)(u_begin - (int64_t)fi * nb);
      uint64_t pol;
      asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
      for (int i = 0; i < n_units; ++i) {
        const int st = i % kNS;
        if (i >= kNS) ptx::mbar_wait((uint32_t)__cvta_generic_to_shared(&empty[st]), (uint32_t)((i / kNS - 1) & 1));
        const FrameDesc& fd = a.frames[fi];
        const int H = fd.H, rb16 = (3 * fd.W + 15) & ~15;
        int y[3];
#pragma unroll
        for (int j = 0; j < 3; ++j)
          y[j] = a.ybounds ? __ldg(a.ybounds + 2 * bi + j) : (int)(((uint32_t)(2 * bi + j) * (uint32_t)H) / (uint32_t)sdd_h);
        ybnd[st][0] = y[0];
        ybnd[st][1] = y[1];
        ybnd[st][2] = y[2];
        unit_f[st] = fi;
        unit_b[st] = bi;
        if (bi == 0 && a.stats) atomicAdd(a.stats + (int64_t)fd.slot * NSTAT + 0, 1ull);
        const int rows = y[2] - y[0];
        // the unit's rows of R (L2-resident, 600 B at the default grid) ride along in the same stage
        const int r0 = 2 * bi * 3 * sdd_w, r16 = r0 & ~15;
        const int rbytes = (r0 - r16 + 6 * sdd_w + 15) & ~15;
        unit_roff[st] = r0 - r16;
        const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&full[st]);
        mbar_expect_tx(bar, (uint32_t)(rows * rb16 + rbytes));  // release: the unit's ybnd / unit_* writes above
        const uint32_t dst = (uint32_t)__cvta_generic_to_shared(stage + (size_t)st * a.stage_bytes);
        ptx::bulk_g2s_hint(dst + r_base, fd.ref + r16, (uint32_t)rbytes, bar, pol);
        const uint8_t* src = fd.pixels + (int64_t)y[0] * fd.pitch;
        if (fd.pitch == rb16) {
          ptx::bulk_g2s_hint(dst, src, (uint32_t)(rows * rb16), bar, pol);
        } else {
          for (int yy = 0; yy < rows; ++yy)
            ptx::bulk_g2s_hint(dst + yy * rb16, src + (int64_t)yy * fd.pitch, (uint32_t)rb16, bar, pol);
        }
        if (++bi == nb) {
          bi = 0;
          ++fi;
        }
      }
    }
    return;
  }

  // ---------------- consumer warps
  const int g = warp / kSegWarps, ws = warp - g * kSegWarps;
  const int k0 = ws * half_w / kSegWarps, k1 = (ws + 1) * half_w / kSegWarps;  // this warp's 50-cells
  const int ncell = 2 * (k1 - k0);                                             // 100-cells per row
  uint16_t* cs_w = colsum + (size_t)warp * 2 * 512;                            // [2][512] this warp's column sums
  // per frame width (recomputed when it changes): the window's first chunk, this lane's cell's word range
  int cur_w = -1, win_c0 = 0, win_n = 0;
  int c_word = 0, c_nw = 0, c_q = 0, c_e0 = -1, c_e2 = -1;  // relative word index, count, residue, lone columns
  uint32_t c_wd = 0, c_w50 = 0;                             // cell width, its 50-cell's width (pixels)
  int cur_f = -1, cur_slot = 0;
  uint8_t cur_mode = 0, cur_metric = 0;
  const uint8_t* cur_ref = nullptr;
  uint8_t* cur_d50 = nullptr;
  uint32_t ssd_acc = 0;
  const int cx = 2 * k0 + lane;  // this lane's 100-grid cell column (valid if lane < ncell)
  const bool has_cell = lane < ncell;

  for (int i = g; i < n_units; i += kG) {
    const int st = i % kNS;
    const uint32_t fb = (uint32_t)__cvta_generic_to_shared(&full[st]);
    ptx::mbar_wait(fb, (uint32_t)((i / kNS) & 1));
    const int f = unit_f[st], b = unit_b[st], roff = unit_roff[st];
    const int y0 = ybnd[st][0], y1 = ybnd[st][1], y2 = ybnd[st][2];
    if (f != cur_f) {  // warp-uniform
      if (cur_f >= 0) {
        uint32_t v = ssd_acc;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
        if (lane == 0 && v) {
          atomicAdd(a.acc_ssd + cur_f, (unsigned long long)v);
          if (a.stats) atomicAdd(a.stats + (int64_t)cur_slot * NSTAT + 3, (unsigned long long)v);
        }
        ssd_acc = 0;
      }
      cur_f = f;
      const FrameDesc& fd = a.frames[f];
      cur_slot = fd.slot;
      cur_mode = fd.mode;
      cur_metric = fd.metric;
      cur_ref = fd.ref;
      cur_d50 = a.d50 + (a.d50_index ? (int64_t)__ldg(a.d50_index + f) : (int64_t)f) * a.d50_stride;
      const int W = fd.W;
      if (W != cur_w) {
        auto xbd = [&](int c) { return (int)(((uint32_t)c * (uint32_t)W) / (uint32_t)sdd_w); };
        const int X0 = xbd(2 * k0), X1 = xbd(2 * k1);
        win_c0 = (3 * X0) >> 4;
        win_n = ((3 * X1 + 15) >> 4) - win_c0;
        const int x0 = xbd(cx), x1 = xbd(cx + 1);
        int s = 3 * x0, e = 3 * x1;  // absolute columns
        c_e0 = (s & 1) ? s++ - 16 * win_c0 : -1;
        c_e2 = (e & 1) ? --e - 16 * win_c0 : -1;
        c_word = (s >> 1) - 8 * win_c0;
        c_nw = (e - s) >> 1;
        c_q = (s >> 1) % 3;
        c_wd = (uint32_t)(x1 - x0);
        c_w50 = (uint32_t)(xbd(2 * (k0 + (lane >> 1)) + 2) - xbd(2 * (k0 + (lane >> 1))));
        cur_w = W;
      }
    }
    const int rb16 = (3 * cur_w + 15) & ~15;
    // R of this lane's cell in both rows, from the stage
    uint32_t rv[2][3] = {{0, 0, 0}, {0, 0, 0}};
    if (has_cell) {
      const uint8_t* rp = stage + (size_t)st * a.stage_bytes + r_base + roff + cx * 3;
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        rv[0][c] = rp[c];
        rv[1][c] = rp[3 * sdd_w + c];
      }
    }

    // ---- column phase: lane = chunk of the window, both 100-grid rows
    const uint8_t* sp = stage + (size_t)st * a.stage_bytes;
    if (lane < win_n) {
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        const int ylo = (r ? y1 : y0) - y0, yn = (r ? y2 - y1 : y1 - y0);
        const uint8_t* p = sp + 16 * (win_c0 + lane) + ylo * rb16;
        uint32_t acc[8] = {0u, 0u, 0u, 0u, 0u, 0u, 0u, 0u};
#pragma unroll
        for (int yy = 0; yy < kMaxRows; yy += 2) {
          if (yy + 1 < yn)
            acc16x2(acc, *reinterpret_cast<const uint4*>(p + yy * rb16), *reinterpret_cast<const uint4*>(p + (yy + 1) * rb16));
          else if (yy < yn)
            acc16(acc, *reinterpret_cast<const uint4*>(p + yy * rb16));
        }
        store_colsum(reinterpret_cast<uint32_t*>(cs_w + r * 512), lane, acc);
      }
    }
    __syncwarp();
    // the stage is consumed by this warp
    if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(&empty[st])) : "memory");

    // ---- cell phase: lane = 100-grid cell, rows A then B; the 50-cell sums accumulate in the lane
    uint32_t s50[3] = {0, 0, 0};
    if (has_cell) {
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        const uint16_t* cs = cs_w + r * 512;
        const uint32_t* w = reinterpret_cast<const uint32_t*>(cs) + c_word;
        uint32_t bb[3] = {0u, 0u, 0u};
#pragma unroll
        for (int k = 0; k < kW1; ++k)
          if (k < kW0 || k < c_nw) bb[k % 3] += w[k];
        const uint32_t b0 = bb[0], b1 = bb[1], b2 = bb[2];
        const uint32_t A0 = c_q == 0 ? b0 : (c_q == 1 ? b2 : b1);
        const uint32_t A1 = c_q == 0 ? b1 : (c_q == 1 ? b0 : b2);
        const uint32_t A2 = c_q == 0 ? b2 : (c_q == 1 ? b1 : b0);
        const uint32_t c0 = (A0 & 0xFFFFu) + (A1 >> 16) + (c_e0 >= 0 ? (uint32_t)cs[c_e0] : 0u);
        const uint32_t c1 = (A0 >> 16) + (A2 & 0xFFFFu);
        const uint32_t c2 = (A1 & 0xFFFFu) + (A2 >> 16) + (c_e2 >= 0 ? (uint32_t)cs[c_e2] : 0u);
        s50[0] += c0;
        s50[1] += c1;
        s50[2] += c2;
        const uint32_t n = c_wd * (uint32_t)(r ? y2 - y1 : y1 - y0);
        const uint32_t m = magic[n];
        const uint32_t d0 = __umulhi(c0 + (n >> 1), m), d1 = __umulhi(c1 + (n >> 1), m), d2 = __umulhi(c2 + (n >> 1), m);
        const int e0 = (int)d0 - (int)rv[r][0], e1 = (int)d1 - (int)rv[r][1], e2 = (int)d2 - (int)rv[r][2];
        if (cur_mode != kRefPrevious) {  // PREVIOUS mode: K2 measures against the previous frame's D100
          if (cur_metric == kDistSad) ssd_acc += (uint32_t)(abs(e0) + abs(e1) + abs(e2));
          else ssd_acc += (uint32_t)(e0 * e0 + e1 * e1 + e2 * e2);
        }
        if (a.d100) {
          uint8_t* o = a.d100 + (int64_t)cur_f * sdd_h * 3 * sdd_w + ((int64_t)(2 * b + r) * sdd_w + cx) * 3;
          o[0] = (uint8_t)d0;
          o[1] = (uint8_t)d1;
          o[2] = (uint8_t)d2;
        }
      }
    }
    // ---- D50: horizontal pair (lanes 2m, 2m + 1) by one shuffle per channel; even lanes emit the 50-cell
#pragma unroll
    for (int c = 0; c < 3; ++c) s50[c] += __shfl_xor_sync(0xffffffffu, s50[c], 1);
    if (has_cell && !(lane & 1)) {
      const uint32_t n50 = c_w50 * (uint32_t)(y2 - y0);
      const uint32_t m50 = magic[n50];
      uint8_t* o = cur_d50 + ((int64_t)b * half_w + k0 + (lane >> 1)) * 3;
#pragma unroll
      for (int c = 0; c < 3; ++c) o[c] = (uint8_t)__umulhi(s50[c] + (n50 >> 1), m50);
    }
  }
  if (cur_f >= 0) {
    uint32_t v = ssd_acc;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
    if (lane == 0 && v) {
      atomicAdd(a.acc_ssd + cur_f, (unsigned long long)v);
      if (a.stats) atomicAdd(a.stats + (int64_t)cur_slot * NSTAT + 3, (unsigned long long)v);
    }
  }
}

// Reference image R: one rounding of the mean over k frames x box. One thread per value.
__global__ void reference_kernel(const uint8_t* __restrict__ frames, int32_t k, int64_t frame_stride, int32_t W,
                                 int32_t H, int64_t pitch, int32_t sdd_w, int32_t sdd_h, uint8_t* __restrict__ out) {
  const int o = blockIdx.x * blockDim.x + threadIdx.x;
  if (o >= 3 * sdd_w * sdd_h) return;
  const int oy = o / (3 * sdd_w), r = o - oy * 3 * sdd_w, ox = r / 3, ch = r - 3 * ox;
  const int64_t y0 = ((int64_t)oy * H) / sdd_h, y1 = ((int64_t)(oy + 1) * H) / sdd_h;
  const int64_t x0 = ((int64_t)ox * W) / sdd_w, x1 = ((int64_t)(ox + 1) * W) / sdd_w;
  unsigned long long s = 0;
  for (int j = 0; j < k; ++j)
    for (int64_t y = y0; y < y1; ++y) {
      const uint8_t* row = frames + (int64_t)j * frame_stride + y * pitch + ch;
      for (int64_t x = x0; x < x1; ++x) s += row[3 * x];
    }
  const unsigned long long n = (unsigned long long)k * (unsigned long long)((y1 - y0) * (x1 - x0));
  out[o] = (uint8_t)((s + n / 2) / n);
}

// K2: distance of a PREVIOUS-mode frame's D100 to its stream's previous D100 (or R for the stream's first frame
// of the batch). One CTA per frame; 16-byte loads of two L2-resident 30 KB images (K1 wrote them just before).
constexpr int kPrevThreads = 256;
__global__ void __launch_bounds__(kPrevThreads) sdd_prev_kernel(PrevArgs a) {
  __shared__ unsigned long long red[kPrevThreads / 32];
  const int f = a.pairs[2 * blockIdx.x], prev = a.pairs[2 * blockIdx.x + 1];
  const FrameDesc& fd = a.frames[f];
  const uint8_t* x = a.d100 + (int64_t)f * a.n_values;
  const uint8_t* r = prev >= 0 ? a.d100 + (int64_t)prev * a.n_values : fd.ref;
  const bool sad = fd.metric == kDistSad;
  // u64 sums: one CTA covers a whole frame, and grids up to 4096x4096 would wrap a 32-bit sum (a 16-byte chunk's
  // partial, <= 16 * 255^2, is the only 32-bit quantity)
  unsigned long long acc = 0;
  const int nv16 = a.n_values >> 4;  // n_values = 3*sdd_w*sdd_h, sdd_w and sdd_h even: a multiple of 4 only
  if ((a.n_values & 15) == 0) {
    for (int i = threadIdx.x; i < nv16; i += kPrevThreads) {
      const uint4 u = reinterpret_cast<const uint4*>(x)[i], v = reinterpret_cast<const uint4*>(r)[i];
      const uint32_t uw[4] = {u.x, u.y, u.z, u.w}, vw[4] = {v.x, v.y, v.z, v.w};
      uint32_t part = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        if (sad) {
          part = __vsadu4(uw[k], vw[k]) + part;
        } else {
#pragma unroll
          for (int b = 0; b < 4; ++b) {
            const int d = (int)((uw[k] >> (8 * b)) & 255u) - (int)((vw[k] >> (8 * b)) & 255u);
            part += (uint32_t)(d * d);
          }
        }
      }
      acc += part;
    }
  } else {
    for (int i = threadIdx.x; i < a.n_values; i += kPrevThreads) acc += dist_term((int)x[i] - (int)r[i], fd.metric);
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int w = 0; w < kPrevThreads / 32; ++w) t += red[w];
    atomicAdd(a.acc_ssd + f, t);
    if (a.stats) atomicAdd(a.stats + (int64_t)fd.slot * NSTAT + 3, t);
  }
}

// K2b: the stream's reference becomes the D100 of its last frame in the batch (runs after every K2 read of R).
__global__ void __launch_bounds__(kPrevThreads) ref_update_kernel(PrevArgs a) {
  const int f = a.last[blockIdx.x];
  const uint8_t* src = a.d100 + (int64_t)f * a.n_values;
  uint8_t* dst = const_cast<uint8_t*>(a.frames[f].ref);
  if ((a.n_values & 15) == 0) {
    for (int i = threadIdx.x; i < (a.n_values >> 4); i += kPrevThreads)
      reinterpret_cast<uint4*>(dst)[i] = reinterpret_cast<const uint4*>(src)[i];
  } else {
    for (int i = threadIdx.x; i < a.n_values; i += kPrevThreads) dst[i] = src[i];
  }
}

__global__ void fill_nan_kernel(float* p, int32_t n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = __int_as_float(0x7fc00000);
}

}  // namespace

size_t sdd_smem_bytes(int max_chunks, int sdd_w) {
  return (size_t)4 * 16 * max_chunks + (size_t)8 * 3 * sdd_w + (size_t)4 * (sdd_w + 1);
}

int sdd_threads(int max_chunks) {
  int t = ((max_chunks + 31) / 32) * 32;
  if (t < 64) t = 64;
  if (t > 512) t = 512;
  return t;
}

size_t sdd_bulk_smem_bytes(int stage_bytes, int sdd_w) {
  return (size_t)stage_bytes + (size_t)4 * (3 * (sdd_w / 2) + sdd_w + 1) + (size_t)((3 * sdd_w + 3) & ~3);
}

int sdd_bulk_stage_bytes(int W, int H, int sdd_h) {
  const int rb16 = (3 * W + 15) & ~15;
  int rows = (H + sdd_h - 1) / sdd_h;  // max source rows of one 100-grid row
  if (rows < 2) rows = 2;              // the stage also holds the 2*rb16-byte column sums
  return rows * rb16;
}

bool sdd_bulk_ok(int max_chunks, int stage_bytes) {
  return max_chunks <= 2 * kBulkThreads && stage_bytes <= kBulkMaxStage;
}

void sdd_plan_add(SddPlan& p, int32_t W, int32_t H, int64_t pitch, const void* pixels, int32_t sdd_h) {
  const int rb16 = (3 * W + 15) & ~15;
  p.max_chunks = std::max(p.max_chunks, rb16 >> 4);
  p.pair_stage = std::max(p.pair_stage, sdd_bulk_stage_bytes(W, H, sdd_h));
  // a 50-grid row (two 100-grid rows) spans at most ceil(2H / sdd_h) source rows
  p.seg_stage = std::max(p.seg_stage, ((2 * H + sdd_h - 1) / sdd_h) * rb16);
  p.max_rows100 = std::max(p.max_rows100, (H + sdd_h - 1) / sdd_h);
  p.max_w = std::max(p.max_w, W);
  p.min_w = p.min_w ? std::min(p.min_w, W) : W;
  if ((pitch & 15) || ((uintptr_t)pixels & 15)) p.vec16 = false;
}

int k1_variant(int max_chunks, int sdd_w);
constexpr int kK1Band2 = 1282;  // k1_variant id of sdd_band2_kernel_impl (rows of <= 128 chunks)

int sdd_seg_magic_n(const SddPlan& p, int sdd_w) {  // largest box area + 1: a 50-grid cell of 2 x 2 100-grid cells
  return 4 * p.max_rows100 * ((p.max_w + sdd_w - 1) / sdd_w) + 1;
}

// (groups of 5 consumer warps, stages) of the warp-segment kernel, measured on M1 (profiles/r02/k1_m1_ab.md):
// 2 groups x 5 stages, two CTAs per SM; FFSVA_K1_SEG="g,ns" selects another instantiated pair (A/B)
struct SegCfg {
  int g, ns;
};
SegCfg seg_cfg() {
  SegCfg c{2, 5};
  if (const char* e = std::getenv("FFSVA_K1_SEG")) {
    int g = 0, ns = 0;
    if (std::sscanf(e, "%d,%d", &g, &ns) == 2 && ((g == 2 && ns == 5) || (g == 3 && ns == 8) || (g == 2 && ns == 4)))
      c = SegCfg{g, ns};
  }
  return c;
}
size_t sdd_seg_smem_bytes(int stage_bytes, int magic_n) {
  const SegCfg c = seg_cfg();
  return (size_t)c.ns * stage_bytes + (size_t)c.g * kSegWarps * 2 * 512 * 2 + (size_t)4 * magic_n;
}
// The warp-segment kernel takes a narrow-row batch when: at most 10 50-cells per warp (half_w <= 50); a segment's
// window of <= 32 chunks (cells of <= 8 px); packed 16-bit lanes that cannot overflow (every 100-cell channel sum
// <= 65535); cells of >= 2 px (no one-pixel box: the magic table's n = 1 entry is not used); a unit that fits the stage
// budget.
bool sdd_seg_ok(const SddPlan& p, int sdd_w) {
  const int cellw = (p.max_w + sdd_w - 1) / sdd_w;
  return sdd_w / 2 <= 10 * kSegWarps && cellw <= 8 && (int64_t)p.max_rows100 * cellw * 255 <= 65535 &&
         p.max_rows100 <= 16 && p.seg_stage <= 32 * 1024 && p.min_w >= 2 * sdd_w;
}

size_t sdd_band2_smem_bytes(int stage_bytes, int sdd_w) {
  return (size_t)stage_bytes + (size_t)4 * (sdd_w + 1) + (size_t)((6 * sdd_w + 3) & ~3);
}

void sdd_plan_finish(SddPlan& p, int32_t sdd_w, int32_t sdd_h) {
  (void)sdd_h;
  const char* force = std::getenv("FFSVA_SDD_KERNEL");
  const bool pair_ok = p.vec16 && sdd_bulk_ok(p.max_chunks, p.pair_stage);
  p.variant = pair_ok && !(force && !std::strcmp(force, "stream")) ? kSddPair : kSddStream;
  if (p.variant == kSddPair) {
    const char* nt = std::getenv("FFSVA_K1_NT");  // 1282 keeps the one-CTA-per-band kernel (A/B)
    if (k1_variant(p.max_chunks, sdd_w) == kK1Band2 && sdd_seg_ok(p, sdd_w) && !(nt && std::atoi(nt) == kK1Band2)) {
      // source rows, then the 16-byte aligned span of the unit's two rows of R (the kernel's r_base)
      p.stage_bytes = (p.seg_stage + ((6 * sdd_w + 31) & ~15) + 127) & ~127;
      p.smem = sdd_seg_smem_bytes(p.stage_bytes, sdd_seg_magic_n(p, sdd_w));
      p.seg = true;
      } else if (k1_variant(p.max_chunks, sdd_w) == kK1Band2) {  // two rows' sources; then 2 x column sums + 2 x cells
      p.stage_bytes = std::max(2 * p.pair_stage, 64 * p.max_chunks + 24 * sdd_w);
      p.smem = sdd_band2_smem_bytes(p.stage_bytes, sdd_w);
    } else {
      p.stage_bytes = std::max(p.pair_stage, 32 * p.max_chunks + 12 * sdd_w);
      p.smem = sdd_bulk_smem_bytes(p.stage_bytes, sdd_w);
    }
  } else {
    p.stage_bytes = 0;
    p.smem = sdd_smem_bytes(p.max_chunks, sdd_w);
  }
}

void sdd_plan_apply(const SddPlan& p, SddArgs& a) {
  a.seg = p.seg;
  a.max_cellw = (p.max_w + a.sdd_w - 1) / a.sdd_w;
  a.max_rows100 = p.max_rows100;
  a.min_cellw = p.min_w / a.sdd_w;
  a.magic_n = sdd_seg_magic_n(p, a.sdd_w);
  a.max_chunks = p.max_chunks;
  a.vec16 = p.vec16;
  a.bulk = p.variant == kSddPair;
  a.stage_bytes = p.stage_bytes;
}

template <int kNT, int kCh, int kMinB>
cudaError_t k1_set_smem(int smem) {
  cudaError_t e = cudaFuncSetAttribute(sdd_bulk_kernel<true, kNT, kCh, kMinB>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(sdd_bulk_kernel<false, kNT, kCh, kMinB>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             smem);
  return e;
}

template <int kNT, int kCh, int kMinB>
void k1_launch(const SddArgs& b, dim3 grid, size_t smem, cudaStream_t st) {
  if (b.d100) sdd_bulk_kernel<true, kNT, kCh, kMinB><<<grid, kNT, smem, st>>>(b);
  else sdd_bulk_kernel<false, kNT, kCh, kMinB><<<grid, kNT, smem, st>>>(b);
}

// K1 variant (block size) for a batch, measured on B200 (profiles/r01/k1_ab.md): rows of <= 128 16-byte chunks
// (360p) 128 threads; <= 256 chunks (720p) 256 threads with one chunk each at 7 CTAs/SM; 321..384 chunks (1080p)
// 384 threads (one chunk and one 100-grid value per thread: M3 0.93 -> 0.99 of the copy peak); otherwise 256
// threads with two chunks each. Rows of <= 128 chunks run sdd_band2_kernel_impl (both rows of a pair in one CTA).
// FFSVA_K1_NT = 128 (CTA pairs) / 1282 (band of two) / 256 / 384 / 2562 (256 threads, two chunks) overrides (A/B).
int k1_variant(int max_chunks, int sdd_w) {
  const int need = std::max(max_chunks, 3 * sdd_w);
  int v = max_chunks <= 128 ? kK1Band2 : max_chunks <= 256 ? 256 : (need <= 384) ? 384 : 2562;
  if (const char* e = std::getenv("FFSVA_K1_NT")) {
    const int o = std::atoi(e);
    const int cap = o == 2562 ? 512 : o == kK1Band2 ? 128 : o;
    if ((o == 128 || o == 256 || o == 384 || o == 2562 || o == kK1Band2) && max_chunks <= cap) v = o;
  }
  return v;
}

// warp-segment kernel instantiations: 360p (cells of 6-7 px = 8-10 words, 100-grid rows of 3-4 source rows) and a
// general one (cells <= 8 px, <= 16 source rows)
#define SEG_360(kG, kNS, kMinB) sdd_seg_kernel<kG, kNS, kMinB, 8, 10, 4>
#define SEG_GEN(kG, kNS, kMinB) sdd_seg_kernel<kG, kNS, kMinB, 0, 12, 16>
template <int kG, int kNS, int kMinB>
cudaError_t seg_set_smem(int smem) {
  cudaError_t e = cudaFuncSetAttribute(SEG_360(kG, kNS, kMinB), cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(SEG_GEN(kG, kNS, kMinB), cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  return e;
}

cudaError_t sdd_configure(size_t smem) {
  // per device (the attribute is set on the current device); it is an upper bound for every later launch there, so
  // it never goes below the 48 KB default
  static size_t configured[64] = {};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) dev = 0;
  smem = std::max(smem, (size_t)48 * 1024);
  if (smem <= configured[dev]) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(sdd_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(sdd_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess)
    e = k1_set_smem<128, 1, FFSVA_K1_MINB128>((int)smem);
  if (e == cudaSuccess) e = k1_set_smem<256, 1, 7>((int)smem);
  if (e == cudaSuccess) e = k1_set_smem<256, 2, FFSVA_K1_MINBLOCKS>((int)smem);
  if (e == cudaSuccess) e = k1_set_smem<384, 1, 3>((int)smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(sdd_band2_kernel_impl, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess) e = seg_set_smem<2, 5, 2>((int)smem);
  if (e == cudaSuccess) e = seg_set_smem<3, 8, 1>((int)smem);
  if (e == cudaSuccess) e = seg_set_smem<2, 4, 2>((int)smem);
  if (e == cudaSuccess) configured[dev] = smem;
  return e;
}

// Persistent grid of the warp-segment kernel: every SM filled to its occupancy.
template <typename K>
int seg_grid(K kernel, int threads, size_t smem, int64_t units) {
  int dev = 0, sms = 0, per_sm = 1;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, smem) != cudaSuccess || per_sm < 1)
    per_sm = 1;
  return (int)std::max<int64_t>(1, std::min<int64_t>(units, (int64_t)sms * per_sm));
}

template <int kG, int kNS, int kMinB>
void seg_launch(const SddArgs& a, size_t smem, int64_t units, cudaStream_t st) {
  const int threads = 32 * (kG * kSegWarps + 1);
  if (a.max_rows100 <= 4 && a.max_cellw <= 7 && a.min_cellw >= 6) {  // 360p
    auto k = SEG_360(kG, kNS, kMinB);
    k<<<seg_grid(k, threads, smem, units), threads, smem, st>>>(a);
  } else {
    auto k = SEG_GEN(kG, kNS, kMinB);
    k<<<seg_grid(k, threads, smem, units), threads, smem, st>>>(a);
  }
}

cudaError_t launch_sdd(const SddArgs& a, cudaStream_t st) {
  if (a.n <= 0) return cudaSuccess;
  if (a.bulk && a.seg) {
    const size_t smem = sdd_seg_smem_bytes(a.stage_bytes, a.magic_n);
    const int64_t units = (int64_t)a.n * (a.sdd_h / 2);
    const SegCfg c = seg_cfg();
    if (c.g == 3) seg_launch<3, 8, 1>(a, smem, units, st);
    else if (c.ns == 4) seg_launch<2, 4, 2>(a, smem, units, st);
    else seg_launch<2, 5, 2>(a, smem, units, st);
    return cudaGetLastError();
  }
  if (a.bulk) {
    const int v = k1_variant(a.max_chunks, a.sdd_w);
    const size_t smem = v == kK1Band2 ? sdd_band2_smem_bytes(a.stage_bytes, a.sdd_w)
                                      : sdd_bulk_smem_bytes(a.stage_bytes, a.sdd_w);
    // grid (row, frame); gridDim.y <= 65535, so very large batches take several launches
    for (int32_t f0 = 0; f0 < a.n; f0 += 65535) {
      SddArgs b = a;
      const int32_t cnt = a.n - f0 < 65535 ? a.n - f0 : 65535;
      b.frames += f0;
      b.acc_ssd += f0;
      b.n = cnt;
      if (b.d50_index) b.d50_index += f0;
      else b.d50 += (int64_t)f0 * a.d50_stride;
      if (b.d100) b.d100 += (int64_t)f0 * a.sdd_w * a.sdd_h * 3;
      const dim3 grid((unsigned)a.sdd_h, (unsigned)cnt);
      switch (v) {
        case kK1Band2:
          sdd_band2_kernel_impl<<<dim3((unsigned)(a.sdd_h / 2), (unsigned)cnt), 256, smem, st>>>(b, b.d100 != nullptr);
          break;
        case 128: k1_launch<128, 1, FFSVA_K1_MINB128>(b, grid, smem, st); break;
        case 256: k1_launch<256, 1, 7>(b, grid, smem, st); break;
        case 384: k1_launch<384, 1, 3>(b, grid, smem, st); break;
        default: k1_launch<256, 2, FFSVA_K1_MINBLOCKS>(b, grid, smem, st); break;
      }
    }
    return cudaGetLastError();
  }
  const size_t smem = sdd_smem_bytes(a.max_chunks, a.sdd_w);
  const int threads = sdd_threads(a.max_chunks);
  const unsigned grid = (unsigned)a.n * (unsigned)(a.sdd_h / 2);
  if (a.d100) sdd_kernel<true><<<grid, threads, smem, st>>>(a);
  else sdd_kernel<false><<<grid, threads, smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_reference(const uint8_t* frames, int32_t k, int64_t frame_stride, int32_t W, int32_t H,
                             int64_t pitch, int32_t sdd_w, int32_t sdd_h, uint8_t* out, cudaStream_t st) {
  const int n = 3 * sdd_w * sdd_h;
  reference_kernel<<<(n + 127) / 128, 128, 0, st>>>(frames, k, frame_stride, W, H, pitch, sdd_w, sdd_h, out);
  return cudaGetLastError();
}

cudaError_t launch_prev(const PrevArgs& a, cudaStream_t st) {
  if (a.n_pm <= 0) return cudaSuccess;
  sdd_prev_kernel<<<a.n_pm, kPrevThreads, 0, st>>>(a);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess || a.n_last <= 0) return e;
  ref_update_kernel<<<a.n_last, kPrevThreads, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_fill_nan(float* p, int32_t n, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  fill_nan_kernel<<<(n + 255) / 256, 256, 0, st>>>(p, n);
  return cudaGetLastError();
}

}  // namespace ffsva
