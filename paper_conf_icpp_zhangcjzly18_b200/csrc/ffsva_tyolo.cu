// ffsva_tyolo.cu — K5: the T-YOLO stage on tcgen05 tensor cores.
//
// Method (§3.2.3, §4.2.2): the third filter is Tiny-YOLO-VOC — "9 CONV layers and 6 POOL
// layers" on 416x416 images — shared by all streams; it "divides the input image into a 13*13 grid", "each grid
// cell predicts 5 bounding boxes and confidence scores", a box whose confidence exceeds the threshold (0.2) is one
// target object, and frames with fewer than NumberofObjects targets are filtered out. Readings (DESIGN.md
// Q28-Q32): Q28 resize, x = v/256 (Q29), -inf border of the stride-1 pool (Q30), score = sigmoid(objectness) *
// softmax(classes)[target] without NMS (Q31), bf16 operands / fp32 accumulation / bf16 activations between
// layers (Q32).
//
// B200 mapping — one implicit-GEMM kernel for every layer, activations NHWC bf16 in HBM/L2:
//   * GEMM rows = OUTPUT pixels of the layer (pooled pixels for the pool layers) of the whole batch, 128 per CTA;
//     N = output channels (tile NT <= 256); K = taps x input channels, staged 64 bf16 (128 B) per pipeline step.
//   * Pooling is folded into the MMA like the SNM: for a pool layer the four 2x2 positions are four accumulator
//     chains in four TMEM column groups, so the epilogue max-pools in registers (bias and leaky ReLU commute
//     with max and are applied once after it). The 2x2/1 pool of layer 6 uses the same four chains with the
//     border positions excluded (Q30).
//   * A operands are gathered (im2col on the fly) by 128 producer threads with cp.async zero-fill (padding and
//     K padding are zeros), written straight into the UMMA K-major no-swizzle core-matrix layout; B operands
//     (weights, pre-packed on the host in exactly that layout per (N tile, K step)) arrive by one bulk copy per
//     step. A 2- or 4-stage mbarrier ring overlaps copies with the MMAs, issued by one thread.
//   * The 1x1 head (1024 -> 125) writes its fp32 outputs and counts, per row, the boxes whose score exceeds the
//     threshold into the frame's counter (L171).
#include <algorithm>
#include <cstdlib>

#include "ffsva_internal.h"
#include "ffsva_ptx.h"

namespace ffsva {
namespace {

using namespace ptx;

constexpr int kConvThreads = 320;  // warps 0-3: A gather, 4: TMEM + MMA issue, 5: B copies, 6-9: epilogue
constexpr int kATile = 128 * 128;  // one stage of A for one chain: 128 rows x 64 bf16
constexpr int kMaxAccBufs = 8;     // TMEM accumulator buffers (small N tiles keep several tiles in flight)

// byte offset of (K group g of 8 bf16, row r) in a 128-row K-major no-swizzle tile: core matrices of 8 rows x 16 B,
// K-adjacent core matrices 2048 B apart (LBO), 8-row groups 128 B apart (SBO)
__device__ __forceinline__ uint32_t a_off(int g, int r) {
  return (uint32_t)(g * 2048 + (r >> 3) * 128 + (r & 7) * 16);
}

// Decode output row m of the layer into (frame, oy, ox).
__device__ __forceinline__ void decode_row(const TyConvArgs& a, int m, int& n, int& oy, int& ox) {
  const int hw = a.Ho * a.Wo;
  n = m / hw;
  const int rem = m - n * hw;
  oy = rem / a.Wo;
  ox = rem - oy * a.Wo;
}

// Gather state of one output row for one tile: the address of its 4x4 input window's origin — rows ry0 .. ry0+3,
// columns rx0 .. rx0+3 with (ry0, rx0) = (2oy-1, 2ox-1) for pool layers (the four pool positions' 3x3 taps and the
// 4x4 patch all lie in it) and (oy-1, ox-1) otherwise — and which window rows / columns lie inside the image.
// Every K group then costs a few instructions: validity = three mask bits, address = origin + two constant offsets.
struct RowWin {
  const char* p0;  // window origin (may point outside the image; only dereferenced for in-image pixels)
  uint32_t mask;   // bit 16: row exists; bits 0-3: window rows inside; bits 4-7: window columns inside
};

__device__ __forceinline__ RowWin row_window(const TyConvArgs& a, int m) {
  RowWin w{reinterpret_cast<const char*>(a.in), 0u};
  if (m >= a.M) return w;
  int n, oy, ox;
  decode_row(a, m, n, oy, ox);
  const int sc = a.pool == 1 ? 2 : 1, ry0 = sc * oy - 1, rx0 = sc * ox - 1;
  uint32_t mask = 1u << 16;
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    if ((unsigned)(ry0 + u) < (unsigned)a.H) mask |= 1u << u;
    if ((unsigned)(rx0 + u) < (unsigned)a.W) mask |= 1u << (4 + u);
  }
  w.p0 = reinterpret_cast<const char*>(a.in) + (((int64_t)n * a.H + ry0) * a.W + rx0) * a.Cp * 2;
  w.mask = mask;
  return w;
}

// One piece of a row's K step: window pixel (du, dv) at byte offset off within it.
__device__ __forceinline__ void gather_piece(const TyConvArgs& a, const RowWin& w, int du, int dv, int off,
                                             int64_t rowb, int pixb, uint32_t dst, bool half, bool ok = true) {
  const bool v = ok && ((w.mask >> 16) & (w.mask >> du) & (w.mask >> (4 + dv)) & 1u);
  const void* src = v ? (const void*)(w.p0 + du * rowb + dv * pixb + off) : (const void*)a.in;
  if (half) cp_async8(dst, src, v);
  else cp_async16(dst, src, v);
}

// Patch mode (pool layers with few input channels): the A row of pooled pixel (oy, ox) is its 4x4 input patch
// (the window) x Cp channels, pixel-major; K step j holds 64 of its values. The four pool positions then differ
// only in their weights (the 3x3 kernel placed at offset (a, b) of the patch), so one A tile feeds all four
// accumulator chains.
__device__ __forceinline__ void gather_patch(const TyConvArgs& a, const RowWin& w, int j, int64_t rowb, int pixb,
                                             uint32_t dst, int r) {
  if (a.Cp == 4) {  // all 16 patch pixels in one K step, two 8-byte pixels per 16-byte K group
#pragma unroll
    for (int p = 0; p < 16; ++p) gather_piece(a, w, p >> 2, p & 3, 0, rowb, pixb, dst + a_off(p >> 1, r) + 8 * (p & 1), true);
  } else {  // Cp = 8 * upp channels: 64 / Cp pixels per K step, upp 16-byte units each
    const int ppc = 64 / a.Cp, upp = a.Cp >> 3;
    for (int pl = 0; pl < ppc; ++pl) {
      const int p = j * ppc + pl;
      for (int u = 0; u < upp; ++u)
        gather_piece(a, w, p >> 2, p & 3, 16 * u, rowb, pixb, dst + a_off(pl * upp + u, r), false);
    }
  }
}

// Per-position / plain gather (Cp a multiple of 64): K step j is one tap (dy, dx) and 64 channels; pool position
// (qa, qb) shifts it inside the window.
__device__ __forceinline__ void gather_tap(const TyConvArgs& a, const RowWin& w, int j, int qa, int qb, int64_t rowb,
                                           int pixb, uint32_t dst, int r) {
  int t, c0;
  if (a.ksize == 1) {
    t = 4;
    c0 = j << 6;
  } else {
    const int sh = a.cp_shift - 6;  // K steps per tap = Cp / 64
    t = j >> sh;
    c0 = (j - (t << sh)) << 6;
  }
  const int du = qa + t / 3, dv = qb + t % 3;
  const bool v = (w.mask >> 16) & (w.mask >> du) & (w.mask >> (4 + dv)) & 1u;
  const char* src = v ? w.p0 + du * rowb + dv * pixb + c0 * 2 : reinterpret_cast<const char*>(a.in);
#pragma unroll
  for (int g = 0; g < 8; ++g) cp_async16(dst + a_off(g, r), src + 16 * g, v);
}

// Persistent, warp-specialised: each CTA walks tiles t = blockIdx.x, + gridDim.x, ... A tile = msub x 128 output
// rows x NT channels (msub = 2 shares every weight stage between two 128-row halves: half the L2 weight traffic
// per MAC for the wide 13x13 layers). One K-step ring (S stages) runs continuously across tiles; the TMEM
// accumulators are double buffered when they fit twice, so the epilogue of tile i overlaps tile i + 1's mainloop.
// Stage = a_tiles A tiles (msub x (patch ? 1 : nq)) + b_tiles B tiles (patch ? nq : 1).
// cp.async.wait_group with a runtime count (the immediate must be a constant): at most n groups stay pending
__device__ __forceinline__ void cp_async_wait_n(int n) {
  switch (n) {
    case 0: cp_async_wait<0>(); break;
    case 1: cp_async_wait<1>(); break;
    case 2: cp_async_wait<2>(); break;
    case 3: cp_async_wait<3>(); break;
    case 4: cp_async_wait<4>(); break;
    case 5: cp_async_wait<5>(); break;
    case 6: cp_async_wait<6>(); break;
    default: cp_async_wait<7>(); break;
  }
}

template <int MS, int NQ, bool PATCH>
__global__ void __launch_bounds__(kConvThreads, 1) tyolo_conv_kernel(TyConvArgs a) {
  extern __shared__ __align__(1024) uint8_t sm[];
  const int S = a.stages, nq = NQ, NT = a.NT, KC = a.kchunks, NB = a.acc_bufs;
  const int a_per_sub = PATCH ? 1 : nq;
  const int b_tiles = PATCH ? nq : 1;
  const uint32_t stage_a = (uint32_t)(MS * a_per_sub) * kATile;
  const uint32_t b_tile = (uint32_t)NT * 128, stage_b = (uint32_t)b_tiles * b_tile;
  const int acc_cols = MS * nq * NT;  // per accumulator buffer
  uint8_t* As = sm;
  uint8_t* Bs = sm + (size_t)S * stage_a;
  uint64_t* bars = reinterpret_cast<uint64_t*>(Bs + (size_t)S * stage_b);
  uint32_t* s_tmem = reinterpret_cast<uint32_t*>(bars + 2 * S + 2 * kMaxAccBufs);
  const uint32_t full0 = smem_addr(bars), empty0 = full0 + 8 * S;
  const uint32_t accf0 = full0 + 16 * S, acce0 = accf0 + 8 * kMaxAccBufs;  // acc_full[NB], acc_empty[NB]
  const uint32_t As0 = smem_addr(As), Bs0 = smem_addr(Bs);
  const int tid = threadIdx.x, lane = tid & 31;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);  // warp-uniform (role branches, MMA issue)
  const int rows_per_tile = 128 * MS;
  const int n_tiles = a.Cout_tiles, tiles = ((a.M + rows_per_tile - 1) / rows_per_tile) * n_tiles;

  if (tid == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(full0 + 8 * s, 129);  // 128 gather threads + the weight copy's expect_tx arrival
      mbar_init(empty0 + 8 * s, 1);
    }
    for (int b = 0; b < NB; ++b) {
      mbar_init(accf0 + 8 * b, 1);
      mbar_init(acce0 + 8 * b, 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 4) tmem_alloc(smem_addr(s_tmem), (uint32_t)a.tmem_cols);
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *s_tmem;

  if (warp < 4) {
    // ---------------- A producers: thread = row r of every 128-row half of the tile
    // Up to `lag` (<= S - 1) steps of copies stay in flight per thread; step g is published (cp.async.wait_group,
    // proxy fence, mbarrier arrive) once step g + lag has been issued. Deadlock-free: the wait for slot g % S needs
    // the MMA of step g - S, published after step g - S + lag <= g - 1 was issued. lag = S - 1 leaves the MMA no
    // slack; lag = 1 measured best (profiles/r01/tyolo_ab.md).
    const int r = tid, lag = a.lag < 1 ? 1 : (a.lag > S - 1 ? S - 1 : a.lag);
    int g = 0;  // global K-step counter (continues across tiles)
    const int64_t rowb = (int64_t)a.W * a.Cp * 2;
    const int pixb = a.Cp * 2;
    for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
      RowWin w[MS];
#pragma unroll
      for (int i = 0; i < MS; ++i) w[i] = row_window(a, (t / n_tiles) * rows_per_tile + i * 128 + r);
      for (int j = 0; j < KC; ++j, ++g) {
        const int s = g % S;
        mbar_wait(empty0 + 8 * s, ((g / S) & 1) ^ 1);
#pragma unroll
        for (int i = 0; i < MS; ++i) {
          const uint32_t base = As0 + (uint32_t)s * stage_a + (uint32_t)(i * a_per_sub) * kATile;
          if (PATCH) {
            gather_patch(a, w[i], j, rowb, pixb, base, r);
          } else {
#pragma unroll
            for (int q = 0; q < NQ; ++q)
              gather_tap(a, w[i], j, NQ == 4 ? (q >> 1) : 0, NQ == 4 ? (q & 1) : 0, rowb, pixb,
                         base + (uint32_t)q * kATile, r);
          }
        }
        cp_async_commit();
        if (g >= lag) {  // step g - lag has landed: publish it to the tensor core (async proxy)
          cp_async_wait_n(lag);
          fence_proxy_async();
          mbar_arrive(full0 + 8 * ((g - lag) % S));
        }
      }
    }
    cp_async_wait<0>();
    fence_proxy_async();
    for (int h = g - lag < 0 ? 0 : g - lag; h < g; ++h) mbar_arrive(full0 + 8 * (h % S));
  } else if (warp == 4) {
    // ---------------- MMA issue (the whole warp, one elected lane issues: ffsva_ptx.h mma_bf16)
    // Descriptors are built once; per MMA only their start-address fields advance (byte offset >> 4 added to the
    // low 14 bits, which cannot carry: shared addresses stay below 256 KB), so the issuing warp spends a few
    // instructions per MMA instead of rebuilding two 64-bit descriptors.
    {
      const uint32_t idesc = idesc_bf16(128, NT);
      const uint64_t a_base = umma_desc(As0, 2048, 128), b_base = umma_desc(Bs0, (uint32_t)NT * 16, 128);
      const uint32_t a_tile16 = (uint32_t)kATile >> 4, b_tile16 = b_tile >> 4, b_ks16 = (uint32_t)(2 * NT * 16) >> 4;
      const int ksteps = a.ksteps;
      int g = 0, it = 0;
      for (int t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
        const int b = it % NB;
        mbar_wait(acce0 + 8 * b, ((it / NB) & 1) ^ 1);  // the epilogue has drained this accumulator
        fence_after();
        const uint32_t acc = tmem + (uint32_t)(b * acc_cols);
        for (int j = 0; j < KC; ++j, ++g) {
          const int s = g % S;
          mbar_wait(full0 + 8 * s, (g / S) & 1);
          fence_after();
          const uint64_t a_s = a_base + (((uint32_t)s * stage_a) >> 4), b_s = b_base + (((uint32_t)s * stage_b) >> 4);
#pragma unroll
          for (int i = 0; i < MS; ++i)
#pragma unroll
            for (int q = 0; q < NQ; ++q) {
              const uint64_t ad = a_s + (uint64_t)((i * (PATCH ? 1 : NQ) + (PATCH ? 0 : q)) * a_tile16);
              const uint64_t bd = b_s + (uint64_t)((PATCH ? q : 0) * b_tile16);
              const uint32_t d = acc + (uint32_t)((i * NQ + q) * NT);
#pragma unroll
              for (int ks = 0; ks < 4; ++ks)
                if (ks < ksteps)
                  mma_bf16(d, ad + (uint64_t)(ks * 256), bd + (uint64_t)(ks * b_ks16), idesc, (j > 0 || ks > 0) ? 1u : 0u);
            }
          mma_commit(empty0 + 8 * s);
        }
        mma_commit(accf0 + 8 * b);
      }
    }
  } else if (warp == 5) {
    // ---------------- weight copies (one thread): all B tiles of a step are one contiguous block
    if (lane == 0) {
      int g = 0;
      for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
        const uint8_t* wsrc = a.wpk + (int64_t)(t % n_tiles) * KC * stage_b;
        for (int j = 0; j < KC; ++j, ++g) {
          const int s = g % S;
          mbar_wait(empty0 + 8 * s, ((g / S) & 1) ^ 1);
          mbar_expect_tx(full0 + 8 * s, stage_b);
          bulk_g2s(Bs0 + (uint32_t)s * stage_b, wsrc + (int64_t)j * stage_b, stage_b, full0 + 8 * s);
        }
      }
    }
  } else {
    // ---------------- epilogue (warps 6-9): TMEM lane quadrant = warp % 4, row = 32 * quadrant + lane
    const int qd = warp & 3, r = 32 * qd + lane;
    int it = 0;
    for (int t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
      const int b = it % NB, nt = t % n_tiles;
      mbar_wait(accf0 + 8 * b, (it / NB) & 1);
      fence_after();
      const int cbase = nt * NT;
      for (int i = 0; i < MS; ++i) {
        const int m = (t / n_tiles) * rows_per_tile + i * 128 + r;
        const bool rv = m < a.M;
        int n = 0, oy = 0, ox = 0;
        if (rv) decode_row(a, m, n, oy, ox);
        const uint32_t trow = tmem + ((uint32_t)(32 * qd) << 16) + (uint32_t)(b * acc_cols + i * nq * NT);
        for (int c0 = 0; c0 < NT; c0 += 16) {
          float v[16];
          if (NQ == 4) {  // the four pool chains: all four loads in flight, one wait
            uint32_t r0[16], r1[16], r2[16], r3[16];
            tmem_ld16(trow + (uint32_t)c0, r0);
            tmem_ld16(trow + (uint32_t)(NT + c0), r1);
            tmem_ld16(trow + (uint32_t)(2 * NT + c0), r2);
            tmem_ld16(trow + (uint32_t)(3 * NT + c0), r3);
            tmem_wait_ld2(r0, r1);
            reg_fence2(r2, r3);
#pragma unroll
            for (int k = 0; k < 16; ++k)
              v[k] = fmaxf(fmaxf(__uint_as_float(r0[k]), __uint_as_float(r1[k])),
                           fmaxf(__uint_as_float(r2[k]), __uint_as_float(r3[k])));
          } else {
            uint32_t rr[16];
            tmem_ld16(trow + (uint32_t)c0, rr);
            tmem_wait_ld(rr);
#pragma unroll
            for (int k = 0; k < 16; ++k) v[k] = __uint_as_float(rr[k]);
          }
          if (!rv) continue;
          const float* bias = a.bias + cbase + c0;
          if (a.head) {
            float* o = a.out_f32 + (int64_t)m * a.Cout + cbase + c0;
#pragma unroll
            for (int k = 0; k < 16; k += 4)
              *reinterpret_cast<float4*>(o + k) =
                  make_float4(v[k] + bias[k], v[k + 1] + bias[k + 1], v[k + 2] + bias[k + 2], v[k + 3] + bias[k + 3]);
          } else {
            uint32_t w[8];
#pragma unroll
            for (int k = 0; k < 8; ++k) {
              float x0 = v[2 * k] + bias[2 * k], x1 = v[2 * k + 1] + bias[2 * k + 1];
              if (a.leaky) {
                x0 = x0 < 0.f ? 0.1f * x0 : x0;
                x1 = x1 < 0.f ? 0.1f * x1 : x1;
              }
              w[k] = pack_bf16(x0, x1);
            }
            uint4* o = reinterpret_cast<uint4*>(a.out + (int64_t)m * a.Cout + cbase + c0);
            o[0] = make_uint4(w[0], w[1], w[2], w[3]);
            o[1] = make_uint4(w[4], w[5], w[6], w[7]);
          }
        }
        if (a.head && rv) {  // L171: count this cell's boxes whose score exceeds the threshold (Q31)
          const float* o = a.out_f32 + (int64_t)m * a.Cout;
          int cnt = 0;
          for (int bx = 0; bx < 5; ++bx) {
            const float* p = o + 25 * bx;
            float mx = p[5];
            for (int k = 1; k < 20; ++k) mx = fmaxf(mx, p[5 + k]);
            float z = 0.f;
            for (int k = 0; k < 20; ++k) z += __expf(p[5 + k] - mx);
            const float score = __expf(p[5 + a.frames[n].target] - mx) / z / (1.f + __expf(-p[4]));
            cnt += score > a.thresh ? 1 : 0;
          }
          if (cnt) atomicAdd(a.counts + n, cnt);
        }
      }
      fence_before();
      mbar_arrive(acce0 + 8 * b);  // this accumulator may be overwritten
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 4) {
    fence_after();
    tmem_dealloc(tmem, (uint32_t)a.tmem_cols);
  }
}

// 2x2 max-pool with stride 1 and a -inf right/bottom border (Q30) on bf16 NHWC, 8 channels per thread. Applied
// after the layer-6 convolution (bf16 rounding is monotone, so pooling the rounded values equals rounding the
// pooled ones).
// planar_stride > 0: write the 13x13 slab layout instead (plane c/8 at planar_stride entries, entry = frame * 225 +
// (y + 1) * 15 + x + 1 of the zero-bordered 15x15 grid; see tyolo_slab_kernel)
__global__ void tyolo_pool_s1_kernel(const __nv_bfloat16* in, __nv_bfloat16* out, int32_t n, int32_t H, int32_t C,
                                     int64_t planar_stride) {
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int c8 = C >> 3;
  const int64_t total = (int64_t)n * H * H * c8;
  if (idx >= total) return;
  const int cg = (int)(idx % c8);
  const int64_t p = idx / c8;
  const int x = (int)(p % H), y = (int)((p / H) % H);
  const int64_t base = p - (int64_t)y * H - x;  // frame's first pixel
  __nv_bfloat162 mx[4];
  const uint4 v0 = *reinterpret_cast<const uint4*>(in + p * C + 8 * cg);
  mx[0] = *reinterpret_cast<const __nv_bfloat162*>(&v0.x);
  mx[1] = *reinterpret_cast<const __nv_bfloat162*>(&v0.y);
  mx[2] = *reinterpret_cast<const __nv_bfloat162*>(&v0.z);
  mx[3] = *reinterpret_cast<const __nv_bfloat162*>(&v0.w);
  for (int d = 1; d < 4; ++d) {
    const int yy = y + (d >> 1), xx = x + (d & 1);
    if (yy >= H || xx >= H) continue;
    const uint4 v = *reinterpret_cast<const uint4*>(in + (base + (int64_t)yy * H + xx) * C + 8 * cg);
    mx[0] = __hmax2(mx[0], *reinterpret_cast<const __nv_bfloat162*>(&v.x));
    mx[1] = __hmax2(mx[1], *reinterpret_cast<const __nv_bfloat162*>(&v.y));
    mx[2] = __hmax2(mx[2], *reinterpret_cast<const __nv_bfloat162*>(&v.z));
    mx[3] = __hmax2(mx[3], *reinterpret_cast<const __nv_bfloat162*>(&v.w));
  }
  uint4 o;
  o.x = *reinterpret_cast<uint32_t*>(&mx[0]);
  o.y = *reinterpret_cast<uint32_t*>(&mx[1]);
  o.z = *reinterpret_cast<uint32_t*>(&mx[2]);
  o.w = *reinterpret_cast<uint32_t*>(&mx[3]);
  if (planar_stride > 0) {
    const int64_t f = p / ((int64_t)H * H);
    *reinterpret_cast<uint4*>(out + ((int64_t)cg * planar_stride + f * 225 + (y + 1) * 15 + x + 1) * 8) = o;
  } else {
    *reinterpret_cast<uint4*>(out + p * C + 8 * cg) = o;
  }
}

// Q28 resize of each raw RGB8 frame to 416x416, x = v / 256 (Q29) as bf16 NHWC with a zero 4th channel. One CTA per
// (frame, group of R output rows): thread 0 bulk-copies the group's source rows (one contiguous span of the frame,
// L2 evict-first) into shared memory against an mbarrier — R is sized on the host so several CTAs per SM keep tens
// of KB each in flight — then each thread box-sums output pixels from shared memory. Frames whose rows are not
// 16-byte aligned (or whose span exceeds the stage) read their bytes straight from global memory.
constexpr int kResizeThreads = 256;
constexpr int kResizeMaxD = 1024;  // output size bound of the column-bound table

// Q28 cell bounds: [floor(i*S/D), max(floor((i+1)*S/D), floor(i*S/D) + 1))
__device__ __forceinline__ int rs_lo(int i, int S, int D) { return (int)(((int64_t)i * S) / D); }
__device__ __forceinline__ int rs_hi(int i, int S, int D) {
  const int lo = rs_lo(i, S, D), hi = (int)(((int64_t)(i + 1) * S) / D);
  return hi > lo ? hi : lo + 1;
}

// floor(a / n) for a < 2^31 with a quotient < 2^16: float estimate + one remainder correction (box means <= 255)
__device__ __forceinline__ uint32_t rs_div(uint32_t a, uint32_t n) {
  uint32_t q = __float2uint_rz(__uint2float_rn(a) * __frcp_rn(__uint2float_rn(n)));
  const int r = (int)(a - q * n);
  if (r < 0) --q;
  else if (r >= (int)n) ++q;
  return q;
}

__global__ void __launch_bounds__(kResizeThreads) tyolo_resize_kernel(const TyFrame* frames, int32_t D, int32_t R,
                                                                     int32_t stage_bytes, __nv_bfloat16* out) {
  extern __shared__ __align__(16) uint8_t rows_sm[];
  __shared__ __align__(8) uint64_t bar;
  __shared__ int2 xcell[kResizeMaxD];  // Q28 column bounds of every output column (32-bit: i * W < 2^31)
  const int f = blockIdx.y;
  const int oy0 = blockIdx.x * R, oy1 = min(oy0 + R, D);
  const TyFrame fr = frames[f];
  const int ylo = rs_lo(oy0, fr.H, D), yhi = rs_hi(oy1 - 1, fr.H, D);
  const int rb = 3 * fr.W, rb16 = (rb + 15) & ~15;
  const bool staged = ((fr.pitch & 15) == 0) && (((uintptr_t)fr.pixels & 15) == 0) && (yhi - ylo) * rb16 <= stage_bytes;
  const uint32_t b = smem_addr(&bar);
  if (staged && threadIdx.x == 0) {
    mbar_init(b, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const uint32_t bytes = (uint32_t)((yhi - ylo) * rb16);
    mbar_expect_tx(b, bytes);
    const uint8_t* src = fr.pixels + (int64_t)ylo * fr.pitch;
    if (fr.pitch == rb16) {
      asm volatile(
          "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
          ::"r"(smem_addr(rows_sm)), "l"(src), "r"(bytes), "r"(b), "l"(pol) : "memory");
    } else {
      for (int y = 0; y < yhi - ylo; ++y)
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
            ::"r"(smem_addr(rows_sm + y * rb16)), "l"(src + (int64_t)y * fr.pitch), "r"((uint32_t)rb16), "r"(b),
            "l"(pol) : "memory");
    }
  }
  for (int i = threadIdx.x; i < D; i += kResizeThreads) {
    const int lo = (int)(((uint32_t)i * (uint32_t)fr.W) / (uint32_t)D);
    const int hi = (int)(((uint32_t)(i + 1) * (uint32_t)fr.W) / (uint32_t)D);
    xcell[i] = make_int2(lo, hi > lo ? hi : lo + 1);
  }
  __syncthreads();  // barrier initialised, column bounds ready
  if (staged) mbar_wait(b, 0);
  const float inv = 1.f / 256.f;
  for (int oy = oy0; oy < oy1; ++oy) {
    const int y0 = (int)(((uint32_t)oy * (uint32_t)fr.H) / (uint32_t)D);
    const int yh = (int)(((uint32_t)(oy + 1) * (uint32_t)fr.H) / (uint32_t)D);
    const int y1 = yh > y0 ? yh : y0 + 1;
    // zero-bordered output [N][D+2][D+2][4] (layer 1 reads it by bulk copies; the border stays zero)
    __nv_bfloat16* orow = out + (((int64_t)f * (D + 2) + oy + 1) * (D + 2) + 1) * 4;
    for (int ox = threadIdx.x; ox < D; ox += kResizeThreads) {
      const int2 xc = xcell[ox];
      uint32_t s0 = 0, s1 = 0, s2 = 0;
      for (int y = y0; y < y1; ++y) {
        const uint8_t* row = staged ? rows_sm + (y - ylo) * rb16 : fr.pixels + (int64_t)y * fr.pitch;
        for (int x = xc.x; x < xc.y; ++x) {
          s0 += row[3 * x];
          s1 += row[3 * x + 1];
          s2 += row[3 * x + 2];
        }
      }
      const uint32_t nn = (uint32_t)((y1 - y0) * (xc.y - xc.x));
      uint2 w;
      w.x = pack_bf16((float)rs_div(s0 + nn / 2, nn) * inv, (float)rs_div(s1 + nn / 2, nn) * inv);
      w.y = pack_bf16((float)rs_div(s2 + nn / 2, nn) * inv, 0.f);
      *reinterpret_cast<uint2*>(orow + ox * 4) = w;
    }
  }
}

// ---------------------------------------------------------------- layer 1 (3 -> 16, 3x3, 2x2/2 pool) by patch views
// The first layer has 3 input channels: the generic kernel's per-row gathers (16 eight-byte pieces per pooled pixel)
// bound it. Here its input is the zero-bordered resize output [N][418][418][4] bf16 (8 bytes per pixel), so a tile =
// 128 consecutive pooled pixels of one pooled row needs four contiguous 2,064-byte input row segments (padded rows
// 2oy .. 2oy+3 from column 2ox0), one bulk copy each, and NO im2col: the A row of pooled pixel ox is its 4x4 patch
// x 4 channel slots, and patch row dy of consecutive pooled pixels is a constant-stride view of segment dy (rows 16 B
// apart: two pixels per pooled step; K-halves 16 B apart; 8-row groups 128 B apart). One A operand feeds N = 64 =
// 4 pool positions x 16 channels with per-position zero-padded 3x3 weights: 4 MMAs (M128 N64 K16) per tile.
// Persistent, warp-specialised: warp 4 lane 0 copies segments through an S-stage ring, warp 5 issues the MMAs into
// four TMEM accumulator buffers, warps 0-3 max-pool / bias / leaky / bf16 and store 32 B per pooled pixel.
constexpr int kL1Pad = 418, kL1Out = 208;
// layer 2's planar, zero-bordered input (= layer 1's output): [N][210 rows][2 column parities][2 channel groups]
// [105 entries][16 B]
constexpr int kL2Pad = 210, kL2Out = 104, kL2Entries = 105;
constexpr int kL2Plane = kL2Entries * 16;       // 1680 B
constexpr int kL2Row = 4 * kL2Plane;            // 6720 B
constexpr int kL1Seg = 258 * 8;                 // 2064 B: input columns 2ox0 .. 2ox0 + 257 of one padded row
constexpr int kL1Stage = 4 * kL1Seg;            // 8256 B
constexpr int kL1Stages = 8;
constexpr int kL1Bufs = 4;                      // TMEM accumulators of 64 columns
constexpr int kL1Threads = 192;
constexpr int kL1WBytes = 4 * 2 * 64 * 16;      // 8192 B of packed weights
constexpr int kL1Smem = kL1WBytes + kL1Stages * kL1Stage + 8 * (2 * kL1Stages + 2 * kL1Bufs + 1) + 16;

__global__ void __launch_bounds__(kL1Threads, 2) tyolo_l1_kernel(TyL1Args a) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* Ws = sm;
  uint8_t* Ss = sm + kL1WBytes;
  uint64_t* bars = reinterpret_cast<uint64_t*>(Ss + kL1Stages * kL1Stage);
  uint32_t* s_tmem = reinterpret_cast<uint32_t*>(bars + 2 * kL1Stages + 2 * kL1Bufs + 1);
  const uint32_t full0 = smem_addr(bars), empty0 = full0 + 8 * kL1Stages;
  const uint32_t accf0 = empty0 + 8 * kL1Stages, acce0 = accf0 + 8 * kL1Bufs, wbar = acce0 + 8 * kL1Bufs;
  const int tid = threadIdx.x, lane = tid & 31;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);
  const int tiles = a.N * kL1Out * 2;  // (frame, pooled row, half of the row)

  if (tid == 0) {
    for (int s = 0; s < kL1Stages; ++s) {
      mbar_init(full0 + 8 * s, 1);
      mbar_init(empty0 + 8 * s, 1);
    }
    for (int b = 0; b < kL1Bufs; ++b) {
      mbar_init(accf0 + 8 * b, 1);
      mbar_init(acce0 + 8 * b, 128);
    }
    mbar_init(wbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    mbar_expect_tx(wbar, kL1WBytes);
    bulk_g2s(smem_addr(Ws), a.w, kL1WBytes, wbar);
  }
  if (warp == 5) tmem_alloc(smem_addr(s_tmem), kL1Bufs * 64);
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *s_tmem;

  if (warp == 4) {
    // ---------------- producer: four row segments per tile
    if (lane == 0) {
      int g = 0;
      for (int t = blockIdx.x; t < tiles; t += gridDim.x, ++g) {
        const int n = t / (2 * kL1Out), rem = t - n * 2 * kL1Out, oy = rem >> 1, half = rem & 1;
        const int s = g % kL1Stages;
        const uint32_t bytes = half ? (uint32_t)(kL1Pad - 2 * 128) * 8 : (uint32_t)kL1Seg;
        mbar_wait(empty0 + 8 * s, ((g / kL1Stages) & 1) ^ 1);
        mbar_expect_tx(full0 + 8 * s, 4 * bytes);
        const char* src = reinterpret_cast<const char*>(a.in) + (((int64_t)n * kL1Pad + 2 * oy) * kL1Pad + 256 * half) * 8;
        for (int dy = 0; dy < 4; ++dy)
          bulk_g2s(smem_addr(Ss + s * kL1Stage + dy * kL1Seg), src + (int64_t)dy * kL1Pad * 8, bytes, full0 + 8 * s);
      }
    }
  } else if (warp == 5) {
    // ---------------- MMA issue (whole warp, one elected lane)
    mbar_wait(wbar, 0);
    const uint32_t idesc = idesc_bf16(128, 64);
    const uint64_t a_base = umma_desc(smem_addr(Ss), 16, 128), b_base = umma_desc(smem_addr(Ws), 64 * 16, 128);
    int g = 0;
    for (int t = blockIdx.x; t < tiles; t += gridDim.x, ++g) {
      const int s = g % kL1Stages, b = g % kL1Bufs;
      mbar_wait(acce0 + 8 * b, ((g / kL1Bufs) & 1) ^ 1);
      mbar_wait(full0 + 8 * s, (g / kL1Stages) & 1);
      fence_after();
#pragma unroll
      for (int dy = 0; dy < 4; ++dy)
        mma_bf16(tmem + (uint32_t)(b * 64), a_base + (uint64_t)((s * kL1Stage + dy * kL1Seg) >> 4),
                 b_base + (uint64_t)((dy * 2 * 64 * 16) >> 4), idesc, dy > 0 ? 1u : 0u);
      mma_commit(empty0 + 8 * s);
      mma_commit(accf0 + 8 * b);
    }
  } else {
    // ---------------- epilogue (warps 0-3): TMEM lane = pooled pixel of the tile
    const int qd = warp & 3, r = 32 * qd + lane;
    float bias[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) bias[k] = __ldg(a.bias + k);
    int g = 0;
    for (int t = blockIdx.x; t < tiles; t += gridDim.x, ++g) {
      const int n = t / (2 * kL1Out), rem = t - n * 2 * kL1Out, oy = rem >> 1, half = rem & 1;
      const int b = g % kL1Bufs;
      mbar_wait(accf0 + 8 * b, (g / kL1Bufs) & 1);
      fence_after();
      uint32_t r0[16], r1[16], r2[16], r3[16];
      const uint32_t trow = tmem + ((uint32_t)(32 * qd) << 16) + (uint32_t)(b * 64);
      tmem_ld16(trow, r0);
      tmem_ld16(trow + 16, r1);
      tmem_ld16(trow + 32, r2);
      tmem_ld16(trow + 48, r3);
      tmem_wait_ld2(r0, r1);
      reg_fence2(r2, r3);
      fence_before();
      mbar_arrive(acce0 + 8 * b);  // the accumulator is in registers: the next tile may overwrite it
      const int ox = 128 * half + r;
      if (ox < kL1Out) {
        uint32_t w[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          float x0 = fmaxf(fmaxf(__uint_as_float(r0[2 * k]), __uint_as_float(r1[2 * k])),
                           fmaxf(__uint_as_float(r2[2 * k]), __uint_as_float(r3[2 * k]))) + bias[2 * k];
          float x1 = fmaxf(fmaxf(__uint_as_float(r0[2 * k + 1]), __uint_as_float(r1[2 * k + 1])),
                           fmaxf(__uint_as_float(r2[2 * k + 1]), __uint_as_float(r3[2 * k + 1]))) + bias[2 * k + 1];
          x0 = x0 < 0.f ? 0.1f * x0 : x0;
          x1 = x1 < 0.f ? 0.1f * x1 : x1;
          w[k] = pack_bf16(x0, x1);
        }
        // layer 2's planar input: padded pixel (Y, X) = (oy + 1, ox + 1), channel group g at plane (X & 1, g)
        const int X = ox + 1;
        uint8_t* o = reinterpret_cast<uint8_t*>(a.out) + ((int64_t)n * kL2Pad + oy + 1) * kL2Row +
                     (X & 1) * 2 * kL2Plane + (X >> 1) * 16;
        *reinterpret_cast<uint4*>(o) = make_uint4(w[0], w[1], w[2], w[3]);
        *reinterpret_cast<uint4*>(o + kL2Plane) = make_uint4(w[4], w[5], w[6], w[7]);
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 5) {
    fence_after();
    tmem_dealloc(tmem, kL1Bufs * 64);
  }
}

// ---------------------------------------------------------------- layer 2 (16 -> 32, 3x3, 2x2/2 pool) by patch views
// Layer 1 writes its output zero-bordered and planar: padded row Y holds four planes (pixel-column parity p, channel
// group g of 8) of 105 sixteen-byte entries (entry e = padded column 2e + p), so a padded row is one contiguous
// 6,720-byte segment and, for patch column u, consecutive pooled pixels (columns 2ox + u) are consecutive entries of
// plane (u & 1, g): a constant-stride view again (rows 16 B apart, the two channel groups one plane apart, 8-row
// groups 128 B apart). A tile = one pooled row (104 pixels in 128 MMA rows), four segment copies; per patch row dy
// and column u one MMA of K16 (16 channels) and N = 128 = 4 pool positions x 32 channels: 16 MMAs per tile.
constexpr int kL2Stages = 5;
constexpr int kL2Bufs = 4;                      // TMEM accumulators of 128 columns
constexpr int kL2Threads = 192;
constexpr int kL2WBytes = 16 * 2 * 128 * 16;    // 65,536 B: [dy][u][channel group][n][8]
constexpr int kL2Stage = 4 * kL2Row;            // 26,880 B
constexpr int kL2Smem = kL2WBytes + kL2Stages * kL2Stage + 512 + 8 * (2 * kL2Stages + 2 * kL2Bufs + 1) + 16;

__global__ void __launch_bounds__(kL2Threads, 1) tyolo_l2_kernel(TyL1Args a) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* Ws = sm;
  uint8_t* Ss = sm + kL2WBytes;
  uint64_t* bars = reinterpret_cast<uint64_t*>(Ss + kL2Stages * kL2Stage + 512);  // + tail read by junk rows
  uint32_t* s_tmem = reinterpret_cast<uint32_t*>(bars + 2 * kL2Stages + 2 * kL2Bufs + 1);
  const uint32_t full0 = smem_addr(bars), empty0 = full0 + 8 * kL2Stages;
  const uint32_t accf0 = empty0 + 8 * kL2Stages, acce0 = accf0 + 8 * kL2Bufs, wbar = acce0 + 8 * kL2Bufs;
  const int tid = threadIdx.x, lane = tid & 31;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);
  const int tiles = a.N * kL2Out;  // (frame, pooled row)

  if (tid == 0) {
    for (int s = 0; s < kL2Stages; ++s) {
      mbar_init(full0 + 8 * s, 1);
      mbar_init(empty0 + 8 * s, 1);
    }
    for (int b = 0; b < kL2Bufs; ++b) {
      mbar_init(accf0 + 8 * b, 1);
      mbar_init(acce0 + 8 * b, 128);
    }
    mbar_init(wbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    mbar_expect_tx(wbar, kL2WBytes);
    bulk_g2s(smem_addr(Ws), a.w, kL2WBytes, wbar);
  }
  if (warp == 5) tmem_alloc(smem_addr(s_tmem), kL2Bufs * 128);
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *s_tmem;

  if (warp == 4) {
    if (lane == 0) {
      int g = 0;
      for (int t = blockIdx.x; t < tiles; t += gridDim.x, ++g) {
        const int n = t / kL2Out, oy = t - n * kL2Out;
        const int s = g % kL2Stages;
        mbar_wait(empty0 + 8 * s, ((g / kL2Stages) & 1) ^ 1);
        mbar_expect_tx(full0 + 8 * s, kL2Stage);
        // padded rows 2oy .. 2oy + 3 are contiguous: one copy of four segments
        bulk_g2s(smem_addr(Ss + s * kL2Stage),
                 reinterpret_cast<const char*>(a.in) + ((int64_t)n * kL2Pad + 2 * oy) * kL2Row, kL2Stage,
                 full0 + 8 * s);
      }
    }
  } else if (warp == 5) {
    mbar_wait(wbar, 0);
    const uint32_t idesc = idesc_bf16(128, 128);
    const uint64_t a_base = umma_desc(smem_addr(Ss), kL2Plane, 128), b_base = umma_desc(smem_addr(Ws), 128 * 16, 128);
    int g = 0;
    for (int t = blockIdx.x; t < tiles; t += gridDim.x, ++g) {
      const int s = g % kL2Stages, b = g % kL2Bufs;
      mbar_wait(acce0 + 8 * b, ((g / kL2Bufs) & 1) ^ 1);
      mbar_wait(full0 + 8 * s, (g / kL2Stages) & 1);
      fence_after();
#pragma unroll
      for (int dy = 0; dy < 4; ++dy)
#pragma unroll
        for (int u = 0; u < 4; ++u)
          mma_bf16(tmem + (uint32_t)(b * 128),
                   a_base + (uint64_t)((s * kL2Stage + dy * kL2Row + (u & 1) * 2 * kL2Plane + (u >> 1) * 16) >> 4),
                   b_base + (uint64_t)(((dy * 4 + u) * 2 * 128 * 16) >> 4), idesc, (dy | u) ? 1u : 0u);
      mma_commit(empty0 + 8 * s);
      mma_commit(accf0 + 8 * b);
    }
  } else {
    const int qd = warp & 3, r = 32 * qd + lane;
    int g = 0;
    for (int t = blockIdx.x; t < tiles; t += gridDim.x, ++g) {
      const int n = t / kL2Out, oy = t - n * kL2Out;
      const int b = g % kL2Bufs;
      mbar_wait(accf0 + 8 * b, (g / kL2Bufs) & 1);
      fence_after();
      const uint32_t trow = tmem + ((uint32_t)(32 * qd) << 16) + (uint32_t)(b * 128);
      uint32_t w[16];
#pragma unroll
      for (int c0 = 0; c0 < 32; c0 += 16) {
        uint32_t r0[16], r1[16], r2[16], r3[16];
        tmem_ld16(trow + (uint32_t)c0, r0);
        tmem_ld16(trow + (uint32_t)(32 + c0), r1);
        tmem_ld16(trow + (uint32_t)(64 + c0), r2);
        tmem_ld16(trow + (uint32_t)(96 + c0), r3);
        tmem_wait_ld2(r0, r1);
        reg_fence2(r2, r3);
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          float x0 = fmaxf(fmaxf(__uint_as_float(r0[2 * k]), __uint_as_float(r1[2 * k])),
                           fmaxf(__uint_as_float(r2[2 * k]), __uint_as_float(r3[2 * k]))) + __ldg(a.bias + c0 + 2 * k);
          float x1 = fmaxf(fmaxf(__uint_as_float(r0[2 * k + 1]), __uint_as_float(r1[2 * k + 1])),
                           fmaxf(__uint_as_float(r2[2 * k + 1]), __uint_as_float(r3[2 * k + 1]))) +
                     __ldg(a.bias + c0 + 2 * k + 1);
          x0 = x0 < 0.f ? 0.1f * x0 : x0;
          x1 = x1 < 0.f ? 0.1f * x1 : x1;
          w[c0 / 2 + k] = pack_bf16(x0, x1);
        }
      }
      fence_before();
      mbar_arrive(acce0 + 8 * b);
      if (r < kL2Out) {
        if (a.out_plane > 0) {  // layer 3's parity-slab input (see tyolo_pslab_kernel): 32 channels, grid 53 x 53
          const int Y = oy + 1, X = r + 1;
          const int64_t e = (int64_t)n * 53 * 53 + (Y >> 1) * 53 + (X >> 1);
          const int par = (Y & 1) * 2 + (X & 1);
#pragma unroll
          for (int cg = 0; cg < 4; ++cg)
            *reinterpret_cast<uint4*>(a.out + (((int64_t)cg * 4 + par) * a.out_plane + e) * 8) =
                make_uint4(w[4 * cg], w[4 * cg + 1], w[4 * cg + 2], w[4 * cg + 3]);
        } else {
          uint4* o = reinterpret_cast<uint4*>(a.out + (((int64_t)n * kL2Out + oy) * kL2Out + r) * 32);
          o[0] = make_uint4(w[0], w[1], w[2], w[3]);
          o[1] = make_uint4(w[4], w[5], w[6], w[7]);
          o[2] = make_uint4(w[8], w[9], w[10], w[11]);
          o[3] = make_uint4(w[12], w[13], w[14], w[15]);
        }
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 5) {
    fence_after();
    tmem_dealloc(tmem, kL2Bufs * 128);
  }
}

// ---------------------------------------------------------------- 13x13 layers (3x3, no pool) by slab views
// Input: zero-bordered "slab" layout: for every 8-channel group a plane of 16-byte entries, entry p = frame * 225 +
// Y * 15 + X over the 15x15 padded grid (frames stacked). Output rows of the GEMM are the padded-grid entries p
// themselves (rows with y or x >= 13 are computed and discarded: 169 of 225 useful), so tap (dy, dx) of consecutive
// rows is the plane read at p + dy*15 + dx: a constant-stride UMMA view (rows 16 B apart, channel groups one plane
// apart, 8-row groups 128 B apart). A tile job = 2 x 128 rows x 128 output channels (two TMEM accumulator buffers); per 64-channel group one slab
// of 160 entries x 8 planes per half is bulk-copied (16 copies) and feeds all nine taps, so the A operand costs
// 40 KB per 9 K steps instead of a 32 KB im2col gather per step; B (the pre-packed weights of the generic kernel's
// layout with NT = 128, K step = tap * (Cin/64) + group) streams through a 6-stage ring. Warp 4 lane 0 copies, warp 5 issues MMAs,
// warps 0-3 drain the accumulators (bias, leaky, bf16) into the next slab layout or NHWC.
constexpr int kSlabEntries = 160;               // 128 rows + the largest tap offset (2 * 15 + 2) rounded up
constexpr int kSlabPlaneBytes = kSlabEntries * 16;  // 2560
constexpr int kSlabHalf = 8 * kSlabPlaneBytes;  // 20,480 B: one half's 64-channel slab
constexpr int kSlabA = 2 * kSlabHalf;           // both halves
constexpr int kSlabAStages = 2, kSlabBStages = 6;
constexpr int kSlabNT = 128;                    // N tile: two accumulator buffers of 2 x 128 columns fit in TMEM
constexpr int kSlabBStage = 64 * kSlabNT * 2;   // 16 KB: one K step of weights for a 128-wide N tile
constexpr int kSlabThreads = 192;
constexpr int kSlabSmem = kSlabAStages * kSlabA + kSlabBStages * kSlabBStage +
                          8 * (2 * kSlabAStages + 2 * kSlabBStages + 4) + 16;

__global__ void __launch_bounds__(kSlabThreads, 1) tyolo_slab_kernel(TySlabArgs a) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* As = sm;
  uint8_t* Bs = sm + kSlabAStages * kSlabA;
  uint64_t* bars = reinterpret_cast<uint64_t*>(Bs + kSlabBStages * kSlabBStage);
  uint32_t* s_tmem = reinterpret_cast<uint32_t*>(bars + 2 * kSlabAStages + 2 * kSlabBStages + 4);
  const uint32_t fullA0 = smem_addr(bars), emptyA0 = fullA0 + 8 * kSlabAStages;
  const uint32_t fullB0 = emptyA0 + 8 * kSlabAStages, emptyB0 = fullB0 + 8 * kSlabBStages;
  const uint32_t accf0 = emptyB0 + 8 * kSlabBStages, acce0 = accf0 + 16;  // two accumulator buffers
  const int tid = threadIdx.x, lane = tid & 31;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);
  const int G = a.Cin >> 6;                       // 64-channel groups
  const int n_nt = a.Cout / kSlabNT;
  const int m_tiles = (a.N * 225 + 255) >> 8;
  const int jobs = m_tiles * n_nt;

  if (tid == 0) {
    for (int s = 0; s < kSlabAStages; ++s) {
      mbar_init(fullA0 + 8 * s, 1);
      mbar_init(emptyA0 + 8 * s, 1);
    }
    for (int s = 0; s < kSlabBStages; ++s) {
      mbar_init(fullB0 + 8 * s, 1);
      mbar_init(emptyB0 + 8 * s, 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(accf0 + 8 * b, 1);
      mbar_init(acce0 + 8 * b, 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 5) tmem_alloc(smem_addr(s_tmem), 512);
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *s_tmem;

  if (warp == 4) {
    // ---------------- producer: per job, G slabs (16 copies each) interleaved with 9 * G weight stages
    if (lane == 0) {
      int ga = 0, gb = 0;
      for (int j = blockIdx.x; j < jobs; j += gridDim.x) {
        const int mt = j / n_nt, nt = j - mt * n_nt;
        const int64_t p0 = (int64_t)mt * 256;
        for (int g = 0; g < G; ++g, ++ga) {
          const int sa = ga % kSlabAStages;
          mbar_wait(emptyA0 + 8 * sa, ((ga / kSlabAStages) & 1) ^ 1);
          mbar_expect_tx(fullA0 + 8 * sa, kSlabA);
          for (int h = 0; h < 2; ++h)
            for (int pl = 0; pl < 8; ++pl)
              bulk_g2s(smem_addr(As + sa * kSlabA + h * kSlabHalf + pl * kSlabPlaneBytes),
                       reinterpret_cast<const char*>(a.in) + ((int64_t)(8 * g + pl) * a.plane + p0 + 128 * h) * 16,
                       kSlabPlaneBytes, fullA0 + 8 * sa);
          for (int t = 0; t < 9; ++t, ++gb) {
            const int sb = gb % kSlabBStages;
            mbar_wait(emptyB0 + 8 * sb, ((gb / kSlabBStages) & 1) ^ 1);
            mbar_expect_tx(fullB0 + 8 * sb, kSlabBStage);
            bulk_g2s(smem_addr(Bs + sb * kSlabBStage),
                     a.wpk + ((int64_t)nt * 9 * G + t * G + g) * kSlabBStage, kSlabBStage, fullB0 + 8 * sb);
          }
        }
      }
    }
  } else if (warp == 5) {
    // ---------------- MMA issue
    const uint32_t idesc = idesc_bf16(128, kSlabNT);
    const uint64_t a_base = umma_desc(smem_addr(As), kSlabPlaneBytes, 128);
    const uint64_t b_base = umma_desc(smem_addr(Bs), kSlabNT * 16, 128);
    int ga = 0, gb = 0, it = 0;
    for (int j = blockIdx.x; j < jobs; j += gridDim.x, ++it) {
      const int ab = it & 1;
      mbar_wait(acce0 + 8 * ab, ((it >> 1) & 1) ^ 1);  // the epilogue has drained this accumulator buffer
      fence_after();
      for (int g = 0; g < G; ++g, ++ga) {
        const int sa = ga % kSlabAStages;
        mbar_wait(fullA0 + 8 * sa, (ga / kSlabAStages) & 1);
        for (int t = 0; t < 9; ++t, ++gb) {
          const int sb = gb % kSlabBStages;
          mbar_wait(fullB0 + 8 * sb, (gb / kSlabBStages) & 1);
          fence_after();
          const int toff = ((t / 3) * 15 + (t % 3)) * 16;  // tap (dy, dx): entries p + 15 dy + dx
#pragma unroll
          for (int h = 0; h < 2; ++h)
#pragma unroll
            for (int k = 0; k < 4; ++k)  // 16 channels = planes 2k, 2k + 1
              mma_bf16(tmem + (uint32_t)(ab * 2 * kSlabNT + h * kSlabNT),
                       a_base + (uint64_t)((sa * kSlabA + h * kSlabHalf + 2 * k * kSlabPlaneBytes + toff) >> 4),
                       b_base + (uint64_t)((sb * kSlabBStage + k * 2 * kSlabNT * 16) >> 4), idesc,
                       (g | t | k) ? 1u : 0u);
          mma_commit(emptyB0 + 8 * sb);
        }
        mma_commit(emptyA0 + 8 * sa);
      }
      mma_commit(accf0 + 8 * ab);
    }
  } else {
    // ---------------- epilogue (warps 0-3): lane = row of each half
    const int qd = warp & 3, r = 32 * qd + lane;
    int it = 0;
    for (int j = blockIdx.x; j < jobs; j += gridDim.x, ++it) {
      const int mt = j / n_nt, nt = j - mt * n_nt;
      const int ab = it & 1;
      mbar_wait(accf0 + 8 * ab, (it >> 1) & 1);
      fence_after();
      for (int h = 0; h < 2; ++h) {
        const int64_t p = (int64_t)mt * 256 + 128 * h + r;
        const int64_t f = p / 225;
        const int q = (int)(p - f * 225), y = q / 15, x = q - 15 * (q / 15);
        const bool valid = f < a.N && y < 13 && x < 13;
        const uint32_t trow = tmem + ((uint32_t)(32 * qd) << 16) + (uint32_t)(ab * 2 * kSlabNT + h * kSlabNT);
        for (int c0 = 0; c0 < kSlabNT; c0 += 16) {
          uint32_t rr[16];
          tmem_ld16(trow + (uint32_t)c0, rr);
          tmem_wait_ld(rr);
          if (!valid) continue;
          const int co = nt * kSlabNT + c0;
          uint32_t w[8];
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            float x0 = __uint_as_float(rr[2 * k]) + __ldg(a.bias + co + 2 * k);
            float x1 = __uint_as_float(rr[2 * k + 1]) + __ldg(a.bias + co + 2 * k + 1);
            x0 = x0 < 0.f ? 0.1f * x0 : x0;
            x1 = x1 < 0.f ? 0.1f * x1 : x1;
            w[k] = pack_bf16(x0, x1);
          }
          if (a.out_plane > 0) {  // next layer's slab layout: (y, x) -> padded (y + 1, x + 1)
            const int64_t e = f * 225 + (y + 1) * 15 + x + 1;
            *reinterpret_cast<uint4*>(a.out + ((int64_t)(co >> 3) * a.out_plane + e) * 8) = make_uint4(w[0], w[1], w[2], w[3]);
            *reinterpret_cast<uint4*>(a.out + ((int64_t)((co >> 3) + 1) * a.out_plane + e) * 8) =
                make_uint4(w[4], w[5], w[6], w[7]);
          } else {
            uint4* o = reinterpret_cast<uint4*>(a.out + (f * 169 + y * 13 + x) * a.Cout + co);
            o[0] = make_uint4(w[0], w[1], w[2], w[3]);
            o[1] = make_uint4(w[4], w[5], w[6], w[7]);
          }
        }
      }
      fence_before();
      mbar_arrive(acce0 + 8 * ab);
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 5) {
    fence_after();
    tmem_dealloc(tmem, 512);
  }
}

// ---------------------------------------------------------------- pool layers 3-5 by parity-slab views
// Input layout ("parity slab") of a layer with C channels on an H x H grid (H even), zero-bordered to (H+2)^2: for
// every 8-channel group cg and padded-coordinate parity (Y & 1, X & 1) a plane of 16-byte entries, entry
// e = frame * Gp^2 + (Y >> 1) * Gp + (X >> 1), Gp = (H + 2) / 2, planes ordered [cg][Y parity][X parity]. GEMM rows
// are the entries e = (frame, py, px) of that Gp x Gp grid read as POOLED output pixels (py, px < H/2 useful: 96 % /
// 93 % / 86 % for layers 3 / 4 / 5). For pool position (a, b) and tap (dy, dx) the input pixel is padded
// (2py + a + dy, 2px + b + dx): plane parity ((a + dy) & 1, (b + dx) & 1) at entry e + ((a + dy) >> 1) * Gp +
// ((b + dx) >> 1) — a constant-stride view for every (position, tap), so the four pool positions are four TMEM
// accumulator chains fed from one staged slab (rows 16 B apart, channel groups four planes apart, 8-row groups
// 128 B apart) and the 3x3 weights are shared by the chains. Per 64-channel group one slab of 128 + Gp + 2 entries
// x 4 parities x 8 groups is bulk-copied (32 copies) and feeds 9 taps x 4 chains; weights (8 KB per tap and group,
// N tile 64) stream through a ring. Warp 4 lane 0 copies, warp 5 issues, warps 0-3 max-pool / bias / leaky / bf16
// into the next layer's parity slab or NHWC.
constexpr int kPsBStages = 6;
constexpr int kPsBStage = 64 * 64 * 2;          // 8 KB: one (tap, 64-channel group) of weights, N tile 64
constexpr int kPsThreads = 192;
constexpr int kPsMaxSlab = 96 * 1024;           // per A stage

__host__ __device__ inline int ps_slab_entries(int Gp) { return (128 + Gp + 2 + 7) & ~7; }

__global__ void __launch_bounds__(kPsThreads, 1) tyolo_pslab_kernel(TyPslabArgs a) {
  extern __shared__ __align__(1024) uint8_t sm[];
  const int Gp = a.Gp, SE = ps_slab_entries(Gp), SEB = SE * 16;
  const int CG = a.Cin >= 64 ? 8 : a.Cin / 8;     // channel groups per slab (64 channels, or all of a smaller Cin)
  const int G = a.Cin >= 64 ? a.Cin / 64 : 1;
  const int slab_bytes = CG * 4 * SEB;
  uint8_t* As = sm;
  uint8_t* Bs = sm + 2 * slab_bytes;
  uint64_t* bars = reinterpret_cast<uint64_t*>(Bs + kPsBStages * kPsBStage);
  uint32_t* s_tmem = reinterpret_cast<uint32_t*>(bars + 4 + 2 * kPsBStages + 4);
  const uint32_t fullA0 = smem_addr(bars), emptyA0 = fullA0 + 16;
  const uint32_t fullB0 = emptyA0 + 16, emptyB0 = fullB0 + 8 * kPsBStages;
  const uint32_t accf0 = emptyB0 + 8 * kPsBStages, acce0 = accf0 + 16;
  const int tid = threadIdx.x, lane = tid & 31;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);
  const int n_nt = a.Cout / 64;
  const int64_t entries = (int64_t)a.N * Gp * Gp;
  const int m_tiles = (int)((entries + 127) / 128);
  const int jobs = m_tiles * n_nt;
  const int Ho = Gp - 1;

  if (tid == 0) {
    for (int s = 0; s < 2; ++s) {
      mbar_init(fullA0 + 8 * s, 1);
      mbar_init(emptyA0 + 8 * s, 1);
    }
    for (int s = 0; s < kPsBStages; ++s) {
      mbar_init(fullB0 + 8 * s, 1);
      mbar_init(emptyB0 + 8 * s, 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(accf0 + 8 * b, 1);
      mbar_init(acce0 + 8 * b, 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 5) tmem_alloc(smem_addr(s_tmem), 512);
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *s_tmem;

  if (warp == 4) {
    if (lane == 0) {
      int ga = 0, gb = 0;
      for (int j = blockIdx.x; j < jobs; j += gridDim.x) {
        const int mt = j / n_nt, nt = j - mt * n_nt;
        const int64_t e0 = (int64_t)mt * 128;
        for (int g = 0; g < G; ++g, ++ga) {
          const int sa = ga & 1;
          mbar_wait(emptyA0 + 8 * sa, ((ga >> 1) & 1) ^ 1);
          mbar_expect_tx(fullA0 + 8 * sa, (uint32_t)slab_bytes);
          for (int pl = 0; pl < CG * 4; ++pl)  // plane pl = cg * 4 + parity of this group
            bulk_g2s(smem_addr(As + sa * slab_bytes + pl * SEB),
                     reinterpret_cast<const char*>(a.in) + ((int64_t)(g * CG * 4 + pl) * a.plane + e0) * 16,
                     (uint32_t)SEB, fullA0 + 8 * sa);
          for (int t = 0; t < 9; ++t, ++gb) {
            const int sb = gb % kPsBStages;
            mbar_wait(emptyB0 + 8 * sb, ((gb / kPsBStages) & 1) ^ 1);
            mbar_expect_tx(fullB0 + 8 * sb, kPsBStage);
            bulk_g2s(smem_addr(Bs + sb * kPsBStage), a.wpk + (((int64_t)nt * G + g) * 9 + t) * kPsBStage, kPsBStage,
                     fullB0 + 8 * sb);
          }
        }
      }
    }
  } else if (warp == 5) {
    const uint32_t idesc = idesc_bf16(128, 64);
    const uint64_t a_base = umma_desc(smem_addr(As), 4 * SEB, 128);      // next channel group = 4 planes on
    const uint64_t b_base = umma_desc(smem_addr(Bs), 64 * 16, 128);
    const int ksteps = CG / 2;                                              // K16 steps per slab
    int ga = 0, gb = 0, it = 0;
    for (int j = blockIdx.x; j < jobs; j += gridDim.x, ++it) {
      const int ab = it & 1;
      mbar_wait(acce0 + 8 * ab, ((it >> 1) & 1) ^ 1);
      fence_after();
      for (int g = 0; g < G; ++g, ++ga) {
        const int sa = ga & 1;
        mbar_wait(fullA0 + 8 * sa, (ga >> 1) & 1);
        for (int t = 0; t < 9; ++t, ++gb) {
          const int sb = gb % kPsBStages;
          mbar_wait(fullB0 + 8 * sb, (gb / kPsBStages) & 1);
          fence_after();
          const int dy = t / 3, dx = t - 3 * (t / 3);
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const int ya = (q >> 1) + dy, xb = (q & 1) + dx;
            const int par = (ya & 1) * 2 + (xb & 1), off = (ya >> 1) * Gp + (xb >> 1);
            for (int k = 0; k < ksteps; ++k)
              mma_bf16(tmem + (uint32_t)(ab * 256 + q * 64),
                       a_base + (uint64_t)((sa * slab_bytes + (2 * k * 4 + par) * SEB + off * 16) >> 4),
                       b_base + (uint64_t)((sb * kPsBStage + k * 2 * 64 * 16) >> 4), idesc, (g | t | k) ? 1u : 0u);
          }
          mma_commit(emptyB0 + 8 * sb);
        }
        mma_commit(emptyA0 + 8 * sa);
      }
      mma_commit(accf0 + 8 * ab);
    }
  } else {
    const int qd = warp & 3, r = 32 * qd + lane;
    int it = 0;
    for (int j = blockIdx.x; j < jobs; j += gridDim.x, ++it) {
      const int mt = j / n_nt, nt = j - mt * n_nt;
      const int ab = it & 1;
      mbar_wait(accf0 + 8 * ab, (it >> 1) & 1);
      fence_after();
      const int64_t e = (int64_t)mt * 128 + r;
      const int64_t f = e / (Gp * Gp);
      const int rem = (int)(e - f * Gp * Gp), py = rem / Gp, px = rem - Gp * (rem / Gp);
      const bool valid = f < a.N && py < Ho && px < Ho;
      const uint32_t trow = tmem + ((uint32_t)(32 * qd) << 16) + (uint32_t)(ab * 256);
      for (int c0 = 0; c0 < 64; c0 += 16) {
        uint32_t r0[16], r1[16], r2[16], r3[16];
        tmem_ld16(trow + (uint32_t)c0, r0);
        tmem_ld16(trow + (uint32_t)(64 + c0), r1);
        tmem_ld16(trow + (uint32_t)(128 + c0), r2);
        tmem_ld16(trow + (uint32_t)(192 + c0), r3);
        tmem_wait_ld2(r0, r1);
        reg_fence2(r2, r3);
        if (!valid) continue;
        const int co = nt * 64 + c0;
        uint32_t w[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          float x0 = fmaxf(fmaxf(__uint_as_float(r0[2 * k]), __uint_as_float(r1[2 * k])),
                           fmaxf(__uint_as_float(r2[2 * k]), __uint_as_float(r3[2 * k]))) + __ldg(a.bias + co + 2 * k);
          float x1 = fmaxf(fmaxf(__uint_as_float(r0[2 * k + 1]), __uint_as_float(r1[2 * k + 1])),
                           fmaxf(__uint_as_float(r2[2 * k + 1]), __uint_as_float(r3[2 * k + 1]))) +
                     __ldg(a.bias + co + 2 * k + 1);
          x0 = x0 < 0.f ? 0.1f * x0 : x0;
          x1 = x1 < 0.f ? 0.1f * x1 : x1;
          w[k] = pack_bf16(x0, x1);
        }
        if (a.out_plane > 0 && a.out_Gp < 0) {  // 13x13 slab layout of tyolo_slab_kernel (padded 15 x 15 grid)
          const int64_t eo = f * 225 + (py + 1) * 15 + px + 1;
          *reinterpret_cast<uint4*>(a.out + ((int64_t)(co >> 3) * a.out_plane + eo) * 8) = make_uint4(w[0], w[1], w[2], w[3]);
          *reinterpret_cast<uint4*>(a.out + ((int64_t)((co >> 3) + 1) * a.out_plane + eo) * 8) =
              make_uint4(w[4], w[5], w[6], w[7]);
        } else if (a.out_plane > 0) {  // the next layer's parity slab (grid Go = Ho / 2 + 1)
          const int Go = a.out_Gp, Y = py + 1, X = px + 1;
          const int64_t eo = f * Go * Go + (Y >> 1) * Go + (X >> 1);
          const int par = (Y & 1) * 2 + (X & 1);
          *reinterpret_cast<uint4*>(a.out + (((int64_t)(co >> 3) * 4 + par) * a.out_plane + eo) * 8) =
              make_uint4(w[0], w[1], w[2], w[3]);
          *reinterpret_cast<uint4*>(a.out + (((int64_t)((co >> 3) + 1) * 4 + par) * a.out_plane + eo) * 8) =
              make_uint4(w[4], w[5], w[6], w[7]);
        } else {
          uint4* o = reinterpret_cast<uint4*>(a.out + ((f * Ho + py) * Ho + px) * a.Cout + co);
          o[0] = make_uint4(w[0], w[1], w[2], w[3]);
          o[1] = make_uint4(w[4], w[5], w[6], w[7]);
        }
      }
      fence_before();
      mbar_arrive(acce0 + 8 * ab);
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 5) {
    fence_after();
    tmem_dealloc(tmem, 512);
  }
}

int ps_smem_bytes(int Cin, int Gp) {
  const int CG = Cin >= 64 ? 8 : Cin / 8;
  return 2 * CG * 4 * ps_slab_entries(Gp) * 16 + kPsBStages * kPsBStage + 8 * (4 + 2 * kPsBStages + 4) + 16;
}

}  // namespace

int tyolo_conv_smem_bytes(int stages, int a_tiles, int b_tiles, int NT) {
  return stages * (a_tiles * kATile + b_tiles * NT * 128) + 8 * (2 * stages + 2 * kMaxAccBufs) + 16;
}

cudaError_t tyolo_configure() {
  const int smem = 227 * 1024;
  {
    cudaError_t e = cudaFuncSetAttribute(tyolo_l1_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kL1Smem);
    if (e == cudaSuccess) e = cudaFuncSetAttribute(tyolo_l2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kL2Smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(tyolo_slab_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSlabSmem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(tyolo_pslab_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    if (e == cudaSuccess)  // the default 48 KB limit also covers static and reserved memory
      e = cudaFuncSetAttribute(tyolo_resize_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    if (e != cudaSuccess) return e;
  }
  cudaError_t e = cudaFuncSetAttribute(tyolo_conv_kernel<1, 4, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tyolo_conv_kernel<1, 4, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tyolo_conv_kernel<2, 1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(tyolo_conv_kernel<1, 1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  return e;
}

cudaError_t launch_tyolo_conv(const TyConvArgs& a, cudaStream_t st) {
  const int rows = 128 * a.msub;
  const int tiles = ((a.M + rows - 1) / rows) * a.Cout_tiles;
  const unsigned grid = (unsigned)(tiles < a.grid ? tiles : a.grid);
  const int a_tiles = a.msub * (a.patch ? 1 : a.nq), b_tiles = a.patch ? a.nq : 1;
  const int smem = tyolo_conv_smem_bytes(a.stages, a_tiles, b_tiles, a.NT);
  // the three shapes of tiny-yolo-voc: pool layers by patch (L1-L3) or per-position gather (L4, L5), and the 13x13
  // layers with two row halves (L6-L9); msub 1 for the A/B knob
  if (a.nq == 4 && a.patch) tyolo_conv_kernel<1, 4, true><<<grid, kConvThreads, smem, st>>>(a);
  else if (a.nq == 4) tyolo_conv_kernel<1, 4, false><<<grid, kConvThreads, smem, st>>>(a);
  else if (a.msub == 2) tyolo_conv_kernel<2, 1, false><<<grid, kConvThreads, smem, st>>>(a);
  else tyolo_conv_kernel<1, 1, false><<<grid, kConvThreads, smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_tyolo_l1(const TyL1Args& a, int num_sms, cudaStream_t st) {
  const int tiles = a.N * kL1Out * 2;
  const int grid = tiles < 2 * num_sms ? tiles : 2 * num_sms;
  tyolo_l1_kernel<<<grid, kL1Threads, kL1Smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_tyolo_l2(const TyL1Args& a, int num_sms, cudaStream_t st) {
  const int tiles = a.N * kL2Out;
  const int grid = tiles < num_sms ? tiles : num_sms;
  tyolo_l2_kernel<<<grid, kL2Threads, kL2Smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_tyolo_pslab(const TyPslabArgs& a, int num_sms, cudaStream_t st) {
  const int smem = ps_smem_bytes(a.Cin, a.Gp);
  if (smem > 227 * 1024 || a.Cout % 64 || (a.Cin < 64 && a.Cin % 16) || (a.Cin >= 64 && a.Cin % 64))
    return cudaErrorInvalidValue;
  const int64_t jobs = (((int64_t)a.N * a.Gp * a.Gp + 127) / 128) * (a.Cout / 64);
  tyolo_pslab_kernel<<<(unsigned)(jobs < num_sms ? jobs : num_sms), kPsThreads, smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_tyolo_slab(const TySlabArgs& a, int num_sms, cudaStream_t st) {
  const int jobs = ((a.N * 225 + 255) / 256) * (a.Cout / kSlabNT);
  tyolo_slab_kernel<<<jobs < num_sms ? jobs : num_sms, kSlabThreads, kSlabSmem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_tyolo_pool_s1(const __nv_bfloat16* in, __nv_bfloat16* out, int32_t n, int32_t H, int32_t C,
                                 int64_t planar_stride, cudaStream_t st) {
  const int64_t total = (int64_t)n * H * H * (C / 8);
  tyolo_pool_s1_kernel<<<(unsigned)((total + 255) / 256), 256, 0, st>>>(in, out, n, H, C, planar_stride);
  return cudaGetLastError();
}

cudaError_t launch_tyolo_resize(const TyFrame* frames, int32_t n, int32_t D, int32_t max_row_bytes, int32_t max_H,
                                __nv_bfloat16* out, cudaStream_t st) {
  // R output rows per CTA: the largest with a stage of <= 24 KB (A/B at 720p: 0.42 ms vs 0.44 at 48 KB and 0.52 at
  // R = 1); a group of R rows spans at most ceil(R*H/D) + 1 source rows (or R rows when H < D)
  const int rb16 = (max_row_bytes + 15) & ~15;
  const char* renv = std::getenv("FFSVA_TYOLO_RESIZE_ROWS");
  auto span = [&](int r) { return std::max((r * max_H + D - 1) / D + 1, r); };
  int R = 1;
  if (renv) R = std::max(1, std::atoi(renv));
  else
    while (R < D && span(R + 1) * rb16 <= 24 * 1024) ++R;
  const int stage = span(R) * rb16;
  if (D > kResizeMaxD || stage > 200 * 1024) return cudaErrorInvalidValue;
  // the >48 KB opt-in is set per device by tyolo_configure (every model load, on the model's device)
  const dim3 grid((unsigned)((D + R - 1) / R), (unsigned)n);
  tyolo_resize_kernel<<<grid, kResizeThreads, stage, st>>>(frames, D, R, stage, out);
  return cudaGetLastError();
}

}  // namespace ffsva
