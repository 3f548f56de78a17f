// ffsva_internal.h — shared declarations of the product library (kernels <-> host runtime).
// Not part of the public ABI (include/ffsva.h is). Nothing here is shared with oracle/.
#pragma once

#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "ffsva.h"

namespace ffsva {

// ------------------------------------------------------------------ per-frame descriptor (device, 64 B)
struct FrameDesc {
  const uint8_t* pixels;   // raw RGB8 frame
  const uint8_t* ref;      // stream's reference image R [sdd_h][sdd_w][3]
  const uint8_t* snm;      // stream's packed SNM weight image (SnmLayout), nullptr for SDD-only batches
  int64_t pitch;           // row pitch in bytes
  uint64_t T;              // SDD threshold: pass iff SSD > T
  int32_t W, H;            // raw size
  float L_t;               // logit threshold for t_pre (Eq. (2)); pass iff logit >= L_t
  float L_low, L_high;     // logit(c_low), logit(c_high) for the class (L159)
  uint16_t slot;           // stream slot (stats row; < 65536 slots per device)
  uint8_t metric;          // SDD distance: kDistMse / kDistSad / kDistNrmse (ffsva_distance)
  uint8_t mode;            // SDD reference: kRefBackground / kRefPrevious (ffsva_ref_mode)
};
constexpr uint8_t kDistMse = 0, kDistSad = 1, kDistNrmse = 2;
constexpr uint8_t kRefBackground = 0, kRefPrevious = 1;
static_assert(sizeof(FrameDesc) == 64, "FrameDesc must stay 64 B");

// ------------------------------------------------------------------ SNM packed weight image (global + smem)
// Exactly the shared-memory image the SNM kernel copies in once per stream change (dynamic batch, L219).
// bf16 B operands are in the tcgen05 K-major no-swizzle canonical layout: [mma][khalf][n][8 k] (16 B rows).
namespace snm {
constexpr int C1 = 16, C2 = 32;
constexpr int IN = 50, P1 = 25, P2 = 12;             // input, pooled conv1, pooled conv2 (floor)
constexpr int NF = C2 * P2 * P2;                    // 4608 FC inputs
constexpr int N_PARAMS = 27 * C1 + C1 + 9 * C1 * C2 + C2 + NF + 1;  // 9697
// conv1 B operands, one per 4x4-patch row dy (the MMA's A rows are pooled pixels' 4x4 input patches, 4 channel
// slots per pixel): N = 64 = [pool position q = 2a + b][16 output channels], K = 16 = [patch column u][4 channel
// slots], value w1[oc][c][dy - a][u - b] where that tap exists (c < 3), else 0. Each is [2 K-halves][64 n][8 k] bf16.
// Patch row 0 only reaches positions a = 0 (n < 32) and row 3 only a = 1 (n >= 32): those two MMAs use N = 32.
constexpr int W1_MMAS = 4;
constexpr int W1_BYTES = W1_MMAS * 2 * 64 * 16;     // 8192
// conv2 B operands, one per MMA of kConv2Mmas. The A operand of an MMA is one 3x3-window cell (Y', X') of the 4x4
// patch around a pooled output pixel (Y', X' in 0..3, 16 input channels = K16); pool position (a, b) reads that cell
// through tap (Y' - a, X' - b), so one A serves every position whose 3x3 window holds the cell: N = 32 x (positions
// in one run of consecutive TMEM column groups, order kConv2Group). Each B is [2 K-halves][N][8] bf16.
struct Conv2Mma {
  int32_t cy, cx;   // patch cell (Y', X')
  int32_t g0, ng;   // first TMEM column group (32 columns each) and number of groups (positions)
  int32_t boff;     // byte offset of the B operand in the W2 region
};
// TMEM column group of pool position (a, b): (0,0) 0, (0,1) 1, (1,1) 2, (1,0) 3 — so the two-position cells of three
// of the four edges are one contiguous run; the (0,0)+(1,0) cells (X' = 0) take two N = 32 MMAs.
__host__ __device__ constexpr int conv2_group(int a, int b) { return a == 0 ? b : 3 - b; }
constexpr int kConv2Mmas = 18;
// MMA i of a conv2 tile (host packing and the kernel's issue loop, constant-folded there)
__host__ __device__ constexpr Conv2Mma conv2_mma(int i) {
  switch (i) {
    // four-position cells first: the first MMA (accumulate = 0) initialises all 128 columns
    case 0: return {1, 1, 0, 4, 0};
    case 1: return {1, 2, 0, 4, 4096};
    case 2: return {2, 1, 0, 4, 8192};
    case 3: return {2, 2, 0, 4, 12288};
    // two-position runs
    case 4: return {0, 1, 0, 2, 16384};   // a = 0: (0,0) (0,1)
    case 5: return {0, 2, 0, 2, 18432};
    case 6: return {3, 1, 2, 2, 20480};   // a = 1: (1,1) (1,0)
    case 7: return {3, 2, 2, 2, 22528};
    case 8: return {1, 3, 1, 2, 24576};   // b = 1: (0,1) (1,1)
    case 9: return {2, 3, 1, 2, 26624};
    case 10: return {1, 0, 0, 1, 28672};  // b = 0: (0,0) | (1,0), not adjacent
    case 11: return {1, 0, 3, 1, 29696};
    case 12: return {2, 0, 0, 1, 30720};
    case 13: return {2, 0, 3, 1, 31744};
    // corners
    case 14: return {0, 0, 0, 1, 32768};
    case 15: return {0, 3, 1, 1, 33792};
    case 16: return {3, 3, 2, 1, 34816};
    default: return {3, 0, 3, 1, 35840};
  }
}
constexpr int W2_BYTES = 36864;                     // 36 position-taps x 32 n x 32 B
constexpr int OFF_W1 = 0;
constexpr int OFF_W2 = OFF_W1 + W1_BYTES;           // 8192
constexpr int OFF_B1 = OFF_W2 + W2_BYTES;           // 45056 (fp32[16])
constexpr int OFF_B2 = OFF_B1 + C1 * 4;             // 45120 (fp32[32])
constexpr int OFF_BFC = OFF_B2 + C2 * 4;            // 45248 (fp32[1] + pad to 16)
constexpr int OFF_WFC = OFF_BFC + 16;               // 45264: fp32 [8 channel quads][144 pixels][4] of bf16 values
constexpr int BLOB_BYTES = OFF_WFC + NF * 4;        // 63696
static_assert(BLOB_BYTES % 16 == 0, "blob must be 16-B granular");
}  // namespace snm

// ------------------------------------------------------------------ launchers (defined in the .cu files)
struct SddArgs {
  const FrameDesc* frames;
  int32_t n;
  int32_t sdd_w, sdd_h;      // grid (uniform over the batch)
  uint8_t* d50;              // [n][d50_stride], or a slot pool addressed through d50_index
  int64_t d50_stride;
  const int32_t* d50_index;  // optional [n]: frame f's D50 goes to slot d50_index[f] (online queues)
  uint8_t* d100;             // optional [n][sdd_h*sdd_w*3]
  unsigned long long* acc_ssd; // [n] per-frame SSD accumulator: zero on entry; K3 reads it and re-zeroes it
  unsigned long long* stats; // [slots][NSTAT] or nullptr
  int32_t max_chunks;        // max over frames of ceil(3W/16)
  bool vec16;                // all frames 16-B aligned with 16-B pitch
  bool bulk;                 // use the bulk-async (TMA engine) + cluster kernel
  int32_t stage_bytes;       // bulk: shared-memory bytes for one 100-grid row's source rows (max over frames)
  const int32_t* xbounds;    // [sdd_w + 1] floor(i*uni_W/sdd_w) for frames of width uni_W, or nullptr
  const int32_t* ybounds;    // [sdd_h + 1] floor(i*uni_H/sdd_h) for frames of height uni_H, or nullptr
  int32_t uni_W, uni_H;
  int32_t cellw;             // widest 100-grid cell of uni_W-wide frames, ceil(uni_W / sdd_w) (0 if mixed)
  bool seg;                  // bulk: the warp-segment pipeline kernel (narrow rows)
  int32_t max_cellw;         // widest 100-grid cell over the batch
  int32_t max_rows100;       // tallest 100-grid row (source rows) over the batch
  int32_t magic_n;           // warp-segment kernel: entries of its box-area reciprocal table
  int32_t min_cellw;         // narrowest 100-grid cell over the batch (floor(min W / sdd_w))
};

// K1 variant choice for one batch (sdd_plan_add per frame, then sdd_plan_finish): the bulk-async CTA-pair kernel
// for 16-B aligned rows whose 100-grid row fits the stage, the register-streaming kernel otherwise;
// FFSVA_SDD_KERNEL=stream forces the latter (tests exercise both).
enum SddVariant : int32_t { kSddStream = 0, kSddPair = 1 };
struct SddPlan {
  int32_t max_chunks = 1, pair_stage = 0;
  int32_t seg_stage = 0;     // warp-segment kernel: max bytes of one 50-grid row's source rows
  int32_t max_rows100 = 0, max_w = 0;  // tallest 100-grid row (source rows), widest frame
  int32_t min_w = 0;         // narrowest frame
  bool vec16 = true;
  int32_t variant = kSddStream, stage_bytes = 0;
  bool seg = false;
  size_t smem = 0;
};
void sdd_plan_add(SddPlan& p, int32_t W, int32_t H, int64_t pitch, const void* pixels, int32_t sdd_h);
void sdd_plan_finish(SddPlan& p, int32_t sdd_w, int32_t sdd_h);
void sdd_plan_apply(const SddPlan& p, SddArgs& a);
cudaError_t launch_sdd(const SddArgs& a, cudaStream_t st);
size_t sdd_smem_bytes(int max_chunks, int sdd_w);
size_t sdd_bulk_smem_bytes(int stage_bytes, int sdd_w);
int sdd_bulk_stage_bytes(int W, int H, int sdd_h);
bool sdd_bulk_ok(int max_chunks, int stage_bytes);
cudaError_t sdd_configure(size_t smem);  // raise the kernels' dynamic smem limit (outside graph capture)
int sdd_threads(int max_chunks);

struct CompactArgs {
  const FrameDesc* frames;   // [n] (threshold T per frame)
  unsigned long long* acc_ssd; // [n] K1's SSD accumulators (read, then re-zeroed for the next launch)
  uint64_t* ssd;             // [n] out
  uint8_t* pass;             // [n] out: SSD > T
  int32_t n;
  const int32_t* perm;       // [n] work (stream-major, stable) order -> frame index
  const int32_t* seg_lo;     // [n_seg + 1] segment boundaries in perm order (one segment per stream)
  int32_t n_seg;
  const int32_t* seg_batch;  // [n_seg] BatchSize of the segment's stream
  const int32_t* seg_slot;   // [n_seg] stats slot of the segment's stream
  unsigned long long* stats; // SNM_BATCHES (pops) counted here; may be nullptr
  int32_t snm_ctas;          // K4 grid size, 0 for SDD-only batches (then no dynamic batches are counted)
  int32_t* survivor_idx;     // [n] out
  int32_t* work;             // [n] out: survivors in work order (frame indices)
  int32_t* posw;             // [n + 1] scratch: exclusive survivor count in perm order
  int32_t* chunks;           // [n + 1] out: pop k = work[chunks[k] .. chunks[k+1]) (one stream, <= BatchSize)
  int32_t* counts;           // [4] out: m, n_chunks, 0, pad
  float* logit;              // [n] initialised here: NaN / 0 / 0 (the SNM kernel overwrites survivors)
  uint8_t* snm_pass;
  uint8_t* snm_class;
};
cudaError_t launch_compact(const CompactArgs& a, cudaStream_t st);

struct SnmArgs {
  const FrameDesc* frames;
  const uint8_t* d50;
  int64_t d50_stride;
  const int32_t* d50_index;  // optional [n]: frame f's D50 image is slot d50_index[f]
  const int32_t* work;
  const int32_t* chunks;
  int32_t* counts;           // m (survivors), n_chunks
  const uint8_t* pop_start;  // optional [n_chunks]: 1 if the unit opens a dynamic batch (online mode counts
                             // SNM_BATCHES here; batch mode counts them in K3)
  float* logit;              // [n] (frame order)
  uint8_t* snm_pass;
  uint8_t* snm_class;
  unsigned long long* stats;
  int32_t grid;              // one CTA per SM at most: CTA c scores survivors [c*m/grid, (c+1)*m/grid) of work order
};
cudaError_t launch_snm(const SnmArgs& a, cudaStream_t st);
constexpr int kSnmCtasPerSm = 1;  // K4 is persistent, one warp-specialised CTA per SM (all 512 TMEM columns, ~182 KB smem)
int snm_smem_bytes();
cudaError_t snm_configure();

// Previous-frame reference (ffsva_ref_mode PREVIOUS, Q25). After K1 has written every frame's D100:
//  K2 sdd_prev_kernel: one CTA per listed frame f, distance of D100[f] against D100[prev] (prev >= 0: the
//     stream's previous frame in the batch) or the stream's R (prev = -1), added to acc_ssd[f] (K1 added 0);
//  K2b ref_update_kernel: R of each listed stream <- D100 of its last frame in the batch.
struct PrevArgs {
  const FrameDesc* frames;
  const uint8_t* d100;       // [n][3*sdd_w*sdd_h]
  int32_t n_values;          // 3*sdd_w*sdd_h
  const int32_t* pairs;      // [n_pm][2]: (frame, prev frame or -1)
  int32_t n_pm;
  const int32_t* last;       // [n_last]: last frame of each PREVIOUS-mode stream (its R is frames[f].ref)
  int32_t n_last;
  unsigned long long* acc_ssd;
  unsigned long long* stats;
};
cudaError_t launch_prev(const PrevArgs& a, cudaStream_t st);  // K2 then K2b (2 launches if n_pm > 0)

// ------------------------------------------------------------------ T-YOLO (f1, ffsva_tyolo.cu)
struct TyFrame {           // raw frame geometry for the 416x416 resize, and the frame's target class (head)
  const uint8_t* pixels;
  int64_t pitch;
  int32_t W, H;
  int32_t target, pad;
};
struct TyConvArgs {
  const __nv_bfloat16* in;   // NHWC [N][H][W][Cp] bf16 (conv input; 'same' convolution keeps H x W)
  __nv_bfloat16* out;        // NHWC [N][Ho][Wo][Cout] bf16 (hidden layers)
  float* out_f32;            // [M][Cout] fp32 (head)
  const uint8_t* wpk;        // weights packed per (N tile, K step) in the UMMA B layout
  const float* bias;         // [Cout] fp32 (zero-padded)
  int32_t N, H, W, Cp;       // batch, conv spatial size, padded input channels (4, 16, 32 or a multiple of 64)
  int32_t Ho, Wo;            // output spatial size (after pooling)
  int32_t Cout, NT, Cout_tiles;  // output channels (row stride of out), N tile, number of N tiles
  int32_t nq, pool, ksize;   // accumulator chains (4 for pool layers), pool 0/1 (2x2/2)/2 (2x2/1), kernel 3 or 1
  int32_t kchunks, ksteps;   // K steps of 64 channels, MMA K16 steps per K step
  int32_t stages, tmem_cols, leaky, M;
  int32_t acc_bufs, grid;    // TMEM accumulator buffers (1 or 2), persistent grid size (CTAs)
  int32_t msub;              // 128-row halves per tile sharing each weight stage (1 or 2)
  int32_t patch;             // pool layers: A row = the pooled pixel's 4x4 input patch, weights per pool position
  int32_t lag;               // K steps of gathers in flight per producer thread before it publishes (1 .. S-1)
  int32_t cp_shift;          // log2(Cp)
  int32_t head;              // head: count boxes of frame f's target class scoring > thresh into counts[f]
  const TyFrame* frames;     // head: per-frame target classes
  float thresh;
  int32_t* counts;
};
cudaError_t launch_tyolo_conv(const TyConvArgs& a, cudaStream_t st);
// Layer 1 by patch views (ffsva_tyolo.cu): zero-bordered resize output [N][418][418][4] -> [N][208][208][16].
struct TyL1Args {
  const __nv_bfloat16* in;
  __nv_bfloat16* out;
  int64_t out_plane;         // layer 2: > 0 writes layer 3's parity slab (entries per plane), else NHWC
  const uint8_t* w;          // 4 patch rows x [2 K-halves][64 n = 16q + oc][8 k = 4u + c] bf16 (8 KB)
  const float* bias;         // [16]
  int32_t N;
};
cudaError_t launch_tyolo_l1(const TyL1Args& a, int num_sms, cudaStream_t st);
// Layer 2 by patch views: layer 1's planar zero-bordered output [N][210][2][2][105][8 ch] -> [N][104][104][32].
// w: 16 (patch row, column) x [2 channel groups][128 n = 32q + oc][8 k] bf16 (64 KB).
cudaError_t launch_tyolo_l2(const TyL1Args& a, int num_sms, cudaStream_t st);
constexpr size_t kTyL2PadBytes = (size_t)210 * 4 * 105 * 16;  // per frame
cudaError_t launch_tyolo_pool_s1(const __nv_bfloat16* in, __nv_bfloat16* out, int32_t n, int32_t H, int32_t C,
                                 int64_t planar_stride, cudaStream_t st);
// 13x13 layers by slab views (ffsva_tyolo.cu tyolo_slab_kernel). Slab layout of C channels: C/8 planes of `plane`
// 16-byte entries, entry = frame * 225 + Y * 15 + X of the zero-bordered 15x15 grid; plane >= round_up(N * 225,
// 256) + 64 (reads past the last frame stay inside the plane).
inline int64_t tyolo_slab_plane(int32_t n) { return (int64_t)((n * 225 + 255) / 256) * 256 + 64; }
struct TySlabArgs {
  const __nv_bfloat16* in;   // slab layout, Cin channels
  int64_t plane;             // entries per input plane
  __nv_bfloat16* out;        // slab layout (out_plane > 0) or NHWC [N][13][13][Cout]
  int64_t out_plane;
  const uint8_t* wpk;        // the generic kernel's packing for this layer (NT = 128, K step = tap * Cin/64 + group)
  const float* bias;
  int32_t N, Cin, Cout;      // Cin % 64 == 0, Cout % 128 == 0
};
cudaError_t launch_tyolo_slab(const TySlabArgs& a, int num_sms, cudaStream_t st);
// Pool layers 3-5 by parity-slab views (tyolo_pslab_kernel). Parity slab of C channels on an H x H grid: planes
// [C/8][Y parity][X parity] of `plane` 16-byte entries, entry = frame * Gp^2 + (Y >> 1) * Gp + (X >> 1) over the
// zero-bordered (H+2)^2 grid, Gp = H/2 + 1; plane >= round_up(N * Gp^2, 128) + Gp + 16.
inline int64_t tyolo_pslab_plane(int32_t n, int32_t Gp) {
  return ((int64_t)n * Gp * Gp + 127) / 128 * 128 + Gp + 16;
}
struct TyPslabArgs {
  const __nv_bfloat16* in;   // parity slab, Cin channels, grid Gp
  int64_t plane;
  __nv_bfloat16* out;        // next layer's parity slab (out_plane > 0, grid out_Gp > 0), 13x13 slab (out_plane > 0,
  int64_t out_plane;         // out_Gp < 0; tyolo_slab_kernel's layout) or NHWC [N][Gp-1][Gp-1][Cout] (out_plane 0)
  int32_t out_Gp;
  const uint8_t* wpk;        // [N tile of 64][64-channel group][tap][8-channel K group][64 n][8] bf16
  const float* bias;
  int32_t N, Cin, Cout, Gp;  // Cin 32 / 64 / 128 ..., Cout % 64 == 0
};
cudaError_t launch_tyolo_pslab(const TyPslabArgs& a, int num_sms, cudaStream_t st);
cudaError_t launch_tyolo_resize(const TyFrame* frames, int32_t n, int32_t D, int32_t max_row_bytes, int32_t max_H,
                                __nv_bfloat16* out, cudaStream_t st);
int tyolo_conv_smem_bytes(int stages, int a_tiles, int b_tiles, int NT);
cudaError_t tyolo_configure();

cudaError_t launch_fill_nan(float* p, int32_t n, cudaStream_t st);
cudaError_t launch_reference(const uint8_t* frames, int32_t k, int64_t frame_stride, int32_t W, int32_t H,
                             int64_t pitch, int32_t sdd_w, int32_t sdd_h, uint8_t* out, cudaStream_t st);

constexpr int NSTAT = 8;   // device statistics table stride (columns FFSVA_STAT_FRAMES .. FFSVA_STAT_SNM_BATCHES)
constexpr int NLAT = 16;   // host latency columns per slot (FFSVA_STAT_DECIDED .. FFSVA_STAT_LAT_BIN0 + 13)
static_assert(NSTAT + NLAT == FFSVA_NSTAT, "statistics row layout (include/ffsva.h)");

}  // namespace ffsva
