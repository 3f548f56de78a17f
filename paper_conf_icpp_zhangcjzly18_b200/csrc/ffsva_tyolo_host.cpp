// ffsva_tyolo_host.cpp — the shared T-YOLO model of a device (f1; one model "shared by all
// streams", L175) and its C-ABI: weight packing into the kernel's UMMA B layout, workspace, the layer sequence.
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <vector>

#include "ffsva_runtime.h"

using namespace ffsva;

namespace {

constexpr int kIn = 416;      // T-YOLO input size (L169)
constexpr int kGrid = 13;     // output grid (L171)
constexpr int kHeadPad = 128; // 125 outputs padded to a 128-column tile
constexpr int kMaxChunk = 256;
// parity slabs of layers 3, 4, 5 (see TyPslabArgs): channels and grid size Gp = H/2 + 1 of their inputs
constexpr int kPsC[3] = {32, 64, 128};
constexpr int kPsGp[3] = {53, 27, 14};

// tiny-yolo-voc: (Cin, Cout, kernel, pool after: 0 none, 1 2x2/2, 2 2x2/1)
constexpr int kNet[9][4] = {{3, 16, 3, 1},     {16, 32, 3, 1},     {32, 64, 3, 1},
                            {64, 128, 3, 1},   {128, 256, 3, 1},   {256, 512, 3, 2},
                            {512, 1024, 3, 0}, {1024, 1024, 3, 0}, {1024, 125, 1, 0}};

struct Layer {
  int Cin, Cout, k, pool;     // pool: the network's (0 none, 1 2x2/2, 2 2x2/1)
  int conv_pool;              // pool folded into the conv kernel (the 2x2/2 layers); 2x2/1 runs as its own kernel
  int Cp, Cout_pad, NT, nq, kchunks, ksteps, stages, tmem_cols, acc_bufs;
  int patch, msub;            // kernel variants (see TyConvArgs)
  int H;                      // conv spatial size (input = output before pooling)
  int Ho;                     // after pooling
  size_t w_off, b_off;        // into the packed weight / bias blobs (bytes / floats)
  size_t w_bytes;
};

uint16_t bf16_bits(float x) { return bf16_bits_rne(x); }

int pow2_at_least(int v) {
  int p = 32;
  while (p < v) p <<= 1;
  return p;
}

}  // namespace

struct ffsva_tyolo {
  DeviceCtx* ctx = nullptr;
  Layer L[9];
  uint8_t* d_w = nullptr;
  float* d_b = nullptr;
  // workspace for up to `cap` frames per chunk
  int cap = 0;
  __nv_bfloat16* d_act[2] = {nullptr, nullptr};
  __nv_bfloat16* d_pad = nullptr;  // zero-bordered resize output [cap][418][418][4] (layer 1's input)
  uint8_t* d_w1v = nullptr;        // layer 1 weights for the patch-view kernel (8 KB)
  __nv_bfloat16* d_pad2 = nullptr; // layer 1's planar zero-bordered output (layer 2's input), kTyL2PadBytes per frame
  uint8_t* d_w2v = nullptr;        // layer 2 weights for the patch-view kernel (64 KB)
  __nv_bfloat16* d_slab[3] = {nullptr, nullptr, nullptr};  // slab layouts of the inputs of layers 7 (512 ch), 8 (1024)
                                                            // and 6 (256 ch)
  int64_t slab_plane = 0;          // entries per slab plane (fixed per workspace: the zero border must not move)
  __nv_bfloat16* d_ps[3] = {nullptr, nullptr, nullptr};  // parity slabs: inputs of layers 3, 4, 5
  int64_t ps_plane[3] = {0, 0, 0};
  uint8_t* d_wps[3] = {nullptr, nullptr, nullptr};       // layers 3-5 weights for the parity-slab kernel
  float* d_raw = nullptr;
  int32_t* d_counts = nullptr;
  TyFrame* d_frames = nullptr;
  TyFrame* h_frames = nullptr;
  int32_t* h_counts = nullptr;
};

namespace {

int env_int(const char* name, int dflt) {
  const char* v = std::getenv(name);
  return v ? std::atoi(v) : dflt;
}

void build_layers(ffsva_tyolo* m) {
  // A/B knobs: patch gather for pool layers with Cp <= FFSVA_TYOLO_PATCH_CP (default 32), and FFSVA_TYOLO_MSUB
  // 128-row halves per tile for the non-pool layers (default 2)
  const int patch_cp = env_int("FFSVA_TYOLO_PATCH_CP", 32), msub = env_int("FFSVA_TYOLO_MSUB", 2);
  int H = kIn;
  size_t w_off = 0, b_off = 0;
  for (int l = 0; l < 9; ++l) {
    Layer& L = m->L[l];
    L.Cin = kNet[l][0];
    L.Cout = kNet[l][1];
    L.k = kNet[l][2];
    L.pool = kNet[l][3];
    L.Cp = L.Cin == 3 ? 4 : L.Cin;
    L.Cout_pad = l == 8 ? kHeadPad : L.Cout;
    L.conv_pool = L.pool == 1 ? 1 : 0;
    L.nq = L.conv_pool ? 4 : 1;
    L.NT = std::min(L.Cout_pad, L.conv_pool ? 128 : 256);
    if (l >= 5 && l <= 7) L.NT = 128;  // layers 6, 7 and 8 run on the slab kernel (N tile 128)
    L.patch = L.conv_pool && L.Cp <= patch_cp ? 1 : 0;
    L.msub = L.conv_pool ? 1 : std::max(1, std::min(2, msub));
    if (L.patch) L.kchunks = 16 * L.Cp / 64 > 0 ? 16 * L.Cp / 64 : 1;  // 4x4 patch x Cp channels
    else if (L.k == 1) L.kchunks = L.Cp / 64;
    else if (L.Cp >= 64) L.kchunks = 9 * L.Cp / 64;
    else if (L.Cp == 4) L.kchunks = 1;
    else L.kchunks = (9 + 64 / L.Cp - 1) / (64 / L.Cp);
    // the first layer's 9 taps x 4 channels = 36 K fit in 3 MMA K16 steps (the patch form uses all 64)
    L.ksteps = (L.Cp == 4 && !L.patch) ? 3 : 4;
    const int a_tiles = L.msub * (L.patch ? 1 : L.nq), b_tiles = L.patch ? L.nq : 1;
    const int stage = a_tiles * 128 * 128 + b_tiles * L.NT * 128;
    L.stages = std::max(2, std::min(8, (227 * 1024 - 1024) / stage));
    // as many TMEM accumulator buffers as fit (up to 8): the epilogue of earlier tiles overlaps later mainloops
    L.acc_bufs = std::max(1, std::min(8, 512 / (L.msub * L.nq * L.NT)));
    L.tmem_cols = pow2_at_least(L.acc_bufs * L.msub * L.nq * L.NT);
    L.H = H;
    L.Ho = L.pool == 1 ? H / 2 : H;
    L.w_off = w_off;
    L.w_bytes = (size_t)(L.Cout_pad / L.NT) * L.kchunks * b_tiles * L.NT * 128;
    w_off += L.w_bytes;
    L.b_off = b_off;
    b_off += L.Cout_pad;
    H = L.Ho;
  }
}

// Pack layer l's weights w[Cout][Cin][k][k] into [N tile][K step][B tile][K group 8][NT rows][8 bf16] (the
// kernel's B tile layout: K-adjacent core matrices NT*16 B apart, 8-row groups 128 B apart). Patch layers have one
// B tile per pool position q = (a, b): patch pixel (u, v) carries tap (u - a, v - b) when that lies in the 3x3.
void pack_layer(const Layer& L, const float* w, uint8_t* dst) {
  uint16_t* out = reinterpret_cast<uint16_t*>(dst);
  const int tiles = L.Cout_pad / L.NT, bt = L.patch ? L.nq : 1;
  for (int t = 0; t < tiles; ++t)
    for (int j = 0; j < L.kchunks; ++j)
      for (int q = 0; q < bt; ++q)
      for (int g = 0; g < 8; ++g)
        for (int nn = 0; nn < L.NT; ++nn)
          for (int e = 0; e < 8; ++e) {
            const int kk = g * 8 + e;
            int tap, c;
            if (L.patch) {
              const int k = j * 64 + kk, px = k / L.Cp, dy = (px >> 2) - (q >> 1), dx = (px & 3) - (q & 1);
              c = k % L.Cp;
              tap = (dy >= 0 && dy < 3 && dx >= 0 && dx < 3) ? dy * 3 + dx : 9;
            } else if (L.k == 1) {
              tap = 4;
              c = j * 64 + kk;
            } else if (L.Cp >= 64) {
              const int cpt = L.Cp / 64;
              tap = j / cpt;
              c = (j % cpt) * 64 + kk;
            } else {
              const int tpc = 64 / L.Cp;
              tap = j * tpc + kk / L.Cp;
              c = kk % L.Cp;
            }
            const int co = t * L.NT + nn;
            float v = 0.f;
            if (tap < 9 && c < L.Cin && co < L.Cout)
              v = L.k == 1 ? w[(size_t)co * L.Cin + c] : w[(((size_t)co * L.Cin + c) * 3 + tap / 3) * 3 + tap % 3];
            const size_t o = (((((size_t)t * L.kchunks + j) * bt + q) * 8 + g) * L.NT + nn) * 8 + e;
            out[o] = bf16_bits(v);
          }
}

ffsva_status ensure_workspace(ffsva_tyolo* m, int n) {
  if (m->cap >= std::min(n, kMaxChunk)) return FFSVA_OK;
  const int cap = std::min(kMaxChunk, std::max(n, 16));
  cudaFree(m->d_act[0]);
  cudaFree(m->d_act[1]);
  cudaFree(m->d_pad);
  cudaFree(m->d_pad2);
  for (auto& p : m->d_slab) cudaFree(p);
  for (auto& p : m->d_ps) cudaFree(p);
  cudaFree(m->d_raw);
  cudaFree(m->d_counts);
  cudaFree(m->d_frames);
  cudaFreeHost(m->h_frames);
  cudaFreeHost(m->h_counts);
  m->cap = 0;
  size_t act = 0;  // largest activation per frame (bytes)
  act = std::max(act, (size_t)kIn * kIn * 4 * 2);
  for (int l = 0; l < 8; ++l) act = std::max(act, (size_t)m->L[l].Ho * m->L[l].Ho * m->L[l].Cout_pad * 2);
  const size_t pad_bytes = (size_t)cap * (kIn + 2) * (kIn + 2) * 4 * 2;
  cudaError_t e = cudaMalloc(&m->d_act[0], act * cap);
  if (e == cudaSuccess) e = cudaMalloc(&m->d_act[1], act * cap);
  if (e == cudaSuccess) e = cudaMalloc(&m->d_pad, pad_bytes);
  if (e == cudaSuccess) e = cudaMemset(m->d_pad, 0, pad_bytes);  // the border is written once, here
  if (e == cudaSuccess) e = cudaMalloc(&m->d_pad2, (size_t)cap * kTyL2PadBytes);
  if (e == cudaSuccess) e = cudaMemset(m->d_pad2, 0, (size_t)cap * kTyL2PadBytes);
  m->slab_plane = tyolo_slab_plane(cap);
  for (int k = 0; k < 3 && e == cudaSuccess; ++k) {  // layers 3, 4, 5: C = 32, 64, 128 on grids 104, 52, 26
    m->ps_plane[k] = tyolo_pslab_plane(cap, kPsGp[k]);
    const size_t bytes = (size_t)(kPsC[k] / 8) * 4 * (size_t)m->ps_plane[k] * 16;
    e = cudaMalloc(&m->d_ps[k], bytes);
    if (e == cudaSuccess) e = cudaMemset(m->d_ps[k], 0, bytes);
  }
  for (int k = 0; k < 3 && e == cudaSuccess; ++k) {
    const size_t bytes = (size_t)(k == 0 ? 512 : k == 1 ? 1024 : 256) / 8 * (size_t)m->slab_plane * 16;
    e = cudaMalloc(&m->d_slab[k], bytes);
    if (e == cudaSuccess) e = cudaMemset(m->d_slab[k], 0, bytes);
  }
  if (e == cudaSuccess) e = cudaMalloc(&m->d_raw, (size_t)cap * kGrid * kGrid * kHeadPad * 4);
  if (e == cudaSuccess) e = cudaMalloc(&m->d_counts, (size_t)cap * 4);
  if (e == cudaSuccess) e = cudaMalloc(&m->d_frames, (size_t)cap * sizeof(TyFrame));
  if (e == cudaSuccess) e = cudaMallocHost(&m->h_frames, (size_t)cap * sizeof(TyFrame));
  if (e == cudaSuccess) e = cudaMallocHost(&m->h_counts, (size_t)cap * 4);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "T-YOLO workspace");
  m->cap = cap;
  return FFSVA_OK;
}

TyConvArgs layer_args(const ffsva_tyolo* m, int l, int n, const __nv_bfloat16* in, __nv_bfloat16* out,
                      float thresh) {
  const Layer& L = m->L[l];
  TyConvArgs a{};
  a.in = in;
  a.out = out;
  a.out_f32 = l == 8 ? m->d_raw : nullptr;
  a.wpk = m->d_w + L.w_off;
  a.bias = m->d_b + L.b_off;
  a.N = n;
  a.H = a.W = L.H;
  a.Cp = L.Cp;
  a.Ho = a.Wo = L.Ho;
  a.Cout = L.Cout_pad;
  a.NT = L.NT;
  a.Cout_tiles = L.Cout_pad / L.NT;
  a.nq = L.nq;
  a.pool = L.conv_pool;
  a.ksize = L.k;
  a.kchunks = L.kchunks;
  a.ksteps = L.ksteps;
  a.stages = L.stages;
  a.tmem_cols = L.tmem_cols;
  a.acc_bufs = L.acc_bufs;
  a.msub = L.msub;
  a.patch = L.patch;
  a.lag = env_int("FFSVA_TYOLO_LAG", 1);
  a.cp_shift = 0;
  while ((1 << a.cp_shift) < L.Cp) ++a.cp_shift;
  a.grid = m->ctx->num_sms;
  a.leaky = l < 8 ? 1 : 0;
  a.M = n * L.Ho * L.Ho;
  a.head = l == 8 ? 1 : 0;
  a.frames = m->d_frames;
  a.thresh = thresh;
  a.counts = m->d_counts;
  return a;
}

// Resize + layers [0, upto] for frames [0, n) (n <= cap), on stream st. ev (optional): 11 events around the
// resize and each layer. *out_buf receives the activation buffer holding the last layer's output.
ffsva_status run_chunk(ffsva_tyolo* m, const ffsva_frame* frames, const int32_t* targets, int n, int upto,
                       float thresh, cudaStream_t st, cudaEvent_t* ev, int* out_buf = nullptr) {
  DeviceCtx* ctx = m->ctx;
  int max_row = 0, max_H = 0;
  for (int i = 0; i < n; ++i) {
    const ffsva_stream_desc& d = frames[i].stream->desc;
    m->h_frames[i] = TyFrame{frames[i].pixels, d.row_pitch, d.width, d.height, targets ? targets[i] : 0, 0};
    max_row = std::max(max_row, 3 * d.width);
    max_H = std::max(max_H, d.height);
  }
  cudaError_t e = cudaMemcpyAsync(m->d_frames, m->h_frames, sizeof(TyFrame) * n, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemsetAsync(m->d_counts, 0, 4 * (size_t)n, st);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "T-YOLO staging");
  if (ev) cudaEventRecord(ev[0], st);
  if ((e = launch_tyolo_resize(m->d_frames, n, kIn, max_row, max_H, m->d_pad, st)) != cudaSuccess)
    return cuda_fail(ctx, e, "T-YOLO resize");
  g_launches += 1;
  if (ev) cudaEventRecord(ev[1], st);
  int cur = -1;  // -1: the padded resize output
  if (upto >= 0) {  // layer 1 by patch views of the padded input, into layer 2's planar padded input
    const TyL1Args a1{m->d_pad, m->d_pad2, 0, m->d_w1v, m->d_b + m->L[0].b_off, n};
    if ((e = launch_tyolo_l1(a1, ctx->num_sms, st)) != cudaSuccess) return cuda_fail(ctx, e, "T-YOLO layer 1");
    g_launches += 1;
    cur = -2;  // -2: the planar layer-1 output
    if (ev) cudaEventRecord(ev[2], st);
  }
  if (upto >= 1) {  // layer 2 by patch views
    const TyL1Args a2{m->d_pad2, m->d_ps[0], m->ps_plane[0], m->d_w2v, m->d_b + m->L[1].b_off, n};
    if ((e = launch_tyolo_l2(a2, ctx->num_sms, st)) != cudaSuccess) return cuda_fail(ctx, e, "T-YOLO layer 2");
    g_launches += 1;
    cur = -10;  // -10 - k: parity slab k (layer 3 + k's input)
    if (ev) cudaEventRecord(ev[3], st);
  }
  for (int l = 2; l <= upto; ++l) {
    if (l <= 4) {  // pool layers 3-5 by parity-slab views: slab 0 -> slab 1 -> slab 2 -> NHWC
      const Layer& L = m->L[l];
      const int k = l - 2;
      TyPslabArgs pa{};
      pa.in = m->d_ps[k];
      pa.plane = m->ps_plane[k];
      pa.out = l < 4 ? m->d_ps[k + 1] : m->d_slab[2];  // layer 5 writes layer 6's 13x13 slab input
      pa.out_plane = l < 4 ? m->ps_plane[k + 1] : m->slab_plane;
      pa.out_Gp = l < 4 ? kPsGp[k + 1] : -15;
      pa.wpk = m->d_wps[k];
      pa.bias = m->d_b + L.b_off;
      pa.N = n;
      pa.Cin = L.Cin;
      pa.Cout = L.Cout_pad;
      pa.Gp = kPsGp[k];
      if ((e = launch_tyolo_pslab(pa, ctx->num_sms, st)) != cudaSuccess)
        return cuda_fail(ctx, e, "T-YOLO parity-slab layer");
      g_launches += 1;
      cur = l < 4 ? -10 - (k + 1) : -5;  // -5: slab 2 (layer 5's output)
      if (ev) cudaEventRecord(ev[2 + l], st);
      continue;
    }
    if (l == 5) {  // 13x13 layer 6 by slab views (slab 2 -> NHWC), then its 2x2/1 max-pool (Q30) into slab 0
      const Layer& L = m->L[l];
      TySlabArgs sa{};
      sa.in = m->d_slab[2];
      sa.plane = m->slab_plane;
      sa.out = m->d_act[1];
      sa.out_plane = 0;
      sa.wpk = m->d_w + L.w_off;
      sa.bias = m->d_b + L.b_off;
      sa.N = n;
      sa.Cin = L.Cin;
      sa.Cout = L.Cout_pad;
      if ((e = launch_tyolo_slab(sa, ctx->num_sms, st)) != cudaSuccess) return cuda_fail(ctx, e, "T-YOLO slab layer");
      if ((e = launch_tyolo_pool_s1(m->d_act[1], m->d_slab[0], n, L.Ho, L.Cout_pad, m->slab_plane, st)) !=
          cudaSuccess)
        return cuda_fail(ctx, e, "T-YOLO 2x2/1 pool");
      g_launches += 2;
      cur = -3;  // -3: slab 0 (layer 6's pooled output)
      if (ev) cudaEventRecord(ev[2 + l], st);
      continue;
    }
    if (l == 6 || l == 7) {  // 13x13 layers 7 and 8 by slab views: slab 0 -> slab 1 -> NHWC
      const Layer& L = m->L[l];
      TySlabArgs sa{};
      sa.in = m->d_slab[l - 6];
      sa.plane = m->slab_plane;
      sa.out = l == 6 ? m->d_slab[1] : m->d_act[0];
      sa.out_plane = l == 6 ? m->slab_plane : 0;
      sa.wpk = m->d_w + L.w_off;
      sa.bias = m->d_b + L.b_off;
      sa.N = n;
      sa.Cin = L.Cin;
      sa.Cout = L.Cout_pad;
      if ((e = launch_tyolo_slab(sa, ctx->num_sms, st)) != cudaSuccess) return cuda_fail(ctx, e, "T-YOLO slab layer");
      g_launches += 1;
      cur = l == 6 ? -4 : 0;  // -4: slab 1 (layer 7's output)
      if (ev) cudaEventRecord(ev[2 + l], st);
      continue;
    }
    const TyConvArgs a = layer_args(m, l, n, m->d_act[cur], m->d_act[cur ^ 1], thresh);
    if ((e = launch_tyolo_conv(a, st)) != cudaSuccess) return cuda_fail(ctx, e, "T-YOLO conv layer");
    g_launches += 1;
    cur ^= 1;
    if (m->L[l].pool == 2) {  // 2x2/1 max-pool (Q30) into layer 7's slab input
      const Layer& L = m->L[l];
      if ((e = launch_tyolo_pool_s1(m->d_act[cur], m->d_slab[0], n, L.Ho, L.Cout_pad, m->slab_plane, st)) !=
          cudaSuccess)
        return cuda_fail(ctx, e, "T-YOLO 2x2/1 pool");
      g_launches += 1;
      cur = -3;  // -3: slab 0 (layer 6's pooled output)
    }
    if (ev) cudaEventRecord(ev[2 + l], st);
  }
  if (out_buf) *out_buf = cur;
  return FFSVA_OK;
}

ffsva_status validate(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n) {
  if (!m || n < 0 || (n > 0 && !frames)) return fail(FFSVA_EINVAL, "bad argument");
  begin_ptr_checks(m->ctx);
  for (int32_t i = 0; i < n; ++i) {
    if (!frames[i].stream || !frames[i].pixels) return fail(FFSVA_EINVAL, "frame without stream or pixels");
    if (frames[i].stream->ctx != m->ctx) return fail(FFSVA_EDEVICE, "frame lives on another device");
    const ffsva_stream_desc& d = frames[i].stream->desc;
    ffsva_status cs = check_device_ptr(m->ctx, frames[i].pixels, (size_t)(d.height - 1) * d.row_pitch + 3 * d.width);
    if (cs != FFSVA_OK) return cs;
  }
  if (m->ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  return FFSVA_OK;
}

}  // namespace

extern "C" {

FFSVA_API ffsva_status ffsva_tyolo_load(int32_t device, const float* params, int64_t n_params, ffsva_tyolo** out) {
  if (!params || !out) return fail(FFSVA_EINVAL, "NULL argument");
  std::unique_ptr<ffsva_tyolo> m(new ffsva_tyolo());
  build_layers(m.get());
  int64_t need = 0;
  for (auto& L : m->L) need += (int64_t)L.Cout * L.Cin * L.k * L.k + L.Cout;
  if (n_params != need) return fail(FFSVA_EINVAL, "n_params != 15,858,717 (tiny-yolo-voc)");
  for (int64_t i = 0; i < n_params; ++i)
    if (!std::isfinite(params[i])) return fail(FFSVA_EINVAL, "non-finite T-YOLO parameter");
  ffsva_status st;
  DeviceCtx* ctx = ctx_acquire(device, &st);
  if (!ctx) return st;
  m->ctx = ctx;
  size_t wbytes = 0, nb = 0;
  for (auto& L : m->L) {
    wbytes += L.w_bytes;
    nb += L.Cout_pad;
  }
  std::vector<uint8_t> hw(wbytes);
  std::vector<float> hb(nb, 0.f);
  const float* p = params;
  for (auto& L : m->L) {
    const size_t nw = (size_t)L.Cout * L.Cin * L.k * L.k;
    pack_layer(L, p, hw.data() + L.w_off);
    std::memcpy(hb.data() + L.b_off, p + nw, sizeof(float) * L.Cout);
    p += nw + L.Cout;
  }
  // layer 1 for the patch-view kernel: B of patch row dy = [K-half h][n = 16q + oc][k = 4(u & 1) + c], u = 2h + (k >> 2)
  // the patch column; pool position q = (qa, qb) puts the 3x3 kernel at patch offset (qa, qb)
  std::vector<uint16_t> w1v(4 * 2 * 64 * 8, 0);
  for (int dy = 0; dy < 4; ++dy)
    for (int q = 0; q < 4; ++q)
      for (int oc = 0; oc < 16; ++oc)
        for (int u = 0; u < 4; ++u)
          for (int c = 0; c < 3; ++c) {
            const int ky = dy - (q >> 1), kx = u - (q & 1);
            if (ky < 0 || ky > 2 || kx < 0 || kx > 2) continue;
            w1v[((dy * 2 + (u >> 1)) * 64 + 16 * q + oc) * 8 + 4 * (u & 1) + c] =
                bf16_bits(params[((oc * 3 + c) * 3 + ky) * 3 + kx]);
          }
  // layers 3-5 for the parity-slab kernel: [N tile of 64][64-channel group][tap][8-channel K group][64 n][8] (K groups
  // past Cin stay zero and are never read)
  std::vector<uint16_t> wps[3];
  {
    const float* wl = params;
    for (int l = 0; l < 5; ++l) {
      const Layer& L = m->L[l];
      if (l >= 2) {
        const int G = std::max(1, L.Cin / 64), nts = L.Cout / 64;
        std::vector<uint16_t>& v = wps[l - 2];
        v.assign((size_t)nts * G * 9 * 8 * 64 * 8, 0);
        for (int nt = 0; nt < nts; ++nt)
          for (int g = 0; g < G; ++g)
            for (int t = 0; t < 9; ++t)
              for (int kg = 0; kg < 8; ++kg)
                for (int nn = 0; nn < 64; ++nn)
                  for (int ee = 0; ee < 8; ++ee) {
                    const int c = 64 * g + 8 * kg + ee, oc = 64 * nt + nn;
                    if (c >= L.Cin) continue;
                    v[(((((size_t)nt * G + g) * 9 + t) * 8 + kg) * 64 + nn) * 8 + ee] =
                        bf16_bits(wl[(((size_t)oc * L.Cin + c) * 3 + t / 3) * 3 + t % 3]);
                  }
      }
      wl += (size_t)L.Cout * L.Cin * L.k * L.k + L.Cout;
    }
  }
  // layer 2 for the patch-view kernel: B of (patch row dy, column u) = [channel group g][n = 32q + oc][8 channels]
  std::vector<uint16_t> w2v(16 * 2 * 128 * 8, 0);
  {
    const float* w2 = params + 16 * 3 * 9 + 16;  // layer 2 follows layer 1's weights and biases
    for (int dy = 0; dy < 4; ++dy)
      for (int u = 0; u < 4; ++u)
        for (int q = 0; q < 4; ++q) {
          const int ky = dy - (q >> 1), kx = u - (q & 1);
          if (ky < 0 || ky > 2 || kx < 0 || kx > 2) continue;
          for (int oc = 0; oc < 32; ++oc)
            for (int c = 0; c < 16; ++c)
              w2v[(((dy * 4 + u) * 2 + (c >> 3)) * 128 + 32 * q + oc) * 8 + (c & 7)] =
                  bf16_bits(w2[((oc * 16 + c) * 3 + ky) * 3 + kx]);
        }
  }
  {
    std::lock_guard<std::mutex> lk(ctx->mu);
    DeviceGuard g(device);
    cudaError_t e = cudaMalloc(&m->d_w, wbytes);
    for (int k = 0; k < 3 && e == cudaSuccess; ++k) {
      e = cudaMalloc(&m->d_wps[k], wps[k].size() * 2);
      if (e == cudaSuccess) e = cudaMemcpy(m->d_wps[k], wps[k].data(), wps[k].size() * 2, cudaMemcpyHostToDevice);
    }
    if (e == cudaSuccess) e = cudaMalloc(&m->d_w2v, w2v.size() * 2);
    if (e == cudaSuccess) e = cudaMemcpy(m->d_w2v, w2v.data(), w2v.size() * 2, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMalloc(&m->d_w1v, w1v.size() * 2);
    if (e == cudaSuccess) e = cudaMemcpy(m->d_w1v, w1v.data(), w1v.size() * 2, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMalloc(&m->d_b, nb * 4);
    if (e == cudaSuccess) e = cudaMemcpy(m->d_w, hw.data(), wbytes, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemcpy(m->d_b, hb.data(), nb * 4, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = tyolo_configure();
    if (e != cudaSuccess) {
      cudaFree(m->d_w);
      cudaFree(m->d_w1v);
      cudaFree(m->d_w2v);
      for (auto& p : m->d_wps) cudaFree(p);
      cudaFree(m->d_b);
      ctx_release(ctx);
      return cuda_fail(nullptr, e, "ffsva_tyolo_load");
    }
  }
  *out = m.release();
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_tyolo_run(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n, int32_t target_class,
                                       float thresh, int32_t number_of_objects, int32_t* counts, uint8_t* pass,
                                       float* raw, void* cuda_stream) {
  if (target_class < 0 || target_class >= 20) return fail(FFSVA_EINVAL, "target_class must be a VOC class 0..19");
  if (n > 0 && !counts && !pass && !raw) return fail(FFSVA_EINVAL, "no output requested");
  if (!m) return fail(FFSVA_EINVAL, "bad argument");
  DeviceCtx* ctx = m->ctx;
  std::lock_guard<std::mutex> lk(ctx->mu);  // taken before validate(): it shares the device's pointer checks
  ffsva_status st = validate(m, frames, n);
  if (st != FFSVA_OK || n == 0) return st;
  DeviceGuard g(ctx->device);
  std::vector<int32_t> targets((size_t)n, target_class);
  return tyolo_run_unlocked(m, frames, n, targets.data(), thresh, number_of_objects, counts, pass, raw,
                            (cudaStream_t)cuda_stream);
}

}  // extern "C"

DeviceCtx* ffsva::tyolo_device_ctx(const ffsva_tyolo* m) { return m->ctx; }

// The run itself, for callers that already hold the device lock (ffsva_tyolo_run, the online runtime's T-YOLO
// cycle): frames in chunks of the workspace capacity, per-frame target classes.
ffsva_status ffsva::tyolo_run_unlocked(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n, const int32_t* targets,
                                       float thresh, int32_t number_of_objects, int32_t* counts, uint8_t* pass,
                                       float* raw, cudaStream_t cs) {
  DeviceCtx* ctx = m->ctx;
  ffsva_status st = ensure_workspace(m, n);
  if (st != FFSVA_OK) return st;
  for (int32_t i0 = 0; i0 < n; i0 += m->cap) {
    const int cnt = std::min(m->cap, n - i0);
    if ((st = run_chunk(m, frames + i0, targets + i0, cnt, 8, thresh, cs, nullptr)) != FFSVA_OK) return st;
    cudaError_t e = cudaMemcpyAsync(m->h_counts, m->d_counts, 4 * (size_t)cnt, cudaMemcpyDeviceToHost, cs);
    if (e == cudaSuccess && raw) {  // [cnt][13][13][125] from the 128-wide padded rows
      e = cudaMemcpy2DAsync(raw + (size_t)i0 * kGrid * kGrid * 125, 125 * 4, m->d_raw, kHeadPad * 4, 125 * 4,
                            (size_t)cnt * kGrid * kGrid, cudaMemcpyDeviceToHost, cs);
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_tyolo_run");
    for (int i = 0; i < cnt; ++i) {
      if (counts) counts[i0 + i] = m->h_counts[i];
      if (pass) pass[i0 + i] = m->h_counts[i] >= number_of_objects ? 1 : 0;  // L195 NumberofObjects
    }
  }
  return FFSVA_OK;
}

extern "C" {

FFSVA_API ffsva_status ffsva_tyolo_layer_output(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n, int32_t layer,
                                                uint16_t* out, void* cuda_stream) {
  if (layer < -1 || layer > 7 || !out) return fail(FFSVA_EINVAL, "layer must be -1 (resized input) .. 7");
  if (!m) return fail(FFSVA_EINVAL, "bad argument");
  DeviceCtx* ctx = m->ctx;
  std::lock_guard<std::mutex> lk(ctx->mu);  // taken before validate(): it shares the device's pointer checks
  ffsva_status st = validate(m, frames, n);
  if (st != FFSVA_OK || n == 0) return st;
  DeviceGuard g(ctx->device);
  if (n > kMaxChunk) return fail(FFSVA_EINVAL, "at most 256 frames");
  if ((st = ensure_workspace(m, n)) != FFSVA_OK) return st;
  cudaStream_t cs = (cudaStream_t)cuda_stream;
  int buf = 0;
  if ((st = run_chunk(m, frames, nullptr, n, layer, 0.2f, cs, nullptr, &buf)) != FFSVA_OK) return st;
  cudaError_t e = cudaSuccess;
  if (buf == -2) {  // layer 1: unpack the planar zero-bordered buffer [n][210][parity][group][105][8] on the host
    std::vector<uint16_t> pl((size_t)n * kTyL2PadBytes / 2);
    e = cudaMemcpyAsync(pl.data(), m->d_pad2, pl.size() * 2, cudaMemcpyDeviceToHost, cs);
    if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_tyolo_layer_output");
    const size_t row = kTyL2PadBytes / 210 / 2, plane = row / 4;  // in bf16 elements
    for (int i = 0; i < n; ++i)
      for (int y = 0; y < 208; ++y)
        for (int x = 0; x < 208; ++x)
          for (int c = 0; c < 16; ++c) {
            const int Y = y + 1, X = x + 1;
            out[(((size_t)i * 208 + y) * 208 + x) * 16 + c] =
                pl[((size_t)i * 210 + Y) * row + ((X & 1) * 2 + (c >> 3)) * plane + (X >> 1) * 8 + (c & 7)];
          }
    return FFSVA_OK;
  }
  if (buf <= -10) {  // parity slab k = -10 - buf: C = 32 / 64 / 128 channels of the H = 104 / 52 / 26 grid
    const int k = -10 - buf, C = kPsC[k], Gp = kPsGp[k], H = 2 * (Gp - 1);
    std::vector<uint16_t> ps((size_t)C / 8 * 4 * m->ps_plane[k] * 8);
    e = cudaMemcpyAsync(ps.data(), m->d_ps[k], ps.size() * 2, cudaMemcpyDeviceToHost, cs);
    if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_tyolo_layer_output");
    for (int i = 0; i < n; ++i)
      for (int y = 0; y < H; ++y)
        for (int x = 0; x < H; ++x)
          for (int c = 0; c < C; ++c) {
            const int Y = y + 1, X = x + 1;
            const size_t pl = (size_t)(c >> 3) * 4 + (Y & 1) * 2 + (X & 1);
            out[(((size_t)i * H + y) * H + x) * C + c] =
                ps[(pl * m->ps_plane[k] + (size_t)i * Gp * Gp + (Y >> 1) * Gp + (X >> 1)) * 8 + (c & 7)];
          }
    return FFSVA_OK;
  }
  if (buf == -3 || buf == -4 || buf == -5) {  // layers 6 / 7 / 5: unpack a 13x13 slab (planes of 8 channels)
    const int si = buf == -3 ? 0 : buf == -4 ? 1 : 2, C = si == 0 ? 512 : si == 1 ? 1024 : 256;
    std::vector<uint16_t> sl((size_t)C / 8 * m->slab_plane * 8);
    e = cudaMemcpyAsync(sl.data(), m->d_slab[si], sl.size() * 2, cudaMemcpyDeviceToHost, cs);
    if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_tyolo_layer_output");
    for (int i = 0; i < n; ++i)
      for (int y = 0; y < 13; ++y)
        for (int x = 0; x < 13; ++x)
          for (int c = 0; c < C; ++c)
            out[(((size_t)i * 13 + y) * 13 + x) * C + c] =
                sl[((size_t)(c >> 3) * m->slab_plane + (size_t)i * 225 + (y + 1) * 15 + x + 1) * 8 + (c & 7)];
    return FFSVA_OK;
  }
  if (buf == -1) {  // the resized input: the interior of the zero-bordered buffer
    const size_t row = (size_t)kIn * 4 * 2, prow = (size_t)(kIn + 2) * 4 * 2;
    for (int i = 0; i < n && e == cudaSuccess; ++i)
      e = cudaMemcpy2DAsync(out + (size_t)i * kIn * kIn * 4, row,
                            reinterpret_cast<const uint8_t*>(m->d_pad) + ((size_t)i * (kIn + 2) + 1) * prow + 4 * 2,
                            prow, row, kIn, cudaMemcpyDeviceToHost, cs);
  } else {
    const size_t bytes = (size_t)n * m->L[layer].Ho * m->L[layer].Ho * m->L[layer].Cout_pad * 2;
    e = cudaMemcpyAsync(out, m->d_act[buf], bytes, cudaMemcpyDeviceToHost, cs);
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
  if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_tyolo_layer_output");
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_tyolo_profile(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n, int32_t iters,
                                           float* ms_out, void* cuda_stream) {
  if (iters < 1 || !ms_out) return fail(FFSVA_EINVAL, "bad argument");
  if (!m) return fail(FFSVA_EINVAL, "bad argument");
  DeviceCtx* ctx = m->ctx;
  std::lock_guard<std::mutex> lk(ctx->mu);  // taken before validate(): it shares the device's pointer checks
  ffsva_status st = validate(m, frames, n);
  if (st != FFSVA_OK || n == 0) return st;
  if (n > kMaxChunk) return fail(FFSVA_EINVAL, "at most 256 frames per profiled chunk");
  DeviceGuard g(ctx->device);
  if ((st = ensure_workspace(m, n)) != FFSVA_OK) return st;
  cudaStream_t cs = (cudaStream_t)cuda_stream;
  cudaEvent_t ev[11];
  for (auto& e : ev) cudaEventCreate(&e);
  double acc[10] = {0};
  for (int it = 0; it < iters && st == FFSVA_OK; ++it) {
    st = run_chunk(m, frames, nullptr, n, 8, 0.2f, cs, ev);
    if (st != FFSVA_OK) break;
    cudaError_t e = cudaEventSynchronize(ev[10]);
    if (e != cudaSuccess) {
      st = cuda_fail(ctx, e, "ffsva_tyolo_profile");
      break;
    }
    for (int k = 0; k < 10; ++k) {
      float t = 0.f;
      cudaEventElapsedTime(&t, ev[k], ev[k + 1]);
      acc[k] += t;
    }
  }
  for (auto& e : ev) cudaEventDestroy(e);
  if (st != FFSVA_OK) return st;
  for (int k = 0; k < 10; ++k) ms_out[k] = (float)(acc[k] / iters);
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_tyolo_destroy(ffsva_tyolo* m) {
  if (!m) return FFSVA_OK;
  DeviceCtx* ctx = m->ctx;
  {
    std::lock_guard<std::mutex> lk(ctx->mu);
    DeviceGuard g(ctx->device);
    cudaDeviceSynchronize();
    cudaFree(m->d_w);
    cudaFree(m->d_b);
    cudaFree(m->d_act[0]);
    cudaFree(m->d_act[1]);
    cudaFree(m->d_pad);
    cudaFree(m->d_w1v);
    cudaFree(m->d_pad2);
    cudaFree(m->d_w2v);
    for (auto& p : m->d_slab) cudaFree(p);
    for (auto& p : m->d_ps) cudaFree(p);
    for (auto& p : m->d_wps) cudaFree(p);
    cudaFree(m->d_raw);
    cudaFree(m->d_counts);
    cudaFree(m->d_frames);
    cudaFreeHost(m->h_frames);
    cudaFreeHost(m->h_counts);
  }
  delete m;
  ctx_release(ctx);
  return FFSVA_OK;
}

}  // extern "C"
