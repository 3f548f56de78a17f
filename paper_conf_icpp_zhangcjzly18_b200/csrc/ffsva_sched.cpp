// ffsva_sched.cpp — online runtime: the FFS-VA queue policy (ffsva_sched_policy.h) driving K1 -> K3 -> K4.
//
// One tick = one SDD cycle + one SNM cycle (§4.3):
//   1. admit SDD-queued frames (feedback: streams whose SNM queue is over q_snm wait), give each a D50 slot;
//   2. K1 writes each admitted frame's 50x50 image into its slot, K3 thresholds the SSD per frame;
//   3. survivors join their stream's SNM queue, dropped frames become events and free their slot;
//   4. every non-empty SNM queue pops min(BatchSize, depth) (dynamic batching); K4 scores all pops in one
//      launch, reading the images from their slots; scored frames become events and free their slots.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstring>
#include <deque>
#include <memory>
#include <unordered_map>
#include <vector>

#include <cstdlib>

#include "ffsva_runtime.h"
#include "ffsva_sched_policy.h"

using namespace ffsva;

namespace {
constexpr int64_t kD50Stride = 7504;
int64_t now_us() {
  return std::chrono::duration_cast<std::chrono::microseconds>(std::chrono::steady_clock::now().time_since_epoch())
      .count();
}
size_t al256(size_t x) { return (x + 255) & ~(size_t)255; }

// Per-cycle staging: one pinned host block mirrored by one device block (a single H2D per stage).
struct Layout {
  size_t desc, index, work, chunks, counts, seg_lo, seg_batch, seg_slot, pop_start, xb, yb, total;
  explicit Layout(size_t n) {
    size_t o = 0;
    desc = o; o += al256(64 * n);
    index = o; o += al256(4 * n);
    work = o; o += al256(4 * n);
    chunks = o; o += al256(4 * (n + 1));
    counts = o; o += al256(16);
    seg_lo = o; o += al256(4 * (n + 1));
    seg_batch = o; o += al256(4 * n);
    seg_slot = o; o += al256(4 * n);
    pop_start = o; o += al256(n);
    xb = o; o += al256(4 * 4097);  // cell boundary tables of a cycle whose frames share W / H (grids <= 4096)
    yb = o; o += al256(4 * 4097);
    total = o;
  }
};
}  // namespace

struct ffsva_sched {
  DeviceCtx* ctx = nullptr;
  std::mutex mu;
  sched::Policy pol;
  std::vector<int32_t> id_of_slot;  // stream slot -> policy id (O(1) per pushed frame)
  std::vector<ffsva_stream*> by_id;
  int32_t lookup(const ffsva_stream* st) const {
    if (st->slot < 0 || st->slot >= (int32_t)id_of_slot.size()) return -1;
    const int32_t id = id_of_slot[st->slot];
    return (id >= 0 && id < (int32_t)by_id.size() && by_id[id] == st) ? id : -1;
  }
  int32_t max_frames = 0, slots = 0, cap = 0;
  int32_t sdd_w = -1, sdd_h = -1;
  std::vector<int32_t> free_slots;
  uint8_t* d_pool = nullptr;  // [slots][7504] D50 images of frames between SDD and SNM
  uint8_t* d_in = nullptr;    // Layout(cap) mirror of h_in
  uint8_t* h_in = nullptr;
  // device scratch / outputs
  void* d_mem = nullptr;
  int32_t *d_perm = nullptr, *d_posw = nullptr, *d_surv = nullptr;
  unsigned long long* d_acc = nullptr;
  uint8_t* d_out = nullptr;   // ssd u64[cap] | logit f32[cap] | pass u8[cap] | snm_pass u8[cap] | snm_class u8[cap]
  uint8_t* h_out = nullptr;   // 2 result buffers (15 * cap bytes each): a cycle's D2H lands in h_out + hb * 15 * cap
  uint8_t* h_out_cur = nullptr;  // the launching cycle's result buffer (enqueue_*_stage)
  // events not yet returned: pending[pend_head ..) (a vector with a consumed prefix, reset when drained)
  std::vector<ffsva_event> pending;
  size_t pend_head = 0;
  std::vector<sched::QFrame> adm;   // this cycle's SDD admissions, reused
  std::vector<sched::QFrame> flat;  // this cycle's SNM pops, reused
  std::vector<int32_t> starts;
  // pipelined mode (ffsva_sched_set_pipeline): the kernels tick k launches are harvested by tick k + 1, so the
  // caller's work between ticks and the next cycle's host preparation overlap them. Host staging and host result
  // buffers are double buffered (hb; the in-flight cycle's is f_hb), the device staging holds separate SDD and SNM
  // regions (stream order separates consecutive cycles). Without a T-YOLO stage tick k launches cycle k before it
  // waits for and harvests cycle k-1, so the GPU never idles on the harvest.
  bool pipelined = false, inflight = false;
  int32_t hb = 0, f_hb = 0;
  cudaEvent_t ev[2] = {nullptr, nullptr};  // ev[b]: the cycle launched with buffers b has finished
  std::vector<sched::QFrame> f_adm, f_flat;  // the in-flight cycle's admissions and pops
  // T-YOLO stage (f1): the device's shared model, its per-cycle extraction and score threshold
  ffsva_tyolo* tyolo = nullptr;
  float ty_thresh = 0.2f;
  std::vector<sched::QFrame> tyflat;
  // per-stage CUDA graphs (updated in place tick to tick); FFSVA_SCHED_GRAPH=0 launches directly (A/B)
  bool use_graph = true;
  cudaGraphExec_t g_sdd = nullptr, g_snm = nullptr;
};

namespace {

void sched_free(ffsva_sched* s) {
  if (s->g_sdd) cudaGraphExecDestroy(s->g_sdd);
  if (s->g_snm) cudaGraphExecDestroy(s->g_snm);
  for (cudaEvent_t e : s->ev)
    if (e) cudaEventDestroy(e);
  cudaFree(s->d_pool);
  cudaFree(s->d_in);
  cudaFree(s->d_mem);
  cudaFreeHost(s->h_in);
  cudaFreeHost(s->h_out);
}

FrameDesc make_desc(const ffsva_stream* st, const void* pixels) {
  FrameDesc d{};
  d.pixels = (const uint8_t*)pixels;
  d.ref = st->d_ref;
  d.snm = st->d_snm;
  d.pitch = st->desc.row_pitch;
  d.T = st->T;
  d.W = st->desc.width;
  d.H = st->desc.height;
  d.L_t = st->L_t;
  d.L_low = st->L_low;
  d.L_high = st->L_high;
  d.slot = (uint16_t)st->slot;
  d.metric = (uint8_t)st->desc.distance;
  d.mode = (uint8_t)st->desc.ref_mode;
  return d;
}

template <typename T>
T* at(uint8_t* base, size_t off) { return reinterpret_cast<T*>(base + off); }

// ---------------------------------------------------------------- cycle phases (shared by both tick modes)
struct SddStage {
  int32_t na = 0, nseg = 0, sdd_w = 0, sdd_h = 0;
  int32_t uni_W = -1, uni_H = -1;  // the admitted frames' common width / height (-1: mixed)
  SddPlan plan;
};
struct SnmStage {
  int32_t m = 0, nch = 0;
};

// SDD admission (feedback: streams whose SNM queue is over q_snm wait) into host staging h: one D50 slot per
// admitted frame, frame descriptors, per-stream segments (admitted frames arrive grouped by stream).
SddStage prep_sdd(ffsva_sched* s, uint8_t* h, const Layout& L, std::vector<sched::QFrame>& adm) {
  NvtxRange r("ffsva sched: SDD admission");
  SddStage sd;
  adm = s->pol.admit_sdd(s->max_frames, (int32_t)s->free_slots.size());
  sd.na = (int32_t)adm.size();
  if (sd.na == 0) return sd;
  FrameDesc* hd = at<FrameDesc>(h, L.desc);
  int32_t* hidx = at<int32_t>(h, L.index);
  int32_t* hseg = at<int32_t>(h, L.seg_lo);
  int32_t* hsegb = at<int32_t>(h, L.seg_batch);
  int32_t* hsegs = at<int32_t>(h, L.seg_slot);
  sd.sdd_w = s->by_id[adm[0].stream]->desc.sdd_w;
  sd.sdd_h = s->by_id[adm[0].stream]->desc.sdd_h;
  for (int32_t i = 0; i < sd.na; ++i) {
    const ffsva_stream* st = s->by_id[adm[i].stream];
    adm[i].slot = s->free_slots.back();
    s->free_slots.pop_back();
    hd[i] = make_desc(st, adm[i].pixels);
    hidx[i] = adm[i].slot;
    if (i == 0 || adm[i].stream != adm[i - 1].stream) {
      hseg[sd.nseg] = i;
      hsegb[sd.nseg] = st->desc.snm_batch;
      hsegs[sd.nseg] = st->slot;
      ++sd.nseg;
    }
    sdd_plan_add(sd.plan, st->desc.width, st->desc.height, st->desc.row_pitch, adm[i].pixels, sd.sdd_h);
  }
  hseg[sd.nseg] = sd.na;
  sdd_plan_finish(sd.plan, sd.sdd_w, sd.sdd_h);
  // cell boundary tables (C1) when every admitted frame has the same width / height: K1 then reads its row and
  // column bounds without waiting for its frame descriptor (as prepared batches do)
  sd.uni_W = s->by_id[adm[0].stream]->desc.width;
  sd.uni_H = s->by_id[adm[0].stream]->desc.height;
  for (int32_t i = 1; i < sd.na && (sd.uni_W > 0 || sd.uni_H > 0); ++i) {
    const ffsva_stream_desc& d = s->by_id[adm[i].stream]->desc;
    if (d.width != sd.uni_W) sd.uni_W = -1;
    if (d.height != sd.uni_H) sd.uni_H = -1;
  }
  if (sd.uni_W > 0) {
    int32_t* hxb = at<int32_t>(h, L.xb);
    for (int32_t i = 0; i <= sd.sdd_w; ++i) hxb[i] = (int32_t)(((int64_t)i * sd.uni_W) / sd.sdd_w);
  }
  if (sd.uni_H > 0) {
    int32_t* hyb = at<int32_t>(h, L.yb);
    for (int32_t i = 0; i <= sd.sdd_h; ++i) hyb[i] = (int32_t)(((int64_t)i * sd.uni_H) / sd.sdd_h);
  }
  return sd;
}

// Upload the SDD staging (used parts only) into device region d, launch K1 (D50 into the slots) and K3 (threshold),
// queue the D2H of distances and pass flags into h_out. Asynchronous on cs.
cudaError_t enqueue_sdd_stage(ffsva_sched* s, uint8_t* h, uint8_t* d, const Layout& L, const SddStage& sd,
                              cudaStream_t cs) {
  DeviceCtx* ctx = s->ctx;
  const size_t n = (size_t)s->cap;
  const int32_t na = sd.na, nseg = sd.nseg;
  cudaError_t e = cudaMemcpyAsync(d + L.desc, h + L.desc, 64 * (size_t)na, cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(d + L.index, h + L.index, 4 * (size_t)na, cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(d + L.seg_lo, h + L.seg_lo, 4 * (size_t)(nseg + 1), cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(d + L.seg_batch, h + L.seg_batch, 4 * (size_t)nseg, cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(d + L.seg_slot, h + L.seg_slot, 4 * (size_t)nseg, cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess && sd.uni_W > 0)
    e = cudaMemcpyAsync(d + L.xb, h + L.xb, 4 * (size_t)(sd.sdd_w + 1), cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess && sd.uni_H > 0)
    e = cudaMemcpyAsync(d + L.yb, h + L.yb, 4 * (size_t)(sd.sdd_h + 1), cudaMemcpyHostToDevice, cs);
  SddArgs sa{};
  sa.frames = at<FrameDesc>(d, L.desc);
  sa.n = na;
  sa.sdd_w = sd.sdd_w;
  sa.sdd_h = sd.sdd_h;
  sa.d50 = s->d_pool;
  sa.d50_stride = kD50Stride;
  sa.d50_index = at<int32_t>(d, L.index);
  sa.acc_ssd = s->d_acc;
  sa.stats = ctx->d_stats;
  sdd_plan_apply(sd.plan, sa);
  sa.uni_W = sd.uni_W;
  sa.uni_H = sd.uni_H;
  sa.cellw = sd.uni_W > 0 ? (sd.uni_W + sd.sdd_w - 1) / sd.sdd_w : 0;
  sa.xbounds = sd.uni_W > 0 ? at<int32_t>(d, L.xb) : nullptr;
  sa.ybounds = sd.uni_H > 0 ? at<int32_t>(d, L.yb) : nullptr;
  if (e == cudaSuccess) e = launch_sdd(sa, cs);
  CompactArgs ca{};  // threshold + per-stream SDD-pass stats; the SNM stage forms its own pops (snm_ctas = 0)
  ca.frames = sa.frames;
  ca.acc_ssd = s->d_acc;
  ca.ssd = at<uint64_t>(s->d_out, 0);
  ca.pass = s->d_out + 12 * n;
  ca.n = na;
  ca.perm = s->d_perm;
  ca.seg_lo = at<int32_t>(d, L.seg_lo);
  ca.n_seg = nseg;
  ca.seg_batch = at<int32_t>(d, L.seg_batch);
  ca.seg_slot = at<int32_t>(d, L.seg_slot);
  ca.stats = ctx->d_stats;
  ca.snm_ctas = 0;
  ca.survivor_idx = s->d_surv;
  ca.work = at<int32_t>(d, L.work);
  ca.posw = s->d_posw;
  ca.chunks = at<int32_t>(d, L.chunks);
  ca.counts = at<int32_t>(d, L.counts);
  ca.logit = at<float>(s->d_out, 8 * n);
  ca.snm_pass = s->d_out + 13 * n;
  ca.snm_class = s->d_out + 14 * n;
  if (e == cudaSuccess) e = launch_compact(ca, cs);
  g_launches += 2;
  if (e == cudaSuccess) e = cudaMemcpyAsync(at<uint64_t>(s->h_out_cur, 0), ca.ssd, 8 * (size_t)na, cudaMemcpyDeviceToHost, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(s->h_out_cur + 12 * n, ca.pass, (size_t)na, cudaMemcpyDeviceToHost, cs);
  return e;
}

// SDD results (in result buffer hout) of admissions adm[0, na): survivors join their SNM queue, dropped frames
// become events.
void harvest_sdd(ffsva_sched* s, const uint8_t* hout, std::vector<sched::QFrame>& adm, int32_t na,
                 ffsva_tick_info& ti) {
  NvtxRange r("ffsva sched: SDD harvest");
  const size_t n = (size_t)s->cap;
  const uint64_t* h_ssd = reinterpret_cast<const uint64_t*>(hout);
  const uint8_t* h_pass = hout + 12 * n;
  const int64_t t_now = now_us();
  for (int32_t i = 0; i < na; ++i) {
    adm[i].ssd = h_ssd[i];
    s->pol.sdd_done(adm[i], h_pass[i] != 0);
    if (h_pass[i]) {
      ++ti.sdd_pass;
      continue;
    }
    ffsva_event ev{};
    ev.stream = s->by_id[adm[i].stream];
    ev.frame_no = adm[i].frame_no;
    ev.result.ssd = h_ssd[i];
    ev.result.logit = NAN;
    ev.result.survivor_idx = -1;
    ev.result.tyolo_count = -1;
    s->pending.push_back(ev);
    s->free_slots.push_back(adm[i].slot);
    record_latency(s->ctx, ev.stream->slot, t_now - adm[i].t_push_us);
  }
}

// SNM cycle: dynamic batching (pops of min(BatchSize, depth) per stream; or the static / feedback-queue fixed-size
// trigger chosen by ffsva_sched_set_policy) into host staging h.
SnmStage prep_snm(ffsva_sched* s, uint8_t* h, const Layout& L, std::vector<sched::QFrame>& flat,
                  std::vector<int32_t>& starts, ffsva_tick_info& ti) {
  SnmStage sn;
  s->pol.pop_snm(flat, starts, (int32_t)s->free_slots.size());
  sn.m = (int32_t)flat.size();
  ti.snm_batches = (int32_t)starts.size() - 1;
  ti.snm_scored = sn.m;
  if (sn.m == 0) return sn;
  const int32_t m = sn.m;
  FrameDesc* hd = at<FrameDesc>(h, L.desc);
  int32_t* hidx = at<int32_t>(h, L.index);
  int32_t* hwork = at<int32_t>(h, L.work);
  int32_t* hch = at<int32_t>(h, L.chunks);
  int32_t* hcnt = at<int32_t>(h, L.counts);
  uint8_t* hpop = h + L.pop_start;
  int32_t nch = 0;
  for (size_t p = 0; p + 1 < starts.size(); ++p) {
    const ffsva_stream* st = s->by_id[flat[starts[p]].stream];
    const FrameDesc d = make_desc(st, nullptr);
    for (int32_t j = starts[p]; j < starts[p + 1]; ++j) {
      const int32_t k = j - starts[p];
      if (k == 0) {  // one chunk per pop (K4 counts SNM_BATCHES per chunk that opens a pop)
        hpop[nch] = 1;
        hch[nch++] = j;
      }
      hd[j] = d;
      hidx[j] = flat[j].slot;
      hwork[j] = j;
    }
  }
  hch[nch] = m;
  hcnt[0] = m;
  hcnt[1] = nch;
  hcnt[2] = 0;
  hcnt[3] = 0;
  sn.nch = nch;
  return sn;
}

// Upload the SNM staging into device region d, launch K4 on the popped frames' slots, queue the D2H of logits,
// decisions and classes into h_out. Asynchronous on cs.
cudaError_t enqueue_snm_stage(ffsva_sched* s, uint8_t* h, uint8_t* d, const Layout& L, const SnmStage& sn,
                              cudaStream_t cs) {
  const size_t n = (size_t)s->cap;
  const int32_t m = sn.m, nch = sn.nch;
  cudaError_t e = cudaMemcpyAsync(d + L.desc, h + L.desc, 64 * (size_t)m, cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(d + L.index, h + L.index, 4 * (size_t)m, cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(d + L.work, h + L.work, 4 * (size_t)m, cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(d + L.chunks, h + L.chunks, 4 * (size_t)(nch + 1), cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(d + L.counts, h + L.counts, 16, cudaMemcpyHostToDevice, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(d + L.pop_start, h + L.pop_start, (size_t)nch, cudaMemcpyHostToDevice, cs);
  SnmArgs na{};
  na.frames = at<FrameDesc>(d, L.desc);
  na.d50 = s->d_pool;
  na.d50_stride = kD50Stride;
  na.d50_index = at<int32_t>(d, L.index);
  na.work = at<int32_t>(d, L.work);
  na.chunks = at<int32_t>(d, L.chunks);
  na.counts = at<int32_t>(d, L.counts);
  na.pop_start = d + L.pop_start;
  na.logit = at<float>(s->d_out, 8 * n);
  na.snm_pass = s->d_out + 13 * n;
  na.snm_class = s->d_out + 14 * n;
  na.stats = s->ctx->d_stats;
  na.grid = std::max(1, std::min(m, kSnmCtasPerSm * s->ctx->num_sms));  // K4: per-CTA ranges of the m pops' frames
  if (e == cudaSuccess) e = launch_snm(na, cs);
  g_launches += 1;
  if (e == cudaSuccess) e = cudaMemcpyAsync(at<float>(s->h_out_cur, 8 * n), na.logit, 4 * (size_t)m, cudaMemcpyDeviceToHost, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(s->h_out_cur + 13 * n, na.snm_pass, (size_t)m, cudaMemcpyDeviceToHost, cs);
  if (e == cudaSuccess) e = cudaMemcpyAsync(s->h_out_cur + 14 * n, na.snm_class, (size_t)m, cudaMemcpyDeviceToHost, cs);
  return e;
}

// A stage's copies and kernels as a CUDA graph (SURVEY.md §3 "steady-state ticks are replayed as a captured CUDA
// graph"): the tick's enqueue is captured, the stage's instantiated graph is updated in place when the topology
// matches (only parameters change from tick to tick: counts, grids, staging offsets) or re-instantiated otherwise,
// and launched as one unit. The legacy NULL stream cannot be captured: ticks on it enqueue directly.
template <typename F>
cudaError_t graph_launch(cudaGraphExec_t& exec, cudaStream_t cs, F&& enqueue) {
  cudaGraph_t g = nullptr;
  cudaError_t e = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal);
  if (e != cudaSuccess) return e;
  const cudaError_t fe = enqueue();
  e = cudaStreamEndCapture(cs, &g);
  if (fe != cudaSuccess) {
    if (g) cudaGraphDestroy(g);
    return fe;
  }
  if (e != cudaSuccess) return e;
  if (exec) {
    cudaGraphExecUpdateResultInfo info;
    if (cudaGraphExecUpdate(exec, g, &info) != cudaSuccess) {  // topology changed: instantiate afresh
      cudaGetLastError();
      cudaGraphExecDestroy(exec);
      exec = nullptr;
    }
  }
  if (!exec) e = cudaGraphInstantiate(&exec, g, 0);
  cudaGraphDestroy(g);
  if (e == cudaSuccess) e = cudaGraphLaunch(exec, cs);
  return e;
}

cudaError_t launch_sdd_stage(ffsva_sched* s, uint8_t* h, uint8_t* d, const Layout& L, const SddStage& sd,
                             cudaStream_t cs) {
  NvtxRange r("ffsva sched: SDD stage launch");
  cudaError_t e = sdd_configure(sd.plan.smem);  // a function attribute: outside any capture
  if (e != cudaSuccess) return e;
  if (!s->use_graph || cs == nullptr) return enqueue_sdd_stage(s, h, d, L, sd, cs);
  return graph_launch(s->g_sdd, cs, [&] { return enqueue_sdd_stage(s, h, d, L, sd, cs); });
}

cudaError_t launch_snm_stage(ffsva_sched* s, uint8_t* h, uint8_t* d, const Layout& L, const SnmStage& sn,
                             cudaStream_t cs) {
  NvtxRange r("ffsva sched: SNM stage launch");
  if (!s->use_graph || cs == nullptr) return enqueue_snm_stage(s, h, d, L, sn, cs);
  return graph_launch(s->g_snm, cs, [&] { return enqueue_snm_stage(s, h, d, L, sn, cs); });
}

// SNM results (in result buffer hout) of pops flat[0, m): slots are freed; survivors with a T-YOLO stage wait in its
// queue, every other frame becomes an event.
void harvest_snm(ffsva_sched* s, const uint8_t* hout, std::vector<sched::QFrame>& flat, int32_t m) {
  NvtxRange r("ffsva sched: SNM harvest");
  const size_t n = (size_t)s->cap;
  const float* h_logit = reinterpret_cast<const float*>(hout + 8 * n);
  const uint8_t* h_snm_pass = hout + 13 * n;
  const uint8_t* h_snm_class = hout + 14 * n;
  const int64_t t_now = now_us();
  for (int32_t k = 0; k < m; ++k) {
    s->free_slots.push_back(flat[k].slot);
    flat[k].logit = h_logit[k];
    flat[k].snm_class = h_snm_class[k];
    if (s->pol.snm_done(flat[k], h_snm_pass[k] != 0)) continue;  // waits in the stream's T-YOLO queue
    ffsva_event ev{};
    ev.stream = s->by_id[flat[k].stream];
    ev.frame_no = flat[k].frame_no;
    ev.result.ssd = flat[k].ssd;
    ev.result.sdd_pass = 1;
    ev.result.snm_pass = h_snm_pass[k];
    ev.result.snm_class = h_snm_class[k];
    ev.result.logit = h_logit[k];
    ev.result.survivor_idx = -1;
    ev.result.tyolo_count = -1;
    s->pending.push_back(ev);
    record_latency(s->ctx, ev.stream->slot, t_now - flat[k].t_push_us);
  }
}

// T-YOLO cycle (f1): at most num_t-yolo frames from each T-YOLO queue (L173), counted with the shared model;
// NumberofObjects per stream (L195). Synchronous on cs.
ffsva_status tyolo_cycle(ffsva_sched* s, cudaStream_t cs, ffsva_tick_info& ti) {
  if (!s->tyolo) return FFSVA_OK;
  NvtxRange r("ffsva sched: T-YOLO cycle");
  std::vector<sched::QFrame>& tf = s->tyflat;
  s->pol.pop_ty(tf);
  const int32_t nt = (int32_t)tf.size();
  ti.tyolo_scored = nt;
  if (nt == 0) return FFSVA_OK;
  std::vector<ffsva_frame> fr((size_t)nt);
  std::vector<int32_t> targets((size_t)nt), counts((size_t)nt);
  for (int32_t i = 0; i < nt; ++i) {
    ffsva_stream* st = s->by_id[tf[i].stream];
    fr[i] = ffsva_frame{st, (const uint8_t*)tf[i].pixels, tf[i].frame_no};
    targets[i] = st->desc.target_class;
  }
  ffsva_status ts = tyolo_run_unlocked(s->tyolo, fr.data(), nt, targets.data(), s->ty_thresh, 0, counts.data(),
                                       nullptr, nullptr, cs);
  if (ts != FFSVA_OK) return ts;
  const int64_t t_now = now_us();
  for (int32_t i = 0; i < nt; ++i) {
    const ffsva_stream* st = s->by_id[tf[i].stream];
    ffsva_event ev{};
    ev.stream = s->by_id[tf[i].stream];
    ev.frame_no = tf[i].frame_no;
    ev.result.ssd = tf[i].ssd;
    ev.result.sdd_pass = 1;
    ev.result.snm_pass = 1;
    ev.result.snm_class = tf[i].snm_class;
    ev.result.logit = tf[i].logit;
    ev.result.survivor_idx = -1;
    ev.result.tyolo_count = counts[i];
    ev.result.tyolo_pass = counts[i] >= st->desc.number_of_objects ? 1 : 0;
    s->pending.push_back(ev);
    record_latency(s->ctx, st->slot, t_now - tf[i].t_push_us);
  }
  return FFSVA_OK;
}

}  // namespace

extern "C" {

FFSVA_API ffsva_status ffsva_sched_create(int32_t device, int32_t max_frames_per_tick, int32_t snm_slots,
                                          ffsva_sched** out) {
  if (!out || max_frames_per_tick < 1 || snm_slots < 1) return fail(FFSVA_EINVAL, "bad argument");
  ffsva_status st;
  DeviceCtx* ctx = ctx_acquire(device, &st);  // the scheduler holds a context reference until destroyed
  if (!ctx) return st;
  std::unique_ptr<ffsva_sched> s(new ffsva_sched());
  s->ctx = ctx;
  s->max_frames = max_frames_per_tick;
  s->slots = snm_slots;
  s->cap = std::max(max_frames_per_tick, snm_slots);
  const size_t n = (size_t)s->cap;
  const Layout L(n);
  DeviceGuard g(device);
  const size_t o_perm = 0, o_posw = al256(4 * n), o_surv = o_posw + al256(4 * (n + 1)),
               o_acc = o_surv + al256(4 * n), o_out = o_acc + al256(8 * n), total = o_out + al256(15 * n);
  cudaError_t e = cudaMalloc(&s->d_mem, total);
  if (e == cudaSuccess) e = cudaMalloc(&s->d_pool, (size_t)snm_slots * kD50Stride);
  if (e == cudaSuccess) e = cudaMalloc(&s->d_in, 2 * L.total);       // SDD region | SNM region
  if (e == cudaSuccess) e = cudaMallocHost(&s->h_in, 4 * L.total);   // 2 buffers x (SDD | SNM)
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&s->ev[0], cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&s->ev[1], cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaMallocHost(&s->h_out, 2 * 15 * n);
  s->h_out_cur = s->h_out;
  if (e == cudaSuccess) {
    uint8_t* b = (uint8_t*)s->d_mem;
    s->d_perm = at<int32_t>(b, o_perm);
    s->d_posw = at<int32_t>(b, o_posw);
    s->d_surv = at<int32_t>(b, o_surv);
    s->d_acc = at<unsigned long long>(b, o_acc);
    s->d_out = b + o_out;
    std::vector<int32_t> ident(n);
    for (size_t i = 0; i < n; ++i) ident[i] = (int32_t)i;
    e = cudaMemcpy(s->d_perm, ident.data(), 4 * n, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemset(s->d_acc, 0, 8 * n);
  }
  if (e != cudaSuccess) {
    sched_free(s.get());
    ctx_release(ctx);
    return cuda_fail(nullptr, e, "ffsva_sched_create");
  }
  for (int32_t i = snm_slots - 1; i >= 0; --i) s->free_slots.push_back(i);
  if (const char* g = std::getenv("FFSVA_SCHED_GRAPH")) s->use_graph = std::atoi(g) != 0;
  *out = s.release();
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_destroy(ffsva_sched* s) {
  if (!s) return FFSVA_OK;
  DeviceCtx* ctx = s->ctx;
  {
    DeviceGuard g(ctx->device);
    cudaDeviceSynchronize();
    sched_free(s);
  }
  delete s;
  ctx_release(ctx);
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_push(ffsva_sched* s, const ffsva_frame* frames, int32_t n, uint8_t* accepted) {
  if (!s || n < 0 || (n > 0 && (!frames || !accepted))) return fail(FFSVA_EINVAL, "bad argument");
  std::lock_guard<std::mutex> lk(s->mu);
  begin_ptr_checks(s->ctx);
  for (int32_t i = 0; i < n; ++i) {  // validate everything before queueing anything
    ffsva_stream* st = frames[i].stream;
    if (!st || !frames[i].pixels) return fail(FFSVA_EINVAL, "frame without stream or pixels");
    if (st->ctx != s->ctx) return fail(FFSVA_EDEVICE, "stream lives on another device");
    // every frame's bytes must be device memory of this device (K1's bulk copies and the T-YOLO resize read them);
    // the range cache makes this one lookup per frame after the first of each allocation
    {
      const ffsva_stream_desc& d = st->desc;
      ffsva_status cs = check_device_ptr(s->ctx, frames[i].pixels, (size_t)(d.height - 1) * d.row_pitch + 3 * d.width);
      if (cs != FFSVA_OK) return cs;
    }
    // an attached stream passed every check below when it attached (its descriptor is immutable, and a reference
    // or SNM, once loaded, stays): consecutive frames of one stream are checked once
    if (i > 0 && st == frames[i - 1].stream) continue;
    if (st->ctx == s->ctx && s->lookup(st) >= 0) continue;
    if (st->ctx != s->ctx) return fail(FFSVA_EDEVICE, "stream lives on another device");
    if (!st->has_ref || !st->has_snm) return fail(FFSVA_ESTATE, "stream has no reference image or no SNM");
    if (st->desc.snm_w != snm::IN || st->desc.snm_h != snm::IN) return fail(FFSVA_EINVAL, "SNM grid must be 50x50");
    if (st->desc.ref_mode != FFSVA_REF_BACKGROUND)
      return fail(FFSVA_EINVAL, "the online scheduler takes background-reference streams only");
    if (s->sdd_w < 0) {  // one SDD grid per scheduler (one K1 launch per cycle)
      s->sdd_w = st->desc.sdd_w;
      s->sdd_h = st->desc.sdd_h;
    }
    if (st->desc.sdd_w != s->sdd_w || st->desc.sdd_h != s->sdd_h)
      return fail(FFSVA_EINVAL, "streams of one scheduler must share the SDD grid");
  }
  const int64_t t_push = now_us();
  for (int32_t i = 0; i < n; ++i) {
    ffsva_stream* st = frames[i].stream;
    int32_t id = s->lookup(st);
    if (id < 0) {
      id = s->pol.add_stream(st->desc.q_sdd, st->desc.q_snm, st->desc.snm_batch, st->desc.q_tyolo);
      if ((int32_t)s->by_id.size() <= id) s->by_id.resize(id + 1, nullptr);
      s->by_id[id] = st;
      if ((int32_t)s->id_of_slot.size() <= st->slot) s->id_of_slot.resize(st->slot + 1, -1);
      s->id_of_slot[st->slot] = id;
    }
    sched::QFrame q;
    q.frame_no = frames[i].frame_no;
    q.pixels = frames[i].pixels;
    q.t_push_us = t_push;
    accepted[i] = s->pol.push(id, q) ? 1 : 0;
  }
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_depth(ffsva_sched* s, ffsva_stream* st, int32_t* sdd_depth, int32_t* snm_depth) {
  if (!s || !st) return fail(FFSVA_EINVAL, "bad argument");
  std::lock_guard<std::mutex> lk(s->mu);
  const int32_t id = s->lookup(st);
  if (sdd_depth) *sdd_depth = id < 0 ? 0 : (int32_t)s->pol.stream(id).sdd.size();
  if (snm_depth) *snm_depth = id < 0 ? 0 : (int32_t)s->pol.stream(id).snm.size();
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_stream_load(ffsva_sched* s, ffsva_stream* st, int32_t reset,
                                               ffsva_stream_load* out) {
  if (!s || !st || !out) return fail(FFSVA_EINVAL, "bad argument");
  std::lock_guard<std::mutex> lk(s->mu);
  std::memset(out, 0, sizeof(*out));
  const int32_t id = s->lookup(st);
  if (id < 0) return FFSVA_OK;  // not attached: idle
  const sched::StreamQ& q = s->pol.stream(id);
  out->sdd_depth = (int32_t)q.sdd.size();
  out->snm_depth = (int32_t)q.snm.size();
  out->max_sdd = q.max_sdd;
  out->max_snm = q.max_snm;
  out->pushed = q.pushed;
  out->refused = q.refused;
  out->sdd_blocked = q.sdd_blocked;
  out->tyolo_depth = (int32_t)q.ty.size();
  out->max_tyolo = q.max_ty;
  out->snm_blocked = q.snm_blocked;
  if (reset) s->pol.reset_counters(id);
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_detach(ffsva_sched* s, ffsva_stream* st) {
  if (!s || !st) return fail(FFSVA_EINVAL, "bad argument");
  std::lock_guard<std::mutex> lk(s->mu);
  const int32_t id = s->lookup(st);
  if (id < 0) return FFSVA_OK;
  const sched::StreamQ& q = s->pol.stream(id);
  if (!q.sdd.empty() || !q.snm.empty() || !q.ty.empty()) return fail(FFSVA_EAGAIN, "stream still has queued frames");
  for (size_t i = s->pend_head; i < s->pending.size(); ++i)
    if (s->pending[i].stream == st) return fail(FFSVA_EAGAIN, "stream still has unreported events");
  if (s->inflight) {
    for (const sched::QFrame& q : s->f_adm)
      if (q.stream == id) return fail(FFSVA_EAGAIN, "stream has frames in flight");
    for (const sched::QFrame& q : s->f_flat)
      if (q.stream == id) return fail(FFSVA_EAGAIN, "stream has frames in flight");
  }
  s->pol.remove_stream(id);
  s->by_id[id] = nullptr;
  s->id_of_slot[st->slot] = -1;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_set_tyolo(ffsva_sched* s, ffsva_tyolo* m, int32_t num_tyolo, float thresh) {
  if (!s || (m && num_tyolo < 1) || !(thresh >= 0.f && thresh <= 1.f)) return fail(FFSVA_EINVAL, "bad argument");
  if (m && tyolo_device_ctx(m) != s->ctx) return fail(FFSVA_EDEVICE, "T-YOLO model lives on another device");
  std::lock_guard<std::mutex> lk(s->mu);
  if (!m && s->pol.queued_ty() > 0) return fail(FFSVA_EAGAIN, "frames still wait in T-YOLO queues");
  s->tyolo = m;
  s->ty_thresh = thresh;
  s->pol.set_tyolo(m != nullptr, num_tyolo);
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_set_policy(ffsva_sched* s, int32_t policy) {
  if (!s || policy < FFSVA_BATCH_DYNAMIC || policy > FFSVA_BATCH_STATIC) return fail(FFSVA_EINVAL, "bad argument");
  std::lock_guard<std::mutex> lk(s->mu);
  s->pol.set_policy((sched::BatchPolicy)policy);
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_set_pipeline(ffsva_sched* s, int32_t on) {
  if (!s) return fail(FFSVA_EINVAL, "bad argument");
  std::lock_guard<std::mutex> lk(s->mu);
  if (!on && s->inflight) return fail(FFSVA_EAGAIN, "a cycle is still in flight (tick once more)");
  s->pipelined = on != 0;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_tick(ffsva_sched* s, void* cuda_stream, ffsva_event* events, int32_t cap,
                                        int32_t* n_events, ffsva_tick_info* info) {
  if (!s || cap < 0 || (cap > 0 && !events) || !n_events) return fail(FFSVA_EINVAL, "bad argument");
  std::lock_guard<std::mutex> lk(s->mu);
  NvtxRange nvtx_tick("ffsva_sched_tick");
  DeviceCtx* ctx = s->ctx;
  if (ctx->sticky) return fail(FFSVA_ECUDA, "device is in a sticky CUDA error state");
  std::lock_guard<std::mutex> dlk(ctx->mu);
  DeviceGuard g(ctx->device);
  cudaStream_t cs = (cudaStream_t)cuda_stream;
  const Layout L((size_t)s->cap);
  ffsva_tick_info ti{};
  const auto t_tick0 = std::chrono::steady_clock::now();
  const uint64_t blocked0 = s->pol.total_sdd_blocked(), snm_blocked0 = s->pol.total_snm_blocked();
  uint8_t* const d_sdd = s->d_in;
  uint8_t* const d_snm = s->d_in + L.total;
  ffsva_status st = FFSVA_OK;
  std::chrono::steady_clock::time_point t_snm0, t_ty0;

  const size_t out_bytes = 15 * (size_t)s->cap;
  if (!s->pipelined) {
    // ---------------- synchronous cycle: SDD (launch, wait, harvest), then SNM on the updated queues
    uint8_t* hs = s->h_in;
    uint8_t* hn = s->h_in + L.total;
    s->h_out_cur = s->h_out;
    SddStage sd = prep_sdd(s, hs, L, s->adm);
    ti.admitted = sd.na;
    if (sd.na > 0) {
      cudaError_t e = launch_sdd_stage(s, hs, d_sdd, L, sd, cs);
      if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
      if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_sched_tick (SDD cycle)");
      harvest_sdd(s, s->h_out, s->adm, sd.na, ti);
    }
    t_snm0 = std::chrono::steady_clock::now();
    SnmStage sn = prep_snm(s, hn, L, s->flat, s->starts, ti);
    if (sn.m > 0) {
      cudaError_t e = launch_snm_stage(s, hn, d_snm, L, sn, cs);
      if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
      if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_sched_tick (SNM cycle)");
      harvest_snm(s, s->h_out, s->flat, sn.m);
    }
    t_ty0 = std::chrono::steady_clock::now();
    if ((st = tyolo_cycle(s, cs, ti)) != FFSVA_OK) return st;
  } else {
    // ---------------- pipelined cycle: prepare this cycle on the host while the previous one runs; without a
    // T-YOLO stage launch it at once, then wait for and harvest the previous one (its results are in the other
    // result buffer); with one, harvest first (the T-YOLO cycle runs on the previous cycle's SNM survivors before
    // this cycle's kernels are queued behind it)
    uint8_t* hs = s->h_in + (size_t)(2 * s->hb) * L.total;
    uint8_t* hn = hs + L.total;
    SddStage sd = prep_sdd(s, hs, L, s->adm);
    ti.admitted = sd.na;
    SnmStage sn = prep_snm(s, hn, L, s->flat, s->starts, ti);
    const bool launch = sd.na > 0 || sn.m > 0;
    auto launch_cycle = [&]() -> cudaError_t {
      s->h_out_cur = s->h_out + (size_t)s->hb * out_bytes;
      cudaError_t e = cudaSuccess;
      if (sd.na > 0) e = launch_sdd_stage(s, hs, d_sdd, L, sd, cs);
      if (e == cudaSuccess && sn.m > 0) e = launch_snm_stage(s, hn, d_snm, L, sn, cs);
      if (e == cudaSuccess) e = cudaEventRecord(s->ev[s->hb], cs);
      return e;
    };
    const bool early = launch && s->tyolo == nullptr;
    if (early) {
      cudaError_t e = launch_cycle();
      if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_sched_tick (launch)");
    }
    if (s->inflight) {
      cudaError_t e = cudaEventSynchronize(s->ev[s->f_hb]);
      if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_sched_tick (in-flight cycle)");
      const uint8_t* hout = s->h_out + (size_t)s->f_hb * out_bytes;
      harvest_sdd(s, hout, s->f_adm, (int32_t)s->f_adm.size(), ti);
      harvest_snm(s, hout, s->f_flat, (int32_t)s->f_flat.size());
      s->inflight = false;
    }
    t_snm0 = std::chrono::steady_clock::now();
    t_ty0 = t_snm0;
    if ((st = tyolo_cycle(s, cs, ti)) != FFSVA_OK) return st;
    if (launch) {
      if (!early) {
        cudaError_t e = launch_cycle();
        if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_sched_tick (launch)");
      }
      s->f_adm.swap(s->adm);
      s->f_adm.resize((size_t)sd.na);
      s->f_flat.swap(s->flat);
      s->f_flat.resize((size_t)sn.m);
      s->f_hb = s->hb;
      s->inflight = true;
      s->hb ^= 1;
    }
  }
  const auto t_ty1 = std::chrono::steady_clock::now();

  ti.sdd_blocked = (int32_t)(s->pol.total_sdd_blocked() - blocked0);
  int32_t k = 0;
  {
    const size_t avail = s->pending.size() - s->pend_head;
    k = (int32_t)std::min<size_t>((size_t)cap, avail);
    if (k > 0) std::memcpy(events, s->pending.data() + s->pend_head, sizeof(ffsva_event) * (size_t)k);
    s->pend_head += (size_t)k;
    if (s->pend_head == s->pending.size()) {
      s->pending.clear();
      s->pend_head = 0;
    }
  }
  *n_events = k;
  ti.sdd_queued = s->pol.queued_sdd();
  ti.snm_queued = s->pol.queued_snm();
  ti.tyolo_queued = s->pol.queued_ty();
  ti.snm_blocked = (int32_t)(s->pol.total_snm_blocked() - snm_blocked0);
  ti.tyolo_ms = std::chrono::duration<float, std::milli>(t_ty1 - t_ty0).count();
  // in-flight frames count as pending events (they will be reported by a later tick)
  ti.events_pending = (int64_t)(s->pending.size() - s->pend_head) + (s->inflight ? (int64_t)(s->f_adm.size() + s->f_flat.size()) : 0);
  const auto t_end = std::chrono::steady_clock::now();
  ti.sdd_ms = std::chrono::duration<float, std::milli>(t_snm0 - t_tick0).count();
  ti.snm_ms = std::chrono::duration<float, std::milli>(t_ty0 - t_snm0).count();
  ti.host_ms = std::chrono::duration<float, std::milli>(t_end - t_tick0).count();
  if (info) *info = ti;
  return FFSVA_OK;
}

FFSVA_API ffsva_status ffsva_sched_inspect(ffsva_sched* s, ffsva_frame* frames, int32_t* stage, uint8_t* d50,
                                           int32_t cap, int32_t* n) {
  if (!s || !n || cap < 0 || (cap > 0 && (!frames || !stage || !d50))) return fail(FFSVA_EINVAL, "bad argument");
  std::lock_guard<std::mutex> lk(s->mu);
  DeviceCtx* ctx = s->ctx;
  std::lock_guard<std::mutex> dlk(ctx->mu);
  DeviceGuard g(ctx->device);
  // the last launched cycle: synchronous mode keeps its admissions / pops in adm / flat; pipelined mode in f_adm /
  // f_flat while in flight (their slots are freed only at the next tick's harvest)
  const std::vector<sched::QFrame>* lists[2] = {&s->adm, &s->flat};
  if (s->pipelined) {
    if (!s->inflight) {
      *n = 0;
      return FFSVA_OK;
    }
    lists[0] = &s->f_adm;
    lists[1] = &s->f_flat;
  }
  cudaError_t e = s->pipelined ? cudaEventSynchronize(s->ev[s->f_hb]) : cudaSuccess;
  int32_t k = 0;
  for (int st = 0; st < 2 && e == cudaSuccess; ++st)
    for (const sched::QFrame& q : *lists[st]) {
      if (k < cap) {
        frames[k] = ffsva_frame{s->by_id[q.stream], (const uint8_t*)q.pixels, q.frame_no};
        stage[k] = st;
        e = cudaMemcpy(d50 + (size_t)k * 7500, s->d_pool + (size_t)q.slot * kD50Stride, 7500, cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) break;
      }
      ++k;
    }
  if (e != cudaSuccess) return cuda_fail(ctx, e, "ffsva_sched_inspect");
  *n = k;
  return FFSVA_OK;
}

}  // extern "C"
