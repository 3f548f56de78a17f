// ffsva_runtime.h — host runtime of the product library (internal).
#pragma once

#include <atomic>
#include <mutex>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "ffsva.h"
#include "ffsva_internal.h"

namespace ffsva {

struct DeviceCtx;

// Error reporting: every public entry point funnels through these.
void set_error(const std::string& msg);
ffsva_status fail(ffsva_status st, const std::string& msg);
ffsva_status cuda_fail(DeviceCtx* ctx, cudaError_t e, const char* what);
extern std::atomic<uint64_t> g_launches;

// One camera stream (SDD and SNM are specialised per stream).
struct StreamState {
  ffsva_stream_desc desc{};
  DeviceCtx* ctx = nullptr;
  int32_t slot = -1;
  uint8_t* d_ref = nullptr;   // R [sdd_h][sdd_w][3]
  uint8_t* d_snm = nullptr;   // packed SNM weight image (snm::BLOB_BYTES)
  bool has_ref = false, has_snm = false;
  uint64_t T = 0;             // SDD threshold on the distance numerator (ffsva_distance)
  uint64_t ref_sum_sq = 0;    // sum R^2 of the reference (NRMSE normaliser)
  float L_t = 0.f, L_low = 0.f, L_high = 0.f;
};

// A prepared batch: device descriptors + all per-batch device buffers; owns a CUDA graph of its kernels.
struct Batch {
  DeviceCtx* ctx = nullptr;
  int32_t n = 0, cap = 0;
  int32_t sdd_w = 0, sdd_h = 0, n_seg = 0;
  bool sdd_only = false, want_d100 = false;
  SddPlan plan;               // K1 variant and its shared-memory layout (sdd_plan_*)
  int32_t uni_W = -1, uni_H = -1;        // common frame size of the batch (-1: mixed)
  int32_t *d_xb = nullptr, *d_yb = nullptr;  // cell boundary tables for uni_W / uni_H (in the input block)
  int32_t *d_pm = nullptr, *d_last = nullptr;  // PREVIOUS-mode plan (input block): (frame, prev) pairs, last frames
  int32_t n_pm = 0, n_last = 0;
  int64_t d50_stride = 0;
  // device buffers (carved from one allocation)
  void* d_mem = nullptr;
  size_t d_bytes = 0;
  FrameDesc* d_desc = nullptr;
  int32_t *d_perm = nullptr, *d_seg_lo = nullptr, *d_seg_batch = nullptr;
  uint8_t* d_d50 = nullptr;
  uint8_t* d_d100 = nullptr;
  unsigned long long* d_acc = nullptr;  // per-frame SSD accumulators (K1 adds, K3 reads + re-zeroes)
  int32_t *d_work = nullptr, *d_posw = nullptr, *d_chunks = nullptr, *d_counts = nullptr;
  // output block (one D2H): ssd u64[n] | logit f32[n] | survivor_idx i32[n] | sdd_pass u8[n] | snm_pass u8[n] |
  // snm_class u8[n]
  uint8_t* d_out = nullptr;
  uint64_t* d_ssd = nullptr;
  float* d_logit = nullptr;
  int32_t* d_surv = nullptr;
  uint8_t *d_pass = nullptr, *d_snm_pass = nullptr, *d_snm_class = nullptr;
  size_t out_bytes = 0;
  // host pinned staging: inputs (desc|perm|seg_lo|seg_batch) and outputs
  uint8_t* h_in = nullptr;
  size_t in_bytes = 0;
  uint8_t* h_out = nullptr;
  // graph
  cudaGraphExec_t graph = nullptr;
  int graph_kernels = 0;
};

struct DeviceCtx {
  int device = 0;
  std::mutex mu;
  int num_sms = 148;
  int nstreams = 0;
  std::vector<int32_t> free_slots;
  int32_t next_slot = 0;
  unsigned long long* d_stats = nullptr;  // [stats_cap][NSTAT] (kernel counters)
  std::mutex lat_mu;                      // guards h_lat (the online runtime records under its own lock)
  std::vector<uint64_t> h_lat;            // [stats_cap][NLAT] (online arrival -> decision latency, a8)
  // pinned snapshot of h_lat for ffsva_stats_copy into device memory: the copy stays asynchronous (no host sync on
  // the caller's stream, e.g. inside a timed region); lat_ev guards the snapshot until its copy has run
  uint64_t* h_lat_pinned = nullptr;
  cudaEvent_t lat_ev = nullptr;
  int32_t stats_cap = 0;
  bool sticky = false;
  Batch* scratch = nullptr;  // reusable batch for ffsva_filter_batch / ffsva_sdd_batch
  // staging ring for host-resident frames (ffsva_filter_batch_host)
  uint8_t* d_ring = nullptr;
  size_t ring_bytes = 0;
  cudaStream_t copy_stream = nullptr;
  // known device allocations [base, base + size) on this device (pointer validation cache). Guarded by its own
  // mutex: the online runtime validates pushed frames under the scheduler's lock, not the device lock. An entry is
  // trusted only within the validation epoch that last confirmed it with the driver (begin_ptr_checks starts an
  // epoch per API call), so a range the caller freed or re-allocated since is looked up again.
  struct Range {
    uintptr_t base;
    size_t size;
    uint64_t epoch;
  };
  std::mutex ranges_mu;
  std::vector<Range> ranges;
  uint64_t range_epoch = 1;
  size_t range_mru = 0;
};

// device context registry
DeviceCtx* ctx_acquire(int device, ffsva_status* st);  // creates lazily, increments nstreams
void ctx_release(DeviceCtx* ctx);                       // decrements; destroys at 0

// helpers
ffsva_status check_device_ptr(DeviceCtx* ctx, const void* p, size_t bytes);
void begin_ptr_checks(DeviceCtx* ctx);   // new validation epoch: cached ranges are re-confirmed once on next use
void clear_ptr_cache(DeviceCtx* ctx);
ffsva_status ensure_stats(DeviceCtx* ctx, int32_t slots);
// a8: one decided frame of stream slot `slot` with arrival -> decision latency `us` (columns 8..23)
void record_latency(DeviceCtx* ctx, int32_t slot, int64_t us);
int latency_bin(int64_t us);
uint64_t exact_threshold(double delta, uint64_t n_values);
uint64_t exact_threshold_sq(double delta, uint64_t q);  // floor(delta^2 * q), exact (NRMSE, Q24)
uint64_t stream_threshold(const ffsva_stream_desc& d, uint64_t ref_sum_sq);  // T of the stream's metric
uint16_t bf16_bits_rne(float x);
void pack_snm_blob(const float* params, uint8_t* blob);
float logit_of(double t);

// batches
ffsva_status batch_build(DeviceCtx* ctx, Batch* b, const ffsva_frame* frames, int32_t n, bool sdd_only,
                         bool want_d100, cudaStream_t st);
ffsva_status batch_run(Batch* b, cudaStream_t st, bool use_graph);
ffsva_status batch_fetch(Batch* b, ffsva_result* results, cudaStream_t st);
ffsva_status batch_profile(Batch* const* batches, int32_t nb, int32_t iters, float* ms_out, cudaStream_t st);
void batch_free(Batch* b);
SddArgs make_sdd_args(Batch* b, int32_t i0, int32_t cnt);  // K1 over frames [i0, i0 + cnt) of the batch
CompactArgs make_compact_args(Batch* b);
SnmArgs make_snm_args(Batch* b);
PrevArgs make_prev_args(Batch* b);
int prev_launches(const Batch* b);  // kernels launch_prev issues for this batch (0, 1 or 2)

// T-YOLO (ffsva_tyolo_host.cpp): run the shared model on n frames with per-frame target classes; the caller holds
// the device lock. counts / pass / raw (host) may be NULL.
DeviceCtx* tyolo_device_ctx(const ffsva_tyolo* m);
ffsva_status tyolo_run_unlocked(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n, const int32_t* targets,
                                float thresh, int32_t number_of_objects, int32_t* counts, uint8_t* pass, float* raw,
                                cudaStream_t cs);

// NVTX range (header-only NVTX3: a no-op unless a tool such as ncu / nsys injects itself)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

// RAII device switch
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

}  // namespace ffsva

struct ffsva_stream : ffsva::StreamState {};
struct ffsva_batch : ffsva::Batch {};
