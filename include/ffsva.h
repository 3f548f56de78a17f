/*
 * ffsva.h — C-ABI of the B200-native FFS-VA prepositive filter cascade (SDD + SNM).
 *
 * The method (Zhang et al., "FFS-VA: A Fast Filtering System for Large-scale Video Analytics", ICPP 2018;
 * /root/reference/PAPER.md line numbers) filters the frames of many concurrent surveillance streams:
 *   SDD  (§3.2.1): downsample each frame to 100x100 (L155, L187), distance to the stream's
 *        reference image (average of background frames, L151) by MSE, drop the frame if MSE <= delta_diff;
 *   queue (L143 §3.1.2): survivors go to the stream's SNM queue in arrival order;
 *   SNM  (L157-L167 §3.2.2): a per-stream three-layer CNN (CONV, CONV, FC; L159) on a 50x50 resize (L167)
 *        outputs the probability c of the target; frames with c >= t_pre pass (L165), where
 *        t_pre = (c_high - c_low) * FilterDegree + c_low (Eq. (2));
 *   dynamic batching (L219-L223 §4.3.2): each SNM cycle pops min(BatchSize, queue depth) frames of a stream.
 * Exact readings of what the paper leaves open are in DESIGN.md "Readings".
 *
 * Conventions for every function:
 *   - returns ffsva_status: FFSVA_OK (0) or a negative error; ffsva_last_error() describes the last error of
 *     the calling thread;
 *   - all argument validation happens before any GPU work; on error nothing is written to outputs;
 *   - FFSVA_ECUDA is sticky per device: after it the caller should close that device's streams;
 *   - calls for one device are serialised by a per-device mutex; a stream handle must not be closed while a
 *     batch that uses it is in flight. Handles are owned by the library.
 *   - frame pixels are RGB8, HWC interleaved, `height` rows of 3*width bytes, rows `row_pitch` bytes apart.
 *     When row_pitch and the pixel pointer are both multiples of 16 the kernels use 16-byte loads and may read
 *     up to row_pitch bytes of every row (so the buffer must hold height*row_pitch bytes); otherwise a
 *     byte-load path reads exactly 3*width bytes per row.
 * The library has no CPU fallback: without a usable sm_100 device every compute call returns FFSVA_ECUDA.
 */
#ifndef FFSVA_H
#define FFSVA_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define FFSVA_API __attribute__((visibility("default")))
#else
#define FFSVA_API
#endif

typedef enum {
  FFSVA_OK = 0,
  FFSVA_EINVAL = -1,  /* bad argument or descriptor */
  FFSVA_ENOMEM = -2,  /* device or pinned host allocation failed */
  FFSVA_ECUDA = -3,   /* CUDA error (sticky per device) or no usable device */
  FFSVA_ESTATE = -4,  /* a frame's stream has no reference image or no SNM loaded */
  FFSVA_EAGAIN = -5,  /* online mode: the stream's SDD queue is over its feedback threshold (L209, L217) */
  FFSVA_EDEVICE = -6  /* frames of one batch live on different devices */
} ffsva_status;

typedef struct ffsva_stream ffsva_stream; /* opaque, owned by the library */
typedef struct ffsva_batch ffsva_batch;   /* opaque prepared batch, owned by the library */
typedef struct ffsva_tyolo ffsva_tyolo;   /* opaque shared T-YOLO model of a device (f1) */

/* Per-stream configuration (SDD and SNM are specialised per stream; L183 thresholds per stream). */
typedef struct {
  int32_t device;          /* CUDA ordinal holding the stream's state and frames */
  int32_t width, height;   /* raw frame size; sdd_w <= width <= 16384, sdd_h <= height <= 256*sdd_h */
  int64_t row_pitch;       /* bytes between rows, >= 3*width */
  int32_t sdd_w, sdd_h;    /* SDD grid, 100 x 100 (L155); even, 2 <= sdd <= 4096 */
  int32_t snm_w, snm_h;    /* SNM grid, 50 x 50 (L167); must equal sdd/2 (the 50-grid cells are unions of
                              2x2 100-grid cells, so one pass produces both resizes) */
  double delta_diff;       /* distance threshold (L151), >= 0; for MSE: pass iff SSD > floor(delta_diff * 3*sdd_w*sdd_h),
                              i.e. iff MSE > delta_diff exactly (other metrics: ffsva_distance) */
  float c_low, c_high;     /* SNM class thresholds (L159), 0 <= c_low <= c_high <= 1 */
  float filter_degree;     /* Eq. (2) (L193); must lie in [0, 1] ("cases t_pre < c_low, t_pre > c_high are not
                              considered") */
  int32_t snm_batch;       /* BatchSize (L219-L223), >= 1; default 30 */
  int32_t q_sdd, q_snm;    /* feedback-queue depth thresholds in frames (L217), default 2 and 10 */
  int32_t distance;        /* SDD distance (L151 "MSE, NRMSE, or SAD"), an ffsva_distance; 0 = MSE */
  int32_t ref_mode;        /* SDD reference (L151), an ffsva_ref_mode; 0 = background reference image */
  int32_t number_of_objects; /* NumberofObjects (L195): the T-YOLO stage keeps a frame iff it counts at least this
                                many target objects; >= 0 (online runtime with a T-YOLO model attached) */
  int32_t target_class;    /* the stream's target object, a VOC class 0..19 for T-YOLO (L139: "the target events to
                              detect, such as the occurrences of cars, persons, etc. ... are predefined by users") */
  int32_t q_tyolo;         /* T-YOLO queue depth threshold in frames (L217), default 2 */
} ffsva_stream_desc;

/* SDD distance metrics ("The distance between two video frames can be characterized by Mean
 * Square Error (MSE), Normalized Root Mean Square Error (NRMSE), or Sum of Absolute Differences (SAD)").
 * D = the frame's sdd_h x sdd_w x 3 resize, R = the reference, N = 3*sdd_w*sdd_h values. ffsva_result.ssd
 * carries the integer distance numerator the threshold is applied to; every test is exact (Q5,
 * Q23, Q24):
 *   MSE   : ssd = sum (D-R)^2;  pass iff ssd/N > delta_diff          <=> ssd > floor(delta_diff * N)
 *   SAD   : ssd = sum |D-R|;    pass iff ssd > delta_diff            <=> ssd > floor(delta_diff)
 *   NRMSE : ssd = sum (D-R)^2;  pass iff sqrt(ssd / sum R^2) > delta_diff <=> ssd > floor(delta_diff^2 * sum R^2)
 *           (Euclidean normalisation; the threshold is recomputed by every ffsva_set_reference. Prepared batches
 *           snapshot it at ffsva_batch_prepare.) */
typedef enum { FFSVA_DIST_MSE = 0, FFSVA_DIST_SAD = 1, FFSVA_DIST_NRMSE = 2 } ffsva_distance;

/* SDD reference (the reference image "is usually computed as the average of dozens of background
 * frames"; Q25 for the alternative):
 *   BACKGROUND: R is the image ffsva_set_reference built; it changes only when that is called again.
 *   PREVIOUS  : each frame is compared with the resize of its stream's previous frame. Within a batch
 *               "previous" follows input order among the stream's frames; the first frame of a batch uses R,
 *               and after the batch R holds the resize of the stream's last frame of that batch (so consecutive
 *               batches chain, and ffsva_set_reference seeds the first comparison). MSE and SAD only (NRMSE's
 *               normaliser would change per frame: EINVAL); batch API only (the online scheduler rejects it). */
typedef enum { FFSVA_REF_BACKGROUND = 0, FFSVA_REF_PREVIOUS = 1 } ffsva_ref_mode;

/* SNM topology (L159: CONV, CONV, FC). The kernels implement c1 = 16, c2 = 32 on a 50x50 input. */
typedef struct {
  int32_t c1, c2;
} ffsva_snm_desc;

/* One input frame of a batch. `pixels` is a device pointer on the stream's device. */
typedef struct {
  ffsva_stream* stream;
  const uint8_t* pixels;
  int64_t frame_no;        /* caller's frame number (carried through, not interpreted) */
} ffsva_frame;

/* Per-frame result, in input order. */
typedef struct {
  uint64_t ssd;            /* SDD distance numerator over the 3*sdd_w*sdd_h values: sum (D100 - R)^2 (MSE, NRMSE;
                              MSE = ssd / (3*sdd_w*sdd_h)) or sum |D100 - R| (SAD) — see ffsva_distance */
  uint8_t sdd_pass;        /* 1 iff the distance exceeds delta_diff (L151), e.g. MSE > delta_diff */
  uint8_t snm_pass;        /* 1 iff sdd_pass and c >= t_pre (L165) */
  uint8_t snm_class;       /* 0: c < c_low, 1: unsure, 2: c > c_high (L159); 0 if !sdd_pass */
  uint8_t tyolo_pass;      /* online runtime with T-YOLO: 1 iff tyolo_count >= NumberofObjects (L195); else 0 */
  float logit;             /* SNM output logit, c = 1/(1+exp(-logit)); NaN if !sdd_pass */
  int32_t survivor_idx;    /* rank among this batch's SDD survivors in input order, -1 if !sdd_pass */
  int32_t tyolo_count;     /* target objects T-YOLO counted (L171); -1 if the frame did not reach T-YOLO */
  int32_t reserved;
} ffsva_result;

/* Counters per stream slot, ffsva_stats_copy() layout: u64[slots][FFSVA_NSTAT] (a8; the per-filter frame ratios of
 * PAPER.md L253 Fig. 5 and the arrival -> decision latency of the online runtime). Columns 0-7 are kept by the
 * kernels (batch and online paths alike); columns 8-23 by the online runtime (ffsva_sched_*): a frame "arrives"
 * when ffsva_sched_push accepts it and is "decided" when the tick that reports its event harvests it (dropped by
 * SDD, scored by SNM, or counted by T-YOLO). Latency bins: bin 0 < 1 ms, bin k (1..12) in [2^(k-1), 2^k) ms,
 * bin 13 >= 4096 ms. */
enum {
  FFSVA_STAT_FRAMES = 0,   /* frames through SDD */
  FFSVA_STAT_SDD_PASS = 1, /* SDD survivors */
  FFSVA_STAT_SNM_PASS = 2, /* SNM survivors (c >= t_pre) */
  FFSVA_STAT_SSD_SUM = 3,  /* sum of SSD over all frames */
  FFSVA_STAT_CLASS0 = 4,   /* SNM class counts (L159) */
  FFSVA_STAT_CLASS1 = 5,
  FFSVA_STAT_CLASS2 = 6,
  FFSVA_STAT_SNM_BATCHES = 7, /* SNM weight loads = dynamic batches executed (L219) */
  FFSVA_STAT_DECIDED = 8,  /* online runtime: frames whose fate was reported (= sum of the latency bins) */
  FFSVA_STAT_LAT_SUM_US = 9, /* online runtime: sum of their arrival -> decision latencies, microseconds */
  FFSVA_STAT_LAT_BIN0 = 10, /* 14 latency bins, columns 10..23 */
  FFSVA_NSTAT = 24
};

/* Create a stream (a camera) with its own SDD/SNM state on desc->device. The first stream of a device creates
 * the device context (lazy); the last close destroys it. *out receives the handle. Errors: EINVAL (bad desc,
 * out NULL), ECUDA, ENOMEM. */
FFSVA_API ffsva_status ffsva_open_stream(const ffsva_stream_desc* desc, ffsva_stream** out);

/* Build the stream's SDD reference image R ("average of dozens of background frames"): k >= 1
 * background frames, frame j at frames + j*frame_stride (host or device memory; frame_stride >= height*pitch;
 * each frame laid out like the stream's frames). R = round-half-up of the mean over all k*box samples of each
 * 100-grid cell (one rounding). The input is copied; the caller may free it on return. Synchronous. */
FFSVA_API ffsva_status ffsva_set_reference(ffsva_stream* s, const uint8_t* frames, int32_t k, int64_t frame_stride);

/* Load the stream's SNM parameters (host fp32, packed w1[c1][3][3][3], b1[c1], w2[c2][c1][3][3], b2[c2],
 * wfc[c2*12*12], bfc[1]; n_params = 27c1 + c1 + 9c1c2 + c2 + 144c2 + 1 = 9697 for 16/32). The weights w1, w2,
 * wfc are rounded to bf16 (RNE) at load; biases stay fp32. Copied; synchronous. Errors: EINVAL (d not 16/32,
 * n_params mismatch, NULL). */
FFSVA_API ffsva_status ffsva_snm_load(ffsva_stream* s, const ffsva_snm_desc* d, const float* params,
                                      int64_t n_params);

/* Run the whole cascade on n frames and write n results (host memory, input order). Synchronous on
 * cuda_stream (NULL = legacy default stream). Frames may come from any mix of open streams of ONE device and
 * any mix of resolutions; survivors of one stream are scored in dynamic batches of at most snm_batch frames
 * (L223). Errors: EINVAL, ESTATE, EDEVICE, ECUDA, ENOMEM. n = 0 is a no-op. */
FFSVA_API ffsva_status ffsva_filter_batch(const ffsva_frame* frames, int32_t n, ffsva_result* results,
                                          void* cuda_stream);

/* Same cascade for frames held in HOST memory (`pixels` host pointers, pinned or pageable): the library stages
 * them through a device ring with copies overlapped against the kernels. Synchronous. */
FFSVA_API ffsva_status ffsva_filter_batch_host(const ffsva_frame* frames, int32_t n, ffsva_result* results,
                                               void* cuda_stream);

/* Prepared batches: upload the descriptors of n device frames once, then launch the cascade asynchronously
 * any number of times (the kernel sequence is captured into a CUDA graph on the first launch and replayed),
 * and fetch results when needed. The frames' bytes may change between launches; their addresses may not.
 * ffsva_batch_launch enqueues on cuda_stream and returns immediately; ffsva_batch_fetch copies the results of
 * the last launch to host (results may be NULL) and synchronises cuda_stream. */
FFSVA_API ffsva_status ffsva_batch_prepare(const ffsva_frame* frames, int32_t n, ffsva_batch** out);
FFSVA_API ffsva_status ffsva_batch_launch(ffsva_batch* b, void* cuda_stream);
FFSVA_API ffsva_status ffsva_batch_fetch(ffsva_batch* b, ffsva_result* results, void* cuda_stream);
/* Device views of a prepared batch's outputs (valid until destroy): ssd u64[n], sdd_pass u8[n], survivor_idx
 * i32[n], logit f32[n], snm_pass u8[n], snm_class u8[n], d50 u8[n][snm_h][snm_w][3] (stride d50_stride bytes),
 * survivor count i32[1]. Any pointer argument may be NULL. */
FFSVA_API ffsva_status ffsva_batch_device_outputs(ffsva_batch* b, uint64_t** ssd, uint8_t** sdd_pass,
                                                  int32_t** survivor_idx, float** logit, uint8_t** snm_pass,
                                                  uint8_t** snm_class, uint8_t** d50, int64_t* d50_stride,
                                                  int32_t** n_survivors);
FFSVA_API ffsva_status ffsva_batch_destroy(ffsva_batch* b);

/* Measurement hook: launch the cascade of each of the nb prepared batches in turn, iters times over the list,
 * directly (no graph) with CUDA events recorded on cuda_stream around every kernel; ms_out[0..2] receive the
 * mean device time per launch of K1 (ingest/downsample/SDD), K3 (compaction) and K4 (SNM). Synchronous. */
FFSVA_API ffsva_status ffsva_batch_profile(ffsva_batch* const* batches, int32_t nb, int32_t iters,
                                           float* ms_out, void* cuda_stream);

/* SDD stage alone (for inspection and tests): D100 (sdd_h*sdd_w*3 u8 per frame, may be NULL), D50
 * (snm_h*snm_w*3 per frame, may be NULL), SSD and pass per frame, written to HOST arrays in input order.
 * Needs only a reference image (no SNM). Synchronous. */
FFSVA_API ffsva_status ffsva_sdd_batch(const ffsva_frame* frames, int32_t n, uint8_t* d100, uint8_t* d50,
                                       uint64_t* ssd, uint8_t* sdd_pass, void* cuda_stream);

/* Copy the stream's reference image R (sdd_h*sdd_w*3 u8) to host memory. */
FFSVA_API ffsva_status ffsva_get_reference(ffsva_stream* s, uint8_t* out);

/* Stream slot id (index into the device's stats table) and device ordinal. */
FFSVA_API ffsva_status ffsva_stream_info(ffsva_stream* s, int32_t* slot, int32_t* device);

/* Per-stream statistics of `device` (a8): copy u64[slots][FFSVA_NSTAT] to dst (device memory on `device`, e.g.
 * a torch tensor later all-gathered over NCCL, or host memory if dst_is_host). *slots receives the table size
 * (max slot + 1); dst must hold max_slots*FFSVA_NSTAT values. reset != 0 zeroes the table afterwards. */
FFSVA_API ffsva_status ffsva_stats_copy(int32_t device, uint64_t* dst, int32_t max_slots, int32_t* slots,
                                        int32_t dst_is_host, int32_t reset, void* cuda_stream);

/* ---------------------------------------------------------------------------------------------------------
 * Online runtime (§4.3): per-stream SDD and SNM queues (L143), the global feedback queue (L209, L217)
 * and dynamic batching (L223), driving the same kernels cycle by cycle.
 *   push  — a stream's prefetcher hands over frames; a frame is refused (accepted[i] = 0, the caller keeps it:
 *           the prefetcher is "blocked") while that stream's SDD queue holds more than q_sdd frames;
 *   tick  — one cycle: the SDD stage admits queued frames round-robin (at most max_frames_per_tick, at most the
 *           free SNM slots), skipping a stream while its SNM queue holds more than q_snm frames; survivors join
 *           the stream's SNM queue (their 50x50 images stay in a device slot pool); then every non-empty SNM
 *           queue pops min(BatchSize, depth) frames and the SNM scores all pops in one launch. Frames whose fate
 *           is decided (dropped by SDD, or scored by SNM) are reported as events, oldest first; events beyond
 *           `cap` are kept for the next tick. Synchronous on cuda_stream.
 * Without a T-YOLO model attached nothing blocks the SNM stage; with one (ffsva_sched_set_tyolo, f1) SNM survivors
 * wait in per-stream T-YOLO queues and the SNM stage skips a stream whose T-YOLO queue is over q_tyolo (L209).
 * push validates every frame's pixels as device memory of the scheduler's device. Frames must stay valid
 * until their event is reported. Streams must be open on the scheduler's device and carry a reference and an
 * SNM; a stream is attached on its first push and must not be closed while it has queued frames. */
typedef struct ffsva_sched ffsva_sched;
typedef struct {
  ffsva_stream* stream;
  int64_t frame_no;
  ffsva_result result;       /* survivor_idx = -1 (ranks are a batch notion) */
} ffsva_event;
typedef struct {
  int32_t admitted;          /* frames through SDD this cycle */
  int32_t sdd_pass;          /* of which survivors */
  int32_t snm_scored;        /* frames scored by the SNM this cycle */
  int32_t snm_batches;       /* dynamic batches (pops) this cycle */
  int32_t sdd_blocked;       /* streams skipped by the SDD stage because their SNM queue was over q_snm */
  int64_t sdd_queued;        /* frames waiting in SDD queues after the cycle */
  int64_t snm_queued;        /* frames waiting in SNM queues after the cycle */
  int64_t events_pending;    /* events not yet returned */
  float sdd_ms, snm_ms;      /* wall time of the SDD / SNM cycle (host work + kernels + copies) */
  float host_ms;             /* wall time of the whole tick */
  int32_t pad;
  int32_t tyolo_scored;      /* frames T-YOLO scored this cycle (0 without a T-YOLO model) */
  int32_t snm_blocked;       /* streams the SNM stage skipped because their T-YOLO queue was over q_tyolo (L209) */
  int64_t tyolo_queued;      /* frames waiting in T-YOLO queues after the cycle */
  float tyolo_ms;            /* wall time of the T-YOLO cycle */
  int32_t pad2;
} ffsva_tick_info;

FFSVA_API ffsva_status ffsva_sched_create(int32_t device, int32_t max_frames_per_tick, int32_t snm_slots,
                                          ffsva_sched** out);
FFSVA_API ffsva_status ffsva_sched_push(ffsva_sched* s, const ffsva_frame* frames, int32_t n, uint8_t* accepted);
FFSVA_API ffsva_status ffsva_sched_tick(ffsva_sched* s, void* cuda_stream, ffsva_event* events, int32_t cap,
                                        int32_t* n_events, ffsva_tick_info* info);
FFSVA_API ffsva_status ffsva_sched_depth(ffsva_sched* s, ffsva_stream* st, int32_t* sdd_depth, int32_t* snm_depth);
FFSVA_API ffsva_status ffsva_sched_destroy(ffsva_sched* s);

/* SNM batch trigger of the online runtime, for the paper's batch-mechanism comparison (§4.3.2,
 * §5.4; Q26):
 *   DYNAMIC  (default, the paper's method, L223): each cycle pops min(BatchSize, depth) frames per stream;
 *   FEEDBACK : fixed-size batches under the feedback queue: a stream pops BatchSize frames only once its SNM
 *              queue holds that many, or its whole queue once that queue blocks its SDD stage (depth > q_snm);
 *   STATIC   : fixed-size batches without SNM->SDD feedback (q_snm ignored; the slot pool bounds the queues).
 * Under FEEDBACK / STATIC, a cycle in which nothing can pop while every D50 slot is taken pops the fullest queue
 * (no deadlock). Frames left in partial batches at the end of input are drained by switching back to DYNAMIC. */
typedef enum { FFSVA_BATCH_DYNAMIC = 0, FFSVA_BATCH_FEEDBACK = 1, FFSVA_BATCH_STATIC = 2 } ffsva_batch_policy;
FFSVA_API ffsva_status ffsva_sched_set_policy(ffsva_sched* s, int32_t policy);

/* Pipelined ticks (on != 0; default off = synchronous ticks as described above). The paper runs its stages as
 * concurrent threads linked by queues (§3.1.2); here the host half of a cycle (admission,
 * batch assembly, event reporting) and the caller's work between ticks overlap the kernels of the previous cycle:
 * tick k prepares cycle k on the host, waits for cycle k-1's kernels, harvests their results (events, SNM queue
 * updates), runs the T-YOLO cycle, and launches cycle k's kernels without waiting for them. SNM pops of cycle k
 * therefore see SDD survivors of cycles <= k-2 (survivors of cycle k-1 join the SNM queues at tick k's harvest),
 * and every decision is reported one tick later than in synchronous mode; ffsva_tick_info.events_pending counts
 * in-flight frames too. Frames in flight hold their D50 slots, so size snm_slots for two cycles. Turning the mode
 * off while a cycle is in flight returns FFSVA_EAGAIN (tick once more first). Errors: EINVAL. */
FFSVA_API ffsva_status ffsva_sched_set_pipeline(ffsva_sched* s, int32_t on);

/* Inspection (tests): the frames of the most recently launched cycle — its SDD admissions (stage 0) and its SNM
 * pops (stage 1), in cycle order — with the 50x50x3 image each holds in the scheduler's device slot pool (the SNM's
 * input: written by K1 when the frame was admitted, possibly several cycles earlier for a pop). Synchronous mode:
 * the cycle of the last tick; pipelined mode: the cycle in flight (waited for), none if idle. Writes min(n, cap)
 * entries: frames[k], stage[k], d50[k*7500 .. +7500) (host memory); *n = the cycle's frame count. */
FFSVA_API ffsva_status ffsva_sched_inspect(ffsva_sched* s, ffsva_frame* frames, int32_t* stage, uint8_t* d50,
                                           int32_t cap, int32_t* n);

/* ---------------------------------------------------------------------------------------------------------
 * Admission control and stream re-forwarding between instances (§4.3.1: "when any queue of
 * T-YOLO or SNM is longer than its predefined threshold ... the corresponding video stream is re-forwarded to
 * another FFS-VA instance with spare capacity immediately"; L225: "load balancing can also be achieved by the
 * re-forwarding of video streams between FFS-VAs instances"). One instance = one GPU process; the decision logic
 * and the transport (NCCL point-to-point over NVLink) live in the Python layer (dist.py); these calls move a
 * stream's whole state and report the per-stream overload signals.
 *
 * Stream image: a self-contained byte image of a stream — its descriptor, thresholds, reference image R, packed
 * SNM weights and its per-stream statistics row — so the stream continues bit-identically elsewhere.
 *   ffsva_stream_image_bytes: size of s's image (57,280 B at the default 100x100 grid);
 *   ffsva_stream_export: write the image to dst (host memory, or device memory on s's device when dst_is_host
 *     is 0 — e.g. a buffer about to be sent over NCCL); synchronous on cuda_stream;
 *   ffsva_stream_import: open a new stream on `device` from an image (host memory, or device memory on `device`
 *     when src_is_host is 0); the stream's statistics row continues from the exported counters. The source
 *     stream is untouched (close it after the handover). Errors: EINVAL (bad image, version or descriptor). */
FFSVA_API ffsva_status ffsva_stream_image_bytes(ffsva_stream* s, int64_t* bytes);
FFSVA_API ffsva_status ffsva_stream_export(ffsva_stream* s, void* dst, int64_t cap, int32_t dst_is_host,
                                           void* cuda_stream);
FFSVA_API ffsva_status ffsva_stream_import(int32_t device, const void* src, int64_t bytes, int32_t src_is_host,
                                           ffsva_stream** out);

/* Per-stream overload signals of the online runtime since the previous reset (L213: "when any queue of T-YOLO or
 * SNM is longer than its predefined threshold ... the FFS-VA instance overloads"): a stream overloads its instance
 * when its SNM queue went over q_snm (the SDD stage had to skip it: sdd_blocked > 0), its T-YOLO queue over q_tyolo
 * (the SNM stage had to skip it: snm_blocked > 0) or its prefetcher was refused (SDD queue over q_sdd: refused > 0). */
typedef struct {
  int32_t sdd_depth, snm_depth;   /* current queue depths (frames) */
  int32_t max_sdd, max_snm;       /* maxima since the reset */
  uint64_t pushed, refused;       /* frames accepted / refused by the SDD queue since the reset */
  uint64_t sdd_blocked;           /* SDD cycles that skipped the stream (SNM queue over q_snm) since the reset */
  int32_t tyolo_depth, max_tyolo; /* T-YOLO queue depth now / maximum since the reset (f1 stage attached) */
  uint64_t snm_blocked;           /* SNM cycles that skipped the stream (T-YOLO queue over q_tyolo) since the reset */
} ffsva_stream_load;
/* Attach the device's shared T-YOLO model (ffsva_tyolo_load) to the online runtime as its third stage (f1; NULL
 * detaches): SNM survivors then wait in per-stream T-YOLO queues; the SNM stage skips a stream while its T-YOLO
 * queue holds more than q_tyolo frames (L209); each tick ends with a T-YOLO cycle that takes at most num_tyolo
 * frames from every non-empty T-YOLO queue (L173), counts each frame's target objects (its stream's
 * target_class, boxes scoring > thresh) and reports tyolo_count / tyolo_pass in its event. The model must outlive
 * the attachment and live on the scheduler's device. */
FFSVA_API ffsva_status ffsva_sched_set_tyolo(ffsva_sched* s, ffsva_tyolo* m, int32_t num_tyolo, float thresh);

FFSVA_API ffsva_status ffsva_sched_stream_load(ffsva_sched* s, ffsva_stream* st, int32_t reset,
                                               ffsva_stream_load* out);
/* Detach a stream from the scheduler (before re-forwarding or closing it): FFSVA_EAGAIN while it still has
 * queued frames or unreported events (keep ticking), FFSVA_OK once removed (or if it was never attached). */
FFSVA_API ffsva_status ffsva_sched_detach(ffsva_sched* s, ffsva_stream* st);

/* ---------------------------------------------------------------------------------------------------------
 * T-YOLO stage (§3.2.3, §4.2.2). The third filter: Tiny-YOLO-VOC
 * ("9 CONV layers and 6 POOL layers", 416x416 input, VOC's 20 classes; L169), one model shared by all streams of a
 * device (L175). Each frame is resized to 416x416 (Q28), scaled by 1/256 (Q29) and run through the nine
 * layers on tcgen05 tensor cores (bf16 operands, fp32 accumulation, bf16 activations between layers: Q32). The
 * 13x13x125 head is decoded per box as score = sigmoid(objectness) * softmax(class logits)[target_class]; a box
 * whose score exceeds `thresh` (0.2 in the paper, L171) is one target object (Q31, no NMS), and a frame passes
 * iff its count >= number_of_objects (NumberofObjects, L195).
 *   ffsva_tyolo_load: params = the nine layers' w[Cout][Cin][k][k] then b[Cout] (fp32, batch norm folded into b;
 *     15,858,717 values); weights are rounded to bf16 at load. The model holds a reference on the device context.
 *   ffsva_tyolo_run: n frames (device pixels; each frame's stream supplies its geometry); outputs (host, may be
 *     NULL, not all): counts[n], pass[n], raw[n][13][13][125] fp32 head outputs. Synchronous on cuda_stream.
 *   ffsva_tyolo_layer_output (diagnostic): run the resize and layers 0..layer on n <= 256 frames and copy that
 *     layer's bf16 NHWC activation (layer -1: the resized input, 416x416x4) to host `out` (bf16 bit patterns).
 *   ffsva_tyolo_profile (measurement): mean device ms of the resize and of each of the nine layers over iters runs
 *     of n <= 256 frames, CUDA events on cuda_stream; ms_out[10]. */
FFSVA_API ffsva_status ffsva_tyolo_load(int32_t device, const float* params, int64_t n_params, ffsva_tyolo** out);
FFSVA_API ffsva_status ffsva_tyolo_run(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n, int32_t target_class,
                                       float thresh, int32_t number_of_objects, int32_t* counts, uint8_t* pass,
                                       float* raw, void* cuda_stream);
FFSVA_API ffsva_status ffsva_tyolo_layer_output(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n, int32_t layer,
                                                uint16_t* out, void* cuda_stream);
FFSVA_API ffsva_status ffsva_tyolo_profile(ffsva_tyolo* m, const ffsva_frame* frames, int32_t n, int32_t iters,
                                           float* ms_out, void* cuda_stream);
FFSVA_API ffsva_status ffsva_tyolo_destroy(ffsva_tyolo* m);

/* Close a stream (NULL is a no-op). */
FFSVA_API ffsva_status ffsva_close(ffsva_stream* s);

/* Human-readable description of the calling thread's last error ("" if none). */
FFSVA_API const char* ffsva_last_error(void);

/* Number of kernels this process has launched through the library (all devices), for launch accounting. */
FFSVA_API uint64_t ffsva_kernel_launches(void);

/* Library version string. */
FFSVA_API const char* ffsva_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FFSVA_H */
