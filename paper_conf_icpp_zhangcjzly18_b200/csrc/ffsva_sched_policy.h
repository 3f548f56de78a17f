// ffsva_sched_policy.h — the online queue policy of FFS-VA (§4.3), host-only and CUDA-free (unit-tested
// on CPU by tests/test_sched_policy.py through tests/sched_policy_test.cpp).
//
//   * per-stream queues between consecutive stages (L143): an SDD queue (frames waiting for SDD) and an SNM
//     queue (SDD survivors waiting for the SNM);
//   * global feedback queue (L209, L217): a stage stops pulling from its input while the queue of the stage
//     after it holds more than that queue's depth threshold. Thresholds are per stream, in frames (reading
//     Q18): the prefetcher is refused while the SDD queue holds more than q_sdd frames (default 2); the SDD
//     stage skips a stream while its SNM queue holds more than q_snm frames (default 10). The SNM stage feeds
//     T-YOLO, which is out of scope, so nothing blocks it;
//   * dynamic batching (L223): each SNM cycle pops min(BatchSize, depth) frames of every non-empty stream;
//   * T-YOLO stage (f1, when a T-YOLO model is attached): SNM survivors join the stream's T-YOLO queue; the SNM
//     stage skips a stream while its T-YOLO queue holds more than q_ty frames ("when the T-YOLO queue depth
//     exceeds a threshold, the SNM thread ... stops pushing frames to the T-YOLO queue", L209; default 2, L217);
//     each T-YOLO cycle traverses the streams' T-YOLO queues and extracts at most num_t-yolo frames from each,
//     skipping empty queues (L173, L211).
// Streams are visited round-robin (the start rotates every cycle) so a per-cycle frame budget is shared fairly.
//
// The two batch mechanisms the paper compares dynamic batching with (§4.3.2, §5.4; f4) are
// selectable for that study (BatchPolicy, Q26):
//   * STATIC  — "a triggering strategy based on a fixed number of input frames per batch": the SNM pops exactly
//               BatchSize frames of a stream once its queue holds that many; no feedback from the SNM queue to
//               the SDD stage (q_snm is ignored; the device slot pool is the only bound);
//   * FEEDBACK — the same fixed-size trigger under the feedback queue (the SDD stage skips a stream whose SNM
//               queue holds more than q_snm frames). "When the batch size is greater than the queue depth
//               threshold, video frames have to wait in the SNM" (L221): a stream whose SDD stage is blocked
//               (depth > q_snm) has its queue popped whole, otherwise it would wait forever;
//   * DYNAMIC — the paper's method (default).
// Under STATIC and FEEDBACK, when no stream can pop and the slot pool is exhausted (every slot holds a partial
// batch) the fullest queue is popped, so the runtime cannot deadlock. To drain at the end of input, switch the
// policy back to DYNAMIC.
#pragma once

#include <algorithm>
#include <cstdint>
#include <vector>

namespace ffsva {
namespace sched {

struct QFrame {
  int32_t stream = -1;        // policy stream id
  int64_t frame_no = 0;       // caller's frame number
  const void* pixels = nullptr;
  int32_t slot = -1;          // device D50 slot while the frame sits in the SNM queue
  uint64_t ssd = 0;           // SDD distance, carried to the frame's final event
  float logit = 0.f;          // SNM result, carried through the T-YOLO queue
  uint8_t snm_class = 0;
  int64_t t_push_us = 0;      // steady-clock microseconds when the push was accepted (a8 latency)
};

enum class BatchPolicy : int32_t { DYNAMIC = 0, FEEDBACK = 1, STATIC = 2 };

// FIFO of frames: a vector with a head index (pops advance the head; the storage is reset when the queue empties
// and compacted when the dead prefix dominates). An empty queue owns no memory, so tens of thousands of streams
// cost a few cache lines each (std::deque allocates a 512-byte chunk per queue up front).
class Fifo {
 public:
  using const_iterator = std::vector<QFrame>::const_iterator;
  size_t size() const { return v_.size() - h_; }
  bool empty() const { return h_ == v_.size(); }
  const QFrame& front() const { return v_[h_]; }
  void push_back(const QFrame& f) { v_.push_back(f); }
  void pop_front() { erase_front(1); }
  void erase_front(size_t n) {
    h_ += n;
    if (h_ == v_.size()) {
      v_.clear();
      h_ = 0;
    } else if (h_ >= 64 && 2 * h_ >= v_.size()) {
      v_.erase(v_.begin(), v_.begin() + (std::ptrdiff_t)h_);
      h_ = 0;
    }
  }
  const_iterator begin() const { return v_.begin() + (std::ptrdiff_t)h_; }
  const_iterator end() const { return v_.end(); }

 private:
  std::vector<QFrame> v_;
  size_t h_ = 0;
};

struct StreamQ {
  int32_t q_sdd = 2, q_snm = 10, batch = 30, q_ty = 2;
  bool live = false;
  Fifo sdd, snm, ty;
  uint64_t pushed = 0, refused = 0, sdd_blocked = 0, snm_blocked = 0;
  int32_t max_sdd = 0, max_snm = 0, max_ty = 0;
};

class Policy {
 public:
  int32_t add_stream(int32_t q_sdd, int32_t q_snm, int32_t batch, int32_t q_ty = 2) {
    int32_t id = -1;
    if (!free_ids_.empty()) {  // reuse a removed stream's id (O(1): attaching S streams is O(S), not O(S^2))
      id = free_ids_.back();
      free_ids_.pop_back();
    }
    if (id < 0) {
      id = (int32_t)st_.size();
      st_.emplace_back();
      nsdd_.push_back(0);
      nsnm_.push_back(0);
      nty_.push_back(0);
    }
    StreamQ& s = st_[id];
    s = StreamQ();
    s.q_sdd = q_sdd;
    s.q_snm = q_snm;
    s.q_ty = q_ty;
    s.batch = batch < 1 ? 1 : batch;
    s.live = true;
    return id;
  }

  // Frames still queued are returned so the caller can release their device slots.
  std::vector<QFrame> remove_stream(int32_t id) {
    std::vector<QFrame> out;
    if (id < 0 || id >= (int32_t)st_.size()) return out;
    StreamQ& s = st_[id];
    out.insert(out.end(), s.sdd.begin(), s.sdd.end());
    out.insert(out.end(), s.snm.begin(), s.snm.end());
    out.insert(out.end(), s.ty.begin(), s.ty.end());
    nq_sdd_ -= (int64_t)s.sdd.size();
    nq_snm_ -= (int64_t)s.snm.size();
    nq_ty_ -= (int64_t)s.ty.size();
    nsdd_[id] = nsnm_[id] = nty_[id] = 0;
    if (s.live) free_ids_.push_back(id);
    s = StreamQ();
    return out;
  }

  bool live(int32_t id) const { return id >= 0 && id < (int32_t)st_.size() && st_[id].live; }

  // The prefetcher of a stream is blocked while its SDD queue holds more than q_sdd frames (L209, L217).
  bool push(int32_t id, const QFrame& f) {
    StreamQ& s = st_[id];
    if ((int32_t)s.sdd.size() > s.q_sdd) {
      ++s.refused;
      return false;
    }
    QFrame g = f;
    g.stream = id;
    s.sdd.push_back(g);
    ++nsdd_[id];
    ++nq_sdd_;
    ++s.pushed;
    s.max_sdd = std::max(s.max_sdd, (int32_t)s.sdd.size());
    return true;
  }

  // SDD stage of one cycle: round-robin over streams; a stream whose SNM queue holds more than q_snm frames is
  // skipped (feedback, L209); otherwise its queued frames are admitted in order, at most `budget` in total and
  // at most `snm_room` that could still land in the SNM queue (device D50 slots).
  std::vector<QFrame> admit_sdd(int32_t budget, int32_t snm_room) {
    std::vector<QFrame> out;
    const int32_t n = (int32_t)st_.size();
    if (n == 0) return out;
    int32_t limit = std::min(budget, snm_room);
    for (int32_t k = 0, i = rr_; k < n && limit > 0; ++k, i = (i + 1 == n ? 0 : i + 1)) {
      if (nsdd_[i] == 0) continue;  // compact depth mirror: idle streams cost 4 bytes of scan
      StreamQ& s = st_[i];
      if (policy_ != BatchPolicy::STATIC && nsnm_[i] > s.q_snm) {
        ++s.sdd_blocked;
        ++tot_sdd_blocked_;
        continue;
      }
      while (!s.sdd.empty() && limit > 0) {
        out.push_back(s.sdd.front());
        s.sdd.pop_front();
        --nsdd_[i];
        --nq_sdd_;
        --limit;
      }
    }
    rr_ = (rr_ + 1) % n;
    return out;
  }

  // An admitted frame's SDD verdict: survivors join their stream's SNM queue in arrival order (L143).
  void sdd_done(const QFrame& f, bool pass) {
    if (!pass) return;
    StreamQ& s = st_[f.stream];
    s.snm.push_back(f);
    ++nsnm_[f.stream];
    ++nq_snm_;
    s.max_snm = std::max(s.max_snm, (int32_t)s.snm.size());
  }

  // SNM stage of one cycle. DYNAMIC (L223): every non-empty stream pops min(BatchSize, depth). STATIC /
  // FEEDBACK: a stream pops BatchSize frames only when it holds that many (FEEDBACK also pops a stream whose
  // SDD stage it blocks). `slots_free` = free device D50 slots (deadlock guard, see above).
  // The pops are appended to `flat`; pop p is flat[starts[p] .. starts[p+1]) (starts gets a final sentinel).
  void pop_snm(std::vector<QFrame>& flat, std::vector<int32_t>& starts, int32_t slots_free = 1 << 30) {
    flat.clear();
    starts.clear();
    const int32_t n = (int32_t)st_.size();
    auto take_from = [&](int32_t k, int32_t take) {
      StreamQ& s = st_[k];
      starts.push_back((int32_t)flat.size());
      flat.insert(flat.end(), s.snm.begin(), s.snm.begin() + take);
      s.snm.erase_front((size_t)take);
      nsnm_[k] -= take;
      nq_snm_ -= take;
    };
    for (int32_t k = 0; k < n; ++k) {
      if (nsnm_[k] == 0) continue;
      StreamQ& s = st_[k];
      if (tyolo_ && nty_[k] > s.q_ty) {  // T-YOLO -> SNM feedback (L209)
        ++s.snm_blocked;
        ++tot_snm_blocked_;
        continue;
      }
      const int32_t depth = (int32_t)s.snm.size();
      if (policy_ == BatchPolicy::DYNAMIC) {
        take_from(k, std::min(s.batch, depth));
      } else if (depth >= s.batch) {
        take_from(k, s.batch);
      } else if (policy_ == BatchPolicy::FEEDBACK && depth > s.q_snm) {
        take_from(k, depth);
      }
    }
    if (flat.empty() && slots_free <= 0) {  // every slot holds a partial batch: pop the fullest queue
      int32_t best = -1;
      for (int32_t k = 0; k < n; ++k)
        if (st_[k].live && !st_[k].snm.empty() && (best < 0 || st_[k].snm.size() > st_[best].snm.size())) best = k;
      if (best >= 0) take_from(best, std::min(st_[best].batch, (int32_t)st_[best].snm.size()));
    }
    starts.push_back((int32_t)flat.size());
  }

  // An SNM-scored frame: with the T-YOLO stage attached, a survivor joins the stream's T-YOLO queue (returns true:
  // its event waits for T-YOLO); otherwise its SNM result is final (false).
  bool snm_done(const QFrame& f, bool pass) {
    if (!tyolo_ || !pass) return false;
    StreamQ& s = st_[f.stream];
    s.ty.push_back(f);
    ++nty_[f.stream];
    ++nq_ty_;
    s.max_ty = std::max(s.max_ty, (int32_t)s.ty.size());
    return true;
  }

  // T-YOLO cycle (L173): every non-empty T-YOLO queue gives at most num_t-yolo frames, oldest first.
  void pop_ty(std::vector<QFrame>& flat) {
    flat.clear();
    for (int32_t k = 0; k < (int32_t)st_.size(); ++k) {
      if (nty_[k] == 0) continue;
      StreamQ& s = st_[k];
      const int32_t take = std::min<int32_t>(ty_take_, (int32_t)s.ty.size());
      flat.insert(flat.end(), s.ty.begin(), s.ty.begin() + take);
      s.ty.erase_front((size_t)take);
      nty_[k] -= take;
      nq_ty_ -= take;
    }
  }

  void set_tyolo(bool on, int32_t per_stream) {
    tyolo_ = on;
    ty_take_ = per_stream < 1 ? 1 : per_stream;
  }
  bool tyolo() const { return tyolo_; }

  void set_policy(BatchPolicy p) { policy_ = p; }
  BatchPolicy policy() const { return policy_; }

  std::vector<std::vector<QFrame>> pop_snm(int32_t slots_free = 1 << 30) {  // convenience form for tests
    std::vector<QFrame> flat;
    std::vector<int32_t> starts;
    pop_snm(flat, starts, slots_free);
    std::vector<std::vector<QFrame>> pops;
    for (size_t p = 0; p + 1 < starts.size(); ++p)
      pops.emplace_back(flat.begin() + starts[p], flat.begin() + starts[p + 1]);
    return pops;
  }

  const StreamQ& stream(int32_t id) const { return st_[id]; }
  // Zero a stream's overload counters (re-forwarding window, L213); depths are state, not counters.
  void reset_counters(int32_t id) {
    StreamQ& s = st_[id];
    s.pushed = s.refused = s.sdd_blocked = s.snm_blocked = 0;
    s.max_sdd = (int32_t)s.sdd.size();
    s.max_snm = (int32_t)s.snm.size();
    s.max_ty = (int32_t)s.ty.size();
  }
  int32_t n_streams() const { return (int32_t)st_.size(); }
  // queue totals and blocking counters over all streams, maintained incrementally (O(1) per tick)
  int64_t queued_sdd() const { return nq_sdd_; }
  int64_t queued_snm() const { return nq_snm_; }
  int64_t queued_ty() const { return nq_ty_; }
  uint64_t total_sdd_blocked() const { return tot_sdd_blocked_; }
  uint64_t total_snm_blocked() const { return tot_snm_blocked_; }

 private:
  std::vector<StreamQ> st_;
  std::vector<int32_t> nsdd_, nsnm_, nty_;  // per-stream queue depths (compact mirror of the FIFOs)
  std::vector<int32_t> free_ids_;           // ids of removed streams, reused by add_stream
  int64_t nq_sdd_ = 0, nq_snm_ = 0, nq_ty_ = 0;
  uint64_t tot_sdd_blocked_ = 0, tot_snm_blocked_ = 0;
  int32_t rr_ = 0;
  BatchPolicy policy_ = BatchPolicy::DYNAMIC;
  bool tyolo_ = false;
  int32_t ty_take_ = 4;
};

}  // namespace sched
}  // namespace ffsva
