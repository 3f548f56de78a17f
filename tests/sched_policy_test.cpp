// Hand traces of the online queue policy (§4.3: feedback queue L209/L217, dynamic batching L223).
// Built and run by tests/test_sched_policy.py with g++ (no CUDA).
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_icpp_zhangcjzly18_b200/csrc/ffsva_sched_policy.h"

using ffsva::sched::Policy;
using ffsva::sched::QFrame;

static int failures = 0;
#define CHECK(c)                                                      \
  do {                                                                \
    if (!(c)) {                                                       \
      std::printf("FAIL line %d: %s\n", __LINE__, #c);                \
      ++failures;                                                     \
    }                                                                 \
  } while (0)

static QFrame fr(int64_t no) {
  QFrame q;
  q.frame_no = no;
  q.pixels = (const void*)0x1000;
  return q;
}

int main() {
  {  // the prefetcher is refused while the SDD queue holds more than q_sdd = 2 frames
    Policy p;
    int s = p.add_stream(2, 10, 30);
    CHECK(p.push(s, fr(0)) && p.push(s, fr(1)) && p.push(s, fr(2)));
    CHECK(!p.push(s, fr(3)));                      // depth 3 > 2: blocked
    CHECK(p.stream(s).refused == 1 && p.stream(s).max_sdd == 3);
    auto a = p.admit_sdd(100, 100);
    CHECK(a.size() == 3 && a[0].frame_no == 0 && a[2].frame_no == 2);  // arrival order
    CHECK(p.push(s, fr(3)));                       // drained: accepted again
  }
  {  // the SDD stage skips a stream while its SNM queue holds more than q_snm = 2 frames
    Policy p;
    int s = p.add_stream(100, 2, 2);
    for (int i = 0; i < 5; ++i) p.push(s, fr(i));
    auto a = p.admit_sdd(100, 100);
    CHECK(a.size() == 5);
    for (auto& f : a) p.sdd_done(f, true);         // all survive: SNM depth 5
    CHECK(p.stream(s).snm.size() == 5);
    p.push(s, fr(5));
    CHECK(p.admit_sdd(100, 100).empty());          // 5 > 2: blocked
    CHECK(p.stream(s).sdd_blocked == 1);
    auto pops = p.pop_snm();                       // BatchSize 2
    CHECK(pops.size() == 1 && pops[0].size() == 2 && pops[0][0].frame_no == 0);
    CHECK(p.admit_sdd(100, 100).empty());          // depth 3 > 2: still blocked
    p.pop_snm();                                   // depth 1
    auto b = p.admit_sdd(100, 100);
    CHECK(b.size() == 1 && b[0].frame_no == 5);    // resumes once depth <= threshold
  }
  {  // dynamic batching: each cycle pops min(BatchSize, depth), survivors in order, dropped frames never queue
    Policy p;
    int s = p.add_stream(100, 100, 3);
    for (int i = 0; i < 9; ++i) p.push(s, fr(i));
    auto a = p.admit_sdd(100, 100);
    for (auto& f : a) p.sdd_done(f, f.frame_no % 4 != 0);  // frames 0, 4, 8 dropped: 6 survivors
    CHECK(p.queued_snm() == 6);
    auto p1 = p.pop_snm();
    CHECK(p1.size() == 1 && p1[0].size() == 3 && p1[0][0].frame_no == 1 && p1[0][2].frame_no == 3);
    auto p2 = p.pop_snm();
    CHECK(p2[0].size() == 3 && p2[0][0].frame_no == 5 && p2[0][2].frame_no == 7);
    CHECK(p.pop_snm().empty());
  }
  {  // a per-cycle budget is shared round-robin; the start stream rotates every cycle
    Policy p;
    int s0 = p.add_stream(100, 100, 30), s1 = p.add_stream(100, 100, 30), s2 = p.add_stream(100, 100, 30);
    for (int i = 0; i < 2; ++i) {
      p.push(s0, fr(i));
      p.push(s1, fr(10 + i));
      p.push(s2, fr(20 + i));
    }
    auto c1 = p.admit_sdd(3, 100);
    CHECK(c1.size() == 3 && c1[0].stream == s0 && c1[1].stream == s0 && c1[2].stream == s1);
    auto c2 = p.admit_sdd(3, 100);
    CHECK(c2.size() == 3 && c2[0].stream == s1 && c2[1].stream == s2 && c2[2].stream == s2);
    CHECK(p.queued_sdd() == 0);
  }
  {  // admission never exceeds the free SNM slots
    Policy p;
    int s = p.add_stream(100, 100, 30);
    for (int i = 0; i < 10; ++i) p.push(s, fr(i));
    CHECK(p.admit_sdd(100, 4).size() == 4);
    CHECK(p.queued_sdd() == 6);
  }
  {  // removing a stream hands back its queued frames; its id is reused
    Policy p;
    int s = p.add_stream(100, 100, 30);
    p.push(s, fr(0));
    auto a = p.admit_sdd(100, 100);
    p.sdd_done(a[0], true);
    p.push(s, fr(1));
    auto left = p.remove_stream(s);
    CHECK(left.size() == 2 && !p.live(s));
    CHECK(p.add_stream(1, 1, 1) == s);
  }
  {  // STATIC (L221 "a triggering strategy based on a fixed number of input frames per batch"): no pop until
     // BatchSize frames are queued, exactly BatchSize per pop, and the SNM queue never blocks the SDD stage
    Policy p;
    p.set_policy(ffsva::sched::BatchPolicy::STATIC);
    int s = p.add_stream(100, 2, 4);
    for (int i = 0; i < 3; ++i) p.push(s, fr(i));
    for (auto& f : p.admit_sdd(100, 100)) p.sdd_done(f, true);
    CHECK(p.pop_snm().empty());                    // 3 < 4 frames: wait (the latency cost, L221)
    for (int i = 3; i < 9; ++i) p.push(s, fr(i));
    auto a = p.admit_sdd(100, 100);
    CHECK(a.size() == 6);                          // depth 3 > q_snm = 2 would block FEEDBACK, not STATIC
    for (auto& f : a) p.sdd_done(f, true);
    auto pops = p.pop_snm();
    CHECK(pops.size() == 1 && pops[0].size() == 4 && pops[0][0].frame_no == 0 && pops[0][3].frame_no == 3);
    pops = p.pop_snm();
    CHECK(pops.size() == 1 && pops[0].size() == 4 && pops[0][0].frame_no == 4);
    CHECK(p.pop_snm().empty() && p.queued_snm() == 1);  // frame 8 waits for a full batch
    CHECK(p.pop_snm(0).size() == 1);               // unless the slot pool is exhausted (deadlock guard)
  }
  {  // FEEDBACK: fixed-size trigger under the feedback queue; a queue that blocks its SDD stage (depth > q_snm)
     // is popped whole even below BatchSize (L221: BatchSize > threshold would otherwise wait forever)
    Policy p;
    p.set_policy(ffsva::sched::BatchPolicy::FEEDBACK);
    int s = p.add_stream(100, 2, 5);
    for (int i = 0; i < 2; ++i) p.push(s, fr(i));
    for (auto& f : p.admit_sdd(100, 100)) p.sdd_done(f, true);
    CHECK(p.pop_snm().empty());                    // depth 2 <= q_snm, < BatchSize: wait
    p.push(s, fr(2));
    for (auto& f : p.admit_sdd(100, 100)) p.sdd_done(f, true);
    p.push(s, fr(3));
    CHECK(p.admit_sdd(100, 100).empty());          // depth 3 > 2: SDD blocked
    auto pops = p.pop_snm();
    CHECK(pops.size() == 1 && pops[0].size() == 3 && pops[0][2].frame_no == 2);
    auto b = p.admit_sdd(100, 100);
    CHECK(b.size() == 1 && b[0].frame_no == 3);    // unblocked
    // switching back to DYNAMIC drains partial batches (end of input)
    p.sdd_done(b[0], true);
    CHECK(p.pop_snm().empty());
    p.set_policy(ffsva::sched::BatchPolicy::DYNAMIC);
    pops = p.pop_snm();
    CHECK(pops.size() == 1 && pops[0].size() == 1 && pops[0][0].frame_no == 3);
  }
  {  // T-YOLO stage (L173, L209, L217): survivors of the SNM wait in the T-YOLO queue; each cycle takes at most
     // num_t-yolo per stream; the SNM stage skips a stream whose T-YOLO queue holds more than q_ty = 2 frames
    Policy p;
    p.set_tyolo(true, 2);
    int s0 = p.add_stream(100, 100, 5, 2), s1 = p.add_stream(100, 100, 5, 2);
    for (int i = 0; i < 5; ++i) p.push(s0, fr(i));
    p.push(s1, fr(100));
    for (auto& f : p.admit_sdd(100, 100)) p.sdd_done(f, true);
    auto pops = p.pop_snm();                       // s0: 5 frames, s1: 1 frame
    CHECK(pops.size() == 2 && pops[0].size() == 5 && pops[1].size() == 1);
    for (auto& pop : pops)  // frame 3 is dropped by the SNM: its result is final, it never queues
      for (auto& f : pop) CHECK(p.snm_done(f, f.frame_no != 3) == (f.frame_no != 3));
    CHECK(p.queued_ty() == 5);                     // s0: 0, 1, 2, 4; s1: 100
    std::vector<QFrame> ty;
    p.pop_ty(ty);
    CHECK(ty.size() == 3 && ty[0].frame_no == 0 && ty[1].frame_no == 1 && ty[2].frame_no == 100);
    CHECK(p.queued_ty() == 2);                     // s0: 2, 4 (depth 2, not over q_ty)
    for (int i = 5; i < 8; ++i) p.push(s0, fr(i));
    for (auto& f : p.admit_sdd(100, 100)) p.sdd_done(f, true);
    pops = p.pop_snm();                            // s0 T-YOLO depth 2 <= 2: may pop
    CHECK(pops.size() == 1 && pops[0].size() == 3);
    for (auto& f : pops[0]) p.snm_done(f, true);   // T-YOLO depth 5 > 2
    p.push(s0, fr(8));
    for (auto& f : p.admit_sdd(100, 100)) p.sdd_done(f, true);
    CHECK(p.pop_snm().empty());                    // blocked by the T-YOLO queue (L209)
    CHECK(p.stream(s0).snm_blocked == 1 && p.stream(s0).max_ty == 5);
    p.pop_ty(ty);
    CHECK(ty.size() == 2 && ty[0].frame_no == 2 && ty[1].frame_no == 4);
    p.pop_ty(ty);                                  // depth 1 <= 2: unblocked
    CHECK(p.pop_snm().size() == 1);
  }
  {  // the incremental totals (queued_*, total_*_blocked) equal the per-stream sums after a random trace
    Policy p;
    p.set_tyolo(true, 2);
    uint32_t h = 12345u;
    auto rnd = [&](uint32_t m) { h = h * 1664525u + 1013904223u; return (h >> 8) % m; };
    std::vector<int> ids;
    for (int i = 0; i < 7; ++i) ids.push_back(p.add_stream(1 + (int)rnd(3), 1 + (int)rnd(4), 1 + (int)rnd(5), 1 + (int)rnd(2)));
    int64_t no = 0;
    for (int step = 0; step < 400; ++step) {
      for (int k = 0; k < 6; ++k) p.push(ids[rnd(7)], fr(no++));
      for (auto& f : p.admit_sdd(1 + (int)rnd(20), 1 + (int)rnd(30))) p.sdd_done(f, rnd(3) != 0);
      for (auto& pop : p.pop_snm()) for (auto& f : pop) p.snm_done(f, rnd(2) != 0);
      if (rnd(2)) { std::vector<QFrame> ty; p.pop_ty(ty); }
      if (step == 200) { p.remove_stream(ids[3]); ids[3] = p.add_stream(2, 2, 3, 1); }
      int64_t qs = 0, qn = 0, qt = 0;
      uint64_t bs = 0, bn = 0;
      for (int i = 0; i < p.n_streams(); ++i) {
        qs += (int64_t)p.stream(i).sdd.size();
        qn += (int64_t)p.stream(i).snm.size();
        qt += (int64_t)p.stream(i).ty.size();
        bs += p.stream(i).sdd_blocked;
        bn += p.stream(i).snm_blocked;
      }
      CHECK(qs == p.queued_sdd() && qn == p.queued_snm() && qt == p.queued_ty());
      if (step < 200) CHECK(bs == p.total_sdd_blocked() && bn == p.total_snm_blocked());  // until a removal
    }
  }
  if (failures == 0) std::printf("ALL PASS\n");
  return failures == 0 ? 0 : 1;
}
