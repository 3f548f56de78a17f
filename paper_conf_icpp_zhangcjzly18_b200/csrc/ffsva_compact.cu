// ffsva_compact.cu — K3: survivor compaction and dynamic-batch formation.
//
// Method: SDD survivors are pushed to the stream's SNM queue in arrival order (L143 §3.1.2);
// "if there are enough video frames in the SNM queue, SNM pops out a batch of (BatchSize) images from the
// queue ... otherwise, the frames are popped from the SNM queue until the queue is empty" (L223 §4.3.2).
// Readings: stable batch order for survivor ranks (Q16), per-stream pops of min(BatchSize, q)
// (Q17).
//
// One CTA of 1024 threads, tiles of 4096 flags (4 per thread, one 32-bit load). Within a warp the prefix
// sum is four __ballot_sync + __popc (lane-mask) steps; warp totals are scanned in shared memory.
//   pass 1 (input order)      -> survivor_idx[i] = rank of i among survivors, or -1
//   pass 2 (stream-major perm) -> work[] = survivors grouped by stream, posw[] = exclusive counts
//   pass 3 (segments)          -> pop list: each stream's queue split into pops of <= BatchSize frames (chunks[k] =
//                                 first work position of pop k), counts[0] = m survivors for K4's per-CTA ranges
#include "ffsva_internal.h"

namespace ffsva {
namespace {

constexpr int kThreads = 1024;
constexpr int kWarps = kThreads / 32;

// Exclusive block scan of one int per thread; returns the exclusive prefix, *total = block sum.
__device__ __forceinline__ int block_exclusive_scan(int v, int* s_warp, int* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  int incl = v;
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    int t = __shfl_up_sync(0xffffffffu, incl, off);
    if (lane >= off) incl += t;
  }
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    int w = lane < kWarps ? s_warp[lane] : 0;
    int wi = w;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      int t = __shfl_up_sync(0xffffffffu, wi, off);
      if (lane >= off) wi += t;
    }
    s_warp[lane] = wi - w;          // exclusive warp offsets
    if (lane == 31) s_warp[32] = wi;
  }
  __syncthreads();
  const int r = s_warp[warp] + incl - v;
  *total = s_warp[32];
  __syncthreads();
  return r;
}

// Ballot/popc rank inside a warp for 4 consecutive flags per thread (thread-major order): returns the number
// of set flags held by lower lanes and writes the warp total to *wtotal.
__device__ __forceinline__ int warp_rank4(const bool (&f)[4], int* wtotal) {
  const unsigned lt = (1u << (threadIdx.x & 31)) - 1u;
  int rank = 0, tot = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const unsigned b = __ballot_sync(0xffffffffu, f[j]);
    rank += __popc(b & lt);
    tot += __popc(b);
  }
  *wtotal = tot;
  return rank;
}

__global__ void __launch_bounds__(kThreads) compact_kernel(CompactArgs a) {
  __shared__ int s_warp[33];
  __shared__ int s_wbase[kWarps + 1];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int n = a.n;

  // ---------------- pass 1: SDD threshold (L151: MSE > delta_diff <=> SSD > T) and ranks in input order
  int carry = 0;
  for (int base = 0; base < n; base += 4 * kThreads) {
    const int i0 = base + 4 * threadIdx.x;
    bool f[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      f[j] = false;
      if (i0 + j < n) {
        const unsigned long long s = a.acc_ssd[i0 + j];
        f[j] = s > a.frames[i0 + j].T;
        a.ssd[i0 + j] = s;
        a.pass[i0 + j] = f[j] ? 1 : 0;
        a.acc_ssd[i0 + j] = 0ull;  // ready for the next launch of this batch
      }
    }
    int wtot;
    const int wr = warp_rank4(f, &wtot);
    if (lane == 0) s_wbase[warp] = wtot;
    __syncthreads();
    if (warp == 0) {
      int w = s_wbase[lane], wi = w;
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        int t = __shfl_up_sync(0xffffffffu, wi, off);
        if (lane >= off) wi += t;
      }
      s_wbase[lane] = wi - w;
      if (lane == 31) s_wbase[kWarps] = wi;
    }
    __syncthreads();
    int r = carry + s_wbase[warp] + wr;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      // wr counts every flag of lower lanes; this thread's own earlier items are added one by one
      if (i0 + j < n) {
        a.survivor_idx[i0 + j] = f[j] ? r : -1;
        a.logit[i0 + j] = __int_as_float(0x7fc00000);  // NaN until the SNM scores the frame
        a.snm_pass[i0 + j] = 0;
        a.snm_class[i0 + j] = 0;
      }
      r += f[j];
    }
    carry += s_wbase[kWarps];
    __syncthreads();
  }
  const int m = carry;

  // ---------------- pass 2: stream-major work order
  carry = 0;
  for (int base = 0; base < n; base += 4 * kThreads) {
    const int k0 = base + 4 * threadIdx.x;
    bool f[4];
    int fi[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      fi[j] = (k0 + j < n) ? a.perm[k0 + j] : -1;
      f[j] = fi[j] >= 0 && a.pass[fi[j]];
    }
    int wtot;
    const int wr = warp_rank4(f, &wtot);
    if (lane == 0) s_wbase[warp] = wtot;
    __syncthreads();
    if (warp == 0) {
      int w = s_wbase[lane], wi = w;
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        int t = __shfl_up_sync(0xffffffffu, wi, off);
        if (lane >= off) wi += t;
      }
      s_wbase[lane] = wi - w;
      if (lane == 31) s_wbase[kWarps] = wi;
    }
    __syncthreads();
    int r = carry + s_wbase[warp] + wr;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (k0 + j < n) {
        a.posw[k0 + j] = r;
        if (f[j]) a.work[r] = fi[j];
      }
      r += f[j];
    }
    carry += s_wbase[kWarps];
    __syncthreads();
  }
  if (threadIdx.x == 0) a.posw[n] = carry;
  __syncthreads();

  // ---------------- pass 3: per-stream pops of <= BatchSize (dynamic batching, L223); K4 loads a stream's weights
  // once per run of its frames in work order, so a pop's frames share one weight image
  int chunk_carry = 0;
  for (int base = 0; base < a.n_seg; base += kThreads) {
    const int s = base + threadIdx.x;
    int q = 0, B = 1, lo_pos = 0;
    if (s < a.n_seg) {
      lo_pos = a.posw[a.seg_lo[s]];
      q = a.posw[a.seg_lo[s + 1]] - lo_pos;  // this stream's SNM queue depth
      B = a.seg_batch[s];
      if (a.stats && q > 0) {
        unsigned long long* st = a.stats + (int64_t)a.seg_slot[s] * NSTAT;
        atomicAdd(st + 1, (unsigned long long)q);                    // SDD survivors
        if (a.snm_ctas > 0) atomicAdd(st + 7, (unsigned long long)((q + B - 1) / B));  // dynamic batches
      }
    }
    const int nch = (q + B - 1) / B;
    int total;
    const int off = chunk_carry + block_exclusive_scan(nch, s_warp, &total);
    int k = off;
    for (int p = 0; p < nch; ++p) a.chunks[k++] = lo_pos + p * B;
    chunk_carry += total;
  }
  if (threadIdx.x == 0) {
    a.chunks[chunk_carry] = m;
    a.counts[0] = m;
    a.counts[1] = chunk_carry;
    a.counts[2] = 0;
  }
}

}  // namespace

cudaError_t launch_compact(const CompactArgs& a, cudaStream_t st) {
  compact_kernel<<<1, kThreads, 0, st>>>(a);
  return cudaGetLastError();
}

}  // namespace ffsva
