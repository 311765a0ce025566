// be_tpacf.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- tpacf (Parboil, Table II)
// NEXT-3, two-point angular correlation histogram (DESIGN.md §2 reading 16):
//   count[bin(a_i . b_j)] += 1 over all pairs (cross) or over i < j (self, b = a),
//   bin(d) = #{k : d < edges[k]},  d = ((ax bx + ay by) + az bz) in fp32 without FMA.
// Block = 128 points of a (thread t owns a_i) x a chunk of 2048 points of b (so even a 16k-point
// self correlation has ~1000 blocks to spread over the SMs); b is staged through shared memory
// 512 points at a time (as float4); the bin is a branch-free binary search over the edges (strictly
// decreasing, held in shared memory: distinct edges sit in distinct banks, so the search loads
// never conflict); every thread counts into its own shared-memory column hist[bin][t]
// (conflict-free shared atomics whose result is unused, so no load-use chain per pair), and the block adds its column sums to the global
// u32 counters with one atomicAdd per bin.  Integer counts: any order gives the same bits.
template <> struct BeBody<TACKER_BE_TPACF> {
  static constexpr int kStage = 512;          // b points per shared-memory stage
  static constexpr int kJChunk = 2048;        // b points per original block
  static constexpr int kMaxEdges = 31;
  static constexpr int kEdgeSlots = 32;
  static constexpr uint32_t kSmem = kStage * 16 + kEdgeSlots * 4 + (kMaxEdges + 1) * kVbThreads * 4;
  static __host__ __device__ int64_t jblocks(const tacker_be_tpacf &p) { return (p.nb + kJChunk - 1) / kJChunk; }
  static __host__ __device__ int64_t num_blocks(const tacker_be_tpacf &p) {
    return (int64_t)((p.na + 127) / 128) * jblocks(p);
  }
  static __device__ __forceinline__ int bin_of(const float *se, float d) {
    // #{k : d < e_k} for decreasing e: the first index whose edge is <= d
    int lo = 0;
#pragma unroll
    for (int step = 16; step >= 1; step >>= 1)
      if (se[lo + step - 1] > d) lo += step;
    return lo;
  }
  static __device__ __forceinline__ void run(const tacker_be_tpacf &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    float4 *sb = reinterpret_cast<float4 *>(smem);   // b points as (x, y, z, -): one 16-byte load per pair
    float *se = reinterpret_cast<float *>(sb + kStage);
    uint32_t *hist = reinterpret_cast<uint32_t *>(se + kEdgeSlots);
    const int nbins = p.nedges + 1;
    const int64_t nj = jblocks(p);
    const int ib = (int)(vb / nj), jb = (int)(vb % nj);
    const int i0 = ib * 128, i = i0 + tid;
    const int jlo = jb * kJChunk, jhi = min(p.nb, jlo + kJChunk);
    // self pairs: only j > i; a chunk entirely at or below this block's points has no pair
    const int j_begin = p.self_pairs ? max(jlo, i0 + 1) : jlo;
    if (j_begin >= jhi) return;                 // uniform per block: no barrier is skipped by part of it
    named_bar_sync(bar, kVbThreads);            // previous block of this slot has read its histogram
    for (int k = tid; k < kEdgeSlots; k += kVbThreads) se[k] = k < p.nedges ? p.edges[k] : -INFINITY;
    for (int b = 0; b < nbins; ++b) hist[b * kVbThreads + tid] = 0u;
    const bool live = i < p.na;
    const float ax = live ? p.a[3 * i] : 0.f, ay = live ? p.a[3 * i + 1] : 0.f, az = live ? p.a[3 * i + 2] : 0.f;
    uint32_t *col = hist + tid;
    for (int j0 = j_begin; j0 < jhi; j0 += kStage) {
      const int n = min(kStage, jhi - j0);
      named_bar_sync(bar, kVbThreads);
      for (int t = tid; t < n; t += kVbThreads)
        sb[t] = make_float4(p.b[3 * (j0 + t)], p.b[3 * (j0 + t) + 1], p.b[3 * (j0 + t) + 2], 0.f);
      named_bar_sync(bar, kVbThreads);
      if (!live) continue;
      int t = p.self_pairs ? max(0, i + 1 - j0) : 0;
      // two independent pairs per iteration (two search chains in flight); the counters are
      // this thread's own column, bumped with fire-and-forget shared atomics (no load-use chain)
      for (; t + 1 < n; t += 2) {
        const float4 b0p = sb[t], b1p = sb[t + 1];
        const float d0 = __fadd_rn(__fadd_rn(__fmul_rn(ax, b0p.x), __fmul_rn(ay, b0p.y)), __fmul_rn(az, b0p.z));
        const float d1 = __fadd_rn(__fadd_rn(__fmul_rn(ax, b1p.x), __fmul_rn(ay, b1p.y)), __fmul_rn(az, b1p.z));
        const int b0 = bin_of(se, d0), b1 = bin_of(se, d1);
        atomicAdd(col + b0 * kVbThreads, 1u);
        atomicAdd(col + b1 * kVbThreads, 1u);
      }
      if (t < n) {
        const float4 b0p = sb[t];
        const float d0 = __fadd_rn(__fadd_rn(__fmul_rn(ax, b0p.x), __fmul_rn(ay, b0p.y)), __fmul_rn(az, b0p.z));
        atomicAdd(col + bin_of(se, d0) * kVbThreads, 1u);
      }
    }
    named_bar_sync(bar, kVbThreads);
    for (int b = tid; b < nbins; b += kVbThreads) {
      uint32_t s = 0;
      for (int t = 0; t < kVbThreads; ++t) s += hist[b * kVbThreads + ((t + b) & (kVbThreads - 1))];
      if (s) atomicAdd(p.count + b, s);
    }
  }
};

}  // namespace tk
