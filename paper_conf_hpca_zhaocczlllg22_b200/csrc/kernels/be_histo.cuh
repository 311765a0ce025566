// be_histo.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- histo
// Block = 32768 inputs: a private u32 histogram of nbins (<= 8192) in shared memory, then one
// global atomicAdd per non-empty bin.  Integer adds commute: bit-exact whatever the order.
template <> struct BeBody<TACKER_BE_HISTO> {
  static constexpr int PER_BLOCK = 32768;
  static constexpr uint32_t kSmem = 8192 * 4;
  static __host__ __device__ int64_t num_blocks(const tacker_be_histo &p) {
    return ((int64_t)p.n + PER_BLOCK - 1) / PER_BLOCK;
  }
  static __device__ __forceinline__ void run(const tacker_be_histo &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    uint32_t *h = reinterpret_cast<uint32_t *>(smem);
    for (int b = tid; b < p.nbins; b += kVbThreads) h[b] = 0;
    named_bar_sync(bar, kVbThreads);
    const int64_t base = vb * PER_BLOCK;
    const int64_t end = min((int64_t)p.n, base + PER_BLOCK);
    if (base + PER_BLOCK <= p.n && (p.n & 3) == 0) {
      const uint4 *in4 = reinterpret_cast<const uint4 *>(p.in + base);
#pragma unroll 4
      for (int i = tid; i < PER_BLOCK / 4; i += kVbThreads) {
        const uint4 v = __ldg(in4 + i);
        atomicAdd(&h[v.x], 1u);
        atomicAdd(&h[v.y], 1u);
        atomicAdd(&h[v.z], 1u);
        atomicAdd(&h[v.w], 1u);
      }
    } else {
      for (int64_t i = base + tid; i < end; i += kVbThreads) atomicAdd(&h[__ldg(p.in + i)], 1u);
    }
    named_bar_sync(bar, kVbThreads);
    for (int b = tid; b < p.nbins; b += kVbThreads) {
      const uint32_t c = h[b];
      if (c) atomicAdd(p.count + b, c);
    }
    named_bar_sync(bar, kVbThreads);  // shared histogram reusable by the next block
  }
};

}  // namespace tk
