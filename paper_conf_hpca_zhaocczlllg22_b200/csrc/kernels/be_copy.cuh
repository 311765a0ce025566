// be_copy.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- copy (query I/O)
// 16 KiB per block, 16-byte vectors, 8 independent loads in flight per thread.
template <> struct BeBody<TACKER_BE_COPY> {
  static constexpr uint32_t kSmem = 0;
  static constexpr int64_t kBlockBytes = 16384;
  static __host__ __device__ int64_t num_blocks(const tacker_be_copy &p) {
    return (p.bytes + kBlockBytes - 1) / kBlockBytes;
  }
  static __device__ __forceinline__ void run(const tacker_be_copy &p, int64_t vb, int tid, uint32_t, uint8_t *) {
    const uint4 *src = reinterpret_cast<const uint4 *>(p.src);
    uint4 *dst = reinterpret_cast<uint4 *>(p.dst);
    const int64_t n16 = p.bytes / 16;
    const int64_t base = vb * (kBlockBytes / 16);
    uint4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t i = base + u * 128 + tid;
      if (i < n16) v[u] = src[i];
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t i = base + u * 128 + tid;
      if (i < n16) dst[i] = v[u];
    }
  }
};

}  // namespace tk
