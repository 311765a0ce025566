// be_spmv.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- spmv JDS (Parboil)
// Thread per JDS row i (block = 128 rows): y[perm[i]] = sum_{d<row_len[i]} val*x[col] at
// jds_ptr[d]+i, d ascending; consecutive i touch consecutive addresses of each diagonal.
template <> struct BeBody<TACKER_BE_SPMV_JDS> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_spmv &p) { return (p.rows + 127) / 128; }
  static __device__ __forceinline__ void run(const tacker_be_spmv &p, int64_t vb, int tid, uint32_t, uint8_t *) {
    const int64_t i = vb * 128 + tid;
    if (i >= p.rows) return;
    const int len = p.row_len[i];
    float acc = 0.f;
    for (int d = 0; d < len; ++d) {
      const int64_t e = (int64_t)__ldg(p.jds_ptr + d) + i;
      acc = __fmaf_rn(__ldg(p.val + e), __ldg(p.x + __ldg(p.col + e)), acc);
    }
    p.y[p.perm[i]] = acc;
  }
};

}  // namespace tk
