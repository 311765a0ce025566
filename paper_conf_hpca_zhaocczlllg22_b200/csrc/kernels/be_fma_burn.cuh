// be_fma_burn.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- fma_burn ("Kc", §III-B)
// Register-only FMA chains: thread g = vb*128+tid runs x_j <- fma(x_j, a, (j+1) b), j < 4,
// from x_j = (g%97 + j)/128, for `iters` steps; out[g] = ((x0+x1)+x2)+x3.
template <> struct BeBody<TACKER_BE_FMA_BURN> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_fma_burn &p) {
    return (p.n_threads + kVbThreads - 1) / kVbThreads;
  }
  static __device__ __forceinline__ void run(const tacker_be_fma_burn &p, int64_t vb, int tid, uint32_t,
                                             uint8_t *) {
    const int64_t g = vb * kVbThreads + tid;
    if (g >= p.n_threads) return;
    const float base = (float)(g % 97);
    float x0 = __fdiv_rn(base + 0.f, 128.f), x1 = __fdiv_rn(base + 1.f, 128.f);
    float x2 = __fdiv_rn(base + 2.f, 128.f), x3 = __fdiv_rn(base + 3.f, 128.f);
    const float a = p.a, b0 = p.b, b1 = __fmul_rn(2.f, p.b), b2 = __fmul_rn(3.f, p.b), b3 = __fmul_rn(4.f, p.b);
#pragma unroll 4
    for (int it = 0; it < p.iters; ++it) {
      x0 = __fmaf_rn(x0, a, b0);
      x1 = __fmaf_rn(x1, a, b1);
      x2 = __fmaf_rn(x2, a, b2);
      x3 = __fmaf_rn(x3, a, b3);
    }
    p.out[g] = __fadd_rn(__fadd_rn(__fadd_rn(x0, x1), x2), x3);
  }
};

}  // namespace tk
