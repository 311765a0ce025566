// be_sgemm.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- sgemm (Parboil)
// C[M,N] = alpha * A[M,K] . B[K,N] + beta * C, row-major fp32.  Block = 64x64 tile of C,
// thread (ty = tid/16, tx = tid%16) owns rows 8ty..8ty+7, cols 4tx..4tx+3.  K is staged in
// chunks of 16 through double-buffered shared memory.  acc = fma(a_k, b_k, acc), k ascending.
template <> struct BeBody<TACKER_BE_SGEMM> {
  static constexpr int BM = 64, BN = 64, BK = 16;
  static constexpr uint32_t kSmem = 2 * BK * (BM + 4) * 4 + 2 * BK * BN * 4;
  static __host__ __device__ int64_t num_blocks(const tacker_be_sgemm &p) {
    return (int64_t)((p.M + BM - 1) / BM) * ((p.N + BN - 1) / BN);
  }
  static __device__ __forceinline__ void run(const tacker_be_sgemm &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    float(*As)[BK][BM + 4] = reinterpret_cast<float(*)[BK][BM + 4]>(smem);
    float(*Bs)[BK][BN] = reinterpret_cast<float(*)[BK][BN]>(smem + 2 * BK * (BM + 4) * 4);
    const int tiles_n = (p.N + BN - 1) / BN;
    const int m0 = (int)(vb / tiles_n) * BM, n0 = (int)(vb % tiles_n) * BN;
    const int ty = tid >> 4, tx = tid & 15;
    float acc[8][4];
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;

    float4 ra[2], rb[2];
    auto load = [&](int k0) {
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int idx = tid + h * 128;          // 256 float4 per operand tile
        const int ar = idx >> 2, ac = (idx & 3) * 4;   // A: 64 rows x 4 float4
        const int gm = m0 + ar, gk = k0 + ac;
        ra[h] = (gm < p.M && gk < p.K) ? __ldg(reinterpret_cast<const float4 *>(p.A + (size_t)gm * p.K + gk))
                                      : make_float4(0.f, 0.f, 0.f, 0.f);
        const int br = idx >> 4, bc = (idx & 15) * 4;  // B: 16 rows x 16 float4
        const int gk2 = k0 + br, gn = n0 + bc;
        rb[h] = (gk2 < p.K && gn < p.N) ? __ldg(reinterpret_cast<const float4 *>(p.B + (size_t)gk2 * p.N + gn))
                                       : make_float4(0.f, 0.f, 0.f, 0.f);
      }
    };
    auto store = [&](int buf) {
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int idx = tid + h * 128;
        const int ar = idx >> 2, ac = (idx & 3) * 4;
        As[buf][ac + 0][ar] = ra[h].x;
        As[buf][ac + 1][ar] = ra[h].y;
        As[buf][ac + 2][ar] = ra[h].z;
        As[buf][ac + 3][ar] = ra[h].w;
        const int br = idx >> 4, bc = (idx & 15) * 4;
        *reinterpret_cast<float4 *>(&Bs[buf][br][bc]) = rb[h];
      }
    };
    const int nk = (p.K + BK - 1) / BK;
    load(0);
    store(0);
    named_bar_sync(bar, kVbThreads);
    for (int kc = 0; kc < nk; ++kc) {
      const int buf = kc & 1;
      if (kc + 1 < nk) load((kc + 1) * BK);
#pragma unroll
      for (int k = 0; k < BK; ++k) {
        const float4 a0 = *reinterpret_cast<const float4 *>(&As[buf][k][ty * 8]);
        const float4 a1 = *reinterpret_cast<const float4 *>(&As[buf][k][ty * 8 + 4]);
        const float4 b = *reinterpret_cast<const float4 *>(&Bs[buf][k][tx * 4]);
        const float av[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const float bv[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) acc[i][j] = __fmaf_rn(av[i], bv[j], acc[i][j]);
      }
      if (kc + 1 < nk) store(buf ^ 1);
      named_bar_sync(bar, kVbThreads);
    }
    const int gn = n0 + tx * 4;
    if (gn >= p.N) return;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int gm = m0 + ty * 8 + i;
      if (gm >= p.M) break;
      float *c = p.C + (size_t)gm * p.N + gn;
      float4 o;
      if (p.beta != 0.f) {
        const float4 ci = *reinterpret_cast<const float4 *>(c);
        o.x = __fadd_rn(__fmul_rn(p.alpha, acc[i][0]), __fmul_rn(p.beta, ci.x));
        o.y = __fadd_rn(__fmul_rn(p.alpha, acc[i][1]), __fmul_rn(p.beta, ci.y));
        o.z = __fadd_rn(__fmul_rn(p.alpha, acc[i][2]), __fmul_rn(p.beta, ci.z));
        o.w = __fadd_rn(__fmul_rn(p.alpha, acc[i][3]), __fmul_rn(p.beta, ci.w));
      } else {
        o.x = __fmul_rn(p.alpha, acc[i][0]);
        o.y = __fmul_rn(p.alpha, acc[i][1]);
        o.z = __fmul_rn(p.alpha, acc[i][2]);
        o.w = __fmul_rn(p.alpha, acc[i][3]);
      }
      *reinterpret_cast<float4 *>(c) = o;
    }
  }
};

}  // namespace tk
