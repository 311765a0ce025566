// be_mrifhd.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- mri-fhd (Parboil, Table II)
// NEXT-3.  The paper does not define the kernel (DESIGN.md §2 reading 14): ComputeRhoPhi is the
// complex product conj(phi) d, ComputeFH the adjoint non-uniform Fourier sum F^H (rho phi) over
// one k chunk.  FH has mri-q's shape with a complex weight (2 MUFU + 4 FMA per voxel-k pair
// instead of 2 + 2), so it reuses mri-q's mapping: a block is 32 voxels x 4 k-lanes, k staged in
// shared memory 512 at a time, each voxel's sum kept as 4 partial sums over k mod 4 combined as
// F_in + ((s0 + s1) + (s2 + s3)), and coarsened in fused CTAs with a static even split.
template <> struct BeBody<TACKER_BE_MRIFHD_RHOPHI> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_mrifhd_rhophi &p) { return (p.numK + 511) / 512; }
  static __device__ __forceinline__ void run(const tacker_be_mrifhd_rhophi &p, int64_t vb, int tid, uint32_t,
                                             uint8_t *) {
#pragma unroll
    for (int h = 0; h < 4; ++h) {
      const int64_t k = vb * 512 + h * 128 + tid;
      if (k < p.numK) {
        const float pr = p.phiR[k], pi = p.phiI[k], dr = p.dR[k], di = p.dI[k];
        p.rRhoPhi[k] = __fadd_rn(__fmul_rn(pr, dr), __fmul_rn(pi, di));
        p.iRhoPhi[k] = __fsub_rn(__fmul_rn(pr, di), __fmul_rn(pi, dr));
      }
    }
  }
};

template <> struct BeBody<TACKER_BE_MRIFHD_FH> {
  static constexpr int KC = 512;
  static constexpr int kKChains = 4;
  static constexpr int kVoxels = kVbThreads / kKChains;
  static constexpr int kCoarsen = TK_MRIQ_COARSEN;
  static constexpr uint32_t kSmem = KC * 16 + KC * 4;   // float4 (kx, ky, kz, rRhoPhi) + iRhoPhi
  static __host__ __device__ int64_t num_blocks(const tacker_be_mrifhd_fh &p) {
    return (p.numX + kVoxels - 1) / kVoxels;
  }
  static __device__ __forceinline__ void run(const tacker_be_mrifhd_fh &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    run_v<1>(p, vb, 1, tid, bar, smem);
  }
  static __device__ __forceinline__ void run_coarse(const tacker_be_mrifhd_fh &p, int64_t vb, int nb, int tid,
                                                    uint32_t bar, uint8_t *smem) {
    static_assert(kCoarsen >= 1 && kCoarsen <= 4, "run_coarse dispatches 1..4 blocks per thread");
    if (kCoarsen >= 4 && nb >= 4) run_v<(kCoarsen >= 4 ? 4 : 1)>(p, vb, 4, tid, bar, smem);
    else if (kCoarsen >= 3 && nb == 3) run_v<(kCoarsen >= 3 ? 3 : 1)>(p, vb, 3, tid, bar, smem);
    else if (kCoarsen >= 2 && nb >= 2) run_v<(kCoarsen >= 2 ? 2 : 1)>(p, vb, 2, tid, bar, smem);
    else run_v<1>(p, vb, 1, tid, bar, smem);
  }
  // rF += rRho cos - iRho sin; iF += iRho cos + rRho sin (each as two rounded FMAs, fixed order)
  static __device__ __forceinline__ void term(const float4 kv, float ri, float x, float y, float z, float &fr,
                                              float &fi) {
    const float kTwoPi = 6.2831853071795864769f;
    float t = __fmaf_rn(kv.z, z, __fmaf_rn(kv.y, y, __fmul_rn(kv.x, x)));
#if TK_MRIQ_REDUCE
    const float kMagic = 12582912.0f;   // 1.5 * 2^23: (t + M) - M == rint(t) for |t| < 2^22
    t = __fsub_rn(t, __fsub_rn(__fadd_rn(t, kMagic), kMagic));
#endif
    float s, c;
    __sincosf(__fmul_rn(kTwoPi, t), &s, &c);
    fr = __fmaf_rn(-ri, s, __fmaf_rn(kv.w, c, fr));
    fi = __fmaf_rn(kv.w, s, __fmaf_rn(ri, c, fi));
  }
  template <int VPT>
  static __device__ __forceinline__ void run_v(const tacker_be_mrifhd_fh &p, int64_t vb, int nb, int tid, uint32_t bar,
                                               uint8_t *smem) {
    float4 *ks = reinterpret_cast<float4 *>(smem);
    float *ris = reinterpret_cast<float *>(smem + KC * 16);
    const int j = tid % kKChains, lv = tid / kKChains;
    int64_t v[VPT];
    float xs[VPT], ys[VPT], zs[VPT], fr[VPT], fi[VPT];
#pragma unroll
    for (int h = 0; h < VPT; ++h) {
      v[h] = h < nb ? (vb + h) * kVoxels + lv : (int64_t)p.numX;
      const bool ok = v[h] < p.numX;
      xs[h] = ok ? p.x[v[h]] : 0.f;
      ys[h] = ok ? p.y[v[h]] : 0.f;
      zs[h] = ok ? p.z[v[h]] : 0.f;
      fr[h] = fi[h] = 0.f;
    }
    static_assert(KC % kKChains == 0, "chunk starts keep k mod kKChains");
    for (int k0 = 0; k0 < p.numK; k0 += KC) {
      const int kn = min(KC, p.numK - k0);
      named_bar_sync(bar, kVbThreads);  // previous chunk fully consumed
      for (int k = tid; k < kn; k += kVbThreads) {
        ks[k] = make_float4(p.kx[k0 + k], p.ky[k0 + k], p.kz[k0 + k], p.rRhoPhi[k0 + k]);
        ris[k] = p.iRhoPhi[k0 + k];
      }
      named_bar_sync(bar, kVbThreads);
#pragma unroll 4
      for (int k = j; k < kn; k += kKChains) {
        const float4 kv = ks[k];
        const float ri = ris[k];
#pragma unroll
        for (int h = 0; h < VPT; ++h) term(kv, ri, xs[h], ys[h], zs[h], fr[h], fi[h]);
      }
    }
    static_assert(kKChains == 4, "the butterfly below combines 4 chains: (s0 + s1) + (s2 + s3)");
#pragma unroll
    for (int h = 0; h < VPT; ++h) {
      float r = __fadd_rn(fr[h], __shfl_xor_sync(0xffffffffu, fr[h], 1));
      float i = __fadd_rn(fi[h], __shfl_xor_sync(0xffffffffu, fi[h], 1));
      r = __fadd_rn(r, __shfl_xor_sync(0xffffffffu, r, 2));
      i = __fadd_rn(i, __shfl_xor_sync(0xffffffffu, i, 2));
      if (j == 0 && v[h] < p.numX) {
        p.rFhD[v[h]] = __fadd_rn(p.rFhD[v[h]], r);
        p.iFhD[v[h]] = __fadd_rn(p.iFhD[v[h]], i);
      }
    }
  }
};

}  // namespace tk
