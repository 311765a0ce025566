// be_mriq.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- mri-q (Parboil)
template <> struct BeBody<TACKER_BE_MRIQ_PHIMAG> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_mriq_phimag &p) { return (p.numK + 511) / 512; }
  static __device__ __forceinline__ void run(const tacker_be_mriq_phimag &p, int64_t vb, int tid, uint32_t,
                                             uint8_t *) {
#pragma unroll
    for (int h = 0; h < 4; ++h) {
      const int64_t k = vb * 512 + h * 128 + tid;
      if (k < p.numK) {
        const float r = p.phiR[k], i = p.phiI[k];
        p.phiMag[k] = __fadd_rn(__fmul_rn(r, r), __fmul_rn(i, i));
      }
    }
  }
};

// Q: original block = 32 voxels x 4 k-chains: thread tid owns voxel 32 vb + tid/4 and the terms
// k = j (mod 4), j = tid % 4, accumulated in increasing k; the four partial sums of a voxel are
// combined as Q_in + ((s0 + s1) + (s2 + s3)) through two butterfly shuffles.  k is staged through
// shared memory in chunks of 512 as float4 (kx, ky, kz, phiMag); MUFU sin/cos of 2*pi*t with
// t = kx x + ky y + kz z (optionally range-reduced to t - rint(t) first, TK_MRIQ_REDUCE).
// Splitting each voxel's k-sum over 4 lanes cuts one block's sequential MUFU chain to K/4 terms,
// so a short PTB slice of this kernel is not stuck on a one-block latency floor (reading 13);
// the order is fixed per voxel, so fused and original launches stay bit-identical.
template <> struct BeBody<TACKER_BE_MRIQ_Q> {
  static constexpr int KC = 512;
  static constexpr int kKChains = 4;
  static constexpr int kVoxels = kVbThreads / kKChains;   // voxels per original block
  // at most this many original blocks per fused virtual block at once (independent chains per
  // thread where the fused CTA has few BE warps); the fused PTB loop gives every CTA an even
  // share, see be_ptb_loop
  static constexpr int kCoarsen = TK_MRIQ_COARSEN;
  static constexpr uint32_t kSmem = KC * 16;
  static __host__ __device__ int64_t num_blocks(const tacker_be_mriq_q &p) {
    return (p.numX + kVoxels - 1) / kVoxels;
  }
  static __device__ __forceinline__ void run(const tacker_be_mriq_q &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    run_v<1>(p, vb, 1, tid, bar, smem);
  }
  // fused virtual block = up to kCoarsen consecutive original blocks, one voxel chain of each per
  // thread; each voxel's arithmetic is unchanged, so results stay bit-identical.
  static __device__ __forceinline__ void run_coarse(const tacker_be_mriq_q &p, int64_t vb, int nb, int tid,
                                                    uint32_t bar, uint8_t *smem) {
    static_assert(kCoarsen >= 1 && kCoarsen <= 4, "run_coarse dispatches 1..4 blocks per thread");
    if (kCoarsen >= 4 && nb >= 4) run_v<(kCoarsen >= 4 ? 4 : 1)>(p, vb, 4, tid, bar, smem);
    else if (kCoarsen >= 3 && nb == 3) run_v<(kCoarsen >= 3 ? 3 : 1)>(p, vb, 3, tid, bar, smem);
    else if (kCoarsen >= 2 && nb >= 2) run_v<(kCoarsen >= 2 ? 2 : 1)>(p, vb, 2, tid, bar, smem);
    else run_v<1>(p, vb, 1, tid, bar, smem);
  }
  static __device__ __forceinline__ void term(const float4 kv, float x, float y, float z, float &qr, float &qi) {
    const float kTwoPi = 6.2831853071795864769f;
    float t = __fmaf_rn(kv.z, z, __fmaf_rn(kv.y, y, __fmul_rn(kv.x, x)));
#if TK_MRIQ_REDUCE
#if TK_MRIQ_RINT
    t = __fsub_rn(t, rintf(t));         // FRND: the same value as the magic-number form, one instruction
#else
    const float kMagic = 12582912.0f;   // 1.5 * 2^23: (t + M) - M == rint(t) for |t| < 2^22
    t = __fsub_rn(t, __fsub_rn(__fadd_rn(t, kMagic), kMagic));
#endif
#endif
    float s, c;
    __sincosf(__fmul_rn(kTwoPi, t), &s, &c);
    qr = __fmaf_rn(kv.w, c, qr);
    qi = __fmaf_rn(kv.w, s, qi);
  }
  template <int VPT>
  static __device__ __forceinline__ void run_v(const tacker_be_mriq_q &p, int64_t vb, int nb, int tid, uint32_t bar,
                                               uint8_t *smem) {
    float4 *ks = reinterpret_cast<float4 *>(smem);
    const int j = tid % kKChains, lv = tid / kKChains;
    int64_t v[VPT];
    float xs[VPT], ys[VPT], zs[VPT], qr[VPT], qi[VPT];
#pragma unroll
    for (int h = 0; h < VPT; ++h) {
      v[h] = h < nb ? (vb + h) * kVoxels + lv : (int64_t)p.numX;
      const bool ok = v[h] < p.numX;
      xs[h] = ok ? p.x[v[h]] : 0.f;
      ys[h] = ok ? p.y[v[h]] : 0.f;
      zs[h] = ok ? p.z[v[h]] : 0.f;
      qr[h] = qi[h] = 0.f;
    }
    static_assert(KC % kKChains == 0, "chunk starts keep k mod kKChains");
    for (int k0 = 0; k0 < p.numK; k0 += KC) {
      const int kn = min(KC, p.numK - k0);
      named_bar_sync(bar, kVbThreads);  // previous chunk fully consumed
      for (int k = tid; k < kn; k += kVbThreads)
        ks[k] = make_float4(p.kx[k0 + k], p.ky[k0 + k], p.kz[k0 + k], p.phiMag[k0 + k]);
      named_bar_sync(bar, kVbThreads);
#pragma unroll 4
      for (int k = j; k < kn; k += kKChains) {
        const float4 kv = ks[k];
#pragma unroll
        for (int h = 0; h < VPT; ++h) term(kv, xs[h], ys[h], zs[h], qr[h], qi[h]);
      }
    }
    static_assert(kKChains == 4, "the butterfly below combines 4 chains: (s0 + s1) + (s2 + s3)");
#pragma unroll
    for (int h = 0; h < VPT; ++h) {
      // IEEE addition is commutative, so both lanes of each pair hold the same bits
      float r = __fadd_rn(qr[h], __shfl_xor_sync(0xffffffffu, qr[h], 1));
      float i = __fadd_rn(qi[h], __shfl_xor_sync(0xffffffffu, qi[h], 1));
      r = __fadd_rn(r, __shfl_xor_sync(0xffffffffu, r, 2));
      i = __fadd_rn(i, __shfl_xor_sync(0xffffffffu, i, 2));
      if (j == 0 && v[h] < p.numX) {
        p.Qr[v[h]] = __fadd_rn(p.Qr[v[h]], r);
        p.Qi[v[h]] = __fadd_rn(p.Qi[v[h]], i);
      }
    }
  }
};

}  // namespace tk
