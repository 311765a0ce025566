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

// Q: block = 512 voxels (thread owns tid + 128h, h < 4); k staged through shared memory in
// chunks of 512 as float4 (kx, ky, kz, phiMag).  Phase in turns t = kx x + ky y + kz z is
// range-reduced exactly (t - rint(t), Sterbenz; rint by the 1.5*2^23 magic add so the XU pipe
// only runs the two MUFU ops) before the MUFU sin/cos of 2*pi*t.
template <> struct BeBody<TACKER_BE_MRIQ_Q> {
  static constexpr int KC = 512;
  // at most this many original blocks per fused virtual block at once (independent MUFU chains
  // per thread; the fused PTB loop gives every CTA an even share, see be_ptb_loop)
  static constexpr int kCoarsen = TK_MRIQ_COARSEN;
  static constexpr uint32_t kSmem = KC * 16;
  static __host__ __device__ int64_t num_blocks(const tacker_be_mriq_q &p) { return (p.numX + 127) / 128; }
  // original block = 128 voxels, one per thread
  static __device__ __forceinline__ void run(const tacker_be_mriq_q &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    run_v<1>(p, vb, 1, tid, bar, smem);
  }
  // fused virtual block = up to kCoarsen consecutive original blocks, thread owns one voxel of
  // each (more independent MUFU chains per thread where the fused CTA has few BE warps); each
  // voxel's k-ordered accumulation is unchanged, so results stay bit-identical.
  static __device__ __forceinline__ void run_coarse(const tacker_be_mriq_q &p, int64_t vb, int nb, int tid,
                                                    uint32_t bar, uint8_t *smem) {
    // exact chain count (a masked voxel would still spend its MUFU slots)
    static_assert(kCoarsen <= 4, "run_coarse dispatches 1..4 voxels per thread");
    if (nb >= 4) run_v<4>(p, vb, 4, tid, bar, smem);
    else if (nb == 3) run_v<3>(p, vb, 3, tid, bar, smem);
    else if (nb == 2) run_v<2>(p, vb, 2, tid, bar, smem);
    else run_v<1>(p, vb, 1, tid, bar, smem);
  }
  template <int VPT>
  static __device__ __forceinline__ void run_v(const tacker_be_mriq_q &p, int64_t vb, int nb, int tid, uint32_t bar,
                                               uint8_t *smem) {
    float4 *ks = reinterpret_cast<float4 *>(smem);
    const float kTwoPi = 6.2831853071795864769f;
    const float kMagic = 12582912.0f;   // 1.5 * 2^23: (t + M) - M == rint(t) for |t| < 2^22
    int64_t v[VPT];
    float xs[VPT], ys[VPT], zs[VPT], qr[VPT], qi[VPT];
#pragma unroll
    for (int h = 0; h < VPT; ++h) v[h] = h < nb ? (vb + h) * 128 + tid : (int64_t)p.numX;
#pragma unroll
    for (int h = 0; h < VPT; ++h) {
      const bool ok = v[h] < p.numX;
      xs[h] = ok ? p.x[v[h]] : 0.f;
      ys[h] = ok ? p.y[v[h]] : 0.f;
      zs[h] = ok ? p.z[v[h]] : 0.f;
      qr[h] = ok ? p.Qr[v[h]] : 0.f;
      qi[h] = ok ? p.Qi[v[h]] : 0.f;
    }
    for (int k0 = 0; k0 < p.numK; k0 += KC) {
      const int kn = min(KC, p.numK - k0);
      named_bar_sync(bar, kVbThreads);  // previous chunk fully consumed
      for (int k = tid; k < kn; k += kVbThreads)
        ks[k] = make_float4(p.kx[k0 + k], p.ky[k0 + k], p.kz[k0 + k], p.phiMag[k0 + k]);
      named_bar_sync(bar, kVbThreads);
#pragma unroll 2
      for (int k = 0; k < kn; ++k) {
        const float4 kv = ks[k];
#pragma unroll
        for (int h = 0; h < VPT; ++h) {
          float t = __fmaf_rn(kv.z, zs[h], __fmaf_rn(kv.y, ys[h], __fmul_rn(kv.x, xs[h])));
#if TK_MRIQ_REDUCE
          const float r = __fsub_rn(__fadd_rn(t, kMagic), kMagic);
          t = __fsub_rn(t, r);
#endif
          const float arg = __fmul_rn(kTwoPi, t);
          float s, c;
          __sincosf(arg, &s, &c);
          qr[h] = __fmaf_rn(kv.w, c, qr[h]);
          qi[h] = __fmaf_rn(kv.w, s, qi[h]);
        }
      }
    }
#pragma unroll
    for (int h = 0; h < VPT; ++h)
      if (v[h] < p.numX) {
        p.Qr[v[h]] = qr[h];
        p.Qi[v[h]] = qi[h];
      }
  }
};

}  // namespace tk
