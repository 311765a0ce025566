// be_im2col.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- im2col (LC CUDA-core helper)
// Explicit im2col as in the paper's conv->GEMM lowering (cudnnIm2col, §VIII-H):
// block = 1024 groups of 8 consecutive output columns (16 B); with C % 8 == 0 a group is one
// filter tap's 8 channels, copied as one 16-byte load (zero outside the image / past R*S*C).
template <> struct BeBody<TACKER_BE_IM2COL> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t rows(const tacker_be_im2col &p) {
    const int P = (p.h + 2 * p.pad - p.r) / p.stride + 1, Q = (p.w + 2 * p.pad - p.s) / p.stride + 1;
    return (int64_t)p.n * P * Q;
  }
  static __host__ __device__ int64_t num_blocks(const tacker_be_im2col &p) {
    return (rows(p) * (p.Kpad / 8) + 1023) / 1024;
  }
  static __device__ __forceinline__ void run(const tacker_be_im2col &p, int64_t vb, int tid, uint32_t, uint8_t *) {
    // 32-bit index math (the host bounds rows * Kpad / 8 < 2^31); (r, s, c) of a group's 8
    // columns is stepped incrementally instead of divided per element
    const uint32_t P = (uint32_t)((p.h + 2 * p.pad - p.r) / p.stride + 1);
    const uint32_t Q = (uint32_t)((p.w + 2 * p.pad - p.s) / p.stride + 1);
    const uint32_t gpr = (uint32_t)(p.Kpad / 8);
    const uint32_t total = (uint32_t)p.n * P * Q * gpr;
    const int Kreal = p.r * p.s * p.c;
    const __half *x = reinterpret_cast<const __half *>(p.x);
    __half *out = reinterpret_cast<__half *>(p.out);
#pragma unroll 2
    for (int u = 0; u < 8; ++u) {
      const uint32_t g = (uint32_t)vb * 1024u + (uint32_t)(u * 128 + tid);
      if (g >= total) return;
      const uint32_t m = g / gpr;
      const int kk0 = (int)(g - m * gpr) * 8;
      const uint32_t mq = m / Q;
      const int q = (int)(m - mq * Q), pp = (int)(mq % P), n = (int)(mq / P);
      const int h0 = pp * p.stride - p.pad, w0 = q * p.stride - p.pad;
      const __half *xn = x + (int64_t)n * p.h * p.w * p.c;
      uint4 v = make_uint4(0, 0, 0, 0);
      if ((p.c & 7) == 0) {
        if (kk0 < Kreal) {
          const int c = kk0 % p.c, rs = kk0 / p.c, s = rs % p.s, r = rs / p.s;
          const int hi = h0 + r, wi = w0 + s;
          if (hi >= 0 && hi < p.h && wi >= 0 && wi < p.w)
            v = __ldg(reinterpret_cast<const uint4 *>(xn + ((int64_t)hi * p.w + wi) * p.c + c));
        }
      } else {
        __align__(16) __half e[8];
        int c = kk0 % p.c, rs = kk0 / p.c;
        int s = rs % p.s, r = rs / p.s;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          e[j] = __float2half(0.f);
          const int hi = h0 + r, wi = w0 + s;
          if (kk0 + j < Kreal && hi >= 0 && hi < p.h && wi >= 0 && wi < p.w) e[j] = xn[((int64_t)hi * p.w + wi) * p.c + c];
          if (++c == p.c) {
            c = 0;
            if (++s == p.s) {
              s = 0;
              ++r;
            }
          }
        }
        v = *reinterpret_cast<uint4 *>(e);
      }
      *reinterpret_cast<uint4 *>(out + (int64_t)m * p.Kpad + kk0) = v;
    }
  }
};

}  // namespace tk
