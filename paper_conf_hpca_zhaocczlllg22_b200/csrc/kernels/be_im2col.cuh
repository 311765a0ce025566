// be_im2col.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- im2col (LC CUDA-core helper)
// Explicit im2col as in the paper's conv->GEMM lowering (cudnnIm2col, §VIII-H):
// block = 1024 groups of 8 consecutive output columns (16 B); with C % 8 == 0 a group is one
// filter tap's 8 channels, copied as one 16-byte load (zero outside the image / past R*S*C).
template <> struct BeBody<TACKER_BE_IM2COL> {
  static constexpr int kMaxGroups = 1024;                 // Kpad / 8 <= 1024 (Kpad <= 8192)
  static constexpr uint32_t kSmem = kMaxGroups * 4;       // per-column-group tap table
  static __host__ __device__ int64_t rows(const tacker_be_im2col &p) {
    const int P = (p.h + 2 * p.pad - p.r) / p.stride + 1, Q = (p.w + 2 * p.pad - p.s) / p.stride + 1;
    return (int64_t)p.n * P * Q;
  }
  static __host__ __device__ int64_t num_blocks(const tacker_be_im2col &p) {
    return (rows(p) * (p.Kpad / 8) + 1023) / 1024;
  }
  // Thread tid handles groups g = 1024 vb + 128 u + tid, u < 8, in order.  The (r, s, c) of a
  // column group is the same in every row, so the block first tabulates it in shared memory
  // (packed r | s << 8 | c << 16; 0xffffffff = padding past R*S*C), and a thread divides only
  // once for its first group, then steps (row m -> (n, p, q), column j) incrementally.  32-bit
  // indices (the host bounds rows * Kpad / 8 < 2^31).
  static __device__ __forceinline__ void run(const tacker_be_im2col &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    const uint32_t P = (uint32_t)((p.h + 2 * p.pad - p.r) / p.stride + 1);
    const uint32_t Q = (uint32_t)((p.w + 2 * p.pad - p.s) / p.stride + 1);
    const uint32_t gpr = (uint32_t)(p.Kpad / 8);
    const uint32_t total = (uint32_t)p.n * P * Q * gpr;
    const int Kreal = p.r * p.s * p.c;
    uint32_t *tab = reinterpret_cast<uint32_t *>(smem);
    const bool vec = (p.c & 7) == 0;
    named_bar_sync(bar, kVbThreads);   // the previous block of this slot is done with the table
    if (vec)
      for (uint32_t jj = tid; jj < gpr; jj += kVbThreads) {
        const int kk = (int)jj * 8;
        uint32_t e = 0xffffffffu;
        if (kk < Kreal) {
          const int c = kk % p.c, rs = kk / p.c;
          e = (uint32_t)(rs / p.s) | ((uint32_t)(rs % p.s) << 8) | ((uint32_t)c << 16);
        }
        tab[jj] = e;
      }
    named_bar_sync(bar, kVbThreads);
    const __half *x = reinterpret_cast<const __half *>(p.x);
    __half *out = reinterpret_cast<__half *>(p.out);
    uint32_t g = (uint32_t)vb * 1024u + (uint32_t)tid;
    if (g >= total) return;
    uint32_t m = g / gpr, j = g - m * gpr;
    uint32_t q = m % Q, t = m / Q, pp = t % P, n = t / P;
    // pass 1: the 8 groups' source (or none) and destination; pass 2: all loads in flight, then
    // all stores (8 independent 16-byte gathers per thread instead of a load-store chain)
    const uint4 *src[8];
    uint32_t dst[8];     // in 16-byte units (rows * Kpad / 8 < 2^31)
    int cnt = 0;
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int h0 = (int)pp * p.stride - p.pad, w0 = (int)q * p.stride - p.pad;
      const int kk0 = (int)j * 8;
      src[u] = nullptr;
      if (vec) {
        const uint32_t e = tab[j];
        if (e != 0xffffffffu) {
          const int hi = h0 + (int)(e & 0xff), wi = w0 + (int)((e >> 8) & 0xff);
          if (hi >= 0 && hi < p.h && wi >= 0 && wi < p.w)
            src[u] = reinterpret_cast<const uint4 *>(x + (((int64_t)n * p.h + hi) * p.w + wi) * p.c + (e >> 16));
        }
        dst[u] = m * gpr + j;
      } else {
        __align__(16) __half ev[8];
        int c = kk0 % p.c, rs = kk0 / p.c;
        int s_ = rs % p.s, r = rs / p.s;
        const __half *xn = x + (int64_t)n * p.h * p.w * p.c;
#pragma unroll
        for (int jv = 0; jv < 8; ++jv) {
          ev[jv] = __float2half(0.f);
          const int hi = h0 + r, wi = w0 + s_;
          if (kk0 + jv < Kreal && hi >= 0 && hi < p.h && wi >= 0 && wi < p.w) ev[jv] = xn[((int64_t)hi * p.w + wi) * p.c + c];
          if (++c == p.c) {
            c = 0;
            if (++s_ == p.s) {
              s_ = 0;
              ++r;
            }
          }
        }
        reinterpret_cast<uint4 *>(out)[(int64_t)m * gpr + j] = *reinterpret_cast<uint4 *>(ev);
      }
      ++cnt;
      // next group of this thread: 128 columns further
      g += kVbThreads;
      if (u == 7 || g >= total) break;
      j += kVbThreads;
      if (j >= gpr) {
        const uint32_t adv = j / gpr;
        j -= adv * gpr;
        m += adv;
        if (adv == 1) {
          if (++q == Q) {
            q = 0;
            if (++pp == P) {
              pp = 0;
              ++n;
            }
          }
        } else {
          q = m % Q;
          t = m / Q;
          pp = t % P;
          n = t / P;
        }
      }
    }
    if (!vec) return;
    uint4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = (u < cnt && src[u]) ? __ldg(src[u]) : make_uint4(0, 0, 0, 0);
    uint4 *o = reinterpret_cast<uint4 *>(out);
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (u < cnt) o[dst[u]] = v[u];
  }
};

}  // namespace tk
