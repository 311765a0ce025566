// be_fft.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- fft (Parboil, Table II)
// NEXT-3, the GEMM-fft pair of Fig. 10.  Batched forward complex DFT of a
// power-of-two length n (DESIGN.md §2 reading 15): X[k] = sum_j x[j] exp(-2 pi i j k / n).
//
// Twiddle table (TACKER_BE_FFT_TWIDDLE, the "plan" step, one launch per n):
//   w[m] = (cospi(2m/n), -sinpi(2m/n)), m < n, with the accurate sincospi (not the MUFU).
// Transform (TACKER_BE_FFT): one original block = kT transforms (2), Stockham autosort: one
// radix-2/4/8/16 pass, then radix-8 passes (n = 1024: 16, 8, 8), so input and output are both
// in natural order; the first pass reads x from global memory and the last writes y to it
// (coalesced 8-byte accesses), intermediate results sit in shared memory (8n bytes).
// Pass with sub-transform size Ns (1, R, R^2, ...), butterfly j < n/R, k = j mod Ns:
//   v_r = x[j + r n/R] * w[(r k n / (Ns R)) mod n],  V = DFT_R(v),
//   out[(j / Ns) Ns R + k + r Ns] = V_r,   r < R.
// A pass reads all its inputs into registers, synchronises, then writes in place.  The twiddles
// of a radix-R butterfly are w, w^2, ..., w^(R-1) with w = w[k n / (Ns R)] from the table, the
// powers formed by complex products (one table load per butterfly; a few ulp, far inside the
// gate; radix 16 loads w, w^4, w^8, w^12 and forms the rest with at most two products).
// DFT_8 = two DFT_4 combined with W8^k; DFT_16 = 4 x 4 with W16^(n2 k1) between the stages.
template <> struct BeBody<TACKER_BE_FFT_TWIDDLE> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_fft &p) { return (p.n + 127) / 128; }
  static __device__ __forceinline__ void run(const tacker_be_fft &p, int64_t vb, int tid, uint32_t, uint8_t *) {
    const int m = (int)vb * 128 + tid;
    if (m < p.n) {
      float s, c;
      sincospif(__fdiv_rn(2.f * (float)m, (float)p.n), &s, &c);   // 2m/n is exact (n a power of 2)
      reinterpret_cast<float2 *>(p.twiddle)[m] = make_float2(c, -s);
    }
  }
};

template <> struct BeBody<TACKER_BE_FFT> {
  static constexpr int kMaxN = TK_FFT_MAXN;   // register arrays of one radix-16 butterfly per thread (1024)
  // shared layout XOR-swizzled in 16-complex (128-byte) rows: index i lives at i ^ ((i >> 4) & 15).
  // Consecutive indices stay within their aligned 16-block (reads and staging conflict-free);
  // the Stockham writes of the first pass (stride 4 complex) spread over all 16 slots instead of
  // 4, those of Ns >= 16 stay conflict-free, Ns = 4 drops from 8-way to 4-way.
  // kT transforms per original block (TK_FFT_PER_BLOCK): with 2, a radix-16 pass of n = 1024 keeps
  // all 128 threads busy (64 butterflies per transform) and every thread has twice the loads
  // in flight, so a vblock of the fused kernel (fewer resident warps) hides more latency.
  static constexpr int kT = TK_FFT_PER_BLOCK;
#if TK_FFT_ODD_FIRST
  static_assert(kMaxN == 1024, "run() dispatches the static plans of n = 2 .. 1024");
#endif
  static constexpr uint32_t kSmem = kT * kMaxN * 8;
  static __device__ __forceinline__ int pad(int i) { return i ^ ((i >> 4) & 15); }
  static __host__ __device__ int64_t num_blocks(const tacker_be_fft &p) { return (p.batch + kT - 1) / kT; }

  // complex product, contracted to two FMUL + two FFMA (the gate is 1e-5 of the signal scale)
  static __device__ __forceinline__ float2 cmul(float2 a, float2 w) {
    return make_float2(fmaf(a.x, w.x, -(a.y * w.y)), fmaf(a.x, w.y, a.y * w.x));
  }
  static __device__ __forceinline__ float2 add(float2 a, float2 b) { return make_float2(__fadd_rn(a.x, b.x), __fadd_rn(a.y, b.y)); }
  static __device__ __forceinline__ float2 sub(float2 a, float2 b) { return make_float2(__fsub_rn(a.x, b.x), __fsub_rn(a.y, b.y)); }
  // multiply by -i (forward transform)
  static __device__ __forceinline__ float2 mul_mi(float2 a) { return make_float2(a.y, -a.x); }

  // DFT_4 (forward): Y0 = (b0+b2)+(b1+b3), Y1 = (b0-b2) - i(b1-b3), Y2 = (b0+b2)-(b1+b3), Y3 = (b0-b2) + i(b1-b3)
  static __device__ __forceinline__ void dft4(float2 b0, float2 b1, float2 b2, float2 b3, float2 (&y)[4]) {
    const float2 t0 = add(b0, b2), t1 = sub(b0, b2), t2 = add(b1, b3), t3 = mul_mi(sub(b1, b3));
    y[0] = add(t0, t2);
    y[1] = add(t1, t3);
    y[2] = sub(t0, t2);
    y[3] = sub(t1, t3);
  }

  // W16^m = exp(-2 pi i m / 16) products used inside DFT_16 (m in {1, 2, 3, 4, 6, 9})
  static constexpr float kC1 = 0.92387953251128674f, kS1 = 0.38268343236508978f, kH = 0.70710678118654752f;
  static __device__ __forceinline__ float2 w16_2(float2 a) {   // (h, -h)
    return make_float2(__fmul_rn(__fadd_rn(a.x, a.y), kH), __fmul_rn(__fsub_rn(a.y, a.x), kH));
  }
  static __device__ __forceinline__ float2 w16_6(float2 a) {   // (-h, -h)
    return make_float2(__fmul_rn(__fsub_rn(a.y, a.x), kH), __fmul_rn(-__fadd_rn(a.x, a.y), kH));
  }

  // y[r] = sum_m v[m] W_R^(m r) for R in {2, 4, 8, 16}
  template <int R>
  static __device__ __forceinline__ void dft(const float2 (&v)[R], float2 (&y)[R]) {
    if constexpr (R == 16) {
      // n = 4 n1 + n2, k = k1 + 4 k2:  X[k] = DFT_4 over n2 of W16^(n2 k1) * DFT_4 over n1 of v[4 n1 + n2]
      float2 a[4][4];
#pragma unroll
      for (int n2 = 0; n2 < 4; ++n2) dft4(v[n2], v[n2 + 4], v[n2 + 8], v[n2 + 12], a[n2]);
      a[1][1] = cmul(a[1][1], make_float2(kC1, -kS1));
      a[1][2] = w16_2(a[1][2]);
      a[1][3] = cmul(a[1][3], make_float2(kS1, -kC1));
      a[2][1] = w16_2(a[2][1]);
      a[2][2] = mul_mi(a[2][2]);
      a[2][3] = w16_6(a[2][3]);
      a[3][1] = cmul(a[3][1], make_float2(kS1, -kC1));
      a[3][2] = w16_6(a[3][2]);
      a[3][3] = cmul(a[3][3], make_float2(-kC1, kS1));
#pragma unroll
      for (int k1 = 0; k1 < 4; ++k1) {
        float2 z[4];
        dft4(a[0][k1], a[1][k1], a[2][k1], a[3][k1], z);
#pragma unroll
        for (int k2 = 0; k2 < 4; ++k2) y[k1 + 4 * k2] = z[k2];
      }
    } else if constexpr (R == 8) {
      // DFT_8 = two DFT_4 (even / odd inputs) combined with W8^k, W8 = exp(-2 pi i / 8)
      float2 e[4], d[4];
      dft4(v[0], v[2], v[4], v[6], e);
      dft4(v[1], v[3], v[5], v[7], d);
      const float2 d1 = w16_2(d[1]), d2 = mul_mi(d[2]), d3 = w16_6(d[3]);
      y[0] = add(e[0], d[0]);
      y[1] = add(e[1], d1);
      y[2] = add(e[2], d2);
      y[3] = add(e[3], d3);
      y[4] = sub(e[0], d[0]);
      y[5] = sub(e[1], d1);
      y[6] = sub(e[2], d2);
      y[7] = sub(e[3], d3);
    } else if constexpr (R == 4) {
      dft4(v[0], v[1], v[2], v[3], y);
    } else {
      y[0] = add(v[0], v[1]);
      y[1] = sub(v[0], v[1]);
    }
  }

  // One Stockham pass.  kIn: the first pass (Ns = 1, no twiddles) reads x straight from global
  // memory (thread j loads x[j + r n/R]: consecutive j, coalesced); kOut: the last pass
  // (Ns = n/R, o = j) writes y[j + r Ns] straight to global memory.  In-between results live in
  // shared memory, so a transform moves 16n bytes through shared memory per middle boundary and
  // none for staging.  The shared buffer is free on entry to a kIn pass (run_n's leading barrier).
  // Butterfly g < nt n/R of the block's nt transforms: transform h = g / (n/R), j = g mod (n/R);
  // transform h lives at s + h n in shared memory and at gx + h n, gy + h n in global memory.
  template <int R, int NMAX, bool kIn, bool kOut>
  static __device__ __forceinline__ void pass(float2 *s0, const float2 *gx0, float2 *gy0, const float2 *tw, int n,
                                              int nt, int Ns, int tid, uint32_t bar) {
    constexpr int kMaxBf = kT * NMAX / R / kVbThreads > 0 ? kT * NMAX / R / kVbThreads : 1;   // per thread
    // n, Ns, R are powers of two: shifts and masks instead of integer division
    constexpr int lR = R == 2 ? 1 : R == 4 ? 2 : R == 8 ? 3 : 4;
    const int ln = __ffs(n) - 1, ls = __ffs(Ns) - 1;
    const int nbf = n >> lR, q = nbf, lbf = ln - lR;
    float2 v[kMaxBf][R];
#pragma unroll
    for (int u = 0; u < kMaxBf; ++u) {
      const int g = tid + u * kVbThreads;
      const int j = g & (nbf - 1), hn = (g >> lbf) * n;
      const float2 *gx = gx0 + hn;
      const float2 *s = s0 + hn;
      if (g < nt * nbf) {
        if constexpr (kIn) {
#pragma unroll
          for (int r = 0; r < R; ++r) v[u][r] = __ldg(gx + j + r * q);
        } else {
          const int k = j & (Ns - 1);
          const int tstep = k << (ln - ls - lR);           // twiddle index step: k n / (Ns R)
#pragma unroll
          for (int r = 0; r < R; ++r) v[u][r] = s[pad(j + r * q)];
          const float2 w1 = __ldg(tw + tstep);
          if constexpr (R == 16) {
            // w^(4a + b) = w^(4a) w^b: table loads of w, w^4, w^8, w^12, at most two products each
            const float2 w2 = cmul(w1, w1), w3 = cmul(w2, w1);
#pragma unroll
            for (int a4 = 0; a4 < 4; ++a4) {
              const float2 wa = a4 == 0 ? make_float2(1.f, 0.f) : __ldg(tw + 4 * a4 * tstep);
              if (a4) v[u][4 * a4] = cmul(v[u][4 * a4], wa);
              v[u][4 * a4 + 1] = cmul(v[u][4 * a4 + 1], a4 ? cmul(wa, w1) : w1);
              v[u][4 * a4 + 2] = cmul(v[u][4 * a4 + 2], a4 ? cmul(wa, w2) : w2);
              v[u][4 * a4 + 3] = cmul(v[u][4 * a4 + 3], a4 ? cmul(wa, w3) : w3);
            }
          } else {
            // one table load per butterfly: w^r = w^(r-1) w (complex products)
            float2 w = w1;
#pragma unroll
            for (int r = 1; r < R; ++r) {
              v[u][r] = cmul(v[u][r], w);
              w = cmul(w, w1);
            }
          }
        }
      }
    }
    if constexpr (!kIn) named_bar_sync(bar, kVbThreads);   // every read done before the in-place writes
#pragma unroll
    for (int u = 0; u < kMaxBf; ++u) {
      const int g = tid + u * kVbThreads;
      const int j = g & (nbf - 1), hn = (g >> lbf) * n;
      float2 *gy = gy0 + hn;
      float2 *s = s0 + hn;
      if (g < nt * nbf) {
        const int k = j & (Ns - 1);
        const int o = ((j >> ls) << (ls + lR)) + k;
        float2 y[R];
        dft<R>(v[u], y);
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if constexpr (kOut) gy[o + r * Ns] = y[r];
          else s[pad(o + r * Ns)] = y[r];
        }
      }
    }
    if constexpr (!kOut) named_bar_sync(bar, kVbThreads);
  }

  template <int R, int NMAX>
  static __device__ __forceinline__ void last_pass(bool first, float2 *s, const float2 *gx, float2 *gy,
                                                   const float2 *tw, int n, int nt, int Ns, int tid, uint32_t bar) {
    if (first) pass<R, NMAX, true, true>(s, gx, gy, tw, n, nt, Ns, tid, bar);
    else pass<R, NMAX, false, true>(s, gx, gy, tw, n, nt, Ns, tid, bar);
  }

  static __device__ __forceinline__ void run(const tacker_be_fft &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
#if TK_FFT_ODD_FIRST
    // one straight-line pass sequence per n (compile-time plan): inside the fused PTB loop the
    // generic plan (a runtime loop over radix-8 passes and a radix switch, nested in the block loop)
    // was register-allocated to 2.4 KB of spills per thread at any cap; the static sequences are not
    switch (p.n) {
      case 2: run_static<1>(p, vb, tid, bar, smem); return;
      case 4: run_static<2>(p, vb, tid, bar, smem); return;
      case 8: run_static<3>(p, vb, tid, bar, smem); return;
      case 16: run_static<4>(p, vb, tid, bar, smem); return;
      case 32: run_static<5>(p, vb, tid, bar, smem); return;
      case 64: run_static<6>(p, vb, tid, bar, smem); return;
      case 128: run_static<7>(p, vb, tid, bar, smem); return;
      case 256: run_static<8>(p, vb, tid, bar, smem); return;
      case 512: run_static<9>(p, vb, tid, bar, smem); return;
      default: run_static<10>(p, vb, tid, bar, smem); return;   // 1024 (validated on the host)
    }
#else
    if (p.n <= 512) run_n<(kMaxN < 512 ? kMaxN : 512)>(p, vb, tid, bar, smem);
    else if (p.n <= 1024) run_n<(kMaxN < 1024 ? kMaxN : 1024)>(p, vb, tid, bar, smem);
    else run_n<kMaxN>(p, vb, tid, bar, smem);
#endif
  }
  // The same plan as run_n (radix-2^f pass first, then p8 radix-8 passes) with n = 2^L fixed at
  // compile time: identical butterflies in identical order, so identical results.
  template <int L>
  static __device__ __forceinline__ void run_static(const tacker_be_fft &p, int64_t vb, int tid, uint32_t bar,
                                                    uint8_t *smem) {
    constexpr int N = 1 << L;
    constexpr int P8 = L <= 4 ? 0 : L % 3 == 0 ? L / 3 - 1 : L % 3 == 1 ? (L - 4) / 3 : (L - 2) / 3;
    constexpr int F = L <= 4 ? L : L % 3 == 0 ? 3 : L % 3 == 1 ? 4 : 2;
    constexpr int R0 = 1 << F;
    float2 *s = reinterpret_cast<float2 *>(smem);
    const float2 *tw = reinterpret_cast<const float2 *>(p.twiddle);
    const int nt = p.batch - vb * kT < kT ? (int)(p.batch - vb * kT) : kT;
    const float2 *gx = reinterpret_cast<const float2 *>(p.x) + vb * kT * N;
    float2 *gy = reinterpret_cast<float2 *>(p.y) + vb * kT * N;
    named_bar_sync(bar, kVbThreads);        // the previous transform of this slot is done with s
    if constexpr (P8 == 0) {
      pass<R0, N, true, true>(s, gx, gy, tw, N, nt, 1, tid, bar);
    } else {
      pass<R0, N, true, false>(s, gx, gy, tw, N, nt, 1, tid, bar);
      radix8_passes<N, P8 - 1>(s, gx, gy, tw, nt, R0, tid, bar);
    }
  }
  // M middle radix-8 passes from sub-transform size Ns, then the last one (writes global memory)
  template <int N, int M>
  static __device__ __forceinline__ void radix8_passes(float2 *s, const float2 *gx, float2 *gy, const float2 *tw,
                                                       int nt, int Ns, int tid, uint32_t bar) {
    if constexpr (M == 0) {
      pass<8, N, false, true>(s, gx, gy, tw, N, nt, Ns, tid, bar);
    } else {
      pass<8, N, false, false>(s, gx, gy, tw, N, nt, Ns, tid, bar);
      radix8_passes<N, M - 1>(s, gx, gy, tw, nt, Ns * 8, tid, bar);
    }
  }
  // Pass plan for n = 2^L: one radix-2^f pass (f in {1, 2, 3, 4}) and p8 radix-8 passes, the
  // radix-2^f one first (TK_FFT_ODD_FIRST) or last; n = 1024: 16, 8, 8 — two shared-memory
  // boundaries (was 8, 8, 8, 2 with staging: 110 -> 56 us for 16384 x 1024, 0.73 of HBM).
  template <int NMAX>
  static __device__ __forceinline__ void run_n(const tacker_be_fft &p, int64_t vb, int tid, uint32_t bar,
                                               uint8_t *smem) {
    float2 *s = reinterpret_cast<float2 *>(smem);
    const float2 *tw = reinterpret_cast<const float2 *>(p.twiddle);
    const int n = p.n;
    const int nt = p.batch - vb * kT < kT ? (int)(p.batch - vb * kT) : kT;   // transforms of this block
    const float2 *gx = reinterpret_cast<const float2 *>(p.x) + vb * kT * n;
    float2 *gy = reinterpret_cast<float2 *>(p.y) + vb * kT * n;
    const int L = __ffs(n) - 1;
    int p8, f;
    if (L <= 4) p8 = 0, f = L;
    else if (L % 3 == 0) p8 = L / 3 - 1, f = 3;
    else if (L % 3 == 1) p8 = (L - 4) / 3, f = 4;
    else p8 = (L - 2) / 3, f = 2;
    named_bar_sync(bar, kVbThreads);        // the previous transform of this slot is done with s
#if TK_FFT_ODD_FIRST
    if (p8 > 0) {
      // the radix-2^f pass first (reads global), then the radix-8 passes (the last one writes global)
      switch (f) {
        case 1: pass<2, NMAX, true, false>(s, gx, gy, tw, n, nt, 1, tid, bar); break;
        case 2: pass<4, NMAX, true, false>(s, gx, gy, tw, n, nt, 1, tid, bar); break;
        case 3: pass<8, NMAX, true, false>(s, gx, gy, tw, n, nt, 1, tid, bar); break;
        default: pass<16, NMAX, true, false>(s, gx, gy, tw, n, nt, 1, tid, bar); break;
      }
      int Ns = 1 << f;
      for (int i = 0; i < p8 - 1; ++i, Ns *= 8) pass<8, NMAX, false, false>(s, gx, gy, tw, n, nt, Ns, tid, bar);
      pass<8, NMAX, false, true>(s, gx, gy, tw, n, nt, Ns, tid, bar);
      return;
    }
#endif
    int Ns = 1;
    for (int i = 0; i < p8; ++i, Ns *= 8) {
      if (i == 0) pass<8, NMAX, true, false>(s, gx, gy, tw, n, nt, Ns, tid, bar);
      else pass<8, NMAX, false, false>(s, gx, gy, tw, n, nt, Ns, tid, bar);
    }
    const bool first = p8 == 0;
    switch (f) {
      case 1: last_pass<2, NMAX>(first, s, gx, gy, tw, n, nt, Ns, tid, bar); break;
      case 2: last_pass<4, NMAX>(first, s, gx, gy, tw, n, nt, Ns, tid, bar); break;
      case 3: last_pass<8, NMAX>(first, s, gx, gy, tw, n, nt, Ns, tid, bar); break;
      default: last_pass<16, NMAX>(first, s, gx, gy, tw, n, nt, Ns, tid, bar); break;
    }
  }
};

}  // namespace tk
