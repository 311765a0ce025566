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
// Transform (TACKER_BE_FFT): one original block = one transform, held in shared memory (8n
// bytes), Stockham autosort radix-8 passes (a final radix-4 or radix-2 pass), so input
// and output are both in natural order and every global access is a coalesced 16-byte vector.
// Pass with sub-transform size Ns (1, R, R^2, ...), butterfly j < n/R, k = j mod Ns:
//   v_r = x[j + r n/R] * w[(r k n / (Ns R)) mod n],  V = DFT_R(v),
//   out[(j / Ns) Ns R + k + r Ns] = V_r,   r < R.
// A pass reads all its inputs into registers, synchronises, then writes in place.  The twiddles
// of a radix-R butterfly are w, w^2, ..., w^(R-1) with w = w[k n / (Ns R)] from the table, the
// powers formed by complex products (one table load per butterfly; a few ulp, far inside the
// gate).  DFT_8 = two DFT_4 combined with W8^k (n = 1024: passes 8, 8, 8, 2).
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
  static constexpr int kMaxN = TK_FFT_MAXN;   // register arrays of one radix-8 butterfly per thread (1024)
  // shared layout XOR-swizzled in 16-complex (128-byte) rows: index i lives at i ^ ((i >> 4) & 15).
  // Consecutive indices stay within their aligned 16-block (reads and staging conflict-free);
  // the Stockham writes of the first pass (stride 4 complex) spread over all 16 slots instead of
  // 4, those of Ns >= 16 stay conflict-free, Ns = 4 drops from 8-way to 4-way.
  static constexpr uint32_t kSmem = kMaxN * 8;
  static __device__ __forceinline__ int pad(int i) { return i ^ ((i >> 4) & 15); }
  static __host__ __device__ int64_t num_blocks(const tacker_be_fft &p) { return p.batch; }

  static __device__ __forceinline__ float2 cmul(float2 a, float2 w) {
    return make_float2(__fsub_rn(__fmul_rn(a.x, w.x), __fmul_rn(a.y, w.y)),
                       __fadd_rn(__fmul_rn(a.x, w.y), __fmul_rn(a.y, w.x)));
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

  template <int R, int NMAX>
  static __device__ __forceinline__ void pass(float2 *s, const float2 *tw, int n, int Ns, int tid, uint32_t bar) {
    constexpr int kMaxBf = NMAX / R / kVbThreads;    // butterflies per thread at n = NMAX
    const int nbf = n / R, q = n / R;
    float2 v[kMaxBf > 0 ? kMaxBf : 1][R];
#pragma unroll
    for (int u = 0; u < (kMaxBf > 0 ? kMaxBf : 1); ++u) {
      const int j = tid + u * kVbThreads;
      if (j < nbf) {
        const int k = j % Ns;
        const int tstep = k * (n / (Ns * R));            // twiddle index step: k n / (Ns R)
        // one table load per butterfly: w^r = w^(r-1) w (complex products)
        const float2 w1 = __ldg(tw + tstep);
        float2 w = w1;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const float2 a = s[pad(j + r * q)];
          v[u][r] = r == 0 ? a : cmul(a, w);
          if (r >= 1) w = cmul(w, w1);
        }
      }
    }
    named_bar_sync(bar, kVbThreads);
#pragma unroll
    for (int u = 0; u < (kMaxBf > 0 ? kMaxBf : 1); ++u) {
      const int j = tid + u * kVbThreads;
      if (j < nbf) {
        const int k = j % Ns;
        const int o = (j / Ns) * Ns * R + k;
        if constexpr (R == 8) {
          // DFT_8 = two DFT_4 (even / odd inputs) combined with W8^k, W8 = exp(-2 pi i / 8)
          float2 e[4], d[4];
          dft4(v[u][0], v[u][2], v[u][4], v[u][6], e);
          dft4(v[u][1], v[u][3], v[u][5], v[u][7], d);
          const float h = 0.70710678118654752f;   // 1/sqrt(2)
          const float2 d1 = make_float2(__fmul_rn(__fadd_rn(d[1].x, d[1].y), h), __fmul_rn(__fsub_rn(d[1].y, d[1].x), h));
          const float2 d2 = mul_mi(d[2]);
          const float2 d3 = make_float2(__fmul_rn(__fsub_rn(d[3].y, d[3].x), h), __fmul_rn(-__fadd_rn(d[3].x, d[3].y), h));
          s[pad(o)] = add(e[0], d[0]);
          s[pad(o + Ns)] = add(e[1], d1);
          s[pad(o + 2 * Ns)] = add(e[2], d2);
          s[pad(o + 3 * Ns)] = add(e[3], d3);
          s[pad(o + 4 * Ns)] = sub(e[0], d[0]);
          s[pad(o + 5 * Ns)] = sub(e[1], d1);
          s[pad(o + 6 * Ns)] = sub(e[2], d2);
          s[pad(o + 7 * Ns)] = sub(e[3], d3);
        } else if constexpr (R == 4) {
          // DFT_4: X0 = (a0+a2)+(a1+a3), X1 = (a0-a2) - i(a1-a3), X2 = (a0+a2)-(a1+a3), X3 = (a0-a2) + i(a1-a3)
          const float2 t0 = add(v[u][0], v[u][2]), t1 = sub(v[u][0], v[u][2]);
          const float2 t2 = add(v[u][1], v[u][3]), t3 = mul_mi(sub(v[u][1], v[u][3]));
          s[pad(o)] = add(t0, t2);
          s[pad(o + Ns)] = add(t1, t3);
          s[pad(o + 2 * Ns)] = sub(t0, t2);
          s[pad(o + 3 * Ns)] = sub(t1, t3);
        } else {
          s[pad(o)] = add(v[u][0], v[u][1]);
          s[pad(o + Ns)] = sub(v[u][0], v[u][1]);
        }
      }
    }
    named_bar_sync(bar, kVbThreads);
  }

  static __device__ __forceinline__ void run(const tacker_be_fft &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    if (p.n <= 512) run_n<(kMaxN < 512 ? kMaxN : 512)>(p, vb, tid, bar, smem);
    else if (p.n <= 1024) run_n<(kMaxN < 1024 ? kMaxN : 1024)>(p, vb, tid, bar, smem);
    else run_n<kMaxN>(p, vb, tid, bar, smem);
  }
  template <int NMAX>
  static __device__ __forceinline__ void run_n(const tacker_be_fft &p, int64_t vb, int tid, uint32_t bar,
                                               uint8_t *smem) {
    float2 *s = reinterpret_cast<float2 *>(smem);
    const float2 *tw = reinterpret_cast<const float2 *>(p.twiddle);
    const int n = p.n;
    const float4 *x = reinterpret_cast<const float4 *>(p.x) + vb * (n / 2);
    named_bar_sync(bar, kVbThreads);        // the previous transform of this slot is written out
    for (int i = tid; i < n / 2; i += kVbThreads) {
      const float4 v = __ldg(x + i);
      s[pad(2 * i)] = make_float2(v.x, v.y);
      s[pad(2 * i + 1)] = make_float2(v.z, v.w);
    }
    named_bar_sync(bar, kVbThreads);
    int Ns = 1;
    for (; Ns * 8 <= n; Ns *= 8) pass<8, NMAX>(s, tw, n, Ns, tid, bar);
    if (Ns * 4 <= n) {
      pass<4, NMAX>(s, tw, n, Ns, tid, bar);
      Ns *= 4;
    }
    if (Ns < n) pass<2, NMAX>(s, tw, n, Ns, tid, bar);
    float4 *y = reinterpret_cast<float4 *>(p.y) + vb * (n / 2);
    for (int i = tid; i < n / 2; i += kVbThreads) {
      const float2 a = s[pad(2 * i)], b = s[pad(2 * i + 1)];
      y[i] = make_float4(a.x, a.y, b.x, b.y);
    }
  }
};

}  // namespace tk
