// be_bodies.cuh — BE (best-effort, CUDA-core) kernel bodies.
//
// Each body executes ONE original thread block ("virtual block", 128 threads = 4 warps) of a
// Parboil/Rodinia-style kernel given its block id `vb` and the thread id `tid` rebased into
// [0,128) (the "thread_step" of Fig. 5).  Partial-CTA synchronisation uses
// `bar.sync bar_id, 128` (Fig. 9), never __syncthreads().  The same body is
// called by the fused kernel (PTB loop, Fig. 7) and by the original non-persistent kernel,
// so their outputs are bit-identical: all floating-point arithmetic uses explicit
// round-to-nearest intrinsics (no FMA contraction differences between call sites) and a
// per-element order that does not depend on which CTA runs the block.
#pragma once
#include <cuda_fp16.h>
#include <cstdint>

#include "ptx.cuh"
#include "tacker.h"

namespace tk {

constexpr int kVbThreads = 128;
#ifndef TK_STENCIL_ZC
#define TK_STENCIL_ZC 4
#endif
#ifndef TK_MRIQ_COARSEN
#define TK_MRIQ_COARSEN 4
#endif
#ifndef TK_MRIQ_REDUCE
#define TK_MRIQ_REDUCE 0
#endif

template <int KIND> struct BeBody;

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

// ---------------------------------------------------------------- stencil (Parboil)
// One 7-point Jacobi sweep over A0[nz][ny][nx] (x fastest), HBM-bound.  Block = 128 x 4 x 4
// (x,y,z) cells: lane l of warp w owns x = 4l..4l+3 (one float4) of row y = w for ZC = 4 planes.
// The centre column's ZC+2 planes are loaded up front (memory-level parallelism), x+-1 comes
// from the neighbouring lanes' float4 by shuffle, y+-1 rows through L1/L2.
//   interior: An = c1*(((((W+E)+S)+N)+B)+T) - c0*A   (S/N = y-1/y+1, B/T = z-1/z+1)
//   boundary cells (x, y or z on the faces) are copied.
// nx % 4 != 0 uses the scalar path with the same per-element arithmetic.
template <> struct BeBody<TACKER_BE_STENCIL> {
  static constexpr uint32_t kSmem = 0;
  static constexpr int ZC = TK_STENCIL_ZC;
  static __host__ __device__ int64_t num_blocks(const tacker_be_stencil &p) {
    return (int64_t)((p.nx + 127) / 128) * ((p.ny + 3) / 4) * ((p.nz + ZC - 1) / ZC);
  }
  static __device__ __forceinline__ float point(const tacker_be_stencil &p, float w, float e, float s, float n,
                                                float b, float t, float c) {
    float sum = __fadd_rn(w, e);
    sum = __fadd_rn(sum, s);
    sum = __fadd_rn(sum, n);
    sum = __fadd_rn(sum, b);
    sum = __fadd_rn(sum, t);
    return __fsub_rn(__fmul_rn(p.c1, sum), __fmul_rn(p.c0, c));
  }
  static __device__ __forceinline__ void run(const tacker_be_stencil &p, int64_t vb, int tid, uint32_t,
                                             uint8_t *) {
    const int bx = (p.nx + 127) / 128, by = (p.ny + 3) / 4;
    const int zb = (int)(vb / ((int64_t)bx * by));
    const int rem = (int)(vb % ((int64_t)bx * by));
    const int lane = tid & 31;
    const int x0 = (rem % bx) * 128 + 4 * lane;
    const int y = (rem / bx) * 4 + (tid >> 5);
    const int z0 = zb * ZC;
    if (y >= p.ny) return;                     // warp-uniform
    const size_t plane = (size_t)p.nx * p.ny;
    const float *__restrict__ A = p.A0;
    float *__restrict__ An = p.Anext;
    const bool ybord = (y == 0) | (y == p.ny - 1);
    if ((p.nx & 3) == 0) {
      const bool act = x0 < p.nx;
      const size_t row = (size_t)y * p.nx + x0;
      float4 c[ZC + 2];
#pragma unroll
      for (int i = 0; i < ZC + 2; ++i) {
        const int z = z0 - 1 + i;
        c[i] = (act && z >= 0 && z < p.nz) ? __ldg(reinterpret_cast<const float4 *>(A + z * plane + row))
                                           : make_float4(0.f, 0.f, 0.f, 0.f);
      }
#pragma unroll
      for (int i = 0; i < ZC; ++i) {
        const int z = z0 + i;
        if (z >= p.nz) break;                  // warp-uniform
        const float4 cc = c[i + 1];
        float wv = __shfl_up_sync(0xffffffffu, cc.w, 1);
        float ev = __shfl_down_sync(0xffffffffu, cc.x, 1);
        if (!act) continue;
        float4 o = cc;
        const bool zb_ = (z == 0) | (z == p.nz - 1);
        if (!ybord && !zb_) {
          if (lane == 0) wv = x0 > 0 ? __ldg(A + z * plane + row - 1) : 0.f;
          if (lane == 31 || x0 + 4 >= p.nx) ev = x0 + 4 < p.nx ? __ldg(A + z * plane + row + 4) : 0.f;
          const float4 s = __ldg(reinterpret_cast<const float4 *>(A + z * plane + row - p.nx));
          const float4 n = __ldg(reinterpret_cast<const float4 *>(A + z * plane + row + p.nx));
          const float4 b = c[i], t = c[i + 2];
          if (x0 > 0) o.x = point(p, wv, cc.y, s.x, n.x, b.x, t.x, cc.x);
          o.y = point(p, cc.x, cc.z, s.y, n.y, b.y, t.y, cc.y);
          o.z = point(p, cc.y, cc.w, s.z, n.z, b.z, t.z, cc.z);
          if (x0 + 3 < p.nx - 1) o.w = point(p, cc.z, ev, s.w, n.w, b.w, t.w, cc.w);
        }
        *reinterpret_cast<float4 *>(An + z * plane + row) = o;
      }
      return;
    }
    // scalar path (nx % 4 != 0)
    for (int e = 0; e < 4; ++e) {
      const int x = x0 + e;
      if (x >= p.nx) break;
      const size_t col = (size_t)y * p.nx + x;
      for (int z = z0; z < min(z0 + ZC, p.nz); ++z) {
        const size_t o = z * plane + col;
        const bool bord = ybord | (x == 0) | (x == p.nx - 1) | (z == 0) | (z == p.nz - 1);
        An[o] = bord ? A[o]
                     : point(p, A[o - 1], A[o + 1], A[o - p.nx], A[o + p.nx], A[o - plane], A[o + plane], A[o]);
      }
    }
  }
};

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
  // original blocks one fused virtual block runs at once (measured sweep 2/3/4/6 on the bench
  // grid: 4 is fastest; per-thread MUFU ILP outweighs the 86 % unit balance of 512 units)
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
    run_v<kCoarsen>(p, vb, nb, tid, bar, smem);
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

// ---------------------------------------------------------------- cutcp (Parboil)
// Cutoff Coulomb potential.  Block = one atom bin = an 8x8x8 lattice region; thread t owns the
// points (x = t%8, y = (t/8)%8, z = t/64 + 2m), m < 4, sharing dx, dy across its 4 points.
// Neighbour bins within ceil(cutoff / bin side) are visited in (z, y, x) order, their atom slots
// staged through shared memory 512 at a time, summed in slot order (deterministic):
//   r2 = dz^2 + (dy^2 + dx^2);  e = ((q * rsqrt(r2)) * s) * s,  s = 1 - r2/c^2;  for r2 < c^2
//   V = 0 if any r2 < excl^2.
template <> struct BeBody<TACKER_BE_CUTCP> {
  static constexpr int kStage = 512;
  static constexpr uint32_t kSmem = kStage * 16;
  static __host__ __device__ int64_t num_blocks(const tacker_be_cutcp &p) {
    return (int64_t)p.bdim_x * p.bdim_y * p.bdim_z;
  }
  static __device__ __forceinline__ void run(const tacker_be_cutcp &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    float4 *st = reinterpret_cast<float4 *>(smem);
    const int rbx = (int)(vb % p.bdim_x), rby = (int)((vb / p.bdim_x) % p.bdim_y);
    const int rbz = (int)(vb / ((int64_t)p.bdim_x * p.bdim_y));
    const int i = rbx * 8 + (tid & 7), j = rby * 8 + ((tid >> 3) & 7), k0 = rbz * 8 + (tid >> 6);
    const float px = (float)i * p.h, py = (float)j * p.h;
    float pz[4], acc[4] = {0.f, 0.f, 0.f, 0.f};
    bool ex[4] = {false, false, false, false};
#pragma unroll
    for (int m = 0; m < 4; ++m) pz[m] = (float)(k0 + 2 * m) * p.h;
    const float c2 = __fmul_rn(p.cutoff, p.cutoff), e2 = __fmul_rn(p.excl, p.excl);
    const float inv_c2 = __fdiv_rn(1.f, c2);
    const int reach = (int)ceilf(p.cutoff / p.bin_size);
    const int bx0 = max(rbx - reach, 0), bx1 = min(rbx + reach, p.bdim_x - 1);
    const int by0 = max(rby - reach, 0), by1 = min(rby + reach, p.bdim_y - 1);
    const int bz0 = max(rbz - reach, 0), bz1 = min(rbz + reach, p.bdim_z - 1);
    const int nxr = bx1 - bx0 + 1;
    const float4 *bins = reinterpret_cast<const float4 *>(p.bins);
    // one x-row of neighbour bins (<= 7 bins) per round, only their occupied slots, compacted in
    // (bin, slot) order
    for (int bz = bz0; bz <= bz1; ++bz)
    for (int by = by0; by <= by1; ++by) {
      const int64_t row = ((int64_t)bz * p.bdim_y + by) * p.bdim_x;
      int cnt[7], off[7], n = 0;
#pragma unroll
      for (int q = 0; q < 7; ++q) {
        cnt[q] = q < nxr ? min(__ldg(p.count + row + bx0 + q), p.bin_depth) : 0;
        off[q] = n;
        n += cnt[q];
      }
      for (int a = tid; a < n; a += kVbThreads) {
        int q = 0;
#pragma unroll
        for (int u = 1; u < 7; ++u) q += (a >= off[u] && u < nxr) ? 1 : 0;
        st[a] = __ldg(bins + (row + bx0 + q) * p.bin_depth + (a - off[q]));
      }
      named_bar_sync(bar, kVbThreads);
#pragma unroll 4
      for (int a = 0; a < n; ++a) {
        const float4 at = st[a];
        const float dx = __fsub_rn(at.x, px), dy = __fsub_rn(at.y, py);
        const float dxy2 = __fmaf_rn(dy, dy, __fmul_rn(dx, dx));
#pragma unroll
        for (int m = 0; m < 4; ++m) {
          const float dz = __fsub_rn(at.z, pz[m]);
          const float r2 = __fmaf_rn(dz, dz, dxy2);
          const float s = __fmaf_rn(-r2, inv_c2, 1.f);
          const float e = __fmul_rn(__fmul_rn(__fmul_rn(at.w, rsqrtf(r2)), s), s);
          acc[m] = r2 < c2 ? __fadd_rn(acc[m], e) : acc[m];
          ex[m] = ex[m] | (r2 < e2);
        }
      }
      named_bar_sync(bar, kVbThreads);
    }
    if (i < p.nx && j < p.ny) {
#pragma unroll
      for (int m = 0; m < 4; ++m) {
        const int k = k0 + 2 * m;
        if (k < p.nz) p.V[((int64_t)k * p.ny + j) * p.nx + i] = ex[m] ? 0.f : acc[m];
      }
    }
  }
};

// Deterministic binning for cutcp: thread = bin; atoms scanned in index order through shared
// memory, an atom goes to bin (floor(z/bs), floor(y/bs), floor(x/bs)) clamped into the grid.
template <> struct BeBody<TACKER_BE_CUTCP_BIN> {
  static constexpr int kStage = 1024;
  static constexpr uint32_t kSmem = kStage * 16;
  static __host__ __device__ int64_t num_blocks(const tacker_be_cutcp_bin &p) {
    return ((int64_t)p.bdim_x * p.bdim_y * p.bdim_z + 127) / 128;
  }
  static __device__ __forceinline__ void run(const tacker_be_cutcp_bin &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    float4 *st = reinterpret_cast<float4 *>(smem);
    const int64_t nb = (int64_t)p.bdim_x * p.bdim_y * p.bdim_z;
    const int64_t b = vb * 128 + tid;
    const float4 *atoms = reinterpret_cast<const float4 *>(p.atoms);
    float4 *bins = reinterpret_cast<float4 *>(p.bins);
    int cnt = 0;
    for (int c = 0; c < p.natoms; c += kStage) {
      const int n = min(kStage, p.natoms - c);
      named_bar_sync(bar, kVbThreads);
      for (int a = tid; a < n; a += kVbThreads) st[a] = __ldg(atoms + c + a);
      named_bar_sync(bar, kVbThreads);
      if (b < nb) {
        for (int a = 0; a < n; ++a) {
          const float4 at = st[a];
          const int ix = min(max((int)floorf(__fdiv_rn(at.x, p.bin_size)), 0), p.bdim_x - 1);
          const int iy = min(max((int)floorf(__fdiv_rn(at.y, p.bin_size)), 0), p.bdim_y - 1);
          const int iz = min(max((int)floorf(__fdiv_rn(at.z, p.bin_size)), 0), p.bdim_z - 1);
          if (((int64_t)iz * p.bdim_y + iy) * p.bdim_x + ix == b) {
            if (cnt < p.bin_depth) bins[b * p.bin_depth + cnt] = at;
            ++cnt;
          }
        }
      }
    }
    if (b < nb) {
      for (int s = cnt; s < p.bin_depth; ++s) bins[b * p.bin_depth + s] = make_float4(1e30f, 1e30f, 1e30f, 0.f);
      p.count[b] = cnt;
      if (cnt > p.bin_depth) *p.overflow = 1;
    }
  }
};

// ---------------------------------------------------------------- lbm (Parboil)
// D3Q19 BGK push step, SoA src/dst [19][cells], block = 128 consecutive cells (x fastest).
// Direction order C N S E W T B NE NW SE SW NT NB ST SB ET EB WT WB.
__constant__ int8_t kLbmE[19][3] = {{0, 0, 0},  {0, 1, 0},  {0, -1, 0}, {1, 0, 0},   {-1, 0, 0},
                                    {0, 0, 1},  {0, 0, -1}, {1, 1, 0},  {-1, 1, 0},  {1, -1, 0},
                                    {-1, -1, 0}, {0, 1, 1}, {0, 1, -1}, {0, -1, 1},  {0, -1, -1},
                                    {1, 0, 1},  {1, 0, -1}, {-1, 0, 1}, {-1, 0, -1}};
__constant__ int8_t kLbmOpp[19] = {0, 2, 1, 4, 3, 6, 5, 10, 9, 8, 7, 14, 13, 12, 11, 18, 17, 16, 15};

template <> struct BeBody<TACKER_BE_LBM> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_lbm &p) {
    return ((int64_t)p.nx * p.ny * p.nz + 127) / 128;
  }
  static __device__ __forceinline__ void run(const tacker_be_lbm &p, int64_t vb, int tid, uint32_t, uint8_t *) {
    const int64_t cells = (int64_t)p.nx * p.ny * p.nz;
    const int64_t idx = vb * 128 + tid;
    if (idx >= cells) return;
    const int x = (int)(idx % p.nx), y = (int)((idx / p.nx) % p.ny), z = (int)(idx / ((int64_t)p.nx * p.ny));
    const uint32_t flag = p.flags[idx];
    float f[19];
#pragma unroll
    for (int i = 0; i < 19; ++i) f[i] = __ldg(p.src + i * cells + idx);
    const float w[19] = {1.f / 3.f,  1.f / 18.f, 1.f / 18.f, 1.f / 18.f, 1.f / 18.f, 1.f / 18.f, 1.f / 18.f,
                         1.f / 36.f, 1.f / 36.f, 1.f / 36.f, 1.f / 36.f, 1.f / 36.f, 1.f / 36.f, 1.f / 36.f,
                         1.f / 36.f, 1.f / 36.f, 1.f / 36.f, 1.f / 36.f, 1.f / 36.f};
    if (flag == 1u) {  // OBSTACLE: dst_{opp(i)}[x + e_opp(i)] = src_i[x]
#pragma unroll
      for (int i = 0; i < 19; ++i) {
        const int j = kLbmOpp[i];
        const int tx = x + kLbmE[j][0], ty = y + kLbmE[j][1], tz = z + kLbmE[j][2];
        if (tx >= 0 && tx < p.nx && ty >= 0 && ty < p.ny && tz >= 0 && tz < p.nz)
          p.dst[j * cells + ((int64_t)tz * p.ny + ty) * p.nx + tx] = f[i];
      }
      return;
    }
    float rho = 0.f, ux = 0.f, uy = 0.f, uz = 0.f;
#pragma unroll
    for (int i = 0; i < 19; ++i) {
      rho = __fadd_rn(rho, f[i]);
      if (kLbmE[i][0] > 0) ux = __fadd_rn(ux, f[i]);
      if (kLbmE[i][0] < 0) ux = __fsub_rn(ux, f[i]);
      if (kLbmE[i][1] > 0) uy = __fadd_rn(uy, f[i]);
      if (kLbmE[i][1] < 0) uy = __fsub_rn(uy, f[i]);
      if (kLbmE[i][2] > 0) uz = __fadd_rn(uz, f[i]);
      if (kLbmE[i][2] < 0) uz = __fsub_rn(uz, f[i]);
    }
    ux = __fdiv_rn(ux, rho);
    uy = __fdiv_rn(uy, rho);
    uz = __fdiv_rn(uz, rho);
    if (flag == 2u) {  // ACCEL
      ux = 0.005f;
      uy = 0.002f;
      uz = 0.f;
    }
    const float u2 = __fadd_rn(__fadd_rn(__fmul_rn(ux, ux), __fmul_rn(uy, uy)), __fmul_rn(uz, uz));
    const float omega = 1.95f;
    const float one_m = __fsub_rn(1.f, omega);
#pragma unroll
    for (int i = 0; i < 19; ++i) {
      float eu = 0.f;
      if (kLbmE[i][0] != 0) eu = __fadd_rn(eu, kLbmE[i][0] > 0 ? ux : -ux);
      if (kLbmE[i][1] != 0) eu = __fadd_rn(eu, kLbmE[i][1] > 0 ? uy : -uy);
      if (kLbmE[i][2] != 0) eu = __fadd_rn(eu, kLbmE[i][2] > 0 ? uz : -uz);
      // feq = w rho (1 + 3 eu + 4.5 eu^2 - 1.5 u2)
      float poly = __fadd_rn(1.f, __fmul_rn(3.f, eu));
      poly = __fadd_rn(poly, __fmul_rn(4.5f, __fmul_rn(eu, eu)));
      poly = __fsub_rn(poly, __fmul_rn(1.5f, u2));
      const float feq = __fmul_rn(__fmul_rn(w[i], rho), poly);
      const float out = __fadd_rn(__fmul_rn(one_m, f[i]), __fmul_rn(omega, feq));
      const int tx = x + kLbmE[i][0], ty = y + kLbmE[i][1], tz = z + kLbmE[i][2];
      if (tx >= 0 && tx < p.nx && ty >= 0 && ty < p.ny && tz >= 0 && tz < p.nz)
        p.dst[i * cells + ((int64_t)tz * p.ny + ty) * p.nx + tx] = out;
    }
  }
};

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

// ---------------------------------------------------------------- histo
// Block = 32768 inputs: a private u32 histogram of nbins (<= 8192) in shared memory, then one
// global atomicAdd per non-empty bin.  Integer adds commute: bit-exact whatever the order.
template <> struct BeBody<TACKER_BE_HISTO> {
  static constexpr int PER_BLOCK = 32768;
  static constexpr uint32_t kSmem = 8192 * 4;
  static __host__ __device__ int64_t num_blocks(const tacker_be_histo &p) {
    return ((int64_t)p.n + PER_BLOCK - 1) / PER_BLOCK;
  }
  static __device__ __forceinline__ void run(const tacker_be_histo &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    uint32_t *h = reinterpret_cast<uint32_t *>(smem);
    for (int b = tid; b < p.nbins; b += kVbThreads) h[b] = 0;
    named_bar_sync(bar, kVbThreads);
    const int64_t base = vb * PER_BLOCK;
    const int64_t end = min((int64_t)p.n, base + PER_BLOCK);
    if (base + PER_BLOCK <= p.n && (p.n & 3) == 0) {
      const uint4 *in4 = reinterpret_cast<const uint4 *>(p.in + base);
#pragma unroll 4
      for (int i = tid; i < PER_BLOCK / 4; i += kVbThreads) {
        const uint4 v = __ldg(in4 + i);
        atomicAdd(&h[v.x], 1u);
        atomicAdd(&h[v.y], 1u);
        atomicAdd(&h[v.z], 1u);
        atomicAdd(&h[v.w], 1u);
      }
    } else {
      for (int64_t i = base + tid; i < end; i += kVbThreads) atomicAdd(&h[__ldg(p.in + i)], 1u);
    }
    named_bar_sync(bar, kVbThreads);
    for (int b = tid; b < p.nbins; b += kVbThreads) {
      const uint32_t c = h[b];
      if (c) atomicAdd(p.count + b, c);
    }
    named_bar_sync(bar, kVbThreads);  // shared histogram reusable by the next block
  }
};

// ---------------------------------------------------------------- bfs (Rodinia kernels 1 and 2)
template <> struct BeBody<TACKER_BE_BFS_EXPAND> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_bfs_expand &p) { return (p.V + 127) / 128; }
  static __device__ __forceinline__ void run(const tacker_be_bfs_expand &p, int64_t vb, int tid, uint32_t,
                                             uint8_t *) {
    const int64_t v = vb * 128 + tid;
    if (v >= p.V || !p.mask[v]) return;
    p.mask[v] = 0;
    const int lv = p.level[v] + 1;
    for (int e = p.row_ptr[v]; e < p.row_ptr[v + 1]; ++e) {
      const int u = p.col[e];
      if (!p.visited[u]) {
        p.level[u] = lv;
        p.upd[u] = 1;
      }
    }
  }
};
template <> struct BeBody<TACKER_BE_BFS_COMMIT> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_bfs_commit &p) { return (p.V + 127) / 128; }
  static __device__ __forceinline__ void run(const tacker_be_bfs_commit &p, int64_t vb, int tid, uint32_t,
                                             uint8_t *) {
    const int64_t u = vb * 128 + tid;
    if (u >= p.V || !p.upd[u]) return;
    p.mask[u] = 1;
    p.visited[u] = 1;
    p.upd[u] = 0;
    *p.over = 1;
  }
};

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
    const int P = (p.h + 2 * p.pad - p.r) / p.stride + 1, Q = (p.w + 2 * p.pad - p.s) / p.stride + 1;
    const int64_t groups_per_row = p.Kpad / 8;
    const int64_t total = (int64_t)p.n * P * Q * groups_per_row;
    const int Kreal = p.r * p.s * p.c;
    const __half *x = reinterpret_cast<const __half *>(p.x);
    __half *out = reinterpret_cast<__half *>(p.out);
#pragma unroll 2
    for (int u = 0; u < 8; ++u) {
      const int64_t g = vb * 1024 + u * 128 + tid;
      if (g >= total) return;
      const int64_t m = g / groups_per_row;
      const int kk0 = (int)(g % groups_per_row) * 8;
      const int q = (int)(m % Q), pp = (int)((m / Q) % P), n = (int)(m / ((int64_t)P * Q));
      uint4 v = make_uint4(0, 0, 0, 0);
      if ((p.c & 7) == 0) {
        if (kk0 < Kreal) {
          const int c = kk0 % p.c, rs = kk0 / p.c, s = rs % p.s, r = rs / p.s;
          const int hi = pp * p.stride - p.pad + r, wi = q * p.stride - p.pad + s;
          if (hi >= 0 && hi < p.h && wi >= 0 && wi < p.w)
            v = __ldg(reinterpret_cast<const uint4 *>(x + (((int64_t)n * p.h + hi) * p.w + wi) * p.c + c));
        }
      } else {
        __align__(16) __half e[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int kk = kk0 + j;
          e[j] = __float2half(0.f);
          if (kk < Kreal) {
            const int c = kk % p.c, rs = kk / p.c, s = rs % p.s, r = rs / p.s;
            const int hi = pp * p.stride - p.pad + r, wi = q * p.stride - p.pad + s;
            if (hi >= 0 && hi < p.h && wi >= 0 && wi < p.w) e[j] = x[(((int64_t)n * p.h + hi) * p.w + wi) * p.c + c];
          }
        }
        v = *reinterpret_cast<uint4 *>(e);
      }
      *reinterpret_cast<uint4 *>(out + m * p.Kpad + kk0) = v;
    }
  }
};

// ---------------------------------------------------------------- copy (query I/O)
// 16 KiB per block, 16-byte vectors, 8 independent loads in flight per thread.
template <> struct BeBody<TACKER_BE_COPY> {
  static constexpr uint32_t kSmem = 0;
  static constexpr int64_t kBlockBytes = 16384;
  static __host__ __device__ int64_t num_blocks(const tacker_be_copy &p) {
    return (p.bytes + kBlockBytes - 1) / kBlockBytes;
  }
  static __device__ __forceinline__ void run(const tacker_be_copy &p, int64_t vb, int tid, uint32_t, uint8_t *) {
    const uint4 *src = reinterpret_cast<const uint4 *>(p.src);
    uint4 *dst = reinterpret_cast<uint4 *>(p.dst);
    const int64_t n16 = p.bytes / 16;
    const int64_t base = vb * (kBlockBytes / 16);
    uint4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t i = base + u * 128 + tid;
      if (i < n16) v[u] = src[i];
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t i = base + u * 128 + tid;
      if (i < n16) dst[i] = v[u];
    }
  }
};

// ---------------------------------------------------------------- JDS build (spmv input format)
// Stable counting sort of rows by length, descending, ties by row index:
//   COUNT  per 1024-row block b: c[b][L] = #rows of length L in the block
//   SCAN   per L: c[b][L] -> exclusive prefix over blocks; start[L] = #rows longer than L;
//          jds_ptr[d] = sum_{d' < d} #rows longer than d'
//   PERM   row r of block b with length L goes to start[L] + c[b][L] + (#earlier rows of length
//          L in its block): perm[pos] = r, row_len[pos] = L
//   FILL   element (d, i) = d-th nonzero of row perm[i] at jds_ptr[d] + i
constexpr int kJdsMaxLen = 4095;
constexpr int kJdsRows = 1024;
template <> struct BeBody<TACKER_BE_JDS_COUNT> {
  static constexpr uint32_t kSmem = (kJdsMaxLen + 1) * 4;
  static __host__ __device__ int64_t num_blocks(const tacker_be_jds &p) { return (p.rows + kJdsRows - 1) / kJdsRows; }
  static __device__ __forceinline__ void run(const tacker_be_jds &p, int64_t vb, int tid, uint32_t bar, uint8_t *smem) {
    int32_t *cnt = reinterpret_cast<int32_t *>(smem);
    const int M = p.max_len + 1;
    for (int L = tid; L < M; L += kVbThreads) cnt[L] = 0;
    named_bar_sync(bar, kVbThreads);
    for (int u = 0; u < kJdsRows / kVbThreads; ++u) {
      const int64_t r = vb * kJdsRows + u * kVbThreads + tid;
      if (r < p.rows) {
        const int L = __ldg(p.row_ptr + r + 1) - __ldg(p.row_ptr + r);
        if (L > p.max_len) *p.overflow = 1;
        else atomicAdd(&cnt[L], 1);
      }
    }
    named_bar_sync(bar, kVbThreads);
    for (int L = tid; L < M; L += kVbThreads) p.blk_count[vb * M + L] = cnt[L];
    named_bar_sync(bar, kVbThreads);
  }
};
template <> struct BeBody<TACKER_BE_JDS_SCAN> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_jds &) { return 1; }
  static __device__ __forceinline__ void run(const tacker_be_jds &p, int64_t, int tid, uint32_t bar, uint8_t *) {
    const int M = p.max_len + 1;
    const int64_t nb = (p.rows + kJdsRows - 1) / kJdsRows;
    for (int L = tid; L < M; L += kVbThreads) {
      int32_t s = 0;
      for (int64_t b = 0; b < nb; ++b) {
        const int32_t c = p.blk_count[b * M + L];
        p.blk_count[b * M + L] = s;
        s += c;
      }
      p.start[L] = s;   // total rows of length L
    }
    __threadfence_block();
    named_bar_sync(bar, kVbThreads);
    if (tid == 0) {
      int32_t acc = 0;
      for (int L = M - 1; L >= 0; --L) {   // start[L] = #rows longer than L
        const int32_t t = p.start[L];
        p.start[L] = acc;
        acc += t;
      }
      int32_t ptr = 0;
      for (int d = 0; d < p.max_len; ++d) {
        p.jds_ptr[d] = ptr;
        ptr += p.start[d];
      }
      p.jds_ptr[p.max_len] = ptr;
    }
    named_bar_sync(bar, kVbThreads);
  }
};
template <> struct BeBody<TACKER_BE_JDS_PERM> {
  static constexpr uint32_t kSmem = (kJdsMaxLen + 1) * 4 + kJdsRows * 4;
  static __host__ __device__ int64_t num_blocks(const tacker_be_jds &p) { return (p.rows + kJdsRows - 1) / kJdsRows; }
  static __device__ __forceinline__ void run(const tacker_be_jds &p, int64_t vb, int tid, uint32_t bar, uint8_t *smem) {
    int32_t *cnt = reinterpret_cast<int32_t *>(smem);
    int32_t *lens = cnt + kJdsMaxLen + 1;
    const int M = p.max_len + 1;
    for (int L = tid; L < M; L += kVbThreads) cnt[L] = 0;
    for (int u = 0; u < kJdsRows / kVbThreads; ++u) {
      const int64_t r = vb * kJdsRows + u * kVbThreads + tid;
      lens[u * kVbThreads + tid] =
          r < p.rows ? min(__ldg(p.row_ptr + r + 1) - __ldg(p.row_ptr + r), p.max_len) : -1;
    }
    named_bar_sync(bar, kVbThreads);
    if (tid == 0) {   // rank within the block in row order (stable)
      for (int u = 0; u < kJdsRows; ++u) {
        const int L = lens[u];
        if (L < 0) break;
        const int32_t pos = p.start[L] + p.blk_count[vb * M + L] + cnt[L]++;
        p.perm[pos] = (int32_t)(vb * kJdsRows + u);
        p.row_len[pos] = L;
      }
    }
    named_bar_sync(bar, kVbThreads);
  }
};
template <> struct BeBody<TACKER_BE_JDS_FILL> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_jds &p) { return (p.rows + 127) / 128; }
  static __device__ __forceinline__ void run(const tacker_be_jds &p, int64_t vb, int tid, uint32_t, uint8_t *) {
    const int64_t i = vb * 128 + tid;
    if (i >= p.rows) return;
    const int32_t r = p.perm[i], L = p.row_len[i];
    const int32_t base = __ldg(p.row_ptr + r);
    for (int d = 0; d < L; ++d) {
      const int64_t e = (int64_t)p.jds_ptr[d] + i;
      p.jds_col[e] = __ldg(p.col + base + d);
      p.jds_val[e] = __ldg(p.val + base + d);
    }
  }
};

// ---------------------------------------------------------------- dispatch helpers
template <int KIND> struct BeSel;
#define TK_BE_SEL(K, FIELD)                                                            \
  template <> struct BeSel<K> {                                                        \
    static __host__ __device__ const auto &get(const tacker_be_desc &d) { return d.p.FIELD; } \
  };
TK_BE_SEL(TACKER_BE_SGEMM, sgemm)
TK_BE_SEL(TACKER_BE_STENCIL, stencil)
TK_BE_SEL(TACKER_BE_MRIQ_PHIMAG, mriq_phimag)
TK_BE_SEL(TACKER_BE_MRIQ_Q, mriq_q)
TK_BE_SEL(TACKER_BE_LBM, lbm)
TK_BE_SEL(TACKER_BE_SPMV_JDS, spmv)
TK_BE_SEL(TACKER_BE_HISTO, histo)
TK_BE_SEL(TACKER_BE_BFS_EXPAND, bfs_expand)
TK_BE_SEL(TACKER_BE_BFS_COMMIT, bfs_commit)
TK_BE_SEL(TACKER_BE_FMA_BURN, fma_burn)
TK_BE_SEL(TACKER_BE_IM2COL, im2col)
TK_BE_SEL(TACKER_BE_CUTCP, cutcp)
TK_BE_SEL(TACKER_BE_CUTCP_BIN, cutcp_bin)
TK_BE_SEL(TACKER_BE_COPY, copy)
TK_BE_SEL(TACKER_BE_JDS_COUNT, jds)
TK_BE_SEL(TACKER_BE_JDS_SCAN, jds)
TK_BE_SEL(TACKER_BE_JDS_PERM, jds)
TK_BE_SEL(TACKER_BE_JDS_FILL, jds)
#undef TK_BE_SEL

// Maximum BE warps per fused CTA: register-heavy bodies (sgemm's 8x4 register tile) keep the
// CTA at 6+16 warps (80 registers/thread); the others allow 6+24 warps (64 registers/thread).
__host__ __device__ constexpr int be_max_warps(int kind) { return kind == TACKER_BE_SGEMM ? 16 : 24; }

// Body call with the optional per-kind TMA tensor map (only the stencil uses one).
template <int KIND>
__device__ __forceinline__ void be_run(const tacker_be_desc &d, int64_t vb, int tid, uint32_t bar, uint8_t *smem,
                                       const CUtensorMap *tm) {
  (void)tm;
  BeBody<KIND>::run(BeSel<KIND>::get(d), vb, tid, bar, smem);
}
// Thread coarsening of the fused PTB loop: one ticket covers BeCoarsen original blocks.
template <int KIND> struct BeCoarsen { static constexpr int value = 1; };
template <> struct BeCoarsen<TACKER_BE_MRIQ_Q> { static constexpr int value = BeBody<TACKER_BE_MRIQ_Q>::kCoarsen; };
template <int KIND>
__device__ __forceinline__ void be_run_coarse(const tacker_be_desc &d, int64_t vb, int nb, int tid, uint32_t bar,
                                              uint8_t *smem, const CUtensorMap *tm) {
  if constexpr (BeCoarsen<KIND>::value > 1)
    BeBody<KIND>::run_coarse(BeSel<KIND>::get(d), vb, nb, tid, bar, smem);
  else
    be_run<KIND>(d, vb, tid, bar, smem, tm);
}
// One-time per-slot setup hook (persistent shared-memory state of a body; none at present).
template <int KIND>
__device__ __forceinline__ void be_init(uint8_t *, int, uint32_t) {}

// Every implemented BE kind (X-macro used by the host dispatch tables).
#define TK_FOR_EACH_BE(X)                                                                       \
  X(TACKER_BE_SGEMM) X(TACKER_BE_STENCIL) X(TACKER_BE_MRIQ_PHIMAG) X(TACKER_BE_MRIQ_Q)          \
  X(TACKER_BE_LBM) X(TACKER_BE_SPMV_JDS) X(TACKER_BE_HISTO) X(TACKER_BE_BFS_EXPAND)             \
  X(TACKER_BE_BFS_COMMIT) X(TACKER_BE_FMA_BURN) X(TACKER_BE_IM2COL) X(TACKER_BE_CUTCP) X(TACKER_BE_CUTCP_BIN)        \
  X(TACKER_BE_COPY) X(TACKER_BE_JDS_COUNT) X(TACKER_BE_JDS_SCAN) X(TACKER_BE_JDS_PERM) X(TACKER_BE_JDS_FILL)

}  // namespace tk
