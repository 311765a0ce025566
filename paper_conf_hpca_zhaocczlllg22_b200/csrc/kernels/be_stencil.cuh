// be_stencil.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- stencil (Parboil)
// One 7-point Jacobi sweep over A0[nz][ny][nx] (x fastest), HBM-bound.  Block = 128 x 4 x ZC
// (x,y,z) cells: lane l of warp w owns x = 4l..4l+3 (one float4) of row y = w for ZC planes (TK_STENCIL_ZC).
// The centre column's ZC+2 planes are loaded up front (memory-level parallelism), x+-1 comes
// from the neighbouring lanes' float4 by shuffle, y+-1 rows through L1/L2.
//   interior: An = c1*(((((W+E)+S)+N)+B)+T) - c0*A   (S/N = y-1/y+1, B/T = z-1/z+1)
//   boundary cells (x, y or z on the faces) are copied.
// nx % 4 != 0 uses the scalar path with the same per-element arithmetic.
template <> struct BeBody<TACKER_BE_STENCIL> {
  static constexpr uint32_t kSmem = 0;
  static constexpr int ZC = TK_STENCIL_ZC;
  // fused PTB loop: kCoarsen > 1 runs that many consecutive original blocks per turn, split
  // statically (every cell's arithmetic unchanged: fused and original stay bit-identical); measured
  // no faster than one block per ticket at ZC = 2 or 4, so 1 by default
  static constexpr int kCoarsen = TK_STENCIL_COARSEN;
  static __device__ __forceinline__ void run_coarse(const tacker_be_stencil &p, int64_t vb, int nb, int tid,
                                                    uint32_t bar, uint8_t *smem) {
    for (int i = 0; i < nb; ++i) run(p, vb + i, tid, bar, smem);
  }
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
    // block decode in 32-bit arithmetic (the host bounds the block count below 2^31): the 64-bit
    // divisions and per-load 64-bit address products had made the sweep instruction-bound
    const int bx = (p.nx + 127) >> 7, by = (p.ny + 3) >> 2, bxy = bx * by;
    const int v = (int)vb;
    const int zb = v / bxy, rem = v - zb * bxy;
    const int byi = rem / bx, bxi = rem - byi * bx;
    const int lane = tid & 31;
    const int x0 = bxi * 128 + 4 * lane;
    const int y = byi * 4 + (tid >> 5);
    const int z0 = zb * ZC;
    if (y >= p.ny) return;                     // warp-uniform
    const int64_t plane = (int64_t)p.nx * p.ny;
    const float *__restrict__ A = p.A0;
    float *__restrict__ An = p.Anext;
    const bool ybord = (y == 0) | (y == p.ny - 1);
    if ((p.nx & 3) == 0) {
      const bool act = x0 < p.nx;
      const int64_t row = (int64_t)y * p.nx + x0;
      const float *a = A + row + (int64_t)z0 * plane;      // centre column at plane z0
      float *an = An + row + (int64_t)z0 * plane;
      float4 c[ZC + 2];
#pragma unroll
      for (int i = 0; i < ZC + 2; ++i) {
        const int z = z0 - 1 + i;
        c[i] = (act && z >= 0 && z < p.nz) ? __ldg(reinterpret_cast<const float4 *>(a + (i - 1) * plane))
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
        const float *az = a + i * plane;
        if (!ybord && !zb_) {
          if (lane == 0) wv = x0 > 0 ? __ldg(az - 1) : 0.f;
          if (lane == 31 || x0 + 4 >= p.nx) ev = x0 + 4 < p.nx ? __ldg(az + 4) : 0.f;
          const float4 s = __ldg(reinterpret_cast<const float4 *>(az - p.nx));
          const float4 n = __ldg(reinterpret_cast<const float4 *>(az + p.nx));
          const float4 b = c[i], t = c[i + 2];
          if (x0 > 0) o.x = point(p, wv, cc.y, s.x, n.x, b.x, t.x, cc.x);
          o.y = point(p, cc.x, cc.z, s.y, n.y, b.y, t.y, cc.y);
          o.z = point(p, cc.y, cc.w, s.z, n.z, b.z, t.z, cc.z);
          if (x0 + 3 < p.nx - 1) o.w = point(p, cc.z, ev, s.w, n.w, b.w, t.w, cc.w);
        }
        *reinterpret_cast<float4 *>(an + i * plane) = o;
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

}  // namespace tk
