// be_cp.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- cp (Parboil, Table II)
// NEXT-3.  Direct Coulomb summation on one lattice slice (DESIGN.md §2 reading 14):
//   V[j nx + i] += sum_a q_a * rsqrt((i h - x_a)^2 + (j h - y_a)^2 + (z - z_a)^2).
// Block = a 128 x 4 tile of lattice points: lane l of warp w owns row j = 4 by + w and the
// points i = 128 bx + l + 32 u, u < 4 (coalesced 128-byte stores per u).  Atoms are staged in
// shared memory 512 at a time as float4 (x, y, dz^2, q) — dz^2 is computed once per atom per
// slice — and summed in atom-index order per point:
//   dyz = fma(dy, dy, dz^2);  r2 = fma(dx, dx, dyz);  acc = fma(q, rsqrt(r2), acc)
// i.e. 3 FP32-pipe ops + 1 MUFU per point-atom pair (MUFU-bound, like mri-q); V = V_in + acc.
template <> struct BeBody<TACKER_BE_CP> {
  static constexpr int kStage = 512;
  static constexpr int kPtsX = 128, kRows = 4, kUx = 4;
  static constexpr uint32_t kSmem = kStage * 16;
  static __host__ __device__ int64_t num_blocks(const tacker_be_cp &p) {
    return (int64_t)((p.nx + kPtsX - 1) / kPtsX) * ((p.ny + kRows - 1) / kRows);
  }
  static __device__ __forceinline__ void run(const tacker_be_cp &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    float4 *st = reinterpret_cast<float4 *>(smem);
    const int bxs = (p.nx + kPtsX - 1) / kPtsX;
    const int bx = (int)(vb % bxs), by = (int)(vb / bxs);
    const int lane = tid & 31, row = by * kRows + (tid >> 5);
    const float py = __fmul_rn((float)row, p.h);
    float px[kUx], acc[kUx];
#pragma unroll
    for (int u = 0; u < kUx; ++u) {
      px[u] = __fmul_rn((float)(bx * kPtsX + lane + 32 * u), p.h);
      acc[u] = 0.f;
    }
    const float4 *atoms = reinterpret_cast<const float4 *>(p.atoms);
    for (int a0 = 0; a0 < p.natoms; a0 += kStage) {
      const int n = min(kStage, p.natoms - a0);
      named_bar_sync(bar, kVbThreads);   // previous stage fully consumed
      for (int a = tid; a < n; a += kVbThreads) {
        const float4 at = __ldg(atoms + a0 + a);
        const float dz = __fsub_rn(p.z, at.z);
        st[a] = make_float4(at.x, at.y, __fmul_rn(dz, dz), at.w);
      }
      named_bar_sync(bar, kVbThreads);
#pragma unroll 4
      for (int a = 0; a < n; ++a) {
        const float4 at = st[a];
        const float dy = __fsub_rn(py, at.y);
        const float dyz = __fmaf_rn(dy, dy, at.z);
#pragma unroll
        for (int u = 0; u < kUx; ++u) {
          const float dx = __fsub_rn(px[u], at.x);
          acc[u] = __fmaf_rn(at.w, rsqrt_ftz(__fmaf_rn(dx, dx, dyz)), acc[u]);
        }
      }
    }
    if (row < p.ny) {
#pragma unroll
      for (int u = 0; u < kUx; ++u) {
        const int i = bx * kPtsX + lane + 32 * u;
        if (i < p.nx) {
          float *o = p.V + (int64_t)row * p.nx + i;
          *o = __fadd_rn(*o, acc[u]);
        }
      }
    }
  }
};

}  // namespace tk
