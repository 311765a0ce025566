// be_cutcp.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

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
          const float e = __fmul_rn(__fmul_rn(__fmul_rn(at.w, rsqrt_ftz(r2)), s), s);
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

// Deterministic binning for cutcp: an original block owns 32 bins (lane = bin) and its 4 warps
// split the atoms into 4 contiguous index ranges.  Pass 1 counts each warp's atoms per bin; the
// per-warp counts give every warp its write offset inside each bin (warp w after warps < w), so
// pass 2 stores the atoms of every bin in atom-index order without atomics.  An atom's bin
// (floor(z/bs), floor(y/bs), floor(x/bs)) clamped into the grid is computed once per 32 atoms (one
// per lane) and broadcast with shuffles.  Bins past the depth count the overflow; the rest of a
// bin is padded with far-away zero-charge atoms.
template <> struct BeBody<TACKER_BE_CUTCP_BIN> {
  static constexpr uint32_t kSmem = 4 * 32 * 4;
  static __host__ __device__ int64_t num_blocks(const tacker_be_cutcp_bin &p) {
    return ((int64_t)p.bdim_x * p.bdim_y * p.bdim_z + 31) / 32;
  }
  static __device__ __forceinline__ int bin_of(const tacker_be_cutcp_bin &p, float4 at) {
    const int ix = min(max((int)floorf(__fdiv_rn(at.x, p.bin_size)), 0), p.bdim_x - 1);
    const int iy = min(max((int)floorf(__fdiv_rn(at.y, p.bin_size)), 0), p.bdim_y - 1);
    const int iz = min(max((int)floorf(__fdiv_rn(at.z, p.bin_size)), 0), p.bdim_z - 1);
    return (iz * p.bdim_y + iy) * p.bdim_x + ix;
  }
  static __device__ __forceinline__ void run(const tacker_be_cutcp_bin &p, int64_t vb, int tid, uint32_t bar,
                                             uint8_t *smem) {
    int *s_cnt = reinterpret_cast<int *>(smem);   // [4 warps][32 bins]
    const int w = tid >> 5, lane = tid & 31;
    const int nb = p.bdim_x * p.bdim_y * p.bdim_z;
    const int b = (int)(vb * 32) + lane;
    const float4 *atoms = reinterpret_cast<const float4 *>(p.atoms);
    float4 *bins = reinterpret_cast<float4 *>(p.bins);
    const int a0 = (int)((int64_t)p.natoms * w / 4), a1 = (int)((int64_t)p.natoms * (w + 1) / 4);
    int cnt = 0;
    for (int a = a0; a < a1; a += 32) {
      const int n = min(32, a1 - a);
      const int mine = lane < n ? bin_of(p, __ldg(atoms + a + lane)) : -1;
      for (int j = 0; j < n; ++j) cnt += __shfl_sync(0xffffffffu, mine, j) == b ? 1 : 0;
    }
    named_bar_sync(bar, kVbThreads);          // previous block's readers of s_cnt are done
    s_cnt[w * 32 + lane] = cnt;
    named_bar_sync(bar, kVbThreads);
    int k = 0, total = 0;
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int c = s_cnt[u * 32 + lane];
      if (u < w) k += c;
      total += c;
    }
    for (int a = a0; a < a1; a += 32) {
      const int n = min(32, a1 - a);
      const float4 at = lane < n ? __ldg(atoms + a + lane) : make_float4(0.f, 0.f, 0.f, 0.f);
      const int mine = lane < n ? bin_of(p, at) : -1;
      for (int j = 0; j < n; ++j) {
        const int bj = __shfl_sync(0xffffffffu, mine, j);
        if ((unsigned)(bj - (int)(vb * 32)) >= 32u) continue;   // warp-uniform: not one of this block's bins
        const float x = __shfl_sync(0xffffffffu, at.x, j), y = __shfl_sync(0xffffffffu, at.y, j);
        const float z = __shfl_sync(0xffffffffu, at.z, j), q = __shfl_sync(0xffffffffu, at.w, j);
        if (bj == b) {
          if (k < p.bin_depth) bins[(int64_t)b * p.bin_depth + k] = make_float4(x, y, z, q);
          ++k;
        }
      }
    }
    if (w == 0 && b < nb) {
      for (int t = min(total, p.bin_depth); t < p.bin_depth; ++t)
        bins[(int64_t)b * p.bin_depth + t] = make_float4(1e30f, 1e30f, 1e30f, 0.f);
      p.count[b] = total;
      if (total > p.bin_depth) *p.overflow = 1;
    }
  }
};

}  // namespace tk
