// be_lbm.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

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

}  // namespace tk
