// be_dispatch.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"
#include "be_sgemm.cuh"
#include "be_fma_burn.cuh"
#include "be_stencil.cuh"
#include "be_mriq.cuh"
#include "be_cutcp.cuh"
#include "be_lbm.cuh"
#include "be_spmv.cuh"
#include "be_histo.cuh"
#include "be_bfs.cuh"
#include "be_im2col.cuh"
#include "be_copy.cuh"
#include "be_jds.cuh"
#include "be_mrifhd.cuh"
#include "be_cp.cuh"
#include "be_fft.cuh"
#include "be_tpacf.cuh"

namespace tk {

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
TK_BE_SEL(TACKER_BE_MRIFHD_RHOPHI, mrifhd_rhophi)
TK_BE_SEL(TACKER_BE_MRIFHD_FH, mrifhd_fh)
TK_BE_SEL(TACKER_BE_CP, cp)
TK_BE_SEL(TACKER_BE_FFT_TWIDDLE, fft)
TK_BE_SEL(TACKER_BE_FFT, fft)
TK_BE_SEL(TACKER_BE_TPACF, tpacf)
#undef TK_BE_SEL

// Maximum BE warps per fused CTA: register-heavy bodies (sgemm's 8x4 register tile) keep the
// CTA at 6+16 warps (80 registers/thread); the others allow 6+24 warps (64 registers/thread).
// LC-only instantiations (kind NONE) have no BE warps: their launch bound is the 6 LC warps.
__host__ __device__ constexpr int be_max_warps(int kind) {
  return kind == TACKER_BE_NONE ? 0 : kind == TACKER_BE_SGEMM ? 16 : 24;
}
// Minimum resident blocks per SM of an original (standalone) BE launch: caps the registers of
// bodies whose latency hiding needs many blocks (fft: TK_FFT_MIN_BLOCKS = 8 blocks -> <= 64 registers).
__host__ __device__ constexpr int be_orig_min_blocks(int kind) {
  return kind == TACKER_BE_FFT ? TK_FFT_MIN_BLOCKS : kind == TACKER_BE_STENCIL ? TK_STENCIL_MIN_BLOCKS : 1;
}

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
template <> struct BeCoarsen<TACKER_BE_MRIFHD_FH> { static constexpr int value = BeBody<TACKER_BE_MRIFHD_FH>::kCoarsen; };
template <> struct BeCoarsen<TACKER_BE_STENCIL> { static constexpr int value = BeBody<TACKER_BE_STENCIL>::kCoarsen; };
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
  X(TACKER_BE_COPY) X(TACKER_BE_JDS_COUNT) X(TACKER_BE_JDS_SCAN) X(TACKER_BE_JDS_PERM) X(TACKER_BE_JDS_FILL)          \
  X(TACKER_BE_MRIFHD_RHOPHI) X(TACKER_BE_MRIFHD_FH) X(TACKER_BE_CP) X(TACKER_BE_FFT_TWIDDLE) X(TACKER_BE_FFT)       \
  X(TACKER_BE_TPACF)

}  // namespace tk
