// tacker_fuse.cu — fusion planner (a1), tensor-map encoding, fused / original launches (a2-a8).
//
// tacker_fuse implements Tacker's offline fusion step on B200 (§V-B/C P:1117-1309): PTB with
// one persistent CTA per SM, LC budgeted first (SMEM ring stages, TMEM accumulator columns),
// BE virtual blocks added with what remains, and admission by aggregate per-SM resources
// (§VIII-I).  Instead of generating code it selects one of the
// compiled template instantiations fused_kernel<BN, BE_KIND>.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <cmath>
#include <vector>
#include <set>
#include <memory>
#include <string>
#include <unordered_map>

#include "kernels/fused.cuh"
#include "runtime.h"
#include "tacker.h"

using namespace tk;

namespace tkrt {

static thread_local std::string g_err;

void set_error(const char *fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
}

tacker_status cuda_fail(const char *what, int err) {
  set_error("%s: CUDA error %d (%s)", what, err, cudaGetErrorString((cudaError_t)err));
  return TACKER_ECUDA;
}

int sm_count() {
  static int n = -1;
  if (n < 0) {
    int dev = 0, v = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
      cudaGetLastError();
      return 0;
    }
    n = v;
  }
  return n;
}

const char *be_kind_name(int kind) {
  static const char *names[] = {"none",   "sgemm", "stencil", "mriq_phimag", "mriq_q",   "cutcp",
                                "lbm",    "spmv",  "histo",   "bfs_expand",  "bfs_commit", "fma_burn",
                                "im2col", "cutcp_bin", "copy", "jds_count", "jds_scan", "jds_perm", "jds_fill",
                                "mrifhd_rhophi", "mrifhd_fh", "cp", "fft_twiddle", "fft", "tpacf"};
  return (kind >= 0 && kind < TACKER_BE_KIND_COUNT) ? names[kind] : "?";
}

}  // namespace tkrt

using namespace tkrt;

// ============================================================================ constants
#ifndef TACKER_OVERLAP_DEFAULT
#define TACKER_OVERLAP_DEFAULT 2
#endif
static constexpr int kSmemCap = 232448;      // max dynamic SMEM per CTA on sm_100 (227 KB)
static constexpr int kTmemCols = 512;
static constexpr int kMaxWarps = 32;
static constexpr int kMinLcSmem = 120 * 1024;  // forces one LC CTA per SM (TMEM ownership)

// ============================================================================ BE helpers
template <int K>
static int64_t be_blocks_t(const tacker_be_desc &d) {
  return BeBody<K>::num_blocks(BeSel<K>::get(d));
}

static bool be_num_blocks(const tacker_be_desc &d, int64_t *out) {
  switch (d.kind) {
#define C(K) \
  case K: *out = be_blocks_t<K>(d); return true;
    TK_FOR_EACH_BE(C)
#undef C
    default: return false;
  }
}

static uint32_t be_smem_bytes(int kind) {
  switch (kind) {
#define C(K) \
  case K: return BeBody<K>::kSmem;
    TK_FOR_EACH_BE(C)
#undef C
    default: return 0;
  }
}

static tacker_status validate_be(const tacker_be_desc &d, int64_t *blocks) {
  int64_t full = 0;
  if (!be_num_blocks(d, &full)) {
    set_error("BE kind %d not supported", d.kind);
    return TACKER_EUNSUPPORTED;
  }
  switch (d.kind) {
    case TACKER_BE_SGEMM: {
      const auto &p = d.p.sgemm;
      if (p.M < 0 || p.N < 0 || p.K < 0 || !p.A || !p.B || !p.C) return set_error("sgemm: bad args"), TACKER_EINVAL;
      if (p.N % 4 || p.K % 4) return set_error("sgemm: N and K must be multiples of 4"), TACKER_EUNSUPPORTED;
      break;
    }
    case TACKER_BE_STENCIL: {
      const auto &p = d.p.stencil;
      if (p.nx <= 0 || p.ny <= 0 || p.nz <= 0 || !p.A0 || !p.Anext) return set_error("stencil: bad args"), TACKER_EINVAL;
      if (full > 0x7fffffffLL) return set_error("stencil: more than 2^31 - 1 blocks"), TACKER_EUNSUPPORTED;
      break;
    }
    case TACKER_BE_MRIQ_PHIMAG:
      if (d.p.mriq_phimag.numK < 0 || !d.p.mriq_phimag.phiMag) return set_error("mriq_phimag: bad args"), TACKER_EINVAL;
      break;
    case TACKER_BE_MRIQ_Q:
      if (d.p.mriq_q.numX < 0 || d.p.mriq_q.numK < 0 || !d.p.mriq_q.Qr) return set_error("mriq_q: bad args"), TACKER_EINVAL;
      break;
    case TACKER_BE_MRIFHD_RHOPHI: {
      const auto &p = d.p.mrifhd_rhophi;
      if (p.numK < 0 || (p.numK && (!p.phiR || !p.phiI || !p.dR || !p.dI || !p.rRhoPhi || !p.iRhoPhi)))
        return set_error("mrifhd_rhophi: bad args"), TACKER_EINVAL;
      break;
    }
    case TACKER_BE_MRIFHD_FH: {
      const auto &p = d.p.mrifhd_fh;
      if (p.numX < 0 || p.numK < 0 ||
          (p.numX && (!p.x || !p.y || !p.z || !p.rFhD || !p.iFhD)) ||
          (p.numX && p.numK && (!p.kx || !p.ky || !p.kz || !p.rRhoPhi || !p.iRhoPhi)))
        return set_error("mrifhd_fh: bad args"), TACKER_EINVAL;
      break;
    }
    case TACKER_BE_CP: {
      const auto &p = d.p.cp;
      if (p.natoms < 0 || p.nx < 0 || p.ny < 0 || !(p.h > 0) || (p.nx && p.ny && !p.V) || (p.natoms && !p.atoms))
        return set_error("cp: bad args"), TACKER_EINVAL;
      if (reinterpret_cast<uintptr_t>(p.atoms) & 15) return set_error("cp: atoms must be 16-byte aligned float4"), TACKER_EINVAL;
      break;
    }
    case TACKER_BE_FFT_TWIDDLE:
    case TACKER_BE_FFT: {
      const auto &p = d.p.fft;
      if (p.n < 2 || p.n > BeBody<TACKER_BE_FFT>::kMaxN || (p.n & (p.n - 1)))
        return set_error("fft: n must be a power of two in [2, %d]", BeBody<TACKER_BE_FFT>::kMaxN), TACKER_EUNSUPPORTED;
      if (!p.twiddle || (d.kind == TACKER_BE_FFT && (p.batch < 0 || (p.batch && (!p.x || !p.y)))))
        return set_error("fft: bad args"), TACKER_EINVAL;
      if (d.kind == TACKER_BE_FFT && ((reinterpret_cast<uintptr_t>(p.x) | reinterpret_cast<uintptr_t>(p.y)) & 15))
        return set_error("fft: x and y must be 16-byte aligned"), TACKER_EINVAL;
      break;
    }
    case TACKER_BE_TPACF: {
      const auto &p = d.p.tpacf;
      if (p.na < 0 || p.nb < 0 || !p.count || !p.edges || (p.na && !p.a) || (p.nb && !p.b) ||
          (p.self_pairs && (p.a != p.b || p.na != p.nb)))
        return set_error("tpacf: bad args (self_pairs needs b == a)"), TACKER_EINVAL;
      if (p.nedges < 1 || p.nedges > BeBody<TACKER_BE_TPACF>::kMaxEdges)
        return set_error("tpacf: nedges must be in [1, %d]", BeBody<TACKER_BE_TPACF>::kMaxEdges), TACKER_EUNSUPPORTED;
      break;
    }
    case TACKER_BE_LBM:
      if (d.p.lbm.nx <= 0 || !d.p.lbm.src || !d.p.lbm.dst || !d.p.lbm.flags || d.p.lbm.src == d.p.lbm.dst)
        return set_error("lbm: bad args (src and dst must differ)"), TACKER_EINVAL;
      break;
    case TACKER_BE_SPMV_JDS:
      if (d.p.spmv.rows < 0 || !d.p.spmv.y) return set_error("spmv: bad args"), TACKER_EINVAL;
      break;
    case TACKER_BE_HISTO:
      if (d.p.histo.n < 0 || d.p.histo.nbins <= 0 || d.p.histo.nbins > 8192 || !d.p.histo.count)
        return set_error("histo: nbins must be in [1, 8192]"), TACKER_EUNSUPPORTED;
      break;
    case TACKER_BE_BFS_EXPAND:
    case TACKER_BE_BFS_COMMIT:
      break;
    case TACKER_BE_CUTCP: {
      const auto &p = d.p.cutcp;
      if (p.nx <= 0 || p.ny <= 0 || p.nz <= 0 || !(p.h > 0) || !(p.cutoff > 0) || p.bin_depth <= 0 || !p.bins ||
          !p.count || !p.V)
        return set_error("cutcp: bad args"), TACKER_EINVAL;
      if (7 * p.bin_depth > BeBody<TACKER_BE_CUTCP>::kStage)
        return set_error("cutcp: bin_depth must be <= %d", BeBody<TACKER_BE_CUTCP>::kStage / 7), TACKER_EUNSUPPORTED;
      if (p.bin_size != 8.f * p.h || p.bdim_x != (p.nx + 7) / 8 || p.bdim_y != (p.ny + 7) / 8 || p.bdim_z != (p.nz + 7) / 8)
        return set_error("cutcp: bins must be 8 lattice spacings wide covering the lattice"), TACKER_EUNSUPPORTED;
      if (p.cutoff > 3.f * p.bin_size) return set_error("cutcp: cutoff > 3 bins"), TACKER_EUNSUPPORTED;
      break;
    }
    case TACKER_BE_CUTCP_BIN: {
      const auto &p = d.p.cutcp_bin;
      if (p.natoms < 0 || p.bdim_x <= 0 || p.bdim_y <= 0 || p.bdim_z <= 0 || p.bin_depth <= 0 || !(p.bin_size > 0) ||
          !p.bins || !p.count || !p.overflow || (p.natoms > 0 && !p.atoms))
        return set_error("cutcp_bin: bad args"), TACKER_EINVAL;
      break;
    }
    case TACKER_BE_JDS_COUNT:
    case TACKER_BE_JDS_SCAN:
    case TACKER_BE_JDS_PERM:
    case TACKER_BE_JDS_FILL: {
      const auto &p = d.p.jds;
      if (p.rows < 0 || p.max_len < 1 || p.max_len > kJdsMaxLen || !p.row_ptr || !p.blk_count || !p.start ||
          !p.perm || !p.row_len || !p.jds_ptr || !p.overflow || (d.kind == TACKER_BE_JDS_FILL && (!p.col || !p.val ||
                                                                                          !p.jds_col || !p.jds_val)))
        return set_error("jds: bad args (max_len in [1, %d])", kJdsMaxLen), TACKER_EINVAL;
      break;
    }
    case TACKER_BE_COPY: {
      const auto &p = d.p.copy;
      if (p.bytes < 0 || (p.bytes && (!p.src || !p.dst)) || (p.bytes & 15) ||
          ((reinterpret_cast<uintptr_t>(p.src) | reinterpret_cast<uintptr_t>(p.dst)) & 15))
        return set_error("copy: 16-byte aligned pointers and sizes required"), TACKER_EINVAL;
      break;
    }
    case TACKER_BE_IM2COL: {
      const auto &p = d.p.im2col;
      if (p.n <= 0 || p.h <= 0 || p.w <= 0 || p.c <= 0 || p.r <= 0 || p.s <= 0 || p.stride <= 0 || p.pad < 0 ||
          !p.x || !p.out)
        return set_error("im2col: bad args"), TACKER_EINVAL;
      if (p.Kpad % 8 || p.Kpad < p.r * p.s * p.c) return set_error("im2col: Kpad must be a multiple of 8 >= R*S*C"), TACKER_EINVAL;
      if (p.Kpad > 8 * BeBody<TACKER_BE_IM2COL>::kMaxGroups || p.r > 255 || p.s > 255)
        return set_error("im2col: Kpad <= %d and R, S <= 255", 8 * BeBody<TACKER_BE_IM2COL>::kMaxGroups), TACKER_EUNSUPPORTED;
      if (BeBody<TACKER_BE_IM2COL>::rows(p) * (p.Kpad / 8) >= (int64_t)1 << 31)
        return set_error("im2col: rows * Kpad / 8 must be < 2^31"), TACKER_EUNSUPPORTED;
      break;
    }
    case TACKER_BE_FMA_BURN:
      if (d.p.fma_burn.n_threads < 0 || d.p.fma_burn.iters < 0 || !d.p.fma_burn.out)
        return set_error("fma_burn: bad args"), TACKER_EINVAL;
      break;
  }
  if (d.block_offset < 0 || d.block_offset > full || d.orig_blocks < 0 ||
      (int64_t)d.orig_blocks > full - d.block_offset) {
    set_error("PTB slice [%d, %d + %d) outside [0, %lld]", d.block_offset, d.block_offset, d.orig_blocks,
              (long long)full);
    return TACKER_EINVAL;
  }
  if (d.block_offset && d.kind == TACKER_BE_JDS_SCAN)
    return set_error("jds_scan runs as one block and cannot be sliced"), TACKER_EUNSUPPORTED;
  *blocks = d.orig_blocks ? d.orig_blocks : full - d.block_offset;
  return TACKER_OK;
}

// ============================================================================ LC helpers
static tacker_status lc_view(const tacker_lc_desc &d, LcParams &L) {
  memset(&L, 0, sizeof L);
  L.kind = d.kind;
  if (d.kind == TACKER_LC_GEMM_F16) {
    L.M = d.M;
    L.N = d.N;
    L.K = d.K;
  } else if (d.kind == TACKER_LC_CONV_F16) {
    if (d.n <= 0 || d.h <= 0 || d.w <= 0 || d.c <= 0 || d.k <= 0 || d.r <= 0 || d.s <= 0 || d.stride <= 0 || d.pad < 0)
      return set_error("conv: bad shape"), TACKER_EINVAL;
    L.n = d.n; L.h = d.h; L.w = d.w; L.c = d.c; L.k = d.k; L.r = d.r; L.s = d.s; L.stride = d.stride; L.pad = d.pad;
    L.p = (d.h + 2 * d.pad - d.r) / d.stride + 1;
    L.q = (d.w + 2 * d.pad - d.s) / d.stride + 1;
    if (L.p <= 0 || L.q <= 0) return set_error("conv: empty output"), TACKER_EINVAL;
    L.M = d.n * L.p * L.q;
    L.N = d.k;
    L.K = d.c * d.r * d.s;
    L.conv_direct_gemm = (d.r == 1 && d.s == 1 && d.stride == 1 && d.pad == 0);
    if (!L.conv_direct_gemm && d.c % 64 != 0 && d.c != 8)
      return set_error("conv: C must be a multiple of 64 (or 8) for implicit GEMM (got %d)", d.c), TACKER_EUNSUPPORTED;
  } else {
    return set_error("LC kind %d not supported", d.kind), TACKER_EUNSUPPORTED;
  }
  if (L.M <= 0 || L.N <= 0 || L.K <= 0) return set_error("LC: empty GEMM"), TACKER_EINVAL;
  if (L.K % 8 || L.N % 8) return set_error("LC: K and N must be multiples of 8 (16-byte TMA pitch)"), TACKER_EUNSUPPORTED;
  if (!d.A || !d.B || !d.D) return set_error("LC: null pointer"), TACKER_EINVAL;
  if ((d.epi_flags & TACKER_EPI_BIAS) && !d.bias) return set_error("LC: bias flag without bias"), TACKER_EINVAL;
  if ((d.epi_flags & TACKER_EPI_RESIDUAL) && !d.residual) return set_error("LC: residual flag without residual"), TACKER_EINVAL;
  if (d.d_dtype != TACKER_F32 && d.d_dtype != TACKER_F16) return set_error("LC: bad d_dtype"), TACKER_EINVAL;
  // the epilogue moves 8 columns at a time with 16-byte accesses
  if (((uintptr_t)d.D | (uintptr_t)d.bias | (uintptr_t)d.residual) & 15)
    return set_error("LC: D, bias and residual must be 16-byte aligned"), TACKER_EINVAL;
  L.D = d.D;
  L.d_f16 = d.d_dtype == TACKER_F16;
  L.epi = d.epi_flags;
  L.bias = d.bias;
  L.residual = reinterpret_cast<const __half *>(d.residual);
  return TACKER_OK;
}

static int pick_tile_n(const tacker_lc_desc &d, const LcParams &L) {
  if (d.tile_n == 64 || d.tile_n == 128 || d.tile_n == 256) return d.tile_n;
  if (L.N <= 64) return 64;
  const int sms = sm_count() > 0 ? sm_count() : 148;
  if (L.N >= 256 && (int64_t)((L.M + 127) / 128) * ((L.N + 255) / 256) >= 2LL * sms) return 256;
  // deep-K problems (>= kDeepKb k-blocks) with few tiles: 256-wide tiles halve the A traffic per
  // flop through L2 (the bound of these mainloops); split-K (lc_split) then fills the SMs
  static const int deep_kb = [] {
    const char *e = getenv("TACKER_DEEP_KB");
    return e ? atoi(e) : 1 << 30;
  }();
  if (L.N >= 256 && (L.K + kBK - 1) / kBK >= deep_kb) return 256;
  return 128;
}

// TMA-store epilogue for eligible LC-only plans (TACKER_EPI_TMA=0 restores the register path)
static bool tma_store_enabled() {
  static const bool on = [] {
    const char *e = getenv("TACKER_EPI_TMA");
    return !(e && e[0] == '0');
  }();
  return on;
}

static int lc_dbg_flags() {
  static const int f = [] {
    const char *e = getenv("TACKER_LC_DBG");
    return e ? atoi(e) : 0;
  }();
  return f;
}

// Implicit convs load A through the TMA im2col mode (linear 128-pixel M-tiles, no padding of a
// small image to a 128-position window) unless TACKER_CONV_TILED=1 selects the tiled 4-D windows.
static bool conv_im2col_mode() {
  static const bool tiled = [] {
    const char *e = getenv("TACKER_CONV_TILED");
    return e && e[0] == '1';
  }();
  return !tiled;
}

// Halo mode (stride-1 "same" convs, C % 64 == 0, tiles up to 128 wide): one input halo per
// (filter row, channel block) instead of one 128-pixel im2col load per filter tap (S x fewer A
// bytes through L2 and S x 4 MMAs per ring handshake).  TACKER_CONV_HALO=0 disables it.
static bool conv_halo_ok(const LcParams &L, int BN) {
  static const bool on = [] {
    const char *e = getenv("TACKER_CONV_HALO");
    return !(e && e[0] == '0');
  }();
  return on && L.kind == TACKER_LC_CONV_F16 && !L.conv_direct_gemm && L.stride == 1 && L.c % 64 == 0 &&
         L.r == L.s && L.s <= 7 && 2 * L.pad == L.s - 1 && L.p >= 8 && L.q >= 8 && BN <= 128;
}

// Phase-halo mode for stride-2 convs over 8 channels (ResNet-50 conv1: 7x7, 3 channels padded to
// 8), N <= 64: replaces the explicit im2col + GEMM of §VIII-H.  TACKER_CONV_S2C8=0 disables it.
static bool conv_s2c8_ok(const LcParams &L, int BN) {
  static const bool on = [] {
    const char *e = getenv("TACKER_CONV_S2C8");
    return !(e && e[0] == '0');
  }();
  return on && L.kind == TACKER_LC_CONV_F16 && !L.conv_direct_gemm && L.c == 8 && L.stride == 2 &&
         L.r * L.s <= 63 && L.N <= 64 && BN == 64;
}

static void lc_tiles(LcParams &L, int BN) {
  L.tiles_n = (L.N + BN - 1) / BN;
  L.stage_a = kBM * kBK * 2;
  L.stage_bytes = (uint32_t)(kBM + BN) * kBK * 2;
  if (conv_s2c8_ok(L, BN)) {
    L.conv_s2c8 = 1;
    L.tq = 8;
    L.tp = kBM / 8;
    L.tiles_p = (L.p + L.tp - 1) / L.tp;
    L.tiles_q = (L.q + L.tq - 1) / L.tq;
    L.tiles_m = L.n * L.tiles_p * L.tiles_q;
    L.c_blocks = 1;
    L.num_kb = 1;                                   // one stage = every tap of the tile
    const int rows = L.tp + (L.r - 1) / 2, cols = L.tq + (L.s - 1) / 2;
    L.s2_phase_bytes = (uint32_t)rows * cols * 16u;
    L.s2_phase_stride = (L.s2_phase_bytes + 127u) & ~127u;
    L.s2_sbo = (uint32_t)cols * 16u;
    L.stage_a = (4u * L.s2_phase_stride + 1023u) & ~1023u;
    L.stage_bytes = L.stage_a;
    // taps in shared-memory address order, paired into K = 16 MMAs (the second of a pair at a
    // higher address: LBO > 0); an odd tap count ends with a zero-weight chunk reading the
    // neighbouring (finite) pixel
    std::vector<std::pair<uint32_t, int>> taps;
    for (int r = 0; r < L.r; ++r)
      for (int s = 0; s < L.s; ++s)
        taps.emplace_back((uint32_t)((r % 2) * 2 + (s % 2)) * L.s2_phase_stride +
                              (uint32_t)((r / 2) * cols + s / 2) * 16u,
                          r * L.s + s);
    std::sort(taps.begin(), taps.end());
    L.s2_pairs = (int)(taps.size() + 1) / 2;
    for (int u = 0; u < L.s2_pairs; ++u) {
      const auto &t0 = taps[2 * u];
      const bool two = 2 * u + 1 < (int)taps.size();
      L.s2_a_off[u] = (uint16_t)t0.first;
      L.s2_a_lbo[u] = (uint16_t)(two ? taps[2 * u + 1].first - t0.first : 16u);
      L.s2_chunk_tap[2 * u] = (int16_t)t0.second;
      L.s2_chunk_tap[2 * u + 1] = (int16_t)(two ? taps[2 * u + 1].second : -1);
    }
  } else if (conv_halo_ok(L, BN)) {
    L.conv_halo = 1;
    L.tq = 8;
    L.tp = kBM / 8;
    L.tiles_p = (L.p + L.tp - 1) / L.tp;
    L.tiles_q = (L.q + L.tq - 1) / L.tq;
    L.tiles_m = L.n * L.tiles_p * L.tiles_q;
    L.c_blocks = L.c / kBK;
    L.num_kb = L.r * L.c_blocks;               // k-steps: (filter row, channel block)
    L.stage_a = ((uint32_t)L.tp * (L.tq + L.s - 1) * 128u + 1023u) & ~1023u;
    L.stage_bytes = L.stage_a + (uint32_t)L.s * BN * 128u;
  } else if (L.kind == TACKER_LC_CONV_F16 && !L.conv_direct_gemm && L.c == 8) {
    L.conv_im2col = 1;               // C = 8 (conv1 padded): 8 taps per k-block
    L.conv_c8 = 1;
    L.tiles_m = (L.M + kBM - 1) / kBM;
    L.c_blocks = 1;
    L.num_kb = (L.r * L.s + 7) / 8;
  } else if (L.kind == TACKER_LC_CONV_F16 && !L.conv_direct_gemm && conv_im2col_mode()) {
    L.conv_im2col = 1;
    L.tiles_m = (L.M + kBM - 1) / kBM;
    L.c_blocks = L.c / kBK;
    L.num_kb = L.r * L.s * L.c_blocks;
  } else if (L.kind == TACKER_LC_CONV_F16 && !L.conv_direct_gemm) {
    // output tile of 128 positions: tq along q (power of two <= 32 covering q), tp = 128/tq
    int tq = 1;
    while (tq < L.q && tq < 32) tq <<= 1;
    if (tq < 8) tq = 8;
    L.tq = tq;
    L.tp = kBM / tq;
    L.tiles_p = (L.p + L.tp - 1) / L.tp;
    L.tiles_q = (L.q + L.tq - 1) / L.tq;
    L.tiles_m = L.n * L.tiles_p * L.tiles_q;
    L.c_blocks = L.c / kBK;
    L.num_kb = L.r * L.s * L.c_blocks;
  } else {
    L.tiles_m = (L.M + kBM - 1) / kBM;
    L.num_kb = (L.K + kBK - 1) / kBK;
  }
  L.num_tiles = L.tiles_m * L.tiles_n;
  L.splits = 1;
  L.kb_per_split = L.num_kb;
  L.num_units = L.num_tiles;
}

// Split-K for GEMMs with few tiles and a deep K (batch-1 layer3/4 convs: 4-16 tiles of 16-72
// k-blocks would leave >= 132 SMs idle and serialise the k-loop): S splits of >= 2 k-blocks so
// that tiles x S <= #SMs -- every unit gets its own CTA, which the in-kernel fixup requires.
static void lc_split(LcParams &L, int sms) {
  if (L.num_tiles * 2 > sms || L.num_kb < 4) return;
  int S = std::min(sms / L.num_tiles, L.num_kb / 2);
  if (S < 2) return;
  const int kbs = (L.num_kb + S - 1) / S;
  S = (L.num_kb + kbs - 1) / kbs;
  if (S < 2) return;
  L.splits = S;
  L.kb_per_split = kbs;
  L.num_units = L.num_tiles * S;
}

static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

static tacker_status encode_2d(CUtensorMap *m, const void *base, uint64_t inner, uint64_t outer, uint32_t box_inner,
                               uint32_t box_outer) {
  auto enc = get_encode();
  if (!enc) return set_error("cuTensorMapEncodeTiled unavailable"), TACKER_ECUDA;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {inner * 2};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void *>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error("cuTensorMapEncodeTiled(2d) failed: %d", (int)r), TACKER_ECUDA;
  return TACKER_OK;
}

static tacker_status encode_conv_x(CUtensorMap *m, const tacker_lc_desc &d, const LcParams &L) {
  auto enc = get_encode();
  if (!enc) return set_error("cuTensorMapEncodeTiled unavailable"), TACKER_ECUDA;
  cuuint64_t dims[4] = {(cuuint64_t)d.c, (cuuint64_t)d.w, (cuuint64_t)d.h, (cuuint64_t)d.n};
  cuuint64_t strides[3] = {(cuuint64_t)d.c * 2, (cuuint64_t)d.c * d.w * 2, (cuuint64_t)d.c * d.w * d.h * 2};
  cuuint32_t box[4] = {(cuuint32_t)kBK, (cuuint32_t)(L.tq * d.stride), (cuuint32_t)(L.tp * d.stride), 1};
  cuuint32_t es[4] = {1, (cuuint32_t)d.stride, (cuuint32_t)d.stride, 1};
  if (box[1] > 256 || box[2] > 256) return set_error("conv: TMA box too large"), TACKER_EUNSUPPORTED;
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, const_cast<void *>(d.A), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error("cuTensorMapEncodeTiled(conv x) failed: %d", (int)r), TACKER_ECUDA;
  return TACKER_OK;
}

static tacker_status encode_2d_raw(CUtensorMap *m, const void *base, uint64_t inner, uint64_t outer, uint32_t box_inner,
                                   uint32_t box_outer, CUtensorMapSwizzle swz) {
  auto enc = get_encode();
  if (!enc) return set_error("cuTensorMapEncodeTiled unavailable"), TACKER_ECUDA;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {inner * 2};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void *>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error("cuTensorMapEncodeTiled(2d raw) failed: %d", (int)r), TACKER_ECUDA;
  return TACKER_OK;
}

// Phase-halo A (conv_s2c8): NHWC as (C = 8, W, H, N), traversal stride 2 in W and H, box 8 channels x
// 2 cols x 2 rows of the phase (cols x rows pixels of 16 B loaded, unswizzled); out-of-image pixels
// zero-filled = the padding.
static tacker_status encode_conv_s2c8(CUtensorMap *m, const tacker_lc_desc &d, const LcParams &L) {
  auto enc = get_encode();
  if (!enc) return set_error("cuTensorMapEncodeTiled unavailable"), TACKER_ECUDA;
  const int rows = L.tp + (L.r - 1) / 2, cols = L.tq + (L.s - 1) / 2;
  cuuint64_t dims[4] = {8, (cuuint64_t)d.w, (cuuint64_t)d.h, (cuuint64_t)d.n};
  cuuint64_t strides[3] = {16, (cuuint64_t)d.w * 16, (cuuint64_t)d.w * d.h * 16};
  cuuint32_t box[4] = {8, (cuuint32_t)(2 * cols), (cuuint32_t)(2 * rows), 1};
  cuuint32_t es[4] = {1, 2, 2, 1};
  if (box[1] > 256 || box[2] > 256) return set_error("conv s2c8: TMA box too large"), TACKER_EUNSUPPORTED;
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, const_cast<void *>(d.A), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error("cuTensorMapEncodeTiled(conv s2c8) failed: %d", (int)r), TACKER_ECUDA;
  return TACKER_OK;
}

// Halo mode A: NHWC as (C, W, H, N), box 64 channels x (tq + S - 1) columns x tp rows x 1 image,
// SW128 (one 128-byte row per pixel, pixels in (row, column) order); out-of-image = zero padding.
static tacker_status encode_conv_halo(CUtensorMap *m, const tacker_lc_desc &d, const LcParams &L) {
  auto enc = get_encode();
  if (!enc) return set_error("cuTensorMapEncodeTiled unavailable"), TACKER_ECUDA;
  cuuint64_t dims[4] = {(cuuint64_t)d.c, (cuuint64_t)d.w, (cuuint64_t)d.h, (cuuint64_t)d.n};
  cuuint64_t strides[3] = {(cuuint64_t)d.c * 2, (cuuint64_t)d.c * d.w * 2, (cuuint64_t)d.c * d.w * d.h * 2};
  cuuint32_t box[4] = {(cuuint32_t)kBK, (cuuint32_t)(L.tq + L.s - 1), (cuuint32_t)L.tp, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, const_cast<void *>(d.A), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error("cuTensorMapEncodeTiled(conv halo) failed: %d", (int)r), TACKER_ECUDA;
  return TACKER_OK;
}

// TMA-store map of a halo tile's output: NHWC D as (K, Q, P, N), box 64 channels x 8 columns x 4
// rows x 1 image = one epilogue warp's 32 TMEM lanes; rows / columns past P / Q are clipped.
static tacker_status encode_conv_out_4d(CUtensorMap *m, const tacker_lc_desc &d, const LcParams &L) {
  auto enc = get_encode();
  if (!enc) return set_error("cuTensorMapEncodeTiled unavailable"), TACKER_ECUDA;
  cuuint64_t dims[4] = {(cuuint64_t)L.N, (cuuint64_t)L.q, (cuuint64_t)L.p, (cuuint64_t)L.n};
  cuuint64_t strides[3] = {(cuuint64_t)L.N * 2, (cuuint64_t)L.N * L.q * 2, (cuuint64_t)L.N * L.q * L.p * 2};
  cuuint32_t box[4] = {64, (cuuint32_t)L.tq, 4, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, d.D, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error("cuTensorMapEncodeTiled(conv out) failed: %d", (int)r), TACKER_ECUDA;
  return TACKER_OK;
}

using PFN_encodeIm2col = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                       const cuuint64_t *, const int *, const int *, cuuint32_t, cuuint32_t,
                                       const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                       CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static PFN_encodeIm2col get_encode_im2col() {
  static PFN_encodeIm2col fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_encodeIm2col>(p);
  });
  return fn;
}

// A of an implicit conv in im2col mode: NHWC as (C, W, H, N); the pixel bounding box of every
// image is [-pad, W - 1 + pad - (S - 1)] x [-pad, H - 1 + pad - (R - 1)] walked with the conv
// stride, i.e. exactly the P x Q output positions; 64 channels (128 B, SW128) per pixel, 128
// pixels per load.
static tacker_status encode_conv_im2col(CUtensorMap *m, const tacker_lc_desc &d, bool c8 = false) {
  auto enc = get_encode_im2col();
  if (!enc) return set_error("cuTensorMapEncodeIm2col unavailable"), TACKER_ECUDA;
  if (d.pad > 127 || d.pad - (d.s - 1) < -128 || d.pad - (d.r - 1) < -128 || d.r > 256 || d.s > 256)
    return set_error("conv: padding / filter outside the im2col corner range"), TACKER_EUNSUPPORTED;
  cuuint64_t dims[4] = {(cuuint64_t)d.c, (cuuint64_t)d.w, (cuuint64_t)d.h, (cuuint64_t)d.n};
  cuuint64_t strides[3] = {(cuuint64_t)d.c * 2, (cuuint64_t)d.c * d.w * 2, (cuuint64_t)d.c * d.w * d.h * 2};
  int lower[2] = {-d.pad, -d.pad};
  int upper[2] = {d.pad - (d.s - 1), d.pad - (d.r - 1)};
  cuuint32_t es[4] = {1, (cuuint32_t)d.stride, (cuuint32_t)d.stride, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, const_cast<void *>(d.A), dims, strides, lower, upper,
                   c8 ? 8u : (cuuint32_t)kBK, (cuuint32_t)kBM, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   c8 ? CU_TENSOR_MAP_SWIZZLE_NONE : CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error("cuTensorMapEncodeIm2col(conv x) failed: %d", (int)r), TACKER_ECUDA;
  // driver <= 13.1 with a tensor under 128 KiB: clear descriptor bit 85 (as CUTLASS does)
  int drv = 0;
  if (cudaDriverGetVersion(&drv) == cudaSuccess && drv <= 13010 &&
      (uint64_t)d.n * d.h * d.w * d.c * 2 < 131072)
    reinterpret_cast<uint64_t *>(m)[1] &= ~(1ull << 21);
  return TACKER_OK;
}

// BE tensor-map hook: a body that stages its input with TMA gets its tensor map encoded here
// (the stencil's TMA plane-ring variant used it; the current bodies load through L1/L2).
static tacker_status encode_be_tmap(const tacker_be_desc &, CUtensorMap *m) {
  memset(m, 0, sizeof *m);
  return TACKER_OK;
}

// ============================================================================ kernel table
using KernelFn = void (*)(FusedParams);

template <int BN>
static KernelFn fused_fn(int be_kind) {
  switch (be_kind) {
    case TACKER_BE_NONE: return fused_kernel<BN, TACKER_BE_NONE>;
#define C(K) \
  case K: return fused_kernel<BN, K>;
    TK_FOR_EACH_BE(C)
#undef C
    default: return nullptr;
  }
}
// TACKER_RICH=0 disables the register-rich class (A/B measurements)
static bool rich_class_enabled() {
  static const bool on = [] {
    const char *e = getenv("TACKER_RICH");
    return !(e && e[0] == '0');
  }();
  return on;
}
// LC-only kernels compiled for one LC mode and epilogue each (fused_lc.cu)
static bool lc_mode_kernels_on() {   // TACKER_LC_MODE_KERNELS=0: the run-time-mode kernels
  static const bool on = [] {
    const char *e = getenv("TACKER_LC_MODE_KERNELS");
    return !(e && e[0] == '0');
  }();
  return on;
}
static KernelFn pick_lc_only(int BN, int mode, int epi) {
  if (!lc_mode_kernels_on()) return nullptr;
  return reinterpret_cast<KernelFn>(pick_lc_only_kernel(BN, mode, epi));
}
static int lc_mode_of(const LcParams &L) {
  if (L.kind != TACKER_LC_CONV_F16 || L.conv_direct_gemm) return kModeGemm;
  if (L.conv_s2c8) return kModeS2c8;
  if (L.conv_halo) return kModeHalo;
  if (L.conv_c8) return kModeC8;
  if (L.conv_im2col) return kModeIm2col;
  return kModeTiled;
}
static KernelFn pick_fused(int BN, int be_kind) {
  if (BN == 64) return fused_fn<64>(be_kind);
  if (BN == 128) return fused_fn<128>(be_kind);
  if (BN == 256) return fused_fn<256>(be_kind);
  return nullptr;
}

using BeFn = void (*)(BeOrigParams);
static BeFn pick_be_original(int kind) {
  switch (kind) {
#define C(K) \
  case K: return be_original_kernel<K>;
    TK_FOR_EACH_BE(C)
#undef C
    default: return nullptr;
  }
}

// The dynamic-SMEM limit is a per-function attribute shared by every plan of that instantiation:
// only ever raise it (a later, smaller plan must not invalidate the launches of an earlier one).
static tacker_status set_smem_attr(const void *fn, int bytes) {
  static std::mutex mu;
  static std::unordered_map<const void *, int> limit;
  std::lock_guard<std::mutex> g(mu);
  int &cur = limit[fn];
  if (bytes <= cur) return TACKER_OK;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e != cudaSuccess) return cuda_fail("cudaFuncSetAttribute", e);
  cur = bytes;
  return TACKER_OK;
}

// ============================================================================ fused handle
struct tacker_fused_s {
  FusedParams P;
  KernelFn fn;
  tacker_lc_desc lc;
  tacker_be_desc be;
  int warp_split;
  int grid, block, smem;
  int BN;
  int regs;
  int64_t be_full;         // whole-problem BE block count (slice bound)
  std::string lc_key, be_key, pair_key;
};

static std::string lc_key_of(const tacker_lc_desc &d, const LcParams &L, int BN) {
  char b[256];
  if (d.kind == TACKER_LC_GEMM_F16)
    snprintf(b, sizeof b, "lc:gemm:N%d:K%d:bn%d:%s", L.N, L.K, BN, L.d_f16 ? "f16" : "f32");
  else
    snprintf(b, sizeof b, "lc:conv:h%dw%dc%d:k%dr%ds%d:st%dp%d:bn%d", d.h, d.w, d.c, d.k, d.r, d.s, d.stride, d.pad, BN);
  return b;
}

static std::string be_key_of(const tacker_be_desc &d) {
  char b[256];
  switch (d.kind) {
    case TACKER_BE_SGEMM: snprintf(b, sizeof b, "be:sgemm:N%d:K%d", d.p.sgemm.N, d.p.sgemm.K); break;
    case TACKER_BE_STENCIL: snprintf(b, sizeof b, "be:stencil:nz%d", d.p.stencil.nz); break;
    case TACKER_BE_MRIQ_Q: snprintf(b, sizeof b, "be:mriq_q:K%d", d.p.mriq_q.numK); break;
    case TACKER_BE_MRIFHD_FH: snprintf(b, sizeof b, "be:mrifhd_fh:K%d", d.p.mrifhd_fh.numK); break;
    case TACKER_BE_CP: snprintf(b, sizeof b, "be:cp:A%d", d.p.cp.natoms); break;
    case TACKER_BE_FFT: snprintf(b, sizeof b, "be:fft:n%d", d.p.fft.n); break;
    case TACKER_BE_TPACF: snprintf(b, sizeof b, "be:tpacf:nb%d:s%d", d.p.tpacf.nb, d.p.tpacf.self_pairs); break;
    case TACKER_BE_FMA_BURN: snprintf(b, sizeof b, "be:fma_burn:it%d", d.p.fma_burn.iters); break;
    default: snprintf(b, sizeof b, "be:%s", be_kind_name(d.kind)); break;
  }
  return b;
}

static tacker_status plan(const tacker_lc_desc *lc, const tacker_be_desc *be, int warp_split, tacker_ratio ratio,
                          tacker_fused_s &F) {
  memset(&F.P, 0, sizeof F.P);
  const bool has_lc = lc && lc->kind != TACKER_LC_NONE;
  const bool has_be = be && be->kind != TACKER_BE_NONE;
  if (!has_lc) return set_error("tacker_fuse: an LC descriptor is required"), TACKER_EINVAL;
  if (has_be && (warp_split < 4 || warp_split % 4 || warp_split > be_max_warps(be->kind)))
    return set_error("warp_split must be a multiple of 4 in [4, %d] for BE kind %d (got %d)", be_max_warps(be->kind),
                     be->kind, warp_split),
           TACKER_EUNSUPPORTED;
  if (!has_be && warp_split != 0) return set_error("warp_split must be 0 without a BE part"), TACKER_EINVAL;
  const int sms = sm_count();
  if (sms <= 0) return set_error("no CUDA device"), TACKER_ECUDA;

  LcParams &L = F.P.lc;
  tacker_status st = lc_view(*lc, L);
  if (st) return st;
  const int BN = pick_tile_n(*lc, L);
  lc_tiles(L, BN);
  if (!(lc->epi_flags & TACKER_LC_NO_SPLIT)) lc_split(L, sms);
  F.BN = BN;

  int64_t be_blocks = 0;
  int vb = 0;
  uint32_t be_slice = 0;
  F.be_full = 0;
  if (has_be) {
    if ((st = validate_be(*be, &be_blocks))) return st;
    be_num_blocks(*be, &F.be_full);
    vb = warp_split / 4;
    if (ratio.be && ratio.be != vb)
      return set_error("block_ratio.be (%d) must equal warp_split/4 (%d)", ratio.be, vb), TACKER_EUNSUPPORTED;
    if (vb > 14) return set_error("too many BE virtual blocks for named barriers (1..14)"), TACKER_ERESOURCE;
    be_slice = (16 + be_smem_bytes(be->kind) + 127) & ~127u;
    F.P.be = *be;
  }
  const int acc = ratio.lc ? ratio.lc : (2 * BN <= kTmemCols ? 2 : 1);
  if (acc < 1 || acc > 2 || acc * BN > kTmemCols)
    return set_error("block_ratio.lc (TMEM accumulator stages) %d does not fit %d columns", acc, kTmemCols), TACKER_ERESOURCE;
  uint32_t cols = 32;
  while (cols < (uint32_t)(acc * BN)) cols <<= 1;

  // TMA-store epilogue: LC-only fp16 outputs whose GEMM rows are linear in D (plain GEMM, 1x1
  // stride-1 conv, im2col-mode conv), no residual, no split-K; 4 warps x 2 staging boxes of 4 KB
  L.tma_store = !has_be && tma_store_enabled() && lc->d_dtype == TACKER_F16 &&
                !(lc->epi_flags & TACKER_EPI_RESIDUAL) && L.splits == 1 && BN >= 64 && L.N >= 64 &&
                (lc->kind == TACKER_LC_GEMM_F16 || L.conv_direct_gemm || L.conv_im2col || L.conv_halo ||
                 L.conv_s2c8);
  const uint32_t epi_bytes = (L.tma_store ? 4u * 2u * 4096u + 1024u : 0u) +
                             (L.conv_s2c8 ? 2u * L.s2_pairs * 1024u + 1024u : 0u);   // + resident weights
  L.dbg = lc_dbg_flags();
  // LC first (TC-first rule, §V-C): the deepest ring (<= 4 stages fused, <= 8 LC-only,
  // >= 2) that still leaves room for the requested BE virtual blocks.
  const uint32_t stage_bytes = L.stage_bytes;
  const uint32_t bar_bytes = 256 + 4 * 256 + epi_bytes;   // mbarriers + TMEM address + one tile's bias (BN <= 256) + staging
  const uint32_t be_total = (uint32_t)vb * be_slice;
  // LC-only launches take the deepest ring that fits (up to 8 stages: more TMA bytes in flight per
  // SM for the latency-bound implicit-GEMM loads); fused plans stop at 4 so the BE keeps L1
  int stages = 0;
  for (int s = has_be ? 4 : 8; s >= 2; --s) {
    const uint32_t need = 1024 + s * stage_bytes + bar_bytes + be_total;
    if (need <= (uint32_t)kSmemCap) {
      stages = s;
      break;
    }
  }
  if (!stages) {
    set_error("fused budget exceeds one SM: LC ring %u B x2 + BE %d x %u B > %d B", stage_bytes, vb, be_slice, kSmemCap);
    return TACKER_ERESOURCE;
  }
  const int warps = kLcWarps + warp_split;
  if (warps > kMaxWarps) return set_error("too many warps"), TACKER_ERESOURCE;

  F.P.stages = stages;
  F.P.acc_stages = acc;
  F.P.tmem_cols = cols;
  F.P.lc_smem_bytes = (stages * stage_bytes + bar_bytes + 127) & ~127u;
  F.P.epi_stage_off = L.tma_store ? ((uint32_t)stages * stage_bytes + 256u + 4u * 256u + 1023u) & ~1023u : 0u;
  if (L.conv_s2c8) {
    const uint32_t after = L.tma_store ? F.P.epi_stage_off + 4u * 2u * 4096u : (uint32_t)stages * stage_bytes + 1280u;
    L.b_res_off = (after + 1023u) & ~1023u;
  }
  F.P.be_smem_per_vb = be_slice;
  F.P.be_vb_per_cta = vb;
  F.P.be_blocks = be_blocks;
  F.P.be_offset = has_be ? be->block_offset : 0;
  F.P.lc_warps = kLcWarps;
  F.warp_split = warp_split;
  F.block = 32 * warps;
  F.smem = 1024 + F.P.lc_smem_bytes + be_total;
  // An LC-only CTA (6 warps) could otherwise share an SM with a second one (both allocating
  // TMEM); a fused CTA is already alone on its SM through its registers (>= 16 warps x 64
  // regs... a second CTA would exceed 64K), so it keeps the unused shared memory as L1.
  if (!has_be && F.smem < kMinLcSmem) F.smem = kMinLcSmem;
  F.grid = has_be ? sms : (L.num_units < sms ? L.num_units : sms);
  if (F.grid < 1) F.grid = 1;
  // register class: plans with at most 8 BE warps take the register-rich instantiation (up to
  // 128 registers per thread) where one is compiled; wider plans the default class (64)
  F.fn = nullptr;
  if (has_be && warp_split <= 8 && rich_class_enabled()) F.fn = reinterpret_cast<KernelFn>(pick_fused_rich(BN, be->kind));
  if (!F.fn && !has_be) F.fn = pick_lc_only(BN, lc_mode_of(L), L.tma_store && BN >= 64 ? 1 : 2);
  if (!F.fn && has_be && lc_mode_kernels_on())   // default register class, compiled per LC mode
    F.fn = reinterpret_cast<KernelFn>(pick_fused_mode_kernel(BN, be->kind, lc_mode_of(L)));
  if (!F.fn) F.fn = pick_fused(BN, has_be ? be->kind : TACKER_BE_NONE);
  if (!F.fn) return set_error("no kernel instantiation for BN=%d BE=%d", BN, has_be ? be->kind : 0), TACKER_EUNSUPPORTED;

  // TMA tensor maps
  if (lc->kind == TACKER_LC_CONV_F16 && !L.conv_direct_gemm) {
    if ((st = L.conv_s2c8 ? encode_conv_s2c8(&F.P.tmap_a, *lc, L)
              : L.conv_halo ? encode_conv_halo(&F.P.tmap_a, *lc, L)
                            : L.conv_im2col ? encode_conv_im2col(&F.P.tmap_a, *lc, L.conv_c8 != 0)
                                            : encode_conv_x(&F.P.tmap_a, *lc, L)))
      return st;
    if (L.conv_s2c8) {   // weights [N][R S 8]: one 16-byte tap chunk x 64 rows per load, unswizzled
      if ((st = encode_2d_raw(&F.P.tmap_b, lc->B, (uint64_t)L.K, (uint64_t)L.N, 8, 64, CU_TENSOR_MAP_SWIZZLE_NONE)))
        return st;
    } else if ((st = encode_2d(&F.P.tmap_b, lc->B, (uint64_t)L.K, (uint64_t)L.N, kBK, BN))) {
      return st;
    }
  } else {
    if ((st = encode_2d(&F.P.tmap_a, lc->A, (uint64_t)L.K, (uint64_t)L.M, kBK, kBM))) return st;
    if ((st = encode_2d(&F.P.tmap_b, lc->B, (uint64_t)L.K, (uint64_t)L.N, kBK, BN))) return st;
  }
  if (has_be && (st = encode_be_tmap(*be, &F.P.tmap_be))) return st;
  if (L.tma_store && (L.conv_halo || L.conv_s2c8)) {
    if ((st = encode_conv_out_4d(&F.P.tmap_d, *lc, L))) return st;
  } else if (L.tma_store && (st = encode_2d(&F.P.tmap_d, lc->D, (uint64_t)L.N, (uint64_t)L.M, 64, 32))) {
    return st;
  }
  // registers: the whole CTA must fit the 64K register file
  cudaFuncAttributes fa{};
  cudaError_t e = cudaFuncGetAttributes(&fa, reinterpret_cast<const void *>(F.fn));
  if (e != cudaSuccess) return cuda_fail("cudaFuncGetAttributes", e);
  F.regs = fa.numRegs;
  if ((int64_t)fa.numRegs * F.block > 65536) {
    set_error("register budget: %d regs x %d threads > 65536", fa.numRegs, F.block);
    return TACKER_ERESOURCE;
  }
  if ((st = set_smem_attr(reinterpret_cast<const void *>(F.fn), F.smem))) return st;
  F.lc = *lc;
  if (has_be) F.be = *be; else memset(&F.be, 0, sizeof F.be);
  F.lc_key = lc_key_of(*lc, L, BN);
  F.be_key = has_be ? be_key_of(*be) : "";
  char pk[512];
  snprintf(pk, sizeof pk, "pair:%s|%s|ws%d", F.lc_key.c_str(), F.be_key.c_str(), warp_split);
  F.pair_key = pk;
  return TACKER_OK;
}

namespace tkrt {
bool blacklist_op(const std::string &be_key, int op);
}

static std::atomic<int> g_overlap{TACKER_OVERLAP_DEFAULT};

// cudaLaunchKernelEx with programmatic stream serialization (PDL) unless disabled for this
// launch class (be_original: a non-persistent BE grid)
template <typename Param>
static cudaError_t launch_ex(void (*fn)(Param), dim3 grid, dim3 block, int smem, cudaStream_t s, const Param &p,
                             bool be_original = false) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  const int ov = g_overlap.load(std::memory_order_relaxed);
  cfg.numAttrs = (ov == 1 || (ov == 2 && !be_original)) ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, fn, p);
}

// Split-K workspace (partial tiles + counters) of a plan, owned by its handle.
static tacker_status alloc_lc_workspace(tacker_fused_s &F) {
  LcParams &L = F.P.lc;
  L.part = nullptr;
  L.cnt = nullptr;
  if (L.splits <= 1) return TACKER_OK;
  const size_t part = (size_t)L.num_units * kBM * F.BN * sizeof(float);
  void *p = nullptr;
  cudaError_t e = cudaMalloc(&p, part + 2 * (size_t)L.num_tiles * sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaMemset(static_cast<char *>(p) + part, 0, 2 * (size_t)L.num_tiles * sizeof(uint32_t));
  if (e != cudaSuccess) {
    if (p) cudaFree(p);
    return cuda_fail("split-K workspace", e);
  }
  L.part = static_cast<float *>(p);
  L.cnt = reinterpret_cast<uint32_t *>(static_cast<char *>(p) + part);
  return TACKER_OK;
}

static std::atomic<int> g_dbg_launch{0};
static tacker_status launch_params(const tacker_fused_s &F, FusedParams &P, cudaStream_t s) {
  if (P.lc.dbg & 16) P.lc.dbg_id = g_dbg_launch.fetch_add(1) & 255;   // diagnostics slot
  cudaError_t e = launch_ex(F.fn, dim3(F.grid), dim3(F.block), F.smem, s, P);
  if (e != cudaSuccess) return cuda_fail("launch fused_kernel", e);
  return TACKER_OK;
}
static tacker_status launch_plan(tacker_fused_s &F, cudaStream_t s) { return launch_params(F, F.P, s); }

// ============================================================================ C ABI
extern "C" {

const char *tacker_last_error(void) { return g_err.c_str(); }

tacker_status tacker_select_fusion(const tacker_lc_desc *lc, const tacker_be_desc *be, const int32_t *splits,
                                   int32_t n_splits, int32_t reps, tacker_stream_t s, int32_t *best_ws,
                                   double *best_ms, double *seq_ms, double *fused_ms) {
  if (!lc || !be || !splits || n_splits <= 0 || reps <= 0 || !best_ws || !best_ms || !seq_ms)
    return set_error("tacker_select_fusion: bad arguments"), TACKER_EINVAL;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(s);
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto time_it = [&](auto &&launch, double *ms) -> tacker_status {
    if (tacker_status r = launch()) return r;   // warm-up
    cudaEventRecord(e0, st);
    for (int i = 0; i < reps; ++i)
      if (tacker_status r = launch()) return r;
    cudaEventRecord(e1, st);
    cudaError_t e = cudaEventSynchronize(e1);
    if (e != cudaSuccess) return cuda_fail("select_fusion sync", e);
    float f = 0;
    cudaEventElapsedTime(&f, e0, e1);
    *ms = (double)f / reps;
    return TACKER_OK;
  };
  tacker_status r = time_it([&] { return tacker_launch_original(lc, be, s); }, seq_ms);
  *best_ws = 0;
  *best_ms = *seq_ms;
  for (int32_t i = 0; r == TACKER_OK && i < n_splits; ++i) {
    if (fused_ms) fused_ms[i] = NAN;
    tacker_fused_t f = nullptr;
    tacker_status fs = tacker_fuse(lc, be, splits[i], tacker_ratio{0, 0}, &f);
    if (fs == TACKER_ERESOURCE || fs == TACKER_EUNSUPPORTED) continue;   // not a candidate
    if (fs) {
      r = fs;
      break;
    }
    double ms = 0;
    r = time_it([&] { return tacker_launch_fused(f, s); }, &ms);
    tacker_fused_destroy(f);
    if (r) break;
    if (fused_ms) fused_ms[i] = ms;
    if (ms < *best_ms) {
      *best_ms = ms;
      *best_ws = splits[i];
    }
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (r) return r;
  if (*best_ws == 0) tkrt::blacklist_op(be_key_of(*be), 1);
  return TACKER_OK;
}

tacker_status tacker_blacklist(const char *be_key, int32_t op, int32_t *listed) {
  if (!be_key || op < -1 || op > 1) return set_error("tacker_blacklist: bad arguments"), TACKER_EINVAL;
  const bool in = tkrt::blacklist_op(be_key, op);
  if (listed) *listed = in ? 1 : 0;
  return TACKER_OK;
}

tacker_status tacker_blacklist_clear(void) {
  tkrt::blacklist_op("", 2);
  return TACKER_OK;
}

tacker_status tacker_debug_lc_timestamps(uint64_t *out, int64_t n) {
  if (!out || n < 160 * 5 * 16) return set_error("need 12800 uint64 slots"), TACKER_EINVAL;
  cudaError_t e = cudaMemcpyFromSymbol(out, tk::g_lc_ts, sizeof(tk::g_lc_ts));
  if (e != cudaSuccess) return cuda_fail("debug timestamps", e);
  return TACKER_OK;
}

tacker_status tacker_debug_lc_globaltimer(uint64_t *out, int64_t n, int32_t *next_slot) {
  if (!out || n < 256 * 8) return set_error("need 2048 uint64 slots"), TACKER_EINVAL;
  cudaError_t e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpyFromSymbol(out, tk::g_lc_gt, sizeof(tk::g_lc_gt));
  static const unsigned long long zero[256][8] = {};
  if (e == cudaSuccess) e = cudaMemcpyToSymbol(tk::g_lc_gt, zero, sizeof zero);
  if (e != cudaSuccess) return cuda_fail("debug globaltimer", e);
  if (next_slot) *next_slot = g_dbg_launch.exchange(0) & 255;
  return TACKER_OK;
}

tacker_status tacker_set_launch_overlap(int32_t enable) {
  if (enable < 0 || enable > 2) return set_error("launch overlap mode must be 0, 1 or 2"), TACKER_EINVAL;
  g_overlap.store(enable);
  return TACKER_OK;
}
const char *tacker_version(void) { return "tacker-b200 0.1 (sm_100a)"; }
int tacker_device_sm_count(void) { return sm_count(); }

tacker_status tacker_be_num_blocks(const tacker_be_desc *be, int64_t *out) {
  if (!be || !out) return set_error("null argument"), TACKER_EINVAL;
  if (!be_num_blocks(*be, out)) return set_error("BE kind %d not supported", be->kind), TACKER_EUNSUPPORTED;
  return TACKER_OK;
}

tacker_status tacker_lc_num_tiles(const tacker_lc_desc *lc, int32_t tile_n, int64_t *out) {
  if (!lc || !out) return set_error("null argument"), TACKER_EINVAL;
  LcParams L;
  tacker_status st = lc_view(*lc, L);
  if (st) return st;
  int BN = tile_n ? tile_n : pick_tile_n(*lc, L);
  if (BN != 64 && BN != 128 && BN != 256) return set_error("tile_n must be 64/128/256"), TACKER_EINVAL;
  lc_tiles(L, BN);
  *out = L.num_tiles;
  return TACKER_OK;
}

tacker_status tacker_lc_num_waves(const tacker_lc_desc *lc, int32_t tile_n, int64_t *out) {
  if (!lc || !out) return set_error("null argument"), TACKER_EINVAL;
  LcParams L;
  tacker_status st = lc_view(*lc, L);
  if (st) return st;
  int BN = tile_n ? tile_n : pick_tile_n(*lc, L);
  if (BN != 64 && BN != 128 && BN != 256) return set_error("tile_n must be 64/128/256"), TACKER_EINVAL;
  lc_tiles(L, BN);
  const int sms = sm_count() > 0 ? sm_count() : 148;
  if (!(lc->epi_flags & TACKER_LC_NO_SPLIT)) lc_split(L, sms);
  const int grid = L.num_units < sms ? L.num_units : sms;
  *out = (L.num_units + grid - 1) / grid;
  return TACKER_OK;
}

tacker_status tacker_be_prefix_work(const tacker_be_desc *be, int64_t n, double *work) {
  if (!be || !work || n < 0) return set_error("bad argument"), TACKER_EINVAL;
  int64_t full = 0;
  if (!be_num_blocks(*be, &full)) return set_error("bad BE descriptor"), TACKER_EINVAL;
  n = std::min(n, full);
  if (be->kind == TACKER_BE_SPMV_JDS) {
    const tacker_be_spmv &p = be->p.spmv;
    const int64_t rows = std::min<int64_t>((int64_t)p.rows, n * 128);
    std::vector<int32_t> len((size_t)rows);
    cudaError_t e = cudaMemcpy(len.data(), p.row_len, (size_t)rows * 4, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return cuda_fail("prefix work (spmv row lengths)", e);
    double nnz = 0;
    for (int32_t l : len) nnz += l;
    *work = 8.0 * nnz + 16.0 * (double)rows;
    return TACKER_OK;
  }
  if (be->kind == TACKER_BE_CUTCP) {
    const tacker_be_cutcp &p = be->p.cutcp;
    const int64_t nb = (int64_t)p.bdim_x * p.bdim_y * p.bdim_z;
    std::vector<int32_t> cnt((size_t)nb);
    cudaError_t e = cudaMemcpy(cnt.data(), p.count, (size_t)nb * 4, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return cuda_fail("prefix work (cutcp bin counts)", e);
    const int reach = (int)std::ceil(p.cutoff / p.bin_size);
    double w = 0;
    for (int64_t b = 0; b < n; ++b) {   // block b = bin b in (z, y, x) order: its 512 points x neighbour atoms
      const int bx = (int)(b % p.bdim_x), by = (int)((b / p.bdim_x) % p.bdim_y), bz = (int)(b / ((int64_t)p.bdim_x * p.bdim_y));
      int64_t atoms = 0;
      for (int z = std::max(bz - reach, 0); z <= std::min(bz + reach, p.bdim_z - 1); ++z)
        for (int y = std::max(by - reach, 0); y <= std::min(by + reach, p.bdim_y - 1); ++y)
          for (int x = std::max(bx - reach, 0); x <= std::min(bx + reach, p.bdim_x - 1); ++x)
            atoms += std::min(cnt[((size_t)z * p.bdim_y + y) * p.bdim_x + x], p.bin_depth);
      w += 512.0 * (double)atoms;
    }
    *work = w;
    return TACKER_OK;
  }
  *work = (double)n;
  return TACKER_OK;
}

tacker_status tacker_fuse(const tacker_lc_desc *lc, const tacker_be_desc *be, int32_t warp_split, tacker_ratio block_ratio,
                          tacker_fused_t *out) {
  if (!out) return set_error("null out"), TACKER_EINVAL;
  *out = nullptr;
  auto *F = new (std::nothrow) tacker_fused_s();
  if (!F) return set_error("out of host memory"), TACKER_ENOMEM;
  tacker_status st = plan(lc, be, warp_split, block_ratio, *F);
  if (st) {
    delete F;
    return st;
  }
  cudaError_t e = cudaMalloc(&F->P.work, sizeof(BeWork));
  if (e == cudaSuccess) e = cudaMemset(F->P.work, 0, sizeof(BeWork));
  if (e != cudaSuccess) {
    delete F;
    return cuda_fail("workspace", e);
  }
  if ((st = alloc_lc_workspace(*F))) {
    cudaFree(F->P.work);
    delete F;
    return st;
  }
  *out = F;
  return TACKER_OK;
}

tacker_status tacker_fused_destroy(tacker_fused_t f) {
  if (!f) return TACKER_OK;
  if (f->P.work) cudaFree(f->P.work);
  if (f->P.lc.part) cudaFree(f->P.lc.part);
  delete f;
  return TACKER_OK;
}

tacker_status tacker_fused_info(tacker_fused_t f, tacker_fused_info_t *o) {
  if (!f || !o) return set_error("null argument"), TACKER_EINVAL;
  memset(o, 0, sizeof *o);
  o->grid = f->grid;
  o->block_threads = f->block;
  o->smem_bytes = f->smem;
  o->lc_warps = f->P.lc_warps;
  o->be_warps = f->warp_split;
  o->be_vblocks_per_cta = f->P.be_vb_per_cta;
  o->lc_tile_m = kBM;
  o->lc_tile_n = f->BN;
  o->lc_tile_k = kBK;
  o->lc_stages = f->P.stages;
  o->lc_acc_stages = f->P.acc_stages;
  o->tmem_cols = (int32_t)f->P.tmem_cols;
  o->lc_tiles = f->P.lc.num_tiles;
  o->lc_splits = f->P.lc.splits;
  const LcParams &L = f->P.lc;
  const bool implicit = L.kind == TACKER_LC_CONV_F16 && !L.conv_direct_gemm;
  o->lc_mode = !implicit ? TACKER_LC_MODE_GEMM
               : L.conv_s2c8 ? TACKER_LC_MODE_CONV_S2C8
               : L.conv_halo ? TACKER_LC_MODE_CONV_HALO
               : L.conv_c8 ? TACKER_LC_MODE_CONV_C8
               : L.conv_im2col ? TACKER_LC_MODE_CONV_IM2COL : TACKER_LC_MODE_CONV_TILED;
  o->lc_tma_store = L.tma_store;
  o->be_blocks = f->P.be_blocks;
  o->be_smem_per_vblock = (int32_t)f->P.be_smem_per_vb;
  o->regs_per_thread = f->regs;
  return TACKER_OK;
}

tacker_status tacker_fused_keys(tacker_fused_t f, char *lc_key, char *be_key, char *pair_key, size_t n) {
  if (!f || n == 0) return set_error("null argument"), TACKER_EINVAL;
  if (lc_key) snprintf(lc_key, n, "%s", f->lc_key.c_str());
  if (be_key) snprintf(be_key, n, "%s", f->be_key.c_str());
  if (pair_key) snprintf(pair_key, n, "%s", f->pair_key.c_str());
  return TACKER_OK;
}

tacker_status tacker_fused_rebind(tacker_fused_t f, const tacker_lc_desc *lc, const tacker_be_desc *be) {
  if (!f) return set_error("null handle"), TACKER_EINVAL;
  tacker_fused_s tmp;
  tacker_lc_desc l = lc ? *lc : f->lc;
  tacker_be_desc b = be ? *be : f->be;
  tacker_ratio r{(uint8_t)f->P.acc_stages, (uint8_t)f->P.be_vb_per_cta};
  l.tile_n = f->BN;
  tacker_status st = plan(&l, f->be.kind ? &b : nullptr, f->warp_split, r, tmp);
  if (st) return st;
  if (tmp.fn != f->fn || tmp.P.stages != f->P.stages || tmp.smem != f->smem)
    return set_error("rebind changes the plan; call tacker_fuse"), TACKER_EINVAL;
  if (tmp.P.lc.splits != f->P.lc.splits || tmp.P.lc.num_units != f->P.lc.num_units)
    return set_error("rebind changes the split-K plan; call tacker_fuse"), TACKER_EINVAL;
  BeWork *w = f->P.work;
  float *part = f->P.lc.part;
  uint32_t *cnt = f->P.lc.cnt;
  *f = tmp;
  f->P.work = w;
  f->P.lc.part = part;
  f->P.lc.cnt = cnt;
  return TACKER_OK;
}

tacker_status tacker_launch_fused(tacker_fused_t f, tacker_stream_t stream) {
  if (!f) return set_error("null handle"), TACKER_EINVAL;
  return launch_plan(*f, reinterpret_cast<cudaStream_t>(stream));
}

tacker_status tacker_launch_fused_slice(tacker_fused_t f, int64_t block_offset, int64_t n_blocks, tacker_stream_t stream) {
  if (!f) return set_error("null handle"), TACKER_EINVAL;
  if (!f->be.kind) return set_error("handle has no BE part"), TACKER_EINVAL;
  if (f->be.kind == TACKER_BE_JDS_SCAN && (block_offset || n_blocks != f->be_full))
    return set_error("jds_scan runs as one block and cannot be sliced"), TACKER_EUNSUPPORTED;
  if (block_offset < 0 || n_blocks < 0 || block_offset > f->be_full || n_blocks > f->be_full - block_offset)
    return set_error("PTB slice [%lld, +%lld) outside [0, %lld]", (long long)block_offset, (long long)n_blocks,
                     (long long)f->be_full),
           TACKER_EINVAL;
  FusedParams P = f->P;    // by value: the handle itself is not modified (launchable from any thread)
  P.be_offset = block_offset;
  P.be_blocks = n_blocks;
  P.be.block_offset = (int32_t)block_offset;
  P.be.orig_blocks = (int32_t)n_blocks;
  return launch_params(*f, P, reinterpret_cast<cudaStream_t>(stream));
}

tacker_status tacker_launch_original(const tacker_lc_desc *lc, const tacker_be_desc *be, tacker_stream_t stream) {
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  tacker_status st;
  if (lc && lc->kind != TACKER_LC_NONE) {
    // LC-only plans (tensor maps, smem attribute) are cached by descriptor bytes: the manager
    // re-launches the same LC kernels every query.
    // Entries are never evicted: a plan (and its split-K workspace) may still be in use by a
    // launch in flight, and a service has a bounded set of LC descriptors.
    static std::mutex mu;
    static std::unordered_map<std::string, std::unique_ptr<tacker_fused_s>> cache;
    const std::string key(reinterpret_cast<const char *>(lc), sizeof *lc);
    tacker_fused_s *F = nullptr;
    {
      std::lock_guard<std::mutex> g(mu);
      auto it = cache.find(key);
      if (it != cache.end()) F = it->second.get();
    }
    if (!F) {
      auto P = std::make_unique<tacker_fused_s>();
      if ((st = plan(lc, nullptr, 0, tacker_ratio{0, 0}, *P))) return st;
      P->P.work = nullptr;
      if ((st = alloc_lc_workspace(*P))) return st;
      std::lock_guard<std::mutex> g(mu);
      auto it = cache.find(key);   // another thread may have planned the same descriptor meanwhile
      if (it != cache.end()) {
        if (P->P.lc.part) cudaFree(P->P.lc.part);
        F = it->second.get();
      } else {
        F = (cache[key] = std::move(P)).get();
      }
    }
    if ((st = launch_plan(*F, s))) return st;
  }
  if (be && be->kind != TACKER_BE_NONE) {
    int64_t blocks;
    if ((st = validate_be(*be, &blocks))) return st;
    if (blocks == 0) return TACKER_OK;
    BeFn fn = pick_be_original(be->kind);
    const int smem = (int)be_smem_bytes(be->kind);
    if (smem > 48 * 1024 && (st = set_smem_attr(reinterpret_cast<const void *>(fn), smem))) return st;
    BeOrigParams op;
    op.d = *be;
    if ((st = encode_be_tmap(*be, &op.tmap))) return st;
    if (blocks > 0x7fffffffLL) return set_error("too many blocks"), TACKER_EUNSUPPORTED;
    cudaError_t e = launch_ex(fn, dim3((unsigned)blocks), dim3(128), smem, s, op, true);
    if (e != cudaSuccess) return cuda_fail("launch be_original_kernel", e);
  }
  return TACKER_OK;
}

}  // extern "C"

// accessors used by the predictor / manager translation units
namespace tkrt {
// BE-kernel blacklist (NEXT-1): op 1 add, 0 remove, -1 query, 2 clear; returns membership
bool blacklist_op(const std::string &be_key, int op) {
  static std::mutex mu;
  static std::set<std::string> listed;
  std::lock_guard<std::mutex> g(mu);
  if (op == 2) {
    listed.clear();
    return false;
  }
  if (op == 1) listed.insert(be_key);
  if (op == 0) listed.erase(be_key);
  return listed.count(be_key) != 0;
}

const std::string &fused_lc_key(tacker_fused_t f) { return f->lc_key; }
const std::string &fused_be_key(tacker_fused_t f) { return f->be_key; }
const std::string &fused_pair_key(tacker_fused_t f) { return f->pair_key; }
int64_t fused_lc_tiles(tacker_fused_t f) { return f->P.lc.num_tiles; }
int64_t fused_be_blocks(tacker_fused_t f) { return f->P.be_blocks; }

// Model-store keys without building a handle (no GPU needed): the manager's predictions.
bool make_keys(const tacker_lc_desc *lc, const tacker_be_desc *be, int warp_split, std::string *lk, std::string *bk,
               std::string *pk) {
  if (lc) {
    LcParams L;
    if (lc_view(*lc, L) != TACKER_OK) return false;
    const int BN = pick_tile_n(*lc, L);
    *lk = lc_key_of(*lc, L, BN);
  }
  if (be) *bk = be_key_of(*be);
  if (lc && be) {
    char b[512];
    snprintf(b, sizeof b, "pair:%s|%s|ws%d", lk->c_str(), bk->c_str(), warp_split);
    *pk = b;
  }
  return true;
}
}  // namespace tkrt
