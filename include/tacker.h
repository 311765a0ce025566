/*
 * tacker.h — C ABI of the B200-native Tacker hot path (libtacker.so).
 *
 * Tacker (Zhao et al., HPCA'22; /root/reference/PAPER.md, cited P:a-b) co-runs a latency-
 * critical (LC) tensor-core kernel and a best-effort (BE) CUDA-core kernel inside ONE fused
 * kernel so both core types are busy at once (§III-B, §V), predicts the
 * fused duration with a two-stage linear model (§VI) and decides at run time,
 * from each LC query's QoS headroom, whether to launch the fused or the original kernels
 * (§VII).  This header is the boundary: every call below is implemented by
 * hand-written sm_100a CUDA (tcgen05/TMEM/TMA for LC, CUDA-core bodies for BE) and C++ host
 * code; there is no CPU fallback.
 *
 * Conventions (all calls):
 *   Errors     Every call returns tacker_status; nothing throws across the ABI.  The
 *              thread-local message of the last failure is tacker_last_error().  CUDA runtime
 *              failures map to TACKER_ECUDA.
 *   Memory     Pointers inside descriptors are DEVICE pointers owned by the caller (e.g. torch
 *              tensors).  The library never allocates or frees them.  Descriptors are copied at
 *              tacker_fuse(); buffers must outlive every launch of the handle.  Handles own
 *              their own small device workspace.
 *   Streams    tacker_stream_t is a cudaStream_t (NULL = legacy default stream).  Launches are
 *              asynchronous on that stream; predictor calls never touch the GPU.
 *   Threads    Fused handles are immutable after tacker_fuse() and may be launched from any
 *              thread, but a handle owns device workspaces (the BE ticket counters, split-K
 *              partials and counters) that reset themselves at the end of each launch: at most
 *              one launch of a handle may be in flight at a time (launch it on one stream; fuse
 *              a second handle for concurrent streams).  tacker_launch_original's internal LC
 *              plans follow the same rule per LC descriptor.  A manager is single-threaded.
 *              The model store is mutex-protected.
 */
#ifndef TACKER_H
#define TACKER_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *tacker_stream_t;

typedef enum {
  TACKER_OK = 0,
  TACKER_EINVAL = -1,        /* bad argument (null, negative size, inconsistent shape) */
  TACKER_ERESOURCE = -2,     /* fused budget exceeds one SM: do not fuse */
  TACKER_EUNSUPPORTED = -3,  /* shape/alignment/kind the kernels do not implement */
  TACKER_ECUDA = -4,         /* CUDA runtime / driver error */
  TACKER_ENOMODEL = -5,      /* predictor has no fitted model for this key */
  TACKER_ENOMEM = -6
} tacker_status;

const char *tacker_last_error(void);
/* Library version string and the SM count of the current device (0 without a GPU). */
const char *tacker_version(void);
int tacker_device_sm_count(void);

/* ======================================================================== LC descriptors
 * The LC part is the TC kernel "Kt" of the paper: an fp16 GEMM on tensor cores,
 * or a convolution lowered to GEMM (§VIII-H, here as an implicit GEMM).
 *
 * GEMM   D[M,N] = A[M,K] . B[N,K]^T, A and B fp16 row-major with K contiguous ("K-major"),
 *        fp32 accumulation in TMEM.  Constraints: K % 8 == 0 and N % 8 == 0 (16-byte TMA row
 *        pitch), M >= 1 arbitrary (masked epilogue).  D row-major [M,N], fp32 or fp16 (RNE).
 * CONV   out[n,p,q,k] = sum_{c,r,s} x[n, p*stride-pad+r, q*stride-pad+s, c] * w[k,r,s,c], x = 0
 *        outside the image; x NHWC fp16 (A), w KRSC fp16 (B), out NHWC (D).  As a GEMM:
 *        M = n*p*q, N = k, K = c*r*s.  Constraints: c % 64 == 0 or (r == s == 1 and c % 8 == 0)
 *        or c == 8 (conv1 padded); k % 8 == 0.
 * Epilogue (both): D = act(acc + bias[j] + residual[i,j]) with optional fp32 bias [N], fp16
 *        residual with D's layout, ReLU.  D, bias and residual 16-byte aligned (EINVAL).
 */
typedef enum { TACKER_LC_NONE = 0, TACKER_LC_GEMM_F16 = 1, TACKER_LC_CONV_F16 = 2 } tacker_lc_kind;
enum { TACKER_F32 = 0, TACKER_F16 = 1 };
enum { TACKER_EPI_BIAS = 1, TACKER_EPI_RELU = 2, TACKER_EPI_RESIDUAL = 4,
       /* B (weights) is not written by any kernel on the stream: a launch may fetch its first
        * B k-blocks before waiting for the stream predecessor (programmatic dependent launch) */
       TACKER_LC_B_CONST = 8,
       /* never split K (by default a GEMM with <= #SMs/2 tiles and >= 4 k-blocks is split
        * into <= #SMs units with an in-kernel deterministic fixup, see tacker_fused_info) */
       TACKER_LC_NO_SPLIT = 16 };

typedef struct {
  int32_t kind;                       /* tacker_lc_kind */
  int32_t M, N, K;                    /* GEMM shape (ignored for CONV: derived) */
  int32_t n, h, w, c, k, r, s, stride, pad; /* CONV shape */
  const void *A;                      /* GEMM A [M,K] fp16 | CONV x NHWC fp16 */
  const void *B;                      /* GEMM B [N,K] fp16 | CONV w KRSC fp16 */
  void *D;                            /* output, d_dtype */
  const float *bias;                  /* [N] fp32 or NULL (requires TACKER_EPI_BIAS) */
  const void *residual;               /* fp16 like D, or NULL (requires TACKER_EPI_RESIDUAL) */
  int32_t d_dtype;                    /* TACKER_F32 | TACKER_F16 */
  int32_t epi_flags;                  /* TACKER_EPI_* */
  int32_t tile_n;                     /* LC tile N: 0 = auto, else 64 | 128 | 256 */
} tacker_lc_desc;

/* ======================================================================== BE descriptors
 * The BE part is a CUDA-core kernel (Parboil-style, Table II).  Each kind defines
 * its "original block" (one virtual block = 128 threads = 4 warps); `orig_blocks` is the
 * PTB runtime argument of Fig. 7: 0 = the whole problem, else only blocks
 * [0, orig_blocks) run (must not exceed the whole-problem count).  Bodies use fixed
 * per-element arithmetic order, so a fused launch is bit-identical to the original one.
 * `block_offset` shifts the PTB range to [block_offset, block_offset + orig_blocks) (orig_blocks
 * 0 = to the end): a launch runs a SLICE of the original kernel.  Running the slices of a
 * partition of [0, blocks) in order on one stream is bit-identical to the whole kernel for every
 * kind whose blocks write disjoint outputs or commutative integer counts (all kinds except
 * TACKER_BE_JDS_SCAN, whose single block reads every count).  The manager sizes the BE slice of
 * a fused launch to the pair's opportune load ratio (DESIGN.md §2 reading 13).
 */
typedef enum {
  TACKER_BE_NONE = 0,
  TACKER_BE_SGEMM = 1,        /* C = alpha A.B + beta C; block = 64x64 tile of C          */
  TACKER_BE_STENCIL = 2,      /* 7-point Jacobi sweep; block = 32x4 columns, all z        */
  TACKER_BE_MRIQ_PHIMAG = 3,  /* phiMag = phiR^2 + phiI^2; block = 512 k                   */
  TACKER_BE_MRIQ_Q = 4,       /* Qr/Qi += sum_k phiMag cos/sin(2pi k.x); block = 32 voxels x 4 k-lanes */
  TACKER_BE_CUTCP = 5,        /* cutoff Coulomb potential; block = 4x4x8 lattice points    */
  TACKER_BE_LBM = 6,          /* D3Q19 BGK push step; block = 128 cells along x            */
  TACKER_BE_SPMV_JDS = 7,     /* y[perm[i]] = sum_d val*x[col]; block = 128 rows           */
  TACKER_BE_HISTO = 8,        /* count[in[i]] += 1 (u32); block = 8192 inputs              */
  TACKER_BE_BFS_EXPAND = 9,   /* Rodinia BFS kernel 1; block = 128 nodes                   */
  TACKER_BE_BFS_COMMIT = 10,  /* Rodinia BFS kernel 2; block = 128 nodes                   */
  TACKER_BE_FMA_BURN = 11,    /* register-only FMA chains (Kc, §III-B); block = 128 thr.   */
  TACKER_BE_IM2COL = 12,      /* LC CUDA-core helper: explicit im2col (cudnnIm2col, §VIII-H
                                 P:3350-3381) NHWC fp16 -> [M, Kpad] fp16; block = 1024x8 el. */
  TACKER_BE_CUTCP_BIN = 13,   /* cutcp atom binning (deterministic, index order); block = 128 bins */
  TACKER_BE_COPY = 14,        /* byte copy, e.g. a query's H2D/D2H through host-mapped pinned
                                 memory (UVA); block = 16 KiB */
  /* CSR -> JDS (spmv's input format) as a stable counting sort by row length, descending,
   * ties by row index: four kernels run in this order (all deterministic, integer-exact). */
  TACKER_BE_JDS_COUNT = 15,   /* per 1024-row block: row-length counts; block = 1024 rows */
  TACKER_BE_JDS_SCAN = 16,    /* prefix over blocks per length, start offsets, jds_ptr; 1 block */
  TACKER_BE_JDS_PERM = 17,    /* perm / row_len placement; block = 1024 rows */
  TACKER_BE_JDS_FILL = 18,    /* column / value scatter, diagonal-major; block = 128 JDS rows */
  /* NEXT-3: the remaining Parboil BE apps of Table II */
  TACKER_BE_MRIFHD_RHOPHI = 19, /* mri-fhd ComputeRhoPhi: rho*phi = conj(phi) d; block = 512 k      */
  TACKER_BE_MRIFHD_FH = 20,   /* mri-fhd ComputeFH: F^H d over one k chunk; block = 32 voxels x 4 k-lanes */
  TACKER_BE_CP = 21,          /* cp direct Coulomb summation on one lattice slice; block = 128x4 points */
  TACKER_BE_FFT_TWIDDLE = 22, /* fft plan: twiddle table w[m] = exp(-2 pi i m / n); block = 128 entries */
  TACKER_BE_FFT = 23,         /* batched forward complex DFT, length n <= 1024; block = 2 transforms */
  TACKER_BE_TPACF = 24,       /* angular correlation histogram; block = 128 points of a      */
  TACKER_BE_KIND_COUNT = 25
} tacker_be_kind;

typedef struct { int32_t M, N, K; float alpha, beta; const float *A, *B; float *C; } tacker_be_sgemm;
typedef struct { int32_t nx, ny, nz; float c0, c1; const float *A0; float *Anext; } tacker_be_stencil;
typedef struct { int32_t numK; const float *phiR, *phiI; float *phiMag; } tacker_be_mriq_phimag;
typedef struct { int32_t numX, numK; const float *x, *y, *z, *kx, *ky, *kz, *phiMag; float *Qr, *Qi; } tacker_be_mriq_q;
/* mri-fhd (Parboil; Table II, not defined in the paper: DESIGN.md §2 reading 14).
 * RhoPhi: rRhoPhi[k] = phiR dR + phiI dI, iRhoPhi[k] = phiR dI - phiI dR (all fp32 [numK]).
 * FH:     arg = 2pi (kx x + ky y + kz z);
 *         rFhD[v] += sum_k rRhoPhi cos(arg) - iRhoPhi sin(arg),
 *         iFhD[v] += sum_k iRhoPhi cos(arg) + rRhoPhi sin(arg)   (fp32 [numX], accumulated).
 * Same thread mapping, k staging and fixed per-voxel order as TACKER_BE_MRIQ_Q. */
typedef struct { int32_t numK; const float *phiR, *phiI, *dR, *dI; float *rRhoPhi, *iRhoPhi; } tacker_be_mrifhd_rhophi;
typedef struct { int32_t numX, numK; const float *x, *y, *z, *kx, *ky, *kz, *rRhoPhi, *iRhoPhi; float *rFhD, *iFhD; } tacker_be_mrifhd_fh;
/* cp (Parboil; Table II; reading 14): direct Coulomb summation on one lattice slice,
 *   V[j*nx + i] += sum_a q_a * rsqrt((i h - x_a)^2 + (j h - y_a)^2 + (z - z_a)^2)
 * atoms float4 (x, y, z, q) [natoms]; V fp32 [ny][nx] accumulated (one launch per atom chunk, as
 * Parboil's constant-memory chunks).  An atom ON a lattice point gives inf (caller's concern). */
typedef struct { int32_t natoms, nx, ny; float h, z; const float *atoms; float *V; } tacker_be_cp;
/* fft (Parboil; Fig. 10's GEMM-fft pair P:1417-1419; reading 15): y[b, k] = sum_j x[b, j]
 * exp(-2 pi i j k / n), b < batch, complex fp32 interleaved (re, im) [batch][n][2], out of place,
 * x, y 16-byte aligned; n a power of two in [2, 1024].  twiddle [n][2] fp32 is written by
 * TACKER_BE_FFT_TWIDDLE (w[m] = (cos, -sin)(2 pi m / n), accurate sincospi) and read by
 * TACKER_BE_FFT (Stockham radix-16/8/4/2; first pass from and last pass to global memory). */
typedef struct { int32_t n, batch; float *twiddle; const float *x; float *y; } tacker_be_fft;
/* tpacf (Parboil; reading 16): count[bin(a_i . b_j)] += 1 over all (i, j) (self_pairs = 0) or
 * over i < j with b == a (self_pairs = 1); bin(d) = #{k : d < edges[k]}, edges strictly
 * decreasing fp32 cosines, nedges <= 31; d = ((ax bx + ay by) + az bz) in fp32 without FMA;
 * a, b unit vectors fp32 [n][3]; count u32 [nedges + 1], accumulated. */
typedef struct { int32_t na, nb, nedges, self_pairs; const float *a, *b, *edges; uint32_t *count; } tacker_be_tpacf;
/* cutcp: V[p] = sum_{a: d^2 < cutoff^2} q_a / d * (1 - d^2/cutoff^2)^2, V[p] = 0 if any atom has
 * d < excl.  Atoms come binned (TACKER_BE_CUTCP_BIN): bin side = 8*h, so one block (8x8x8
 * lattice points) is one bin and its atoms within the cutoff lie in the bins within
 * ceil(cutoff / bin side) bins in each direction; bins are visited and atoms summed in a fixed
 * order (bit-identical fused vs original). */
typedef struct {
  int32_t nx, ny, nz;        /* lattice points per axis, point (i,j,k) at h*(i,j,k) */
  float h, cutoff, excl;     /* spacing, cutoff radius, exclusion radius (Angstrom) */
  int32_t bdim_x, bdim_y, bdim_z; /* atom bin grid: bdim_* = ceil(n* / 8) */
  float bin_size;            /* must equal 8*h */
  int32_t bin_depth;         /* atom slots per bin; unused slots have q == 0 and far coords */
  const float *bins;         /* float4 (x,y,z,q) [bdim_z][bdim_y][bdim_x][bin_depth] */
  const int32_t *count;      /* atoms per bin (from the binning kernel); only these slots are read */
  float *V;                  /* [nz][ny][nx] */
} tacker_be_cutcp;
/* Binning: bin b = (floor(z/bs)*bdim_y + floor(y/bs))*bdim_x + floor(x/bs) (clamped into the grid)
 * receives its atoms in atom-index order; unused slots get (1e30,1e30,1e30,0); count[b] = atoms
 * in bin b, *overflow set to 1 if any bin holds more than bin_depth atoms (the caller re-bins
 * with a larger depth; no atom is dropped silently). */
typedef struct {
  int32_t natoms;
  const float *atoms;        /* float4 (x,y,z,q) [natoms] */
  int32_t bdim_x, bdim_y, bdim_z, bin_depth;
  float bin_size;
  float *bins;               /* out: float4 [bdim_z*bdim_y*bdim_x*bin_depth] */
  int32_t *count;            /* out: [bins] */
  int32_t *overflow;         /* out: flag */
} tacker_be_cutcp_bin;
typedef struct { int32_t nx, ny, nz; const float *src; float *dst; const uint32_t *flags; } tacker_be_lbm;
typedef struct { int32_t rows; const int32_t *perm, *row_len, *jds_ptr, *col; const float *val, *x; float *y; } tacker_be_spmv;
typedef struct { int32_t n, nbins; const uint32_t *in; uint32_t *count; } tacker_be_histo;
typedef struct { int32_t V; const int32_t *row_ptr, *col; int32_t *level; uint8_t *mask; const uint8_t *visited; uint8_t *upd; } tacker_be_bfs_expand;
typedef struct { int32_t V; uint8_t *mask, *visited, *upd; int32_t *over; } tacker_be_bfs_commit;
typedef struct { int32_t n_threads, iters; float a; float b; float *out; } tacker_be_fma_burn;
/* out[m, kk] = x[n, p*stride-pad+r, q*stride-pad+s, c] with m = (n*P+p)*Q+q, kk = (r*S+s)*C+c,
 * 0 outside the image and for kk >= R*S*C (row padded to Kpad, a multiple of 8). */
typedef struct {
  int32_t n, h, w, c, r, s, stride, pad, Kpad;
  const void *x;   /* fp16 NHWC */
  void *out;       /* fp16 [n*P*Q, Kpad] */
} tacker_be_im2col;
/* dst[0:bytes) = src[0:bytes); both 16-byte aligned, bytes % 16 == 0; either side may be pinned
 * host memory (device-accessible through UVA). */
typedef struct { int64_t bytes; const void *src; void *dst; } tacker_be_copy;
/* JDS build (one struct for the four kinds).  Outputs follow oracle/be.py jds_build: perm[i] =
 * i-th row by (length desc, index asc); row_len[i] = its length; jds_ptr[d] = start of jagged
 * diagonal d (jds_ptr[0] = 0, jds_ptr[d+1]-jds_ptr[d] = #rows longer than d), sized max_len+1;
 * element (d, i) of the JDS arrays is the d-th nonzero of row perm[i].  *overflow = 1 if a row
 * is longer than max_len (outputs then invalid). */
typedef struct {
  int32_t rows, max_len;
  const int32_t *row_ptr, *col;   /* CSR input, columns sorted within a row */
  const float *val;
  int32_t *blk_count;             /* workspace [ceil(rows/1024)][max_len+1] */
  int32_t *start;                 /* workspace [max_len+2] */
  int32_t *perm, *row_len, *jds_ptr, *jds_col;
  float *jds_val;
  int32_t *overflow;
} tacker_be_jds;

typedef struct {
  int32_t kind;              /* tacker_be_kind */
  int32_t orig_blocks;       /* PTB original block count (0 = whole problem / rest) */
  int32_t block_offset;      /* first original block of this launch (0 = from the start) */
  union {
    tacker_be_sgemm sgemm;
    tacker_be_stencil stencil;
    tacker_be_mriq_phimag mriq_phimag;
    tacker_be_mriq_q mriq_q;
    tacker_be_cutcp cutcp;
    tacker_be_lbm lbm;
    tacker_be_spmv spmv;
    tacker_be_histo histo;
    tacker_be_bfs_expand bfs_expand;
    tacker_be_bfs_commit bfs_commit;
    tacker_be_fma_burn fma_burn;
    tacker_be_im2col im2col;
    tacker_be_cutcp_bin cutcp_bin;
    tacker_be_copy copy;
    tacker_be_jds jds;
    tacker_be_mrifhd_rhophi mrifhd_rhophi;
    tacker_be_mrifhd_fh mrifhd_fh;
    tacker_be_cp cp;
    tacker_be_fft fft;
    tacker_be_tpacf tpacf;
    uint8_t _pad[128];
  } p;
} tacker_be_desc;

/* Whole-problem block counts ("number of blocks in non-PTB mode", §VI-C). */
tacker_status tacker_be_num_blocks(const tacker_be_desc *be, int64_t *out);
tacker_status tacker_lc_num_tiles(const tacker_lc_desc *lc, int32_t tile_n, int64_t *out);
/* Per-kernel LR features (§VI-C) that follow the hardware's cost better than a block
 * count.  LC: waves = ceil(work units / CTAs) of the LC-only persistent launch (tiles of one wave run
 * concurrently: the time steps with the wave count, not the tile count).  BE: the algorithmic work
 * of the first n original blocks -- spmv JDS: 8 nnz + 16 rows bytes of those rows (rows sorted by
 * length, the first blocks are the heaviest); cutcp: (lattice point, neighbour-bin atom) pairs of
 * those bins; every other kind: n.  Reads small device arrays (row lengths, bin counts) and
 * synchronises: calibration only. */
tacker_status tacker_lc_num_waves(const tacker_lc_desc *lc, int32_t tile_n, int64_t *out);
tacker_status tacker_be_prefix_work(const tacker_be_desc *be, int64_t n_blocks, double *work);

/* ======================================================================== fusion (a1)
 * tacker_fuse: admission + resource split of one fused kernel (§V-B/C P:1117-1309,
 * §VIII-I).  One fused CTA per SM, persistent (PTB, Fig. 7):
 *   warps [0,6)            LC: warp 0 TMA producer, warp 1 single-thread tcgen05.mma issuer
 *                          (+ TMEM owner), warps 2..5 TMEM->register epilogue
 *   warps [6, 6+warp_split) BE: block_ratio.be virtual blocks of 4 warps, each with its own
 *                          named barrier (bar.sync 1+j, 128; Fig. 9) and SMEM slice
 * warp_split  BE warps per CTA, a multiple of 4 in [4, 24] (0 = LC only; requires be NULL/NONE)
 * block_ratio.lc  LC accumulator pipelines per CTA (TMEM stages, 1 or 2; 0 = auto)
 * block_ratio.be  BE virtual blocks per CTA = warp_split/4 (0 = auto)
 * LC is budgeted first (SMEM ring stages, TMEM columns), BE gets the rest (TC-first, §V-C).
 * Returns TACKER_ERESOURCE when the aggregate does not fit (232,448 B SMEM, 512 TMEM columns,
 * 64K registers, 32 warps, 16 barriers).  The handle owns encoded TMA tensor maps.
 */
typedef struct { uint8_t lc, be; } tacker_ratio;
typedef struct tacker_fused_s *tacker_fused_t;

tacker_status tacker_fuse(const tacker_lc_desc *lc, const tacker_be_desc *be, int32_t warp_split,
                          tacker_ratio block_ratio, tacker_fused_t *out);
tacker_status tacker_fused_destroy(tacker_fused_t f);

typedef struct {
  int32_t grid, block_threads, smem_bytes;
  int32_t lc_warps, be_warps, be_vblocks_per_cta;
  int32_t lc_tile_m, lc_tile_n, lc_tile_k, lc_stages, lc_acc_stages, tmem_cols;
  int64_t lc_tiles, be_blocks;
  int32_t be_smem_per_vblock, regs_per_thread;
  int32_t lc_splits;         /* split-K factor of the LC part (1 = none) */
  int32_t lc_mode;           /* TACKER_LC_MODE_*: how the LC operands are tiled and loaded */
  int32_t lc_tma_store;      /* 1: TMA-store epilogue (LC-only fp16 plans) */
} tacker_fused_info_t;
enum { TACKER_LC_MODE_GEMM = 0, TACKER_LC_MODE_CONV_IM2COL = 1, TACKER_LC_MODE_CONV_TILED = 2,
       TACKER_LC_MODE_CONV_C8 = 3, TACKER_LC_MODE_CONV_HALO = 4, TACKER_LC_MODE_CONV_S2C8 = 5 };
tacker_status tacker_fused_info(tacker_fused_t f, tacker_fused_info_t *out);
/* Model-store keys of the handle's LC kernel, BE kernel and fused pair (for the predictor). */
tacker_status tacker_fused_keys(tacker_fused_t f, char *lc_key, char *be_key, char *pair_key, size_t buflen);

/* Retarget an existing handle to new buffers/PTB block count of the SAME shape class (no
 * re-planning; used by the manager to reuse a plan).  NULL leaves that part unchanged. */
tacker_status tacker_fused_rebind(tacker_fused_t f, const tacker_lc_desc *lc, const tacker_be_desc *be);

/* ======================================================================== launches (a2-a8)
 * tacker_launch_fused    one fused kernel: LC tiles and BE blocks co-run in every CTA.
 * tacker_launch_original the original kernels one after the other on the same stream (LC then
 *                        BE); either may be NULL.  LC original = the same LC device code in a
 *                        persistent LC-only grid; BE original = the same BE body in a
 *                        non-persistent grid of orig_blocks CTAs of 128 threads (Fig. 7 "CD_kernel").
 */
tacker_status tacker_launch_fused(tacker_fused_t f, tacker_stream_t stream);
tacker_status tacker_launch_original(const tacker_lc_desc *lc, const tacker_be_desc *be,
                                     tacker_stream_t stream);
/* Programmatic dependent launch (default mode 2): every launch of this library may begin its
 * prologue (CTA scheduling, barrier / TMEM setup, TACKER_LC_B_CONST weight fetches) while the
 * previous kernel on the stream is still running; each kernel waits for its predecessor
 * (griddepcontrol.wait) before touching any other global memory, so stream order semantics are
 * unchanged.  0 disables it (plain stream serialization); 1 = every launch; 2 (default) = every
 * launch except original BE kernels (their non-persistent grid is then distributed over an
 * idle GPU instead of being parked behind the running kernel).  Process-wide.  EINVAL else. */
tacker_status tacker_set_launch_overlap(int32_t enable);
/* NEXT-1 fusion selection (§V-C): "create all possible fused kernels for two kernels,
 * measure these candidates' performance and two kernels' sequential performance, and choose the
 * best one among them.  If the sequential case shows the best performance, we do not fuse the two
 * kernels."  Candidates are the BE warp splits in splits[0..n) (a split the budget rejects is
 * skipped, fused_ms = NAN); each is timed over `reps` back-to-back launches on stream s (CUDA
 * events, mean), after one warm-up, as is the sequential pair of original launches.  Out:
 * *best_ws = the fastest split, or 0 when sequential is fastest -- the BE kernel is then also
 * blacklisted ("if a CD kernel could not benefit from kernel fusion with one TC
 * kernel, this CD kernel would not be considered for fusion"); *best_ms its time; *seq_ms;
 * fused_ms[i] (nullable) per candidate.  Synchronises the stream (calibration, not the hot path).
 * Buffers: the descriptors' device memory is written by the timed launches. */
tacker_status tacker_select_fusion(const tacker_lc_desc *lc, const tacker_be_desc *be, const int32_t *splits,
                                   int32_t n_splits, int32_t reps, tacker_stream_t s, int32_t *best_ws,
                                   double *best_ms, double *seq_ms, double *fused_ms);
/* The BE-kernel blacklist (keyed by the BE model-store key, see tacker_fused_keys): op 1 adds, 0
 * removes, -1 only queries; *listed (nullable) = membership after the op.  The manager never fuses
 * a blacklisted BE kernel (it is still reordered / run on an idle GPU). */
tacker_status tacker_blacklist(const char *be_key, int32_t op, int32_t *listed);
tacker_status tacker_blacklist_clear(void);

/* Diagnostics: copies the LC role clock64 stamps recorded by plans built with TACKER_LC_DBG bit 3
 * ([160 CTAs][5 events][16 work units], see fused.cuh) into out (>= 12800 slots).  The stamps (and
 * the TACKER_LC_DBG skip switches) exist only in a library built with -DTK_LC_DIAG=1; production
 * builds record nothing (zeros). */
tacker_status tacker_debug_lc_timestamps(uint64_t *out, int64_t n);
/* Diagnostics: synchronises the device, copies the per-launch %globaltimer stamps (ns) recorded by
 * plans built with TACKER_LC_DBG bit 4 (value 16) in a library built with -DTK_LC_GT=1 (zeros
 * otherwise) into out ([256 launch slots][8], >= 2048 slots;
 * slot layout in fused.cuh g_lc_gt), clears them and the slot counter; *next_slot (nullable) = the
 * number of launches recorded since the last call (mod 256). */
tacker_status tacker_debug_lc_globaltimer(uint64_t *out, int64_t n, int32_t *next_slot);

/* One fused launch of handle f whose BE part runs only the PTB slice [block_offset,
 * block_offset + n_blocks) of the handle's BE kernel (the LC part is unchanged; n_blocks 0 = no
 * BE work).  The handle is not modified.  EINVAL if the slice leaves the whole-problem range. */
tacker_status tacker_launch_fused_slice(tacker_fused_t f, int64_t block_offset, int64_t n_blocks,
                                        tacker_stream_t stream);

/* ======================================================================== predictor (a9, a10)
 * Per-kernel LR (§VI-C): X = a * blocks + b, keyed by kernel class.
 * Two-stage fused model (Eqs. 1-6): r = X_cd / X_tc; T = X_tc * max(l1(r), l2(r)),
 * fitted from samples at r in {0.1, 0.2, 1.8, 1.9}, refit online when the error
 * exceeds 10%.  Keys are NUL-terminated strings (< 256 bytes).
 */
tacker_status tacker_model_add_sample(const char *key, double blocks, double ms);
tacker_status tacker_model_fit(const char *key, double *a_out, double *b_out);
tacker_status tacker_model_predict(const char *key, double blocks, double *ms_out);
tacker_status tacker_pair_add_sample(const char *key, double x_tc, double x_cd, double t_fused);
tacker_status tacker_pair_fit(const char *key, double coef_out[4] /* a1,b1,a2,b2; nullable */);
tacker_status tacker_pair_predict(const char *key, double x_tc, double x_cd, double *ms_out);
tacker_status tacker_pair_observe(const char *key, double x_tc, double x_cd, double t_meas, int32_t *refit_out);
tacker_status tacker_model_clear(void);
tacker_status tacker_model_save(const char *path);
tacker_status tacker_model_load(const char *path);
/* Fused duration of a handle: X_tc and X_cd from the kernel LRs of its LC/BE keys at the
 * handle's tile / block counts, then the pair's two-stage model. */
tacker_status tacker_predict_duration(tacker_fused_t f, double *ms_out);

/* ======================================================================== manager (a11)
 * QoS-aware kernel manager (§VII).  Rules: Eq. 9 headroom at the first issue of
 * the newest query; per TC kernel Eq. 8 admission over ready BE heads, max Tgain, then
 * Thr -= Tk_fuse - Ttc; otherwise original launch and reorder of ready BE heads with
 * Ttmp < Thr.  Only the newest query fuses/reorders (params.fuse_older relaxes it, reading 18);
 * CUDA-core LC kernels may fuse with BE tensor-core kernels (NEXT-2, reading 17); Baymax policy =
 * fusion disabled.
 * The manager keeps its own clock: in simulation mode (stream == NULL and simulate != 0)
 * kernels take their predicted duration; otherwise launches go to `stream` and completions
 * are observed with CUDA events.
 */
typedef enum { TACKER_POLICY_TACKER = 0, TACKER_POLICY_BAYMAX = 1 } tacker_policy;
typedef enum {
  TACKER_DEC_FUSED = 0, TACKER_DEC_ORIGINAL_LC = 1, TACKER_DEC_REORDER_BE = 2,
  TACKER_DEC_IDLE_BE = 3, TACKER_DEC_NOTHING = 4
} tacker_action;
#define TACKER_MAX_APPS 64
#define TACKER_MAX_REORDER 64

typedef struct {
  int32_t is_tc;             /* 1: tensor-core kernel (fusable as LC); 0: CUDA-core kernel */
  double t_pred_ms;          /* predicted standalone duration */
  tacker_lc_desc lc;         /* used when is_tc */
  tacker_be_desc cd;         /* used when !is_tc (an LC CUDA-core kernel: launched original, or
                                fused as the CUDA-core part with a BE tensor-core kernel) */
  int32_t warp_split;        /* !is_tc: CUDA-core warps of a reverse-fused launch (0 = 16) */
} tacker_lc_kernel;

typedef struct {
  int32_t n_kernels;
  const tacker_lc_kernel *kernels;   /* copied at submit */
} tacker_lc_query;

typedef struct {
  int32_t is_cd;             /* 1: CUDA-core kernel (fusable as BE) */
  double t_pred_ms;          /* predicted standalone duration of the whole kernel */
  tacker_be_desc be;
  int32_t warp_split;        /* fusion plan for this kernel (0 = library default 16) */
  /* PTB slicing (params.slice_be): the kernel's original blocks [be.block_offset,
   * be.block_offset + n_blocks) may run as several launches.  Per-kernel LR of a slice of n
   * blocks (§VI-C): X_cd(n) = t_floor_ms + t_block_ms * n.  n_blocks <= 1 or
   * t_block_ms <= 0: never sliced. */
  int32_t n_blocks;
  double t_block_ms, t_floor_ms;
  /* NEXT-2 reverse fusion ("LC and BE kernels are not limited to a specified type";
   * DNN-training BE apps, Table II): is_tc = 1 makes this BE kernel the tensor-core
   * GEMM / conv `tc` (is_cd must be 0).  The manager fuses it with an LC CUDA-core kernel under
   * the same Eq. 8 (LC and BE solo times swap roles in the predictor: X_tc = this kernel,
   * X_cd = the LC kernel); it is never sliced. */
  int32_t is_tc;
  tacker_lc_desc tc;
} tacker_be_kernel;

typedef struct {
  int32_t n_kernels;
  const tacker_be_kernel *kernels;   /* copied; the app cycles through them forever */
} tacker_be_app;

typedef struct {
  int32_t action;            /* tacker_action */
  int32_t query, lc_index;   /* LC kernel decided (-1 if none) */
  int32_t fused_app;         /* BE app fused with it (-1 if none); a reverse fusion (LC CUDA-core
                                kernel + BE tensor-core kernel) is FUSED with reverse = 1 */
  int32_t n_reorder;
  int32_t reorder_apps[TACKER_MAX_REORDER];
  double thr_ms;             /* headroom after the decision */
  double gain_ms;            /* Tgain of the fused pair */
  double t_start_ms, t_end_ms; /* manager clock: predicted (sim) or issue time (GPU) */
  int64_t fused_blocks;      /* BE blocks in the fused launch: a PTB slice, or -1 = the whole rest */
  int32_t reverse;           /* FUSED: 1 = LC CUDA-core kernel + BE tensor-core kernel (NEXT-2) */
} tacker_decision;

typedef struct {
  double direct_eps_ms;      /* Thr <= this at first issue -> launch the query directly (direct_rule) */
  double idle_cap_ms;        /* idle GPU: launch BE heads no longer than this (<=0: any) */
  int32_t max_inflight;      /* GPU mode: kernels allowed in flight on the stream (>=1) */
  int32_t simulate;          /* 1: no GPU, durations = predictions */
  /* Tacker policy, B200 reading 13: the BE part of a fused launch is the slice
   * of the head kernel's remaining blocks whose predicted X_cd puts the pair at its opportune
   * load ratio r* (the two-stage model's inflection), or at slice_ratio when > 0.
   * 0: whole BE kernels only (the paper's fusion unit). */
  int32_t slice_be;
  double slice_ratio;
  /* tacker_reorder_rule.  TACKER_REORDER_UNFUSED (0, default, the paper's rule P:2035-2043: "If
   * all the ready BE kernels may not be fused with the current kernel of Q", reorder the ready BE
   * heads with Ttmp < Thr; nothing after a fused launch); TACKER_REORDER_ALWAYS (B200 reading 6,
   * after every LC kernel, fused or not); TACKER_REORDER_NEVER (BE work only fused
   * or on an idle GPU). */
  int32_t reorder_rule;
  /* 1: never fuse an LC CUDA-core kernel with a BE tensor-core kernel (NEXT-2 off) */
  int32_t no_reverse_fusion;
  /* B200 reading 18 (off = the paper's rule: only the newest query fuses / reorders):
   * 1 = an older query may fuse / reorder too, within the smallest headroom of itself and of every
   * later active query (Eq. 9 of each at the current time), so no later query is pushed past the
   * QoS target either; that bound is lowered by older_margin_ms (a guard against the predictor's
   * error and the host running ahead of the GPU). */
  int32_t fuse_older;
  double older_margin_ms;
  /* tacker_direct_rule: "If the Thr of the new query is close to 0, Tacker directly launches all
   * the kernels".  TACKER_DIRECT_MIN_BE (0, default; SURVEY §8(c) c15 reading):
   * close to 0 = Thr <= max(direct_eps_ms, the smallest prediction of a ready BE head) at the
   * query's first issue; TACKER_DIRECT_EPS: Thr <= direct_eps_ms only. */
  int32_t direct_rule;
} tacker_manager_params;
enum { TACKER_REORDER_UNFUSED = 0, TACKER_REORDER_ALWAYS = 1, TACKER_REORDER_NEVER = 2 };
enum { TACKER_DIRECT_MIN_BE = 0, TACKER_DIRECT_EPS = 1 };

typedef struct tacker_manager_s *tacker_manager_t;

tacker_status tacker_manager_create(int32_t policy, const tacker_manager_params *params,
                                    tacker_stream_t stream, tacker_manager_t *out);
tacker_status tacker_manager_destroy(tacker_manager_t m);
tacker_status tacker_manager_submit_lc(tacker_manager_t m, const tacker_lc_query *q, double arrival_ms,
                                       int32_t *query_id_out);
/* n queries of the same kernels q arriving at arrivals_ms[0..n) (a Poisson trace), ids first_id ..
 * first_id + n - 1 in submission order; one call instead of n (a long trace is submitted before
 * its first arrival). */
tacker_status tacker_manager_submit_lc_batch(tacker_manager_t m, const tacker_lc_query *q, const double *arrivals_ms,
                                             int64_t n, int32_t *first_id);
tacker_status tacker_manager_submit_be(tacker_manager_t m, const tacker_be_app *app, int32_t *app_id_out);
/* Register the predicted fused duration for (LC kernel t_pred class, BE app kernel); the
 * manager asks the model store with the pair key of the fused handle it would build. */
tacker_status tacker_manager_set_clock(tacker_manager_t m, double now_ms);
/* One decision at the manager's clock.  headroom_ms (in/out): on input the newest query's
 * headroom, or NAN to use the manager's Eq. 9 value; on output the updated headroom. */
tacker_status tacker_manager_step(tacker_manager_t m, double qos_target_ms, double *headroom_ms,
                                  tacker_decision *out);
/* GPU mode, Tacker policy: build (and cache in the manager) the fused handle of every (TC
 * kernel, BE kernel) pair with a fitted pair model, so no handle is built (tensor maps, a small
 * cudaMalloc) inside a timed run.  q = NULL: the kernels of every submitted query; else the
 * kernels of *q (not submitted; e.g. before arrival times are fixed).  BE apps must be
 * submitted first.  Handles are keyed by the LC operand pointers and the BE kernel.
 * tacker_manager_run calls it with NULL. */
tacker_status tacker_manager_prepare(tacker_manager_t m, const tacker_lc_query *q);
/* Native run loop: steps the manager (launching in GPU mode) until its clock has passed
 * t_end_ms and every submitted query has completed, or max_decisions decisions were taken
 * (<= 0: unbounded).  The host thread spins between decisions (no Python in the loop). */
tacker_status tacker_manager_run(tacker_manager_t m, double qos_target_ms, double t_end_ms, int64_t max_decisions);
/* Steady-state windows (§VIII-B): steps the manager like
 * tacker_manager_run but returns as soon as its clock reaches t_until_ms, WITHOUT draining the
 * queries or synchronising the stream, so a caller can mark a measurement window (an event on
 * the manager stream + tacker_manager_stats_get) inside one continuous Poisson run and resume. */
tacker_status tacker_manager_run_until(tacker_manager_t m, double qos_target_ms, double t_until_ms);

/* Decision trace (for the discrete-event reference's replay of a GPU-mode run, SURVEY §8(c)
 * c15): one record per decision that launched something, with the observations the decision
 * was taken on -- the manager clock, the active queries (arrival order) and, per BE app, the
 * predicted fused duration Tk_fuse Eq. 8 evaluated (NaN where none was evaluated or no model
 * exists).  Records beyond the capacity are counted in *dropped, not stored. */
#define TACKER_TRACE_MAX_APPS 16
typedef struct {
  double t_ms;                                  /* manager clock at the decision */
  int32_t first_active, n_active;               /* active queries: ids first_active .. + n_active - 1
                                                   (admitted in arrival order, retired oldest first) */
  int32_t active_contiguous;                    /* 0 if the active ids were not that range (queries
                                                   submitted out of arrival order): not replayable */
  int32_t direct;                               /* the decided query runs direct (Thr close to 0) */
  int32_t n_apps;
  uint32_t ready_mask;                          /* bit a: BE app a's head was ready (always, on the GPU) */
  double tk_fuse_ms[TACKER_TRACE_MAX_APPS];
  tacker_decision d;                            /* as tacker_manager_step returned it */
} tacker_trace_rec;
/* capacity 0 disables tracing (default); enabling clears the trace */
tacker_status tacker_manager_trace_enable(tacker_manager_t m, int64_t capacity);
tacker_status tacker_manager_trace_count(tacker_manager_t m, int64_t *stored, int64_t *dropped);
tacker_status tacker_manager_trace_get(tacker_manager_t m, int64_t index, tacker_trace_rec *out);
enum { TACKER_CLASS_LC_TC = 0, TACKER_CLASS_LC_CD = 1, TACKER_CLASS_FUSED = 2, TACKER_CLASS_BE = 3 };
typedef struct {
  int64_t lc_queries_done, be_kernels_done, fused_launches, original_lc, reordered_be, idle_be;
  double now_ms;
  int64_t model_refits;      /* GPU mode: two-stage refits triggered by measured fused runs */
  /* GPU mode: device time per launch class (LC tensor-core original, LC CUDA-core original,
   * fused, BE original).  class_launches counts every launch; class_ms is estimated from CUDA
   * events (manager stream) around one launch in 8 of each class (every fused launch), scaled
   * to the count. */
  double class_ms[4];
  int64_t class_launches[4];
  /* GPU mode: sum of |predicted - measured| / measured of the fused duration over pred_err_n
   * timed fused launches (the pair model as it stood when the manager decided) */
  double pred_err_sum;
  int64_t pred_err_n;
  /* sum of the standalone (predicted) durations of the BE kernels issued: BE work in original-
   * kernel milliseconds, so throughput can be normalised across BE apps of different length */
  double be_work_ms;
  /* GPU mode: host time of the manager loop (ms): event polling, CUDA launch + event-record
   * calls, and everything else in tacker_manager_step (decisions, bookkeeping) */
  double host_poll_ms, host_launch_ms, host_decide_ms;
  int64_t host_steps;        /* tacker_manager_step calls */
  int64_t reverse_fused;     /* fused launches that were reverse fusions (included in fused_launches) */
} tacker_manager_stats;
tacker_status tacker_manager_stats_get(tacker_manager_t m, tacker_manager_stats *out);
/* Completion time (manager clock) of a finished query, or -1 if unfinished. */
tacker_status tacker_manager_query_latency(tacker_manager_t m, int32_t query_id, double *latency_ms);

#ifdef __cplusplus
}
#endif
#endif /* TACKER_H */
