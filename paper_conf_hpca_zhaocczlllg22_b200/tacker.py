"""Thin ctypes binding of libtacker.so (include/tacker.h).  Argument marshalling only:
every step of the hot path runs in the library's CUDA kernels / C++ host code.  PyTorch is
used by callers only for device memory and streams; pass tensors (their data_ptr is taken) or
raw integer device pointers.

The library must be built (python -m paper_conf_hpca_zhaocczlllg22_b200.build); importing this
module fails loudly if libtacker.so is missing — there is no CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import math
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TACKER_LIB") or os.path.join(_HERE, "libtacker.so")   # TACKER_LIB: tuning variants

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libtacker.so not built at {LIB_PATH}; run `python -m paper_conf_hpca_zhaocczlllg22_b200.build`")
_lib = C.CDLL(LIB_PATH)

# ----------------------------------------------------------------------------- enums
OK, EINVAL, ERESOURCE, EUNSUPPORTED, ECUDA, ENOMODEL, ENOMEM = 0, -1, -2, -3, -4, -5, -6
STATUS_NAMES = {0: "OK", -1: "EINVAL", -2: "ERESOURCE", -3: "EUNSUPPORTED", -4: "ECUDA", -5: "ENOMODEL", -6: "ENOMEM"}
LC_NONE, LC_GEMM_F16, LC_CONV_F16 = 0, 1, 2
F32, F16 = 0, 1
EPI_BIAS, EPI_RELU, EPI_RESIDUAL, LC_B_CONST, LC_NO_SPLIT = 1, 2, 4, 8, 16
(BE_NONE, BE_SGEMM, BE_STENCIL, BE_MRIQ_PHIMAG, BE_MRIQ_Q, BE_CUTCP, BE_LBM, BE_SPMV_JDS, BE_HISTO,
 BE_BFS_EXPAND, BE_BFS_COMMIT, BE_FMA_BURN, BE_IM2COL, BE_CUTCP_BIN, BE_COPY, BE_JDS_COUNT, BE_JDS_SCAN,
 BE_JDS_PERM, BE_JDS_FILL, BE_MRIFHD_RHOPHI, BE_MRIFHD_FH, BE_CP, BE_FFT_TWIDDLE, BE_FFT, BE_TPACF) = range(25)
POLICY_TACKER, POLICY_BAYMAX = 0, 1
DEC_FUSED, DEC_ORIGINAL_LC, DEC_REORDER_BE, DEC_IDLE_BE, DEC_NOTHING = range(5)
MAX_APPS = 64
MAX_REORDER = 64


class TackerError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    return x.data_ptr()


# ----------------------------------------------------------------------------- structs
class LcDesc(C.Structure):
    _fields_ = [("kind", C.c_int32), ("M", C.c_int32), ("N", C.c_int32), ("K", C.c_int32),
                ("n", C.c_int32), ("h", C.c_int32), ("w", C.c_int32), ("c", C.c_int32), ("k", C.c_int32),
                ("r", C.c_int32), ("s", C.c_int32), ("stride", C.c_int32), ("pad", C.c_int32),
                ("A", C.c_void_p), ("B", C.c_void_p), ("D", C.c_void_p), ("bias", C.c_void_p),
                ("residual", C.c_void_p), ("d_dtype", C.c_int32), ("epi_flags", C.c_int32), ("tile_n", C.c_int32)]


class BeSgemm(C.Structure):
    _fields_ = [("M", C.c_int32), ("N", C.c_int32), ("K", C.c_int32), ("alpha", C.c_float), ("beta", C.c_float),
                ("A", C.c_void_p), ("B", C.c_void_p), ("C", C.c_void_p)]


class BeStencil(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32), ("c0", C.c_float), ("c1", C.c_float),
                ("A0", C.c_void_p), ("Anext", C.c_void_p)]


class BeMriqPhimag(C.Structure):
    _fields_ = [("numK", C.c_int32), ("phiR", C.c_void_p), ("phiI", C.c_void_p), ("phiMag", C.c_void_p)]


class BeMriqQ(C.Structure):
    _fields_ = [("numX", C.c_int32), ("numK", C.c_int32), ("x", C.c_void_p), ("y", C.c_void_p), ("z", C.c_void_p),
                ("kx", C.c_void_p), ("ky", C.c_void_p), ("kz", C.c_void_p), ("phiMag", C.c_void_p),
                ("Qr", C.c_void_p), ("Qi", C.c_void_p)]


class BeCutcp(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32), ("h", C.c_float), ("cutoff", C.c_float),
                ("excl", C.c_float), ("bdim_x", C.c_int32), ("bdim_y", C.c_int32), ("bdim_z", C.c_int32),
                ("bin_size", C.c_float), ("bin_depth", C.c_int32), ("bins", C.c_void_p), ("count", C.c_void_p),
                ("V", C.c_void_p)]


class BeLbm(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("nz", C.c_int32), ("src", C.c_void_p), ("dst", C.c_void_p),
                ("flags", C.c_void_p)]


class BeSpmv(C.Structure):
    _fields_ = [("rows", C.c_int32), ("perm", C.c_void_p), ("row_len", C.c_void_p), ("jds_ptr", C.c_void_p),
                ("col", C.c_void_p), ("val", C.c_void_p), ("x", C.c_void_p), ("y", C.c_void_p)]


class BeHisto(C.Structure):
    _fields_ = [("n", C.c_int32), ("nbins", C.c_int32), ("inp", C.c_void_p), ("count", C.c_void_p)]


class BeBfsExpand(C.Structure):
    _fields_ = [("V", C.c_int32), ("row_ptr", C.c_void_p), ("col", C.c_void_p), ("level", C.c_void_p),
                ("mask", C.c_void_p), ("visited", C.c_void_p), ("upd", C.c_void_p)]


class BeBfsCommit(C.Structure):
    _fields_ = [("V", C.c_int32), ("mask", C.c_void_p), ("visited", C.c_void_p), ("upd", C.c_void_p),
                ("over", C.c_void_p)]


class BeFmaBurn(C.Structure):
    _fields_ = [("n_threads", C.c_int32), ("iters", C.c_int32), ("a", C.c_float), ("b", C.c_float),
                ("out", C.c_void_p)]


class BeIm2col(C.Structure):
    _fields_ = [("n", C.c_int32), ("h", C.c_int32), ("w", C.c_int32), ("c", C.c_int32), ("r", C.c_int32),
                ("s", C.c_int32), ("stride", C.c_int32), ("pad", C.c_int32), ("Kpad", C.c_int32),
                ("x", C.c_void_p), ("out", C.c_void_p)]


class BeCutcpBin(C.Structure):
    _fields_ = [("natoms", C.c_int32), ("atoms", C.c_void_p), ("bdim_x", C.c_int32), ("bdim_y", C.c_int32),
                ("bdim_z", C.c_int32), ("bin_depth", C.c_int32), ("bin_size", C.c_float), ("bins", C.c_void_p),
                ("count", C.c_void_p), ("overflow", C.c_void_p)]


class BeCopy(C.Structure):
    _fields_ = [("bytes", C.c_int64), ("src", C.c_void_p), ("dst", C.c_void_p)]


class BeJds(C.Structure):
    _fields_ = [("rows", C.c_int32), ("max_len", C.c_int32), ("row_ptr", C.c_void_p), ("col", C.c_void_p),
                ("val", C.c_void_p), ("blk_count", C.c_void_p), ("start", C.c_void_p), ("perm", C.c_void_p),
                ("row_len", C.c_void_p), ("jds_ptr", C.c_void_p), ("jds_col", C.c_void_p), ("jds_val", C.c_void_p),
                ("overflow", C.c_void_p)]


class BeMrifhdRhophi(C.Structure):
    _fields_ = [("numK", C.c_int32), ("phiR", C.c_void_p), ("phiI", C.c_void_p), ("dR", C.c_void_p),
                ("dI", C.c_void_p), ("rRhoPhi", C.c_void_p), ("iRhoPhi", C.c_void_p)]


class BeMrifhdFh(C.Structure):
    _fields_ = [("numX", C.c_int32), ("numK", C.c_int32), ("x", C.c_void_p), ("y", C.c_void_p), ("z", C.c_void_p),
                ("kx", C.c_void_p), ("ky", C.c_void_p), ("kz", C.c_void_p), ("rRhoPhi", C.c_void_p),
                ("iRhoPhi", C.c_void_p), ("rFhD", C.c_void_p), ("iFhD", C.c_void_p)]


class BeCp(C.Structure):
    _fields_ = [("natoms", C.c_int32), ("nx", C.c_int32), ("ny", C.c_int32), ("h", C.c_float), ("z", C.c_float),
                ("atoms", C.c_void_p), ("V", C.c_void_p)]


class BeFft(C.Structure):
    _fields_ = [("n", C.c_int32), ("batch", C.c_int32), ("twiddle", C.c_void_p), ("x", C.c_void_p), ("y", C.c_void_p)]


class BeTpacf(C.Structure):
    _fields_ = [("na", C.c_int32), ("nb", C.c_int32), ("nedges", C.c_int32), ("self_pairs", C.c_int32),
                ("a", C.c_void_p), ("b", C.c_void_p), ("edges", C.c_void_p), ("count", C.c_void_p)]


class _BeUnion(C.Union):
    _fields_ = [("sgemm", BeSgemm), ("stencil", BeStencil), ("mriq_phimag", BeMriqPhimag), ("mriq_q", BeMriqQ),
                ("cutcp", BeCutcp), ("lbm", BeLbm), ("spmv", BeSpmv), ("histo", BeHisto),
                ("bfs_expand", BeBfsExpand), ("bfs_commit", BeBfsCommit), ("fma_burn", BeFmaBurn),
                ("im2col", BeIm2col), ("cutcp_bin", BeCutcpBin), ("copy", BeCopy), ("jds", BeJds),
                ("mrifhd_rhophi", BeMrifhdRhophi), ("mrifhd_fh", BeMrifhdFh), ("cp", BeCp), ("fft", BeFft),
                ("tpacf", BeTpacf),
                ("_pad", C.c_uint8 * 128)]


class BeDesc(C.Structure):
    _fields_ = [("kind", C.c_int32), ("orig_blocks", C.c_int32), ("block_offset", C.c_int32), ("p", _BeUnion)]


class Ratio(C.Structure):
    _fields_ = [("lc", C.c_uint8), ("be", C.c_uint8)]


class FusedInfo(C.Structure):
    _fields_ = [("grid", C.c_int32), ("block_threads", C.c_int32), ("smem_bytes", C.c_int32),
                ("lc_warps", C.c_int32), ("be_warps", C.c_int32), ("be_vblocks_per_cta", C.c_int32),
                ("lc_tile_m", C.c_int32), ("lc_tile_n", C.c_int32), ("lc_tile_k", C.c_int32),
                ("lc_stages", C.c_int32), ("lc_acc_stages", C.c_int32), ("tmem_cols", C.c_int32),
                ("lc_tiles", C.c_int64), ("be_blocks", C.c_int64), ("be_smem_per_vblock", C.c_int32),
                ("regs_per_thread", C.c_int32), ("lc_splits", C.c_int32), ("lc_mode", C.c_int32),
                ("lc_tma_store", C.c_int32)]


LC_MODE_GEMM, LC_MODE_CONV_IM2COL, LC_MODE_CONV_TILED, LC_MODE_CONV_C8, LC_MODE_CONV_HALO, LC_MODE_CONV_S2C8 = range(6)


class LcKernel(C.Structure):
    _fields_ = [("is_tc", C.c_int32), ("t_pred_ms", C.c_double), ("lc", LcDesc), ("cd", BeDesc),
                ("warp_split", C.c_int32)]


class LcQuery(C.Structure):
    _fields_ = [("n_kernels", C.c_int32), ("kernels", C.POINTER(LcKernel))]


class BeKernel(C.Structure):
    _fields_ = [("is_cd", C.c_int32), ("t_pred_ms", C.c_double), ("be", BeDesc), ("warp_split", C.c_int32),
                ("n_blocks", C.c_int32), ("t_block_ms", C.c_double), ("t_floor_ms", C.c_double),
                ("is_tc", C.c_int32), ("tc", LcDesc)]


class BeApp(C.Structure):
    _fields_ = [("n_kernels", C.c_int32), ("kernels", C.POINTER(BeKernel))]


class Decision(C.Structure):
    _fields_ = [("action", C.c_int32), ("query", C.c_int32), ("lc_index", C.c_int32), ("fused_app", C.c_int32),
                ("n_reorder", C.c_int32), ("reorder_apps", C.c_int32 * MAX_REORDER), ("thr_ms", C.c_double),
                ("gain_ms", C.c_double), ("t_start_ms", C.c_double), ("t_end_ms", C.c_double),
                ("fused_blocks", C.c_int64), ("reverse", C.c_int32)]


class ManagerParams(C.Structure):
    _fields_ = [("direct_eps_ms", C.c_double), ("idle_cap_ms", C.c_double), ("max_inflight", C.c_int32),
                ("simulate", C.c_int32), ("slice_be", C.c_int32), ("slice_ratio", C.c_double),
                ("reorder_rule", C.c_int32), ("no_reverse_fusion", C.c_int32), ("fuse_older", C.c_int32),
                ("older_margin_ms", C.c_double), ("direct_rule", C.c_int32)]


REORDER_UNFUSED, REORDER_ALWAYS, REORDER_NEVER = 0, 1, 2     # tacker_manager_params.reorder_rule
DIRECT_MIN_BE, DIRECT_EPS = 0, 1                             # tacker_manager_params.direct_rule


class ManagerStats(C.Structure):
    _fields_ = [("lc_queries_done", C.c_int64), ("be_kernels_done", C.c_int64), ("fused_launches", C.c_int64),
                ("original_lc", C.c_int64), ("reordered_be", C.c_int64), ("idle_be", C.c_int64),
                ("now_ms", C.c_double), ("model_refits", C.c_int64), ("class_ms", C.c_double * 4),
                ("class_launches", C.c_int64 * 4), ("pred_err_sum", C.c_double), ("pred_err_n", C.c_int64),
                ("be_work_ms", C.c_double), ("host_poll_ms", C.c_double), ("host_launch_ms", C.c_double),
                ("host_decide_ms", C.c_double), ("host_steps", C.c_int64), ("reverse_fused", C.c_int64)]


CLASS_LC_TC, CLASS_LC_CD, CLASS_FUSED, CLASS_BE = range(4)
TRACE_MAX_APPS = 16


class TraceRec(C.Structure):
    _fields_ = [("t_ms", C.c_double), ("first_active", C.c_int32), ("n_active", C.c_int32),
                ("active_contiguous", C.c_int32), ("direct", C.c_int32), ("n_apps", C.c_int32), ("ready_mask", C.c_uint32),
                ("tk_fuse_ms", C.c_double * TRACE_MAX_APPS),
                ("d", Decision)]


# ----------------------------------------------------------------------------- prototypes
_V, _I32, _I64, _D, _S = C.c_void_p, C.c_int32, C.c_int64, C.c_double, C.c_char_p
_PROTOS = {
    "tacker_last_error": ([], _S), "tacker_version": ([], _S), "tacker_device_sm_count": ([], C.c_int),
    "tacker_be_num_blocks": ([C.POINTER(BeDesc), C.POINTER(_I64)], C.c_int),
    "tacker_lc_num_tiles": ([C.POINTER(LcDesc), _I32, C.POINTER(_I64)], C.c_int),
    "tacker_lc_num_waves": ([C.POINTER(LcDesc), _I32, C.POINTER(_I64)], C.c_int),
    "tacker_be_prefix_work": ([C.POINTER(BeDesc), _I64, C.POINTER(_D)], C.c_int),
    "tacker_fuse": ([C.POINTER(LcDesc), C.POINTER(BeDesc), _I32, Ratio, C.POINTER(_V)], C.c_int),
    "tacker_fused_destroy": ([_V], C.c_int),
    "tacker_fused_info": ([_V, C.POINTER(FusedInfo)], C.c_int),
    "tacker_fused_keys": ([_V, C.c_char_p, C.c_char_p, C.c_char_p, C.c_size_t], C.c_int),
    "tacker_fused_rebind": ([_V, C.POINTER(LcDesc), C.POINTER(BeDesc)], C.c_int),
    "tacker_launch_fused": ([_V, _V], C.c_int),
    "tacker_launch_fused_slice": ([_V, _I64, _I64, _V], C.c_int),
    "tacker_set_launch_overlap": ([_I32], C.c_int),
    "tacker_debug_lc_timestamps": ([C.POINTER(C.c_uint64), _I64], C.c_int),
    "tacker_debug_lc_globaltimer": ([C.POINTER(C.c_uint64), _I64, C.POINTER(C.c_int32)], C.c_int),
    "tacker_select_fusion": ([C.POINTER(LcDesc), C.POINTER(BeDesc), C.POINTER(_I32), _I32, _I32, _V,
                              C.POINTER(_I32), C.POINTER(_D), C.POINTER(_D), C.POINTER(_D)], C.c_int),
    "tacker_blacklist": ([C.c_char_p, _I32, C.POINTER(_I32)], C.c_int),
    "tacker_blacklist_clear": ([], C.c_int),
    "tacker_launch_original": ([C.POINTER(LcDesc), C.POINTER(BeDesc), _V], C.c_int),
    "tacker_model_add_sample": ([_S, _D, _D], C.c_int),
    "tacker_model_fit": ([_S, C.POINTER(_D), C.POINTER(_D)], C.c_int),
    "tacker_model_predict": ([_S, _D, C.POINTER(_D)], C.c_int),
    "tacker_pair_add_sample": ([_S, _D, _D, _D], C.c_int),
    "tacker_pair_fit": ([_S, C.POINTER(_D)], C.c_int),
    "tacker_pair_predict": ([_S, _D, _D, C.POINTER(_D)], C.c_int),
    "tacker_pair_observe": ([_S, _D, _D, _D, C.POINTER(_I32)], C.c_int),
    "tacker_model_clear": ([], C.c_int),
    "tacker_model_save": ([_S], C.c_int), "tacker_model_load": ([_S], C.c_int),
    "tacker_predict_duration": ([_V, C.POINTER(_D)], C.c_int),
    "tacker_manager_create": ([_I32, C.POINTER(ManagerParams), _V, C.POINTER(_V)], C.c_int),
    "tacker_manager_destroy": ([_V], C.c_int),
    "tacker_manager_submit_lc": ([_V, C.POINTER(LcQuery), _D, C.POINTER(_I32)], C.c_int),
    "tacker_manager_submit_be": ([_V, C.POINTER(BeApp), C.POINTER(_I32)], C.c_int),
    "tacker_manager_set_clock": ([_V, _D], C.c_int),
    "tacker_manager_step": ([_V, _D, C.POINTER(_D), C.POINTER(Decision)], C.c_int),
    "tacker_manager_stats_get": ([_V, C.POINTER(ManagerStats)], C.c_int),
    "tacker_manager_run": ([_V, _D, _D, _I64], C.c_int),
    "tacker_manager_prepare": ([_V, _V], C.c_int),
    "tacker_manager_query_latency": ([_V, _I32, C.POINTER(_D)], C.c_int),
    "tacker_manager_run_until": ([_V, _D, _D], C.c_int),
    "tacker_manager_submit_lc_batch": ([_V, C.POINTER(LcQuery), C.POINTER(_D), _I64, C.POINTER(_I32)], C.c_int),
    "tacker_manager_trace_enable": ([_V, _I64], C.c_int),
    "tacker_manager_trace_count": ([_V, C.POINTER(_I64), C.POINTER(_I64)], C.c_int),
    "tacker_manager_trace_get": ([_V, _I64, C.POINTER(TraceRec)], C.c_int),
}
for _name, (_args, _res) in _PROTOS.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _res
EXPORTED = tuple(_PROTOS)


def _chk(st):
    if st != OK:
        raise TackerError(st, _lib.tacker_last_error().decode())
    return st


def _stream(s):
    if s is None:
        return None
    if isinstance(s, int):
        return s
    return s.cuda_stream


# ----------------------------------------------------------------------------- descriptor builders
def lc_gemm(A, B, D, M=None, N=None, K=None, bias=None, relu=False, residual=None, tile_n=0,
            b_const=False) -> LcDesc:
    """D[M,N] = A[M,K] . B[N,K]^T (+bias)(+residual)(relu); A, B fp16; D fp32 or fp16.
    b_const: B is never written by a kernel on the stream (weights; TACKER_LC_B_CONST)."""
    import torch
    M = A.shape[0] if M is None else M
    K = A.shape[1] if K is None else K
    N = B.shape[0] if N is None else N
    d = LcDesc(kind=LC_GEMM_F16, M=M, N=N, K=K, A=_ptr(A), B=_ptr(B), D=_ptr(D),
               d_dtype=F16 if D.dtype == torch.float16 else F32, tile_n=tile_n)
    _epi(d, bias, relu, residual, b_const)
    return d


def lc_conv(x, w, out, stride, pad, bias=None, relu=False, residual=None, tile_n=0, b_const=False) -> LcDesc:
    """NHWC x [n,h,w,c] fp16, KRSC w [k,r,s,c] fp16 -> NHWC out [n,p,q,k]."""
    import torch
    n, h, wd, c = x.shape
    k, r, s, _ = w.shape
    d = LcDesc(kind=LC_CONV_F16, n=n, h=h, w=wd, c=c, k=k, r=r, s=s, stride=stride, pad=pad, A=_ptr(x), B=_ptr(w),
               D=_ptr(out), d_dtype=F16 if out.dtype == torch.float16 else F32, tile_n=tile_n)
    _epi(d, bias, relu, residual, b_const)
    return d


def _epi(d, bias, relu, residual, b_const=False):
    f = LC_B_CONST if b_const else 0
    if bias is not None:
        d.bias = _ptr(bias)
        f |= EPI_BIAS
    if residual is not None:
        d.residual = _ptr(residual)
        f |= EPI_RESIDUAL
    if relu:
        f |= EPI_RELU
    d.epi_flags = f


def be_sgemm(A, B, Cm, alpha=1.0, beta=0.0, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_SGEMM, orig_blocks=orig_blocks)
    d.p.sgemm = BeSgemm(A.shape[0], B.shape[1], A.shape[1], alpha, beta, _ptr(A), _ptr(B), _ptr(Cm))
    return d


def be_stencil(A0, Anext, c0=1.0 / 6.0, c1=1.0 / 36.0, orig_blocks=0) -> BeDesc:
    nz, ny, nx = A0.shape
    d = BeDesc(kind=BE_STENCIL, orig_blocks=orig_blocks)
    d.p.stencil = BeStencil(nx, ny, nz, c0, c1, _ptr(A0), _ptr(Anext))
    return d


def be_mriq_phimag(phiR, phiI, phiMag, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_MRIQ_PHIMAG, orig_blocks=orig_blocks)
    d.p.mriq_phimag = BeMriqPhimag(phiR.numel(), _ptr(phiR), _ptr(phiI), _ptr(phiMag))
    return d


def be_mriq_q(x, y, z, kx, ky, kz, phiMag, Qr, Qi, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_MRIQ_Q, orig_blocks=orig_blocks)
    d.p.mriq_q = BeMriqQ(x.numel(), kx.numel(), _ptr(x), _ptr(y), _ptr(z), _ptr(kx), _ptr(ky), _ptr(kz),
                         _ptr(phiMag), _ptr(Qr), _ptr(Qi))
    return d


def be_mrifhd_rhophi(phiR, phiI, dR, dI, rRhoPhi, iRhoPhi, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_MRIFHD_RHOPHI, orig_blocks=orig_blocks)
    d.p.mrifhd_rhophi = BeMrifhdRhophi(phiR.numel(), _ptr(phiR), _ptr(phiI), _ptr(dR), _ptr(dI), _ptr(rRhoPhi),
                                       _ptr(iRhoPhi))
    return d


def be_mrifhd_fh(x, y, z, kx, ky, kz, rRhoPhi, iRhoPhi, rFhD, iFhD, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_MRIFHD_FH, orig_blocks=orig_blocks)
    d.p.mrifhd_fh = BeMrifhdFh(x.numel(), kx.numel(), _ptr(x), _ptr(y), _ptr(z), _ptr(kx), _ptr(ky), _ptr(kz),
                               _ptr(rRhoPhi), _ptr(iRhoPhi), _ptr(rFhD), _ptr(iFhD))
    return d


def be_cp(atoms, V, h, z, orig_blocks=0) -> BeDesc:
    """atoms: float32 [natoms, 4] (x, y, z, q) device tensor; V: float32 [ny, nx] (accumulated)."""
    ny, nx = V.shape
    d = BeDesc(kind=BE_CP, orig_blocks=orig_blocks)
    d.p.cp = BeCp(atoms.shape[0], nx, ny, h, z, _ptr(atoms), _ptr(V))
    return d


def be_fft_twiddle(twiddle, n, orig_blocks=0) -> BeDesc:
    """twiddle: float32 [n, 2] device tensor (written)."""
    d = BeDesc(kind=BE_FFT_TWIDDLE, orig_blocks=orig_blocks)
    d.p.fft = BeFft(n, 0, _ptr(twiddle), None, None)
    return d


def be_fft(x, y, twiddle, orig_blocks=0) -> BeDesc:
    """x, y: float32 [batch, n, 2] (complex interleaved); twiddle from be_fft_twiddle."""
    batch, n = x.shape[0], x.shape[1]
    d = BeDesc(kind=BE_FFT, orig_blocks=orig_blocks)
    d.p.fft = BeFft(n, batch, _ptr(twiddle), _ptr(x), _ptr(y))
    return d


def be_tpacf(a, b, edges, count, self_pairs=False, orig_blocks=0) -> BeDesc:
    """a, b: float32 [n, 3] unit vectors; edges float32 decreasing; count int32/uint32 [len(edges)+1]."""
    d = BeDesc(kind=BE_TPACF, orig_blocks=orig_blocks)
    d.p.tpacf = BeTpacf(a.shape[0], b.shape[0], edges.numel(), int(bool(self_pairs)), _ptr(a), _ptr(b), _ptr(edges),
                        _ptr(count))
    return d


def be_lbm(src, dst, flags, orig_blocks=0) -> BeDesc:
    nz, ny, nx = flags.shape
    d = BeDesc(kind=BE_LBM, orig_blocks=orig_blocks)
    d.p.lbm = BeLbm(nx, ny, nz, _ptr(src), _ptr(dst), _ptr(flags))
    return d


def be_spmv(perm, row_len, jds_ptr, col, val, x, y, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_SPMV_JDS, orig_blocks=orig_blocks)
    d.p.spmv = BeSpmv(perm.numel(), _ptr(perm), _ptr(row_len), _ptr(jds_ptr), _ptr(col), _ptr(val), _ptr(x), _ptr(y))
    return d


def be_histo(inp, count, nbins, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_HISTO, orig_blocks=orig_blocks)
    d.p.histo = BeHisto(inp.numel(), nbins, _ptr(inp), _ptr(count))
    return d


def be_bfs_expand(row_ptr, col, level, mask, visited, upd, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_BFS_EXPAND, orig_blocks=orig_blocks)
    d.p.bfs_expand = BeBfsExpand(level.numel(), _ptr(row_ptr), _ptr(col), _ptr(level), _ptr(mask), _ptr(visited),
                                 _ptr(upd))
    return d


def be_bfs_commit(mask, visited, upd, over, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_BFS_COMMIT, orig_blocks=orig_blocks)
    d.p.bfs_commit = BeBfsCommit(mask.numel(), _ptr(mask), _ptr(visited), _ptr(upd), _ptr(over))
    return d


def be_fma_burn(out, iters, n_threads=None, a=0.5, b=0.125, orig_blocks=0) -> BeDesc:
    d = BeDesc(kind=BE_FMA_BURN, orig_blocks=orig_blocks)
    d.p.fma_burn = BeFmaBurn(out.numel() if n_threads is None else n_threads, iters, a, b, _ptr(out))
    return d


def be_im2col(x, out, r, s, stride, pad, Kpad=None, orig_blocks=0) -> BeDesc:
    n, h, w, c = x.shape
    d = BeDesc(kind=BE_IM2COL, orig_blocks=orig_blocks)
    d.p.im2col = BeIm2col(n, h, w, c, r, s, stride, pad, out.shape[1] if Kpad is None else Kpad, _ptr(x), _ptr(out))
    return d


def be_copy(src, dst, nbytes=None, orig_blocks=0) -> BeDesc:
    """dst <- src (either may be pinned host memory: the kernel reads/writes it through UVA)."""
    n = nbytes if nbytes is not None else src.numel() * src.element_size()
    d = BeDesc(kind=BE_COPY, orig_blocks=orig_blocks)
    d.p.copy = BeCopy(n, _ptr(src), _ptr(dst))
    return d


class JdsBuffers:
    """Device buffers of a CSR -> JDS build (outputs + workspace); `descs()` returns the four
    BE kernel descriptors (COUNT, SCAN, PERM, FILL) to launch in order."""

    def __init__(self, row_ptr, col, val, max_len=1023):
        import torch
        rows = row_ptr.numel() - 1
        nnz = col.numel()
        dev = row_ptr.device
        i32 = dict(dtype=torch.int32, device=dev)
        self.src = (row_ptr, col, val)
        self.rows, self.max_len = rows, max_len
        self.blk_count = torch.zeros(((rows + 1023) // 1024) * (max_len + 1), **i32)
        self.start = torch.zeros(max_len + 2, **i32)
        self.perm = torch.zeros(max(rows, 1), **i32)
        self.row_len = torch.zeros(max(rows, 1), **i32)
        self.jds_ptr = torch.zeros(max_len + 1, **i32)
        self.jds_col = torch.zeros(max(nnz, 1), **i32)
        self.jds_val = torch.zeros(max(nnz, 1), dtype=torch.float32, device=dev)
        self.overflow = torch.zeros(1, **i32)

    def descs(self):
        out = []
        for kind in (BE_JDS_COUNT, BE_JDS_SCAN, BE_JDS_PERM, BE_JDS_FILL):
            d = BeDesc(kind=kind)
            d.p.jds = BeJds(self.rows, self.max_len, _ptr(self.src[0]), _ptr(self.src[1]), _ptr(self.src[2]),
                            _ptr(self.blk_count), _ptr(self.start), _ptr(self.perm), _ptr(self.row_len),
                            _ptr(self.jds_ptr), _ptr(self.jds_col), _ptr(self.jds_val), _ptr(self.overflow))
            out.append(d)
        return out

    def build(self, stream=None):
        for d in self.descs():
            tacker_launch_original(None, d, stream)
        return self


def cutcp_bin_dims(nx, ny, nz):
    return (nx + 7) // 8, (ny + 7) // 8, (nz + 7) // 8


def be_cutcp_bin(atoms, bins, count, overflow, nx, ny, nz, h, depth, orig_blocks=0) -> BeDesc:
    """Bin atoms (float4 rows) for cutcp: bin side 8*h over the lattice (nx, ny, nz)."""
    bx, by, bz = cutcp_bin_dims(nx, ny, nz)
    d = BeDesc(kind=BE_CUTCP_BIN, orig_blocks=orig_blocks)
    d.p.cutcp_bin = BeCutcpBin(atoms.shape[0], _ptr(atoms), bx, by, bz, depth, 8.0 * h, _ptr(bins), _ptr(count),
                               _ptr(overflow))
    return d


def be_cutcp(bins, count, V, nx, ny, nz, h, depth, cutoff=12.0, excl=1.0, orig_blocks=0) -> BeDesc:
    bx, by, bz = cutcp_bin_dims(nx, ny, nz)
    d = BeDesc(kind=BE_CUTCP, orig_blocks=orig_blocks)
    d.p.cutcp = BeCutcp(nx, ny, nz, h, cutoff, excl, bx, by, bz, 8.0 * h, depth, _ptr(bins), _ptr(count), _ptr(V))
    return d


# ----------------------------------------------------------------------------- C ABI mirrors
def tacker_version() -> str:
    return _lib.tacker_version().decode()


def tacker_device_sm_count() -> int:
    return _lib.tacker_device_sm_count()


def tacker_last_error() -> str:
    return _lib.tacker_last_error().decode()


def tacker_be_num_blocks(be: BeDesc) -> int:
    v = C.c_int64()
    _chk(_lib.tacker_be_num_blocks(C.byref(be), C.byref(v)))
    return v.value


def tacker_lc_num_waves(lc: LcDesc, tile_n: int = 0) -> int:
    v = C.c_int64()
    _chk(_lib.tacker_lc_num_waves(C.byref(lc), tile_n, C.byref(v)))
    return v.value


def tacker_be_prefix_work(be: BeDesc, n_blocks: int) -> float:
    v = C.c_double()
    _chk(_lib.tacker_be_prefix_work(C.byref(be), n_blocks, C.byref(v)))
    return v.value


def tacker_lc_num_tiles(lc: LcDesc, tile_n: int = 0) -> int:
    v = C.c_int64()
    _chk(_lib.tacker_lc_num_tiles(C.byref(lc), tile_n, C.byref(v)))
    return v.value


class Fused:
    """Owning wrapper of a tacker_fused_t handle."""

    def __init__(self, handle, lc, be):
        self.h = handle
        self._keep = (lc, be)

    def __del__(self):
        if getattr(self, "h", None):
            if _lib is not None:   # None during interpreter shutdown
                _lib.tacker_fused_destroy(self.h)
            self.h = None

    def info(self) -> FusedInfo:
        i = FusedInfo()
        _chk(_lib.tacker_fused_info(self.h, C.byref(i)))
        return i

    def keys(self):
        bufs = [C.create_string_buffer(512) for _ in range(3)]
        _chk(_lib.tacker_fused_keys(self.h, bufs[0], bufs[1], bufs[2], 512))
        return tuple(b.value.decode() for b in bufs)

    def launch(self, stream=None):
        _chk(_lib.tacker_launch_fused(self.h, _stream(stream)))

    def launch_slice(self, block_offset, n_blocks, stream=None):
        """The LC part plus BE original blocks [block_offset, block_offset + n_blocks) only."""
        _chk(_lib.tacker_launch_fused_slice(self.h, block_offset, n_blocks, _stream(stream)))

    def rebind(self, lc=None, be=None):
        _chk(_lib.tacker_fused_rebind(self.h, C.byref(lc) if lc is not None else None,
                                      C.byref(be) if be is not None else None))
        self._keep = (lc or self._keep[0], be or self._keep[1])

    def predict(self) -> float:
        v = C.c_double()
        _chk(_lib.tacker_predict_duration(self.h, C.byref(v)))
        return v.value


def tacker_fuse(lc: LcDesc, be: BeDesc | None, warp_split: int, block_ratio=(0, 0)) -> Fused:
    h = C.c_void_p()
    _chk(_lib.tacker_fuse(C.byref(lc), C.byref(be) if be is not None else None, warp_split,
                          Ratio(*block_ratio), C.byref(h)))
    return Fused(h.value, lc, be)


def tacker_launch_fused(f: Fused, stream=None):
    f.launch(stream)


def tacker_select_fusion(lc: LcDesc, be: BeDesc, splits=(24, 20, 16, 12, 8, 4), reps=5, stream=None):
    """NEXT-1: time every fused candidate and the sequential pair; returns
    (best warp split or 0 = do not fuse, best ms, sequential ms, {split: fused ms})."""
    n = len(splits)
    arr = (C.c_int32 * n)(*splits)
    best, bms, sms = C.c_int32(), C.c_double(), C.c_double()
    fms = (C.c_double * n)()
    _chk(_lib.tacker_select_fusion(C.byref(lc), C.byref(be), arr, n, reps, _stream(stream), C.byref(best),
                                   C.byref(bms), C.byref(sms), fms))
    return best.value, bms.value, sms.value, {s: fms[i] for i, s in enumerate(splits) if fms[i] == fms[i]}


def tacker_blacklist(be_key: str, op: int = -1) -> bool:
    """op 1 add, 0 remove, -1 query; returns membership."""
    v = C.c_int32()
    _chk(_lib.tacker_blacklist(be_key.encode(), op, C.byref(v)))
    return bool(v.value)


def tacker_blacklist_clear():
    _chk(_lib.tacker_blacklist_clear())


def tacker_debug_lc_globaltimer():
    """([256][8] %globaltimer stamps per LC launch (plans built with TACKER_LC_DBG bit 4 = 16),
    number of launches recorded); clears the buffer."""
    import numpy as np
    buf = (C.c_uint64 * (256 * 8))()
    n = C.c_int32()
    _chk(_lib.tacker_debug_lc_globaltimer(buf, len(buf), C.byref(n)))
    return np.frombuffer(buf, dtype=np.uint64).reshape(256, 8).copy(), n.value


def tacker_debug_lc_timestamps():
    """[160][5][16] clock64 stamps of the LC roles (plans built with TACKER_LC_DBG bit 3)."""
    import numpy as np
    buf = (C.c_uint64 * (160 * 5 * 16))()
    _chk(_lib.tacker_debug_lc_timestamps(buf, len(buf)))
    return np.frombuffer(buf, dtype=np.uint64).reshape(160, 5, 16).copy()


def tacker_set_launch_overlap(enable):
    """Programmatic dependent launch: False/0 off, True/1 every launch, 2 (the library default)
    every launch except original BE kernels."""
    _chk(_lib.tacker_set_launch_overlap(int(enable)))


def tacker_launch_fused_slice(f: Fused, block_offset: int, n_blocks: int, stream=None):
    f.launch_slice(block_offset, n_blocks, stream)


def tacker_launch_original(lc: LcDesc | None, be: BeDesc | None, stream=None):
    _chk(_lib.tacker_launch_original(C.byref(lc) if lc is not None else None,
                                     C.byref(be) if be is not None else None, _stream(stream)))


def tacker_predict_duration(f: Fused) -> float:
    return f.predict()


def tacker_model_add_sample(key: str, blocks: float, ms: float):
    _chk(_lib.tacker_model_add_sample(key.encode(), blocks, ms))


def tacker_model_fit(key: str):
    a, b = C.c_double(), C.c_double()
    _chk(_lib.tacker_model_fit(key.encode(), C.byref(a), C.byref(b)))
    return a.value, b.value


def tacker_model_predict(key: str, blocks: float) -> float:
    v = C.c_double()
    _chk(_lib.tacker_model_predict(key.encode(), blocks, C.byref(v)))
    return v.value


def tacker_pair_add_sample(key: str, x_tc: float, x_cd: float, t_fused: float):
    _chk(_lib.tacker_pair_add_sample(key.encode(), x_tc, x_cd, t_fused))


def tacker_pair_fit(key: str):
    c = (C.c_double * 4)()
    _chk(_lib.tacker_pair_fit(key.encode(), c))
    return tuple(c)


def tacker_pair_predict(key: str, x_tc: float, x_cd: float) -> float:
    v = C.c_double()
    _chk(_lib.tacker_pair_predict(key.encode(), x_tc, x_cd, C.byref(v)))
    return v.value


def tacker_pair_observe(key: str, x_tc: float, x_cd: float, t_meas: float) -> bool:
    r = C.c_int32()
    _chk(_lib.tacker_pair_observe(key.encode(), x_tc, x_cd, t_meas, C.byref(r)))
    return bool(r.value)


def tacker_model_clear():
    _chk(_lib.tacker_model_clear())


def tacker_model_save(path: str):
    _chk(_lib.tacker_model_save(path.encode()))


def tacker_model_load(path: str):
    _chk(_lib.tacker_model_load(path.encode()))


class Manager:
    """Owning wrapper of tacker_manager_t."""

    def __init__(self, policy=POLICY_TACKER, stream=None, simulate=False, direct_eps_ms=0.0, idle_cap_ms=0.0,
                 max_inflight=2, slice_be=False, slice_ratio=0.0, reorder_rule=REORDER_UNFUSED, reverse_fusion=True,
                 fuse_older=False, older_margin_ms=0.0, direct_rule=DIRECT_MIN_BE):
        self.h = C.c_void_p()
        self.params = ManagerParams(direct_eps_ms, idle_cap_ms, max_inflight, 1 if simulate else 0,
                                    1 if slice_be else 0, slice_ratio, int(reorder_rule),
                                    0 if reverse_fusion else 1, 1 if fuse_older else 0, older_margin_ms,
                                    int(direct_rule))
        _chk(_lib.tacker_manager_create(policy, C.byref(self.params), _stream(stream), C.byref(self.h)))
        self._keep = []

    def __del__(self):
        if getattr(self, "h", None):
            if _lib is not None:
                _lib.tacker_manager_destroy(self.h)
            self.h = None

    def submit_lc(self, kernels, arrival_ms) -> int:
        arr = (LcKernel * len(kernels))(*kernels)
        q = LcQuery(len(kernels), arr)
        qid = C.c_int32()
        _chk(_lib.tacker_manager_submit_lc(self.h, C.byref(q), arrival_ms, C.byref(qid)))
        return qid.value

    def submit_lc_batch(self, kernels, arrivals_ms) -> list:
        """Queries of the same kernels at each arrival time (one C call); returns their ids."""
        arr = (LcKernel * len(kernels))(*kernels)
        q = LcQuery(len(kernels), arr)
        ts = (C.c_double * len(arrivals_ms))(*[float(a) for a in arrivals_ms])
        first = C.c_int32()
        _chk(_lib.tacker_manager_submit_lc_batch(self.h, C.byref(q), ts, len(arrivals_ms), C.byref(first)))
        return list(range(first.value, first.value + len(arrivals_ms)))

    def submit_be(self, kernels) -> int:
        arr = (BeKernel * len(kernels))(*kernels)
        a = BeApp(len(kernels), arr)
        aid = C.c_int32()
        _chk(_lib.tacker_manager_submit_be(self.h, C.byref(a), C.byref(aid)))
        return aid.value

    def set_clock(self, now_ms):
        _chk(_lib.tacker_manager_set_clock(self.h, now_ms))

    def step(self, qos_ms, headroom=math.nan):
        d = Decision()
        thr = C.c_double(headroom)
        _chk(_lib.tacker_manager_step(self.h, qos_ms, C.byref(thr), C.byref(d)))
        return d

    def prepare(self, kernels=None):
        """Build the fused handles of every admissible (TC kernel, BE kernel) pair up front: of
        `kernels` (a query's kernel list, not submitted) or of every submitted query."""
        if kernels is None:
            _chk(_lib.tacker_manager_prepare(self.h, None))
            return
        arr = (LcKernel * len(kernels))(*kernels)
        q = LcQuery(len(kernels), arr)
        _chk(_lib.tacker_manager_prepare(self.h, C.byref(q)))

    def run(self, qos_ms, t_end_ms=0.0, max_decisions=0):
        """Native loop: decide + launch until t_end_ms has passed and all queries completed."""
        _chk(_lib.tacker_manager_run(self.h, qos_ms, t_end_ms, max_decisions))

    def run_until(self, qos_ms, t_until_ms):
        """Native loop up to manager clock t_until_ms, no drain / no sync (measurement windows)."""
        _chk(_lib.tacker_manager_run_until(self.h, qos_ms, t_until_ms))

    def trace_enable(self, capacity):
        _chk(_lib.tacker_manager_trace_enable(self.h, int(capacity)))

    def trace(self):
        """[TraceRec] recorded decisions and the count dropped beyond the capacity."""
        n, dropped = C.c_int64(), C.c_int64()
        _chk(_lib.tacker_manager_trace_count(self.h, C.byref(n), C.byref(dropped)))
        out = []
        for i in range(n.value):
            r = TraceRec()
            _chk(_lib.tacker_manager_trace_get(self.h, i, C.byref(r)))
            out.append(r)
        return out, dropped.value

    def trace_dicts(self):
        """The trace as plain records for oracle/manager_ref.replay: t, active ids, ready apps,
        {app: Tk_fuse}, and the decision (action, query, lc_index, fused_app, reorder, thr)."""
        recs, dropped = self.trace()
        out = []
        for r in recs:
            if not r.active_contiguous:
                raise TackerError(EINVAL, "trace record whose active queries are not an id range")
            tf = {a: r.tk_fuse_ms[a] for a in range(r.n_apps) if not math.isnan(r.tk_fuse_ms[a])}
            d = r.d
            out.append({"t": r.t_ms, "active": list(range(r.first_active, r.first_active + r.n_active)),
                        "ready": [a for a in range(r.n_apps) if (r.ready_mask >> a) & 1], "tk_fuse": tf,
                        "direct": bool(r.direct), "action": d.action, "query": d.query, "lc_index": d.lc_index,
                        "fused_app": d.fused_app, "reorder": list(d.reorder_apps[:d.n_reorder]),
                        "thr": d.thr_ms, "gain": d.gain_ms, "reverse": bool(d.reverse)})
        return out, dropped

    def stats(self) -> ManagerStats:
        s = ManagerStats()
        _chk(_lib.tacker_manager_stats_get(self.h, C.byref(s)))
        return s

    def latency(self, qid) -> float:
        v = C.c_double()
        _chk(_lib.tacker_manager_query_latency(self.h, qid, C.byref(v)))
        return v.value


def tacker_manager_step(m: Manager, qos_target_ms: float, headroom_ms: float = math.nan) -> Decision:
    return m.step(qos_target_ms, headroom_ms)
