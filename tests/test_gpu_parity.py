"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element,
and fused launches bit-identical to the original launches (BASELINE correctness gates)."""
import numpy as np
import pytest
import torch

import synth
from oracle import be as obe, lc as olc
from oracle.metrics import max_rel_err

pytestmark = pytest.mark.gpu

from tests.gpu_helpers import be_case, dev, host, t  # noqa: E402


@pytest.fixture(scope="module")
def tk():
    from paper_conf_hpca_zhaocczlllg22_b200 import tacker
    assert torch.cuda.is_available()
    return tacker


# ------------------------------------------------------------------ LC GEMM (c1)
@pytest.mark.parametrize("M,N,K,bn", [(256, 256, 256, 0), (256, 256, 256, 64), (256, 256, 256, 256),
                                      (300, 136, 200, 128), (1, 8, 8, 64), (129, 264, 72, 256), (1000, 512, 1024, 128)])
def test_lc_gemm_vs_oracle(tk, M, N, K, bn):
    A, B = synth.lc_gemm_inputs(M, N, K, seed=M + N + K)
    D = torch.full((M, N), float("nan"), device=dev())
    tk.tacker_launch_original(tk.lc_gemm(t(A), t(B), D, tile_n=bn), None)
    ref, S = olc.lc_gemm(A, B)
    assert max_rel_err(host(D), ref, S) <= 1e-2
    assert max_rel_err(host(D), ref, S) <= 1e-5   # fp32 accumulation: far inside the gate


@pytest.mark.parametrize("variant", ["int", "identity", "onehot"])
def test_lc_gemm_exact_variants(tk, variant):
    M, N, K = 256, 256, 256
    A, B = synth.lc_gemm_inputs(M, N, K, seed=7, variant=variant)
    D = torch.zeros(M, N, device=dev())
    tk.tacker_launch_original(tk.lc_gemm(t(A), t(B), D), None)
    ref, _ = olc.lc_gemm(A, B)
    assert np.array_equal(host(D).astype(np.float64), ref)


@pytest.mark.parametrize("M,N,K", [(2304, 2176, 128), (4096 + 200, 2048, 192)])
def test_lc_gemm_many_tiles_exact(tk, M, N, K):
    # >= 256 tiles over the persistent grid (several tiles per CTA, ragged M): every tile covered
    # once -- integer inputs, so the whole output is exact; and the fused launch bit-identical to
    # the original (the mode-specialised LC-only kernel vs the run-time-mode fused kernel)
    A, B = synth.lc_gemm_inputs(M, N, K, seed=17, variant="int")
    D = torch.zeros(M, N, device=dev())
    f = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), None, 0)
    assert f.info().lc_tiles >= 256
    tk.tacker_launch_original(tk.lc_gemm(t(A), t(B), D), None)
    ref = A.astype(np.float64) @ B.astype(np.float64).T
    assert np.array_equal(host(D).astype(np.float64), ref)
    c = be_case(tk.BE_SGEMM, seed=3)
    D1 = torch.zeros(M, N, device=dev())
    c["reset"]()
    tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D1), c["desc"], 16).launch()
    assert host(D1).tobytes() == host(D).tobytes()


def test_lc_gemm_f16_epilogue(tk):
    M, N, K = 200, 192, 128
    A, B = synth.lc_gemm_inputs(M, N, K, seed=9)
    bias = np.random.default_rng(0).uniform(-0.5, 0.5, N).astype(np.float32)
    res = np.random.default_rng(1).uniform(-1, 1, (M, N)).astype(np.float16)
    D = torch.zeros(M, N, dtype=torch.float16, device=dev())
    tk.tacker_launch_original(tk.lc_gemm(t(A), t(B), D, bias=t(bias), relu=True, residual=t(res)), None)
    ref, S = olc.lc_gemm(A, B, bias=bias, relu=True, residual=res)
    got = host(D).astype(np.float64)
    assert max_rel_err(got, ref, S + 1e-3) <= 1e-2


# ------------------------------------------------------------------ LC conv (c2)
CONV_CASES = [synth.ConvShape("3x3s1", 1, 14, 14, 64, 64, 3, 3, 1, 1),
              synth.ConvShape("3x3s2", 1, 28, 28, 128, 128, 3, 3, 2, 1),
              synth.ConvShape("1x1s1", 1, 28, 28, 256, 128, 1, 1, 1, 0),
              synth.ConvShape("1x1s2", 1, 56, 56, 64, 256, 1, 1, 2, 0),
              synth.ConvShape("7x7", 1, 7, 7, 512, 512, 3, 3, 1, 1),
              synth.ConvShape("b2", 2, 9, 11, 64, 72, 3, 3, 1, 1),
              synth.ConvShape("c8_conv1", 2, 30, 28, 8, 64, 7, 7, 2, 3)]   # 8-tap k-blocks, unswizzled A


@pytest.mark.parametrize("cs", CONV_CASES, ids=lambda c: c.name)
def test_lc_conv_vs_oracle(tk, cs):
    x, w, b = synth.conv_inputs(cs, seed=3, real_c=3 if cs.c == 8 else None)
    out = torch.zeros(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device=dev())
    tk.tacker_launch_original(tk.lc_conv(t(x), t(w), out, cs.stride, cs.pad, bias=t(b), relu=True), None)
    ref, S = olc.lc_conv(x, w, cs.stride, cs.pad, bias=b, relu=True)
    assert max_rel_err(host(out).astype(np.float64), ref, S) <= 1e-2


# ------------------------------------------------------------------ BE originals (c3-c10)
BE_KINDS = ["BE_SGEMM", "BE_STENCIL", "BE_MRIQ_Q", "BE_MRIQ_PHIMAG", "BE_LBM", "BE_SPMV_JDS", "BE_HISTO", "BE_FMA_BURN",
            "BE_CUTCP", "BE_MRIFHD_RHOPHI", "BE_MRIFHD_FH", "BE_CP", "BE_FFT_TWIDDLE", "BE_FFT", "BE_TPACF"]


@pytest.mark.parametrize("kind", BE_KINDS)
def test_be_original_vs_oracle(tk, kind):
    c = be_case(getattr(tk, kind))
    c["reset"]()
    tk.tacker_launch_original(None, c["desc"])
    c["check"]([host(o) for o in c["outs"]])


@pytest.mark.parametrize("size", ["odd", "mid", "tiny", "single16", "single8", "two"])
def test_fft_lengths_vs_oracle(tk, size):
    c = be_case(tk.BE_FFT, seed=4, size=size)
    c["reset"]()
    tk.tacker_launch_original(None, c["desc"])
    c["check"]([host(o) for o in c["outs"]])


@pytest.mark.parametrize("size", ["small", "odd", "mid", "tiny", "single16", "single8", "two"])
@pytest.mark.parametrize("ws", [8, 24])
def test_fft_lengths_fused_bit_identical(tk, size, ws):
    # the fused fft runs one static pass plan per length in its own PTB loop copy (fused.cuh
    # be_ptb_loop): every length, in the register-rich (ws 8) and the default (ws 24) class
    c = be_case(tk.BE_FFT, seed=4, size=size)
    c["reset"]()
    tk.tacker_launch_original(None, c["desc"])
    orig = [host(o).copy() for o in c["outs"]]
    c["check"](orig)
    A, B = synth.lc_gemm_inputs(256, 128, 128, seed=1)
    D = torch.zeros(256, 128, device=dev())
    f = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), c["desc"], ws)
    c["reset"]()
    f.launch()
    for a, o in zip(orig, c["outs"]):
        assert a.tobytes() == host(o).tobytes()


@pytest.mark.parametrize("variant", ["impulse", "tone"])
def test_fft_closed_form_inputs(tk, variant):
    # impulse -> pure twiddle rows, tone -> n at one bin: vs the oracle's DFT of the same fp32 input
    batch, n = 40, 512
    x = synth.fft_inputs(batch, n, 0, variant)
    tw = torch.zeros(n, 2, device=dev())
    y = torch.zeros(batch, n, 2, device=dev())
    tk.tacker_launch_original(None, tk.be_fft_twiddle(tw, n))
    tk.tacker_launch_original(None, tk.be_fft(t(x), y, tw))
    X, S = obe.fft(x[..., 0].astype(np.float64) + 1j * x[..., 1])
    g = host(y)
    assert max_rel_err(g[..., 0], X.real, S) <= 1e-5 and max_rel_err(g[..., 1], X.imag, S) <= 1e-5


def test_tpacf_cross_and_axis_points(tk):
    e = synth.tpacf_edges()
    A = synth.tpacf_inputs(777, 3)
    B = synth.tpacf_inputs(1500, 4, "uniform")
    cnt = torch.zeros(len(e) + 1, dtype=torch.int32, device=dev())
    tk.tacker_launch_original(None, tk.be_tpacf(t(A), t(B), t(e), cnt))
    assert np.array_equal(host(cnt).astype(np.int64), obe.tpacf(A, B, e, False))
    ax = np.array([[1, 0, 0], [0, 1, 0], [-1, 0, 0]], np.float32)
    cnt.zero_()
    tk.tacker_launch_original(None, tk.be_tpacf(t(ax[:1]), t(ax), t(e), cnt))
    assert np.array_equal(host(cnt).astype(np.int64), obe.tpacf(ax[:1], ax, e, False))


def test_bfs_levels_vs_oracle(tk):
    V = 1 << 14
    rp, col = synth.bfs_inputs(V, seed=5)
    drp, dcol = t(rp), t(col)
    level = torch.full((V,), -1, dtype=torch.int32, device=dev())
    level[0] = 0
    mask = torch.zeros(V, dtype=torch.uint8, device=dev())
    mask[0] = 1
    visited = mask.clone()
    upd = torch.zeros_like(mask)
    over = torch.zeros(1, dtype=torch.int32, device=dev())
    e = tk.be_bfs_expand(drp, dcol, level, mask, visited, upd)
    cm = tk.be_bfs_commit(mask, visited, upd, over)
    for _ in range(V):
        over.zero_()
        tk.tacker_launch_original(None, e)
        tk.tacker_launch_original(None, cm)
        if int(over.item()) == 0:
            break
    assert np.array_equal(host(level), obe.bfs_levels(rp, col))


# ------------------------------------------------------------------ fused (a1-a8)
FUSE_KINDS = ["BE_SGEMM", "BE_STENCIL", "BE_MRIQ_Q", "BE_LBM", "BE_SPMV_JDS", "BE_HISTO", "BE_FMA_BURN", "BE_CUTCP",
              "BE_MRIFHD_RHOPHI", "BE_MRIFHD_FH", "BE_CP", "BE_FFT", "BE_TPACF"]


RICH_KINDS = {"BE_SGEMM", "BE_STENCIL", "BE_MRIQ_Q", "BE_MRIFHD_FH", "BE_CUTCP", "BE_CP", "BE_LBM", "BE_FFT", "BE_TPACF",
              "BE_SPMV_JDS"}


@pytest.mark.parametrize("kind", FUSE_KINDS)
@pytest.mark.parametrize("ws", [4, 8, 16])
def test_fused_bit_identical_to_original(tk, kind, ws):
    M, N, K = 256, 256, 256
    A, B = synth.lc_gemm_inputs(M, N, K, seed=1)
    dA, dB = t(A), t(B)
    D0 = torch.zeros(M, N, device=dev())
    D1 = torch.zeros(M, N, device=dev())
    c = be_case(getattr(tk, kind), seed=2)
    # original launches
    c["reset"]()
    tk.tacker_launch_original(tk.lc_gemm(dA, dB, D0), c["desc"])
    orig = [host(o).copy() for o in c["outs"]]
    c["check"](orig)
    # fused launch, twice (the BE ticket must self-reset)
    f = tk.tacker_fuse(tk.lc_gemm(dA, dB, D1), c["desc"], ws)
    if ws <= 8 and kind in RICH_KINDS:   # register-rich class (fused_rich.cu): above the 64 cap
        assert f.info().regs_per_thread > 64
    for _ in range(2):
        c["reset"]()
        D1.zero_()
        f.launch()
        fused = [host(o) for o in c["outs"]]
        for a, b in zip(orig, fused):
            assert a.tobytes() == b.tobytes()
        assert host(D1).tobytes() == host(D0).tobytes()
    ref, S = olc.lc_gemm(A, B)
    assert max_rel_err(host(D1), ref, S) <= 1e-2


def test_fused_large_lc_many_tiles(tk):
    # more LC tiles than CTAs (persistent tile loop, TMEM double buffer) + sgemm BE
    M, N, K = 4096, 1024, 512
    A, B = synth.lc_gemm_inputs(M, N, K, seed=4)
    D = torch.zeros(M, N, device=dev())
    c = be_case(tk.BE_SGEMM, seed=3, size="large")
    c["reset"]()
    f = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), c["desc"], 8)
    assert f.info().lc_tiles > f.info().grid
    f.launch()
    ref, S = olc.lc_gemm(A, B)
    assert max_rel_err(host(D), ref, S) <= 1e-5
    c["check"]([host(o) for o in c["outs"]])


def test_fused_conv_stencil(tk):
    cs = synth.ConvShape("c", 1, 28, 28, 128, 128, 3, 3, 1, 1)
    x, w, b = synth.conv_inputs(cs, seed=6)
    out = torch.zeros(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device=dev())
    c = be_case(tk.BE_STENCIL, seed=8)
    c["reset"]()
    f = tk.tacker_fuse(tk.lc_conv(t(x), t(w), out, 1, 1, bias=t(b), relu=True), c["desc"], 8)
    f.launch()
    ref, S = olc.lc_conv(x, w, 1, 1, bias=b, relu=True)
    assert max_rel_err(host(out).astype(np.float64), ref, S) <= 1e-2
    c["check"]([host(o) for o in c["outs"]])


def test_ptb_orig_blocks_prefix(tk):
    # orig_blocks < whole problem: only the first blocks run (PTB runtime argument, Fig. 7)
    n, iters = 128 * 64, 10
    out = torch.zeros(n, device=dev())
    A, B = synth.lc_gemm_inputs(128, 128, 64, seed=0)
    D = torch.zeros(128, 128, device=dev())
    f = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), tk.be_fma_burn(out, iters, orig_blocks=10), 4)
    f.launch()
    o = host(out)
    ref = obe.fma_burn(n, iters)
    assert max_rel_err(o[:1280], ref[:1280]) <= 1e-5
    assert np.all(o[1280:] == 0)


@pytest.mark.parametrize("ws", [4, 20])
def test_stencil_scalar_path_and_large(tk, ws):
    # nx % 4 != 0 (scalar path) and the full bench grid (TMA path, 2048 blocks), fused vs original
    for size in ("scalar", "large"):
        c = be_case(tk.BE_STENCIL, seed=5, size=size)
        c["reset"]()
        tk.tacker_launch_original(None, c["desc"])
        orig = host(c["outs"][0]).copy()
        c["check"]([orig])
        A, B = synth.lc_gemm_inputs(256, 128, 64, seed=0)
        D = torch.zeros(256, 128, device=dev())
        f = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), c["desc"], ws)
        c["reset"]()
        f.launch()
        assert host(c["outs"][0]).tobytes() == orig.tobytes()


@pytest.mark.parametrize("ws", [4, 12, 24])
@pytest.mark.parametrize("orig_blocks", [0, 301])
def test_mriq_static_split_chunks(tk, ws, orig_blocks):
    # fused mri-q Q uses the static even split with up to kCoarsen blocks per thread: 2662 blocks
    # of 32 voxels over 148 CTAs gives 17-18 per CTA, several per slot at every split, with
    # coarsened chunks and 1-block tails; orig_blocks = 301 exercises the PTB prefix (2 per CTA,
    # slots with 0 or 1 block)
    N, nk = 44, 256
    d = synth.mriq_inputs(N, nk, 11)
    pm = (d["phiR"].astype(np.float32) ** 2 + d["phiI"].astype(np.float32) ** 2).astype(np.float32)
    dd = {k: t(v) for k, v in d.items()}
    dpm = t(pm)
    outs = [torch.zeros(N ** 3, device=dev()) for _ in range(4)]
    desc_o = tk.be_mriq_q(dd["x"], dd["y"], dd["z"], dd["kx"], dd["ky"], dd["kz"], dpm, outs[0], outs[1],
                          orig_blocks=orig_blocks)
    desc_f = tk.be_mriq_q(dd["x"], dd["y"], dd["z"], dd["kx"], dd["ky"], dd["kz"], dpm, outs[2], outs[3],
                          orig_blocks=orig_blocks)
    tk.tacker_launch_original(None, desc_o)
    A, B = synth.lc_gemm_inputs(256, 128, 64, seed=0)
    D = torch.zeros(256, 128, device=dev())
    f = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), desc_f, ws)
    f.launch()
    qr_o, qi_o, qr_f, qi_f = (host(o) for o in outs)
    assert qr_f.tobytes() == qr_o.tobytes() and qi_f.tobytes() == qi_o.tobytes()
    n = N ** 3 if orig_blocks == 0 else orig_blocks * 32     # 32 voxels per original block
    rr, ri, sr, si = obe.mriq_q(d["x"][:n], d["y"][:n], d["z"][:n], d["kx"], d["ky"], d["kz"], pm)
    assert max_rel_err(qr_o[:n], rr, sr) <= 1e-5 and max_rel_err(qi_o[:n], ri, si) <= 1e-5
    assert np.all(qr_o[n:] == 0) and np.all(qi_o[n:] == 0)


@pytest.mark.parametrize("kind", FUSE_KINDS)
def test_ptb_slices_compose_to_whole_kernel(tk, kind):
    # PTB slices (reading 13): a fused slice, an original slice and a fused slice that partition
    # [0, N) give the whole original kernel's bytes; every slice run once
    import ctypes
    c = be_case(getattr(tk, kind), seed=3)
    c["reset"]()
    tk.tacker_launch_original(None, c["desc"])
    whole = [host(o).copy() for o in c["outs"]]
    c["check"](whole)
    N = tk.tacker_be_num_blocks(c["desc"])
    a, b = max(1, N // 3), max(1, N // 3) + max(1, N // 4)
    assert 0 < a < b < N, (N, a, b)
    A, B = synth.lc_gemm_inputs(256, 256, 128, seed=1)
    D = torch.zeros(256, 256, device=dev())
    f = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), c["desc"], 8)
    mid = tk.BeDesc()
    ctypes.memmove(ctypes.addressof(mid), ctypes.addressof(c["desc"]), ctypes.sizeof(mid))
    mid.block_offset, mid.orig_blocks = a, b - a
    for _ in range(2):
        c["reset"]()
        f.launch_slice(0, a)
        tk.tacker_launch_original(None, mid)
        f.launch_slice(b, N - b)
        for w, o in zip(whole, c["outs"]):
            assert host(o).tobytes() == w.tobytes()
    with pytest.raises(tk.TackerError):
        f.launch_slice(b, N - b + 1)
    ref, S = olc.lc_gemm(A, B)
    assert max_rel_err(host(D), ref, S) <= 1e-2


def test_launch_overlap_keeps_stream_order(tk):
    """Programmatic dependent launch: a chain where every kernel reads its predecessor's output
    (LC GEMM -> LC GEMM on the fp16 result, stencil ping-pong sweeps fused with them, an original
    BE sweep in between) gives the same bytes with overlap on and off."""
    M = N = K = 512
    A, B1 = synth.lc_gemm_inputs(M, N, K, seed=21)
    _, B2 = synth.lc_gemm_inputs(M, N, K, seed=22)
    S = synth.stencil_inputs(132, 64, 40, 23)

    def run():
        dA, dB1, dB2 = t(A), t(B1), t(B2)
        D1 = torch.zeros(M, N, dtype=torch.float16, device=dev())
        D2 = torch.zeros(M, N, dtype=torch.float16, device=dev())
        s0, s1 = t(S), torch.zeros(S.shape, device=dev())
        st01, st10 = tk.be_stencil(s0, s1), tk.be_stencil(s1, s0)
        g1 = tk.lc_gemm(dA, dB1, D1, b_const=True)
        g2 = tk.lc_gemm(D1, dB2, D2, b_const=True)
        f1, f2 = tk.tacker_fuse(g1, st01, 8), tk.tacker_fuse(g2, st10, 8)
        torch.cuda.synchronize()
        for _ in range(5):
            f1.launch()                                   # D1 = A B1 ; s1 = sweep(s0)
            f2.launch()                                   # D2 = D1 B2 ; s0 = sweep(s1)
            tk.tacker_launch_original(None, st01)         # s1 = sweep(s0)
            tk.tacker_launch_original(g2, st10)           # D2 again ; s0 = sweep(s1)
        return host(D2).tobytes(), host(s0).tobytes()

    tk.tacker_set_launch_overlap(False)
    try:
        ref = run()
    finally:
        tk.tacker_set_launch_overlap(2)
    for _ in range(3):
        assert run() == ref                               # default: PDL except original BE launches
    tk.tacker_set_launch_overlap(True)
    try:
        assert run() == ref                               # PDL on every launch
    finally:
        tk.tacker_set_launch_overlap(2)


@pytest.mark.parametrize("M,N,K", [(128, 256, 4096), (130, 264, 4104), (49, 512, 4608)])
def test_lc_split_k_vs_oracle(tk, M, N, K):
    """Split-K (few tiles, deep K): every unit on its own CTA, deterministic in-kernel fixup.
    Against the oracle, against the unsplit kernel, and repeatable (self-resetting counters)."""
    A, B = synth.lc_gemm_inputs(M, N, K, seed=K)
    dA, dB = t(A), t(B)
    D = torch.full((M, N), float("nan"), device=dev())
    D1 = torch.full((M, N), float("nan"), device=dev())
    f = tk.tacker_fuse(tk.lc_gemm(dA, dB, D, b_const=True), None, 0)
    assert f.info().lc_splits > 1 and f.info().grid == f.info().lc_tiles * f.info().lc_splits
    ref, S = olc.lc_gemm(A, B)
    outs = []
    for _ in range(3):
        D.fill_(float("nan"))
        f.launch()
        outs.append(host(D).tobytes())
        assert max_rel_err(host(D), ref, S) <= 1e-5
    assert outs[0] == outs[1] == outs[2]
    nd = tk.lc_gemm(dA, dB, D1)
    nd.epi_flags |= tk.LC_NO_SPLIT
    tk.tacker_launch_original(nd, None)
    assert max_rel_err(host(D1), ref, S) <= 1e-5


def test_fused_split_k_conv_bit_identical(tk):
    # layer4-like 3x3 conv (7x7 output, 4 tiles x 72 k-blocks -> 36 splits) fused with histo
    cs = synth.ConvShape("l4", 1, 7, 7, 512, 512, 3, 3, 1, 1)
    x, w, b = synth.conv_inputs(cs, seed=12)
    dx, dw, db = t(x), t(w), t(b)
    o0 = torch.zeros(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device=dev())
    o1 = torch.zeros_like(o0)
    c = be_case(tk.BE_HISTO, seed=4)
    c["reset"]()
    tk.tacker_launch_original(tk.lc_conv(dx, dw, o0, 1, 1, bias=db, relu=True, b_const=True), c["desc"])
    orig = [host(o).copy() for o in c["outs"]]
    f = tk.tacker_fuse(tk.lc_conv(dx, dw, o1, 1, 1, bias=db, relu=True, b_const=True), c["desc"], 16)
    assert f.info().lc_splits == 36
    for _ in range(2):
        c["reset"]()
        o1.zero_()
        f.launch()
        assert host(o1).tobytes() == host(o0).tobytes()
        for a, g in zip(orig, c["outs"]):
            assert host(g).tobytes() == a.tobytes()
    ref, S = olc.lc_conv(x, w, 1, 1, bias=b, relu=True)
    assert max_rel_err(host(o1).astype(np.float64), ref, S) <= 1e-2


def test_plans_of_one_instantiation_keep_their_smem(tk):
    # two plans of the same fused_kernel<BN, BE> with different SMEM sizes: building the smaller
    # one after the larger must not lower the function's dynamic-SMEM limit under the larger one
    A, B = synth.lc_gemm_inputs(256, 256, 128, seed=2)
    D = torch.zeros(256, 256, device=dev())
    c = be_case(tk.BE_STENCIL, seed=1)
    big = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), c["desc"], 24)
    small = tk.tacker_fuse(tk.lc_gemm(t(A), t(B), D), c["desc"], 4)
    assert big.info().smem_bytes > small.info().smem_bytes
    c["reset"]()
    big.launch()
    small.launch()
    torch.cuda.synchronize()


# ------------------------------------------------------------------ LC conv, halo mode (a5)
HALO_CASES = [synth.ConvShape("h14", 2, 14, 14, 64, 64, 3, 3, 1, 1),          # 76 % useful tiles, ragged p and q
              synth.ConvShape("h9x11", 2, 9, 11, 128, 72, 3, 3, 1, 1),        # 2 channel blocks, N % 64 != 0
              synth.ConvShape("h28", 3, 28, 28, 64, 128, 3, 3, 1, 1),
              synth.ConvShape("h56", 2, 56, 56, 64, 64, 3, 3, 1, 1),          # layer1 geometry
              synth.ConvShape("h14c256", 1, 14, 14, 256, 256, 3, 3, 1, 1),    # b1 layer3: split-K
              synth.ConvShape("h5x5", 1, 20, 17, 64, 64, 5, 5, 1, 2)]         # S = 5: halo 16 x 12


@pytest.mark.parametrize("bn", [64, 128])
@pytest.mark.parametrize("epi", ["bias_relu", "residual"])
@pytest.mark.parametrize("cs", HALO_CASES, ids=lambda c: c.name)
def test_lc_conv_halo_vs_oracle(tk, cs, epi, bn):
    """Halo mode (one input halo per filter row and channel block, tap-shifted UMMA descriptors):
    TMA-store epilogue (bias + ReLU) and the register epilogue (residual), vs the oracle."""
    x, w, b = synth.conv_inputs(cs, seed=5)
    res = np.random.default_rng(2).uniform(-1, 1, size=(cs.n, cs.p, cs.q, cs.k)).astype(np.float16)
    out = torch.zeros(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device=dev())
    lc = tk.lc_conv(t(x), t(w), out, cs.stride, cs.pad, bias=t(b), relu=True,
                    residual=t(res) if epi == "residual" else None, tile_n=bn)
    info = tk.tacker_fuse(lc, None, 0).info()
    assert info.lc_mode == tk.LC_MODE_CONV_HALO
    assert info.lc_tma_store == (1 if epi == "bias_relu" and info.lc_splits == 1 else 0)
    tk.tacker_launch_original(lc, None)
    ref, S = olc.lc_conv(x, w, cs.stride, cs.pad, bias=b, relu=True, residual=res if epi == "residual" else None)
    assert max_rel_err(host(out).astype(np.float64), ref, S) <= 1e-2


def test_lc_conv_halo_fused_bit_identical(tk):
    """A halo-mode conv fused with a BE kernel (register epilogue, BE warps beside the LC roles)
    writes the same bytes as its original launch."""
    cs = HALO_CASES[2]
    x, w, b = synth.conv_inputs(cs, seed=6)
    o0 = torch.zeros(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device=dev())
    o1 = torch.zeros_like(o0)
    c = be_case(tk.BE_SGEMM)
    c["reset"]()
    tk.tacker_launch_original(tk.lc_conv(t(x), t(w), o0, 1, 1, bias=t(b), relu=True, tile_n=64), None)
    f = tk.tacker_fuse(tk.lc_conv(t(x), t(w), o1, 1, 1, bias=t(b), relu=True, tile_n=64), c["desc"], 8)
    assert f.info().lc_mode == tk.LC_MODE_CONV_HALO
    f.launch()
    assert torch.equal(o0, o1)
    c["check"]([host(o) for o in c["outs"]])


# ------------------------------------------------------------------ LC conv, stride-2 phase halo (conv1)
S2C8_CASES = [synth.ConvShape("conv1_b2", 2, 224, 224, 8, 64, 7, 7, 2, 3),   # ResNet-50 conv1 (3 ch padded)
              synth.ConvShape("odd", 3, 30, 27, 8, 64, 7, 7, 2, 3),         # ragged p and q
              synth.ConvShape("5x5", 2, 33, 41, 8, 48, 5, 5, 2, 2),         # N 48 < 64, 13 tap pairs
              synth.ConvShape("3x3", 1, 20, 20, 8, 64, 3, 3, 2, 1)]


@pytest.mark.parametrize("epi", ["bias_relu", "residual"])
@pytest.mark.parametrize("cs", S2C8_CASES, ids=lambda c: c.name)
def test_lc_conv_s2c8_vs_oracle(tk, cs, epi):
    """conv1 as one implicit GEMM (phase-split halo, tap pairs as unswizzled K = 16 MMAs, resident
    weights), TMA-store (bias + ReLU) and register (residual) epilogues, vs the oracle."""
    x, w, b = synth.conv_inputs(cs, seed=7, real_c=3)
    res = np.random.default_rng(4).uniform(-1, 1, size=(cs.n, cs.p, cs.q, cs.k)).astype(np.float16)
    out = torch.zeros(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device=dev())
    lc = tk.lc_conv(t(x), t(w), out, cs.stride, cs.pad, bias=t(b), relu=True,
                    residual=t(res) if epi == "residual" else None)
    assert tk.tacker_fuse(lc, None, 0).info().lc_mode == tk.LC_MODE_CONV_S2C8
    tk.tacker_launch_original(lc, None)
    ref, S = olc.lc_conv(x, w, cs.stride, cs.pad, bias=b, relu=True, residual=res if epi == "residual" else None)
    assert max_rel_err(host(out).astype(np.float64), ref, S) <= 1e-2


def test_lc_conv_s2c8_fused_bit_identical(tk):
    cs = S2C8_CASES[1]
    x, w, b = synth.conv_inputs(cs, seed=8, real_c=3)
    o0 = torch.zeros(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device=dev())
    o1 = torch.zeros_like(o0)
    c = be_case(tk.BE_MRIQ_Q, seed=3)
    c["reset"]()
    tk.tacker_launch_original(tk.lc_conv(t(x), t(w), o0, 2, 3, bias=t(b), relu=True), None)
    f = tk.tacker_fuse(tk.lc_conv(t(x), t(w), o1, 2, 3, bias=t(b), relu=True), c["desc"], 16)
    assert f.info().lc_mode == tk.LC_MODE_CONV_S2C8
    f.launch()
    assert torch.equal(o0, o1)
    c["check"]([host(o) for o in c["outs"]])
