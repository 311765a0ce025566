"""Shared helpers for the -m gpu parity tests (the CUDA path goes through the C ABI)."""
import numpy as np
import torch

import synth
from oracle import be as obe


def dev():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    return torch.device("cuda:0")


def t(a, dtype=None):
    x = torch.from_numpy(np.ascontiguousarray(a))
    if dtype is not None:
        x = x.to(dtype)
    return x.to(dev())


def host(x):
    torch.cuda.synchronize()
    return x.cpu().numpy()


def be_case(kind, seed=0, size="small"):
    """Build (desc_builder, outputs, check) for a BE kind: returns dict with
    'desc' (tacker BeDesc), 'outs' (list of device tensors to compare), 'reset' (callable that
    restores the inputs/outputs before a launch), 'check' (callable(outs_np) -> None)."""
    from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk
    from oracle.metrics import max_rel_err
    g = np.random.default_rng(seed)
    if kind == tk.BE_SGEMM:
        M, N, K = (256, 256, 256) if size == "small" else (1024, 1536, 512)
        A, B = synth.sgemm_inputs(M, N, K, seed)
        dA, dB = t(A), t(B)
        dC = torch.zeros(M, N, device=dev())
        ref, S = obe.sgemm(A, B)

        def check(o):
            assert max_rel_err(o[0], ref, S) <= 1e-5
        return dict(desc=tk.be_sgemm(dA, dB, dC), outs=[dC], reset=lambda: dC.zero_(), check=check,
                    keep=(dA, dB))
    if kind == tk.BE_STENCIL:
        # small: float4 path (nx % 4 == 0) with a partial x tile and partial y / z blocks;
        # scalar: nx % 4 != 0 path
        nx, ny, nz = {"small": (132, 21, 19), "scalar": (70, 37, 9), "large": (512, 512, 64)}[size]
        A = synth.stencil_inputs(nx, ny, nz, seed)
        dA = t(A)
        dN = torch.zeros_like(dA)
        c0, c1 = np.float32(1 / 6), np.float32(1 / 36)
        ref, S = obe.stencil(A, c0, c1)

        def check(o):
            assert max_rel_err(o[0], ref, S) <= 1e-5
        return dict(desc=tk.be_stencil(dA, dN, float(c0), float(c1)), outs=[dN], reset=lambda: dN.zero_(),
                    check=check, keep=(dA,))
    if kind == tk.BE_MRIQ_Q:
        N, nk = (12, 700) if size == "small" else (32, 1024)
        d = synth.mriq_inputs(N, nk, seed)
        pm = (d["phiR"].astype(np.float32) ** 2 + d["phiI"].astype(np.float32) ** 2).astype(np.float32)
        dd = {k: t(v) for k, v in d.items()}
        dpm = t(pm)
        Qr = torch.zeros(N ** 3, device=dev())
        Qi = torch.zeros(N ** 3, device=dev())
        rr, ri, sr, si = obe.mriq_q(d["x"], d["y"], d["z"], d["kx"], d["ky"], d["kz"], pm)

        def check(o):
            assert max_rel_err(o[0], rr, sr) <= 1e-5
            assert max_rel_err(o[1], ri, si) <= 1e-5

        def reset():
            Qr.zero_()
            Qi.zero_()
        desc = tk.be_mriq_q(dd["x"], dd["y"], dd["z"], dd["kx"], dd["ky"], dd["kz"], dpm, Qr, Qi)
        return dict(desc=desc, outs=[Qr, Qi], reset=reset, check=check, keep=(dd, dpm))
    if kind == tk.BE_MRIQ_PHIMAG:
        nk = 3000
        d = synth.mriq_inputs(4, nk, seed)
        r, i = t(d["phiR"]), t(d["phiI"])
        out = torch.zeros(nk, device=dev())
        ref, S = obe.mriq_phimag(d["phiR"], d["phiI"])

        def check(o):
            assert max_rel_err(o[0], ref, S) <= 1e-5
        return dict(desc=tk.be_mriq_phimag(r, i, out), outs=[out], reset=lambda: out.zero_(), check=check,
                    keep=(r, i))
    if kind == tk.BE_LBM:
        nx, ny, nz = (20, 14, 11) if size == "small" else (120, 120, 150)
        f, fl = synth.lbm_inputs(nx, ny, nz, seed)
        df, dfl = t(f), t(fl.astype(np.uint32).view(np.int32))
        dst = torch.zeros_like(df)
        ref, S = obe.lbm_step(f, fl, np.zeros_like(f))
        mask = obe.lbm_written_mask(nx, ny, nz)

        def check(o):
            assert max_rel_err(o[0][mask], ref[mask], S[mask]) <= 1e-5
            assert np.all(o[0][~mask] == 0)
        return dict(desc=tk.be_lbm(df, dst, dfl), outs=[dst], reset=lambda: dst.zero_(), check=check, keep=(df, dfl))
    if kind == tk.BE_SPMV_JDS:
        R = 3000 if size == "small" else 1 << 16
        rp, cols, vals, x = synth.spmv_inputs(R, seed, mean_len=16)
        perm, rl, jp, jc, jv = obe.jds_build(rp, cols, vals)
        ds = [t(a) for a in (perm, rl, jp, jc, jv, x)]
        y = torch.zeros(R, device=dev())
        ref, S = obe.spmv_jds(perm, rl, jp, jc, jv, x)

        def check(o):
            assert max_rel_err(o[0], ref, S) <= 1e-5
        return dict(desc=tk.be_spmv(*ds, y), outs=[y], reset=lambda: y.zero_(), check=check, keep=ds)
    if kind == tk.BE_HISTO:
        n = 1035840 if size == "small" else 1 << 24
        v = synth.histo_inputs(n, 4096, seed, "skewed")
        dv = t(v.view(np.int32))
        cnt = torch.zeros(4096, dtype=torch.int32, device=dev())
        ref = obe.histo(v, 4096)

        def check(o):
            assert np.array_equal(o[0].view(np.uint32), ref)
            assert int(o[0].astype(np.int64).sum()) == n
        return dict(desc=tk.be_histo(dv, cnt, 4096), outs=[cnt], reset=lambda: cnt.zero_(), check=check, keep=(dv,))
    if kind == tk.BE_CUTCP:
        L = 16.0 if size == "small" else 48.0
        d = synth.cutcp_inputs(L, seed)
        nx = d["nx"]
        depth = 32
        bdim = tk.cutcp_bin_dims(nx, nx, nx)
        datoms = t(d["atoms"])
        bins = torch.zeros(bdim[0] * bdim[1] * bdim[2] * depth * 4, device=dev())
        count = torch.zeros(bdim[0] * bdim[1] * bdim[2], dtype=torch.int32, device=dev())
        ovf = torch.zeros(1, dtype=torch.int32, device=dev())
        tk.tacker_launch_original(None, tk.be_cutcp_bin(datoms, bins, count, ovf, nx, nx, nx, 0.5, depth))
        rb, rc = obe.cutcp_bins(d["atoms"], bdim, 4.0, depth)
        assert int(host(ovf)[0]) == 0
        assert np.array_equal(host(count), rc) and host(bins).tobytes() == rb.tobytes()
        V = torch.zeros(nx ** 3, device=dev())
        pts = None if size == "small" else np.random.default_rng(seed).choice(nx ** 3, 4096, replace=False)
        ref, S = obe.cutcp(d["atoms"], nx, nx, nx, 0.5, points=pts)

        def check(o):
            g = o[0] if pts is None else o[0][pts]
            assert max_rel_err(g, ref, S) <= 1e-5
        return dict(desc=tk.be_cutcp(bins, count, V, nx, nx, nx, 0.5, depth), outs=[V], reset=lambda: V.zero_(),
                    check=check, keep=(datoms, bins, count, ovf))
    if kind == tk.BE_MRIFHD_RHOPHI:
        nk = 3000
        d = synth.mrifhd_inputs(4, nk, seed)
        ins = [t(d[k]) for k in ("phiR", "phiI", "dR", "dI")]
        rr, ri = torch.zeros(nk, device=dev()), torch.zeros(nk, device=dev())
        ref_r, ref_i, sr, si = obe.mrifhd_rhophi(d["phiR"], d["phiI"], d["dR"], d["dI"])

        def check(o):
            assert max_rel_err(o[0], ref_r, sr) <= 1e-5
            assert max_rel_err(o[1], ref_i, si) <= 1e-5

        def reset():
            rr.zero_()
            ri.zero_()
        return dict(desc=tk.be_mrifhd_rhophi(*ins, rr, ri), outs=[rr, ri], reset=reset, check=check, keep=ins)
    if kind == tk.BE_MRIFHD_FH:
        N, nk = (12, 700) if size == "small" else (32, 1024)
        d = synth.mrifhd_inputs(N, nk, seed)
        # the FH inputs are fp32 RhoPhi values; both sides take the same fp32 array
        r64, i64, _, _ = obe.mrifhd_rhophi(d["phiR"], d["phiI"], d["dR"], d["dI"])
        rr, ri = r64.astype(np.float32), i64.astype(np.float32)
        dd = {k: t(d[k]) for k in ("x", "y", "z", "kx", "ky", "kz")}
        drr, dri = t(rr), t(ri)
        Fr, Fi = torch.zeros(N ** 3, device=dev()), torch.zeros(N ** 3, device=dev())
        ref_r, ref_i, sr, si = obe.mrifhd_fh(d["x"], d["y"], d["z"], d["kx"], d["ky"], d["kz"], rr, ri)

        def check(o):
            assert max_rel_err(o[0], ref_r, sr) <= 1e-5
            assert max_rel_err(o[1], ref_i, si) <= 1e-5

        def reset():
            Fr.zero_()
            Fi.zero_()
        desc = tk.be_mrifhd_fh(dd["x"], dd["y"], dd["z"], dd["kx"], dd["ky"], dd["kz"], drr, dri, Fr, Fi)
        return dict(desc=desc, outs=[Fr, Fi], reset=reset, check=check, keep=(dd, drr, dri))
    if kind == tk.BE_CP:
        # small: 2 x-tiles (ragged), 4 row blocks (ragged), 2 atom stages (ragged)
        natoms, nx, ny, h = (700, 200, 13, 0.5) if size == "small" else (4000, 256, 256, 0.5)
        at, z = synth.cp_inputs(natoms, nx, ny, h, seed)
        dat = t(at)
        V = torch.zeros(ny, nx, device=dev())
        ref, S = obe.cp(at, nx, ny, h, z)

        def check(o):
            assert max_rel_err(o[0].ravel(), ref, S) <= 1e-5
        return dict(desc=tk.be_cp(dat, V, h, z), outs=[V], reset=lambda: V.zero_(), check=check, keep=(dat,))
    if kind in (tk.BE_FFT, tk.BE_FFT_TWIDDLE):
        # radix passes (first pass reads global, last writes global): small n = 256 (4, 8, 8);
        # "odd" n = 1024 (16, 8, 8); "mid" n = 128 (16, 8); "tiny" n = 2 (2); "single16" n = 16 and
        # "single8" n = 8 (one pass, global in and out); "two" n = 32 (4, 8); large: the bench shape
        # on sampled rows
        batch, n = {"small": (37, 256), "odd": (7, 1024), "mid": (11, 128), "tiny": (3, 2),
                    "single16": (5, 16), "single8": (6, 8), "two": (9, 32),
                    "large": (1 << 14, 1024)}[size]
        x = synth.fft_inputs(batch, n, seed)
        dx = t(x)
        tw = torch.zeros(n, 2, device=dev())
        y = torch.zeros_like(dx)
        if kind == tk.BE_FFT_TWIDDLE:
            # the twiddles are the DFT of impulses at 1: pinned through the oracle's DFT
            X, _ = obe.fft(np.eye(n)[1:2])

            def check(o):
                assert np.max(np.abs(o[0][:, 0] - X[0].real)) <= 2e-7 and np.max(np.abs(o[0][:, 1] - X[0].imag)) <= 2e-7
            return dict(desc=tk.be_fft_twiddle(tw, n), outs=[tw], reset=lambda: tw.zero_(), check=check, keep=())
        tk.tacker_launch_original(None, tk.be_fft_twiddle(tw, n))
        rows = np.arange(batch) if size != "large" else np.random.default_rng(seed).choice(batch, 64, replace=False)
        X, S = obe.fft(x[rows, :, 0].astype(np.float64) + 1j * x[rows, :, 1])

        def check(o):
            g = o[0][rows]
            assert max_rel_err(g[..., 0], X.real, S) <= 1e-5
            assert max_rel_err(g[..., 1], X.imag, S) <= 1e-5
        return dict(desc=tk.be_fft(dx, y, tw), outs=[y], reset=lambda: y.zero_(), check=check, keep=(dx, tw))
    if kind == tk.BE_TPACF:
        # small: self pairs over a ragged point count (3 b stages, 5 blocks); cross pairs below
        n = 600 if size == "small" else 8192
        e = synth.tpacf_edges()
        A = synth.tpacf_inputs(n, seed)
        dA, de = t(A), t(e)
        cnt = torch.zeros(len(e) + 1, dtype=torch.int32, device=dev())
        ref = obe.tpacf(A, A, e, True)

        def check(o):
            assert np.array_equal(o[0].view(np.uint32).astype(np.int64), ref)
        return dict(desc=tk.be_tpacf(dA, dA, de, cnt, self_pairs=True), outs=[cnt], reset=lambda: cnt.zero_(),
                    check=check, keep=(dA, de))
    if kind == tk.BE_FMA_BURN:
        n, iters = 128 * 300, 1000
        out = torch.zeros(n, device=dev())
        ref = obe.fma_burn(n, iters)

        def check(o):
            assert max_rel_err(o[0], ref) <= 1e-5
        return dict(desc=tk.be_fma_burn(out, iters), outs=[out], reset=lambda: out.zero_(), check=check, keep=())
    raise ValueError(kind)
