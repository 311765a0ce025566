"""GPU parity at the bench's own configurations (BASELINE configs[3], the timed run): every conv of
a ResNet-50 batch-32 query at the tile width the bench autotunes AND forced to BN 64 / 256, the
bias + ReLU (+ residual) fp16 epilogue, checked on sampled outputs against the oracle's direct
convolution (oracle/lc.py lc_conv_point) on the same seeded inputs; mri-q and mri-fhd at the
bench's 64^3 voxels with k ~ U[-32, 32) (two 1024-k chunks), sampled voxels against the oracle,
original and fused with a b32 conv (bit-identical)."""
import numpy as np
import pytest
import torch

import synth
from oracle import be as obe, lc as olc
from oracle.metrics import max_rel_err

pytestmark = pytest.mark.gpu

from tests.gpu_helpers import host  # noqa: E402

SEED = 2022           # bench.py's service seed (rank 0)
SAMPLES = 384         # sampled outputs per conv and tile width (plus the last row of the ragged M tail)


@pytest.fixture(scope="module")
def tk():
    from paper_conf_hpca_zhaocczlllg22_b200 import tacker
    assert torch.cuda.is_available()
    return tacker


def _positions(cs, rng, n):
    """Sampled (n, p, q, k) output positions: random ones plus the last output pixel (the ragged
    end of M = N P Q) and the first / last output channel."""
    pos = [(int(rng.integers(cs.n)), int(rng.integers(cs.p)), int(rng.integers(cs.q)), int(rng.integers(cs.k)))
           for _ in range(n)]
    pos += [(cs.n - 1, cs.p - 1, cs.q - 1, 0), (cs.n - 1, cs.p - 1, cs.q - 1, cs.k - 1), (0, 0, 0, cs.k - 1)]
    return pos


def _check_conv(out_np, x, w, b, cs, pos, residual=None, tol=1e-2):
    """max over sampled positions of |g - ref| / max(|ref|, abs-sum), ref = relu(conv + b (+ res))."""
    worst = 0.0
    for (n, p, q, k) in pos:
        acc, ab = olc.lc_conv_point(x, w, cs.stride, cs.pad, n, p, q, k)
        ref, S = acc + float(b[k]), ab + abs(float(b[k]))
        if residual is not None:
            r = float(residual[n, p, q, k])
            ref, S = ref + r, S + abs(r)
        ref = max(ref, 0.0)
        g = float(out_np[n, p, q, k])
        e = abs(g - ref) / max(abs(ref), S, 1e-30)
        worst = max(worst, e)
    assert worst <= tol, (cs.name, worst)
    return worst


def _bn_variants(tk, lc):
    """(label, desc) for the autotuned width (as the bench sets it) and forced BN 64 / 256."""
    import ctypes
    out = [("auto", lc)]
    for bn in (64, 256):
        d = tk.LcDesc()
        ctypes.memmove(ctypes.addressof(d), ctypes.addressof(lc), ctypes.sizeof(d))
        d.tile_n = bn
        out.append((f"bn{bn}", d))
    return out


def test_resnet50_b32_query_every_conv_vs_oracle(tk):
    """The timed run's LC service: all 53 convs (conv1 = im2col + GEMM) of a batch-32 query at
    the autotuned tile width and at BN 64 / 256, each vs the oracle on sampled outputs."""
    from paper_conf_hpca_zhaocczlllg22_b200 import services as sv
    svc = sv.resnet50_service(32, SEED)
    tuned = sv.autotune_tile_n(svc)
    assert len(tuned) == 53
    convs = synth.resnet50_convs(32)
    rng = np.random.default_rng(7)
    ki = 0
    checked = 0
    for i, cs in enumerate(convs):
        x, w, b = synth.conv_inputs(cs, SEED + i, real_c=3 if cs.name == "conv1" else None)
        k = svc.kernels[ki]
        if not k.is_tc:                   # conv1: the im2col kernel, then its GEMM
            tk.tacker_launch_original(None, k.cd)
            ki += 1
            k = svc.kernels[ki]
        assert k.is_tc and k.conv.name == cs.name
        pos = _positions(cs, rng, SAMPLES)
        for label, d in _bn_variants(tk, k.lc):
            k.out.zero_()
            try:
                tk.tacker_launch_original(d, None)
            except tk.TackerError as e:      # a width the planner rejects for this shape
                assert label != "auto", (cs.name, e)
                continue
            o = host(k.out)
            _check_conv(o, x, w, b, cs, pos)
            checked += 1
        ki += 1
    assert ki == len(svc.kernels)
    assert checked >= 53 * 2


@pytest.mark.parametrize("name", ["layer1.0.conv3", "layer2.0.conv2", "layer4.2.conv3"])
def test_b32_conv_residual_epilogue_vs_oracle(tk, name):
    """The bias + residual + ReLU fp16 epilogue at batch 32 (a bottleneck's last conv with its
    shortcut, and a strided 3x3), every tile width, sampled outputs vs the oracle."""
    cs = next(c for c in synth.resnet50_convs(32) if c.name == name)
    x, w, b = synth.conv_inputs(cs, 99)
    res = np.random.default_rng(5).uniform(-1, 1, size=(cs.n, cs.p, cs.q, cs.k)).astype(np.float16)
    dx, dw, db, dr = (torch.from_numpy(a).cuda() for a in (x, w, b, res))
    out = torch.empty(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device="cuda")
    lc = tk.lc_conv(dx, dw, out, cs.stride, cs.pad, bias=db, relu=True, residual=dr, b_const=True)
    pos = _positions(cs, np.random.default_rng(3), SAMPLES)
    for label, d in _bn_variants(tk, lc):
        out.zero_()
        try:
            tk.tacker_launch_original(d, None)
        except tk.TackerError:
            assert label != "auto"
            continue
        _check_conv(host(out), x, w, b, cs, pos, residual=res)


def _sampled(rng, n, nv):
    idx = np.sort(rng.choice(nv, size=n, replace=False))
    return np.unique(np.concatenate([idx, [0, nv - 1]]))


def test_mriq_bench_size_vs_oracle_and_fused(tk):
    """mri-q as the bench runs it: 64^3 voxels, 2048 k ~ U[-32, 32) (|k.x| up to 48 turns), phiMag
    then two accumulating 1024-k chunks; 2048 sampled voxels vs the oracle at the 1e-5 abs-sum
    gate, plus the median error relative to |Q| itself; then the chunks fused with a b32 conv
    must reproduce the original bytes."""
    from paper_conf_hpca_zhaocczlllg22_b200 import services as sv
    app = sv.mriq_app(64, 2048, 1024, SEED)
    Qr, Qi = app.buffers[2], app.buffers[3]
    for k in app.kernels:
        tk.tacker_launch_original(None, k.desc)
    gr, gi = host(Qr).copy(), host(Qi).copy()
    d = synth.mriq_inputs(64, 2048, SEED)
    idx = _sampled(np.random.default_rng(1), 2048, 64 ** 3)
    pm, _ = obe.mriq_phimag(d["phiR"], d["phiI"])
    rr, ri, Sr, Si = obe.mriq_q(d["x"][idx], d["y"][idx], d["z"][idx], d["kx"], d["ky"], d["kz"], pm)
    assert max_rel_err(gr[idx], rr, Sr) <= 1e-5
    assert max_rel_err(gi[idx], ri, Si) <= 1e-5
    # relative to |Q| itself (not the abs-sum): the fp32 phase of |t| <= 48 turns bounds it
    rel = np.abs(gr[idx] - rr) / np.maximum(np.abs(rr), 1e-30)
    assert np.median(rel) <= 1e-4, np.median(rel)
    # fused with a b32 conv: bit-identical to the original launches
    cs = next(c for c in synth.resnet50_convs(32) if c.name == "layer3.1.conv2")
    x, w, b = synth.conv_inputs(cs, 1)
    dx, dw, db = (torch.from_numpy(a).cuda() for a in (x, w, b))
    out = torch.empty(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device="cuda")
    lc = tk.lc_conv(dx, dw, out, cs.stride, cs.pad, bias=db, relu=True, b_const=True)
    Qr.zero_()
    Qi.zero_()
    for k in app.kernels[1:]:
        tk.tacker_fuse(lc, k.desc, 24).launch()
    assert np.array_equal(host(Qr), gr) and np.array_equal(host(Qi), gi)


def test_mrifhd_bench_size_vs_oracle(tk):
    """mri-fhd at the bench's size (64^3, 2048 k ~ U[-32, 32), RhoPhi + two FH chunks)."""
    from paper_conf_hpca_zhaocczlllg22_b200 import services as sv
    app = sv.mrifhd_app(64, 2048, 1024, SEED)
    Fr, Fi = app.buffers[3], app.buffers[4]
    for k in app.kernels:
        tk.tacker_launch_original(None, k.desc)
    gr, gi = host(Fr), host(Fi)
    d = synth.mrifhd_inputs(64, 2048, SEED)
    rho_r, rho_i, _, _ = obe.mrifhd_rhophi(d["phiR"], d["phiI"], d["dR"], d["dI"])
    idx = _sampled(np.random.default_rng(2), 2048, 64 ** 3)
    fr, fi, Sr, Si = obe.mrifhd_fh(d["x"][idx], d["y"][idx], d["z"][idx], d["kx"], d["ky"], d["kz"], rho_r, rho_i)
    assert max_rel_err(gr[idx], fr, Sr) <= 1e-5
    assert max_rel_err(gi[idx], fi, Si) <= 1e-5
