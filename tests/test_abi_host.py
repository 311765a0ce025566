"""CPU tests of the C ABI boundary (no GPU): the library loads and exports every symbol the
header declares, ctypes struct layouts equal the C compiler's, host-only calls (predictor,
simulated manager) agree with the oracle, and GPU-needing calls fail loudly without a GPU."""
import ctypes as C
import json
import math
import os
import re
import subprocess
import tempfile

import numpy as np
import pytest

from oracle import manager_ref as mr, predictor as op

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "tacker.h")


@pytest.fixture(scope="module")
def tk():
    from paper_conf_hpca_zhaocczlllg22_b200 import build, tacker
    build.build()
    return tacker


def header_functions():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(tacker_[a-z_0-9]+)\s*\(", src)))


def test_library_exports_every_declared_symbol(tk):
    lib = C.CDLL(tk.LIB_PATH)
    funcs = header_functions()
    assert len(funcs) >= 30
    for f in funcs:
        assert hasattr(lib, f), f"{f} declared in tacker.h but not exported"
    assert set(funcs) == set(tk.EXPORTED)


STRUCTS = {
    "tacker_lc_desc": "LcDesc", "tacker_be_desc": "BeDesc", "tacker_be_sgemm": "BeSgemm",
    "tacker_be_stencil": "BeStencil", "tacker_be_mriq_q": "BeMriqQ", "tacker_be_cutcp": "BeCutcp",
    "tacker_be_lbm": "BeLbm", "tacker_be_spmv": "BeSpmv", "tacker_be_histo": "BeHisto",
    "tacker_be_bfs_expand": "BeBfsExpand", "tacker_be_bfs_commit": "BeBfsCommit",
    "tacker_be_fma_burn": "BeFmaBurn", "tacker_be_im2col": "BeIm2col", "tacker_be_cutcp_bin": "BeCutcpBin",
    "tacker_be_copy": "BeCopy", "tacker_be_jds": "BeJds", "tacker_be_mrifhd_rhophi": "BeMrifhdRhophi",
    "tacker_be_mrifhd_fh": "BeMrifhdFh", "tacker_be_cp": "BeCp", "tacker_be_fft": "BeFft", "tacker_be_tpacf": "BeTpacf",
    "tacker_fused_info_t": "FusedInfo",
    "tacker_lc_kernel": "LcKernel", "tacker_be_kernel": "BeKernel", "tacker_decision": "Decision",
    "tacker_manager_params": "ManagerParams", "tacker_manager_stats": "ManagerStats", "tacker_ratio": "Ratio",
    "tacker_trace_rec": "TraceRec",
}


def test_struct_layouts_match_c(tk):
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "tacker.h"', "int main(void){"]
    for cs, py in STRUCTS.items():
        lines.append(f'printf("{py} %zu\\n", sizeof({cs}));')
    lines.append('printf("be.p %zu\\n", offsetof(tacker_be_desc, p));')
    lines.append('printf("lc.A %zu\\n", offsetof(tacker_lc_desc, A));')
    lines.append('printf("lk.cd %zu\\n", offsetof(tacker_lc_kernel, cd));')
    lines.append("return 0;}")
    with tempfile.TemporaryDirectory() as d:
        src = os.path.join(d, "l.c")
        exe = os.path.join(d, "l")
        open(src, "w").write("\n".join(lines))
        subprocess.check_call(["gcc", "-I", os.path.dirname(HDR), src, "-o", exe])
        out = subprocess.check_output([exe], text=True).split("\n")
    got = dict(l.split() for l in out if l.strip())
    for cs, py in STRUCTS.items():
        assert int(got[py]) == C.sizeof(getattr(tk, py)), (cs, got[py], C.sizeof(getattr(tk, py)))
    assert int(got["be.p"]) == tk.BeDesc.p.offset
    assert int(got["lc.A"]) == tk.LcDesc.A.offset
    assert int(got["lk.cd"]) == tk.LcKernel.cd.offset


def test_errors_without_gpu(tk):
    assert tk.tacker_device_sm_count() == 0 or tk.tacker_device_sm_count() >= 100
    with pytest.raises(tk.TackerError) as e:
        tk.tacker_fuse(tk.LcDesc(), None, 0)
    assert e.value.status in (tk.EINVAL, tk.EUNSUPPORTED, tk.ECUDA)
    # BE block counts are pure host arithmetic (PTB "original_block_num", Fig. 7)
    d = tk.BeDesc(kind=tk.BE_SGEMM)
    d.p.sgemm = tk.BeSgemm(256, 256, 256, 1.0, 0.0, 1, 1, 1)
    assert tk.tacker_be_num_blocks(d) == 16
    lc = tk.LcDesc(kind=tk.LC_GEMM_F16, M=300, N=136, K=200, A=16, B=16, D=8)
    with pytest.raises(tk.TackerError) as e:      # the epilogue's 16-byte stores need an aligned D
        tk.tacker_lc_num_tiles(lc, 64)
    assert e.value.status == tk.EINVAL
    lc.D = 16
    assert tk.tacker_lc_num_tiles(lc, 64) == 3 * 3
    assert tk.tacker_lc_num_tiles(lc, 128) == 3 * 2
    bad = tk.LcDesc(kind=tk.LC_GEMM_F16, M=16, N=12, K=16, A=1, B=1, D=1)
    with pytest.raises(tk.TackerError) as e:
        tk.tacker_lc_num_tiles(bad, 64)
    assert e.value.status == tk.EUNSUPPORTED   # N % 8 != 0


# ------------------------------------------------------------------ predictor: C vs oracle
def test_kernel_lr_c_matches_oracle(tk):
    tk.tacker_model_clear()
    rng = np.random.default_rng(5)
    m = op.KernelLR()
    for blocks in (16, 48, 100, 333, 512, 1024):
        ms = 0.0031 * blocks + 0.02 + rng.normal(0, 1e-3)
        tk.tacker_model_add_sample("k1", blocks, ms)
        m.add(blocks, ms)
    a, b = tk.tacker_model_fit("k1")
    ra, rb = m.fit()
    assert abs(a - ra) < 1e-12 and abs(b - rb) < 1e-12
    assert abs(tk.tacker_model_predict("k1", 700) - m.predict(700)) < 1e-12


def test_two_stage_c_matches_oracle_and_refits(tk):
    tk.tacker_model_clear()
    m = op.TwoStage()
    rng = np.random.default_rng(6)
    for r in (0.1, 0.2, 1.8, 1.9, 0.05, 2.5):
        xtc = rng.uniform(0.5, 3)
        tau = max(1 + 0.3 * r, 0.55 + 1.0 * r) * (1 + rng.normal(0, 0.01))
        tk.tacker_pair_add_sample("p", xtc, r * xtc, tau * xtc)
        m.add(xtc, r * xtc, tau * xtc)
    c = tk.tacker_pair_fit("p")
    (a1, b1), (a2, b2) = m.fit()
    assert np.allclose(c, (a1, b1, a2, b2), rtol=0, atol=1e-12)
    for r in (0.0, 0.3, 0.7, 1.2, 3.0):
        assert abs(tk.tacker_pair_predict("p", 2.0, 2.0 * r) - m.predict(2.0, 2.0 * r)) < 1e-12
    assert tk.tacker_pair_observe("p", 1.0, 0.5, m.predict(1.0, 0.5) * 1.3) == m.observe(1.0, 0.5, m.predict(1.0, 0.5) * 1.3)
    assert abs(tk.tacker_pair_predict("p", 1.0, 1.0) - m.predict(1.0, 1.0)) < 1e-12


def test_two_stage_inverted_slopes_c_matches_oracle(tk):
    # the single-LR fallback of reading 5 (stage slopes b1 >= b2): C == oracle
    tk.tacker_model_clear()
    m = op.TwoStage()
    for r in (0.2, 0.4, 0.6, 0.8, 1.5, 2.5, 4.0, 6.0):
        tau = 1 + 2.0 * r if r < 1 else 3.0 + (r - 1.0)
        tk.tacker_pair_add_sample("inv", 1.0, r, tau)
        m.add(1.0, r, tau)
    c = tk.tacker_pair_fit("inv")
    (a1, b1), (a2, b2) = m.fit()
    assert np.allclose(c, (a1, b1, a2, b2), rtol=0, atol=1e-12) and c[1] == c[3]
    for r in (0.1, 1.0, 7.0):
        assert abs(tk.tacker_pair_predict("inv", 1.0, r) - m.predict(1.0, r)) < 1e-12


def test_model_save_load_roundtrip(tk, tmp_path):
    tk.tacker_model_clear()
    for x in (1, 2, 3):
        tk.tacker_model_add_sample("a", x, 2 * x + 1)
    tk.tacker_model_fit("a")
    for r in (0.1, 0.2, 1.8, 1.9):
        tk.tacker_pair_add_sample("b", 1.0, r, max(1 + 0.1 * r, r))
    tk.tacker_pair_fit("b")
    p = str(tmp_path / "models.txt")
    tk.tacker_model_save(p)
    before = (tk.tacker_model_predict("a", 10), tk.tacker_pair_predict("b", 1.0, 0.7))
    tk.tacker_model_clear()
    with pytest.raises(tk.TackerError):
        tk.tacker_model_predict("a", 10)
    tk.tacker_model_load(p)
    assert (tk.tacker_model_predict("a", 10), tk.tacker_pair_predict("b", 1.0, 0.7)) == before


# ------------------------------------------------------------------ manager: C (simulated) vs oracle
FAKE = 0x10000


def lc_kernel(tk, is_tc, t):
    k = tk.LcKernel(is_tc=1 if is_tc else 0, t_pred_ms=t)
    if is_tc:
        k.lc = tk.LcDesc(kind=tk.LC_GEMM_F16, M=1024, N=1024, K=1024, A=FAKE, B=FAKE, D=FAKE)
    else:
        k.cd.kind = tk.BE_FMA_BURN
        k.cd.p.fma_burn = tk.BeFmaBurn(128, 10, 0.5, 0.125, FAKE)
    return k


def be_kernel(tk, t, ws=16):
    b = tk.BeKernel(is_cd=1, t_pred_ms=t, warp_split=ws)
    b.be.kind = tk.BE_STENCIL
    b.be.p.stencil = tk.BeStencil(64, 64, 8, 1 / 6, 1 / 36, FAKE, FAKE)
    return b


def be_kernel_tc(tk, t):
    b = tk.BeKernel(is_cd=0, is_tc=1, t_pred_ms=t)
    b.tc = tk.LcDesc(kind=tk.LC_GEMM_F16, M=512, N=512, K=512, A=FAKE, B=FAKE, D=FAKE)
    return b


def fit_reverse_pair_closed_form(tk, tau):
    # reverse pair (NEXT-2): BE gemm 512^3 as the tcgen05 part, the LC fma_burn (it10) as the
    # CUDA-core part, the LC kernel's default 16 warps
    key = "pair:lc:gemm:N512:K512:bn128:f32|be:fma_burn:it10|ws16"
    for r in (0.1, 0.2, 1.8, 1.9):
        tk.tacker_pair_add_sample(key, 1.0, r, tau(r))
    tk.tacker_pair_fit(key)
    return key


def fit_pair_closed_form(tk, tau):
    # the pair key of (gemm 1024^3, stencil nz=8, ws16), fitted exactly to tau(r) = max(l1, l2)
    key = "pair:lc:gemm:N1024:K1024:bn128:f32|be:stencil:nz8|ws16"
    for r in (0.1, 0.2, 1.8, 1.9):
        tk.tacker_pair_add_sample(key, 1.0, r, tau(r))
    tk.tacker_pair_fit(key)
    return key


@pytest.mark.parametrize("policy", ["tacker", "baymax", "tacker_reverse", "tacker_older", "tacker_noreorder",
                                    "tacker_reorder_always", "tacker_older_always", "tacker_direct_eps"])
def test_manager_simulation_matches_reference(tk, policy):
    tk.tacker_model_clear()
    # stage-2 slope != 1 so that Tgain depends on Tcd (with slope 1 every stage-2 pair has the
    # same gain (1 - a2) * Ttc and ties would be decided by rounding noise)
    tau = lambda r: max(1 + 0.25 * r, 0.4 + 0.93 * r)
    fit_pair_closed_form(tk, tau)
    fuse_pred = lambda ttc, tcd: ttc * tau(tcd / ttc)
    reverse = policy == "tacker_reverse"
    tau_r = lambda r: max(1 + 0.35 * r, 0.3 + 0.97 * r)
    fit_reverse_pair_closed_form(tk, tau_r)
    rfuse_pred = lambda xtc, xcd: xtc * tau_r(xcd / xtc)
    rng = np.random.default_rng(11)
    arrivals = np.cumsum(rng.exponential(6.0, 60))
    shapes = [[(True, 1.21), (False, 0.3), (True, 0.83), (True, 1.97)], [(True, 0.52), (True, 0.49)]]
    if reverse:   # LC CUDA-core kernels long enough to hide a BE tensor-core kernel
        shapes = [[(True, 1.21), (False, 1.3), (True, 0.83), (False, 0.61)], [(False, 0.92), (True, 0.49)]]
    app_ts = [[1.53, 0.71], [3.07], [0.43, 0.37, 2.51]]
    tc_apps = [[0.47, 1.12], [0.81]] if reverse else []
    pol = tk.POLICY_BAYMAX if policy == "baymax" else tk.POLICY_TACKER
    older = policy in ("tacker_older", "tacker_noreorder", "tacker_older_always")
    rule = {"tacker_noreorder": mr.REORDER_NEVER, "tacker_reorder_always": mr.REORDER_ALWAYS,
            "tacker_older_always": mr.REORDER_ALWAYS}.get(policy, mr.REORDER_UNFUSED)
    noreorder = rule == mr.REORDER_NEVER
    drule = mr.DIRECT_EPS if policy == "tacker_direct_eps" else mr.DIRECT_MIN_BE
    if older:   # a denser trace so that queries queue behind each other
        arrivals = np.cumsum(rng.exponential(3.3, 60))
    m = tk.Manager(pol, simulate=True, idle_cap_ms=2.0, fuse_older=older, older_margin_ms=0.7 if older else 0.0,
                   reorder_rule=rule, direct_rule=drule)
    qs = []
    for i, t in enumerate(arrivals):
        sh = shapes[i % 2]
        m.submit_lc([lc_kernel(tk, tc, d) for tc, d in sh], float(t))
        qs.append(mr.Query(i, float(t), list(sh)))
    apps = []
    for ts in app_ts:
        m.submit_be([be_kernel(tk, d) for d in ts])
        apps.append(mr.App([(True, d) for d in ts]))
    for ts in tc_apps:
        m.submit_be([be_kernel_tc(tk, d) for d in ts])
        apps.append(mr.App([(mr.BE_TC, d) for d in ts]))
    ref = mr.simulate(qs, apps, 50.0, mr.BAYMAX if policy == "baymax" else mr.TACKER, fuse_pred, idle_cap=2.0,
                      rfuse_pred=rfuse_pred, fuse_older=older, older_margin=0.7 if older else 0.0,
                      reorder_rule=rule, direct_rule=drule)
    if noreorder:
        assert all(not x.reorder for x in ref["decisions"] if x.action != mr.IDLE_BE)
    if older and not noreorder:   # older queries did fuse, which the paper-literal rule forbids
        lit = mr.simulate([mr.Query(q.qid, q.arrival, list(q.kernels)) for q in qs],
                          [mr.App(list(a.kernels)) for a in apps], 50.0, mr.TACKER, fuse_pred, idle_cap=2.0,
                          rfuse_pred=rfuse_pred)
        assert sum(d.action == mr.FUSED for d in ref["decisions"]) > sum(d.action == mr.FUSED for d in lit["decisions"])
    got = []
    for _ in range(100000):
        st = m.stats()
        if st.lc_queries_done == len(arrivals):
            break
        d = m.step(50.0)
        if d.action in (tk.DEC_FUSED, tk.DEC_ORIGINAL_LC, tk.DEC_REORDER_BE, tk.DEC_IDLE_BE):
            got.append((d.action, d.fused_app, tuple(d.reorder_apps[:d.n_reorder]), bool(d.reverse)))
    exp = [(x.action, x.fused_app, tuple(x.reorder), bool(x.reverse)) for x in ref["decisions"]]
    assert got == exp
    for i in range(len(arrivals)):
        assert abs(m.latency(i) - ref["latency"][i]) < 1e-9
    assert max(ref["latency"].values()) <= 50.0
    if policy != "baymax":
        assert m.stats().fused_launches > 0
    assert m.stats().reverse_fused == sum(1 for x in exp if x[3])
    if reverse:
        assert m.stats().reverse_fused > 0 and any(x[0] == mr.FUSED and not x[3] for x in exp)
    # be_work_ms = standalone time of every BE kernel issued, app heads cycling in order
    app_ts = app_ts + tc_apps
    work, pos = 0.0, [0] * len(app_ts)
    for _, fa, ra, _ in exp:
        for a in ([fa] if fa >= 0 else []) + list(ra):
            work += app_ts[a][pos[a] % len(app_ts[a])]
            pos[a] += 1
    assert abs(m.stats().be_work_ms - work) < 1e-9
    m.prepare()            # no-op on the simulated GPU
    m.prepare([lc_kernel(tk, True, 1.0)])


def be_kernel_sliced(tk, t, n, floor, ws=16):
    b = be_kernel(tk, t, ws)
    b.n_blocks, b.t_floor_ms, b.t_block_ms = n, floor, (t - floor) / n
    return b


@pytest.mark.parametrize("mode", ["opportune", "fixed", "opportune_always"])
def test_manager_slicing_matches_reference(tk, mode):
    """PTB slicing (reading 13): the C manager's decisions (incl. slice sizes), latencies and BE
    work equal the discrete-event reference's."""
    tk.tacker_model_clear()
    tau = lambda r: max(1 + 0.25 * r, 0.4 + 0.93 * r)     # r* = 0.6 / 0.68
    fit_pair_closed_form(tk, tau)
    fuse_pred = lambda ttc, tcd: ttc * tau(tcd / ttc)
    ratio = 1.3 if mode == "fixed" else 0.0
    rule = mr.REORDER_ALWAYS if mode == "opportune_always" else mr.REORDER_UNFUSED
    rng = np.random.default_rng(5)
    arrivals = np.cumsum(rng.exponential(7.0, 50))
    shapes = [[(True, 1.21), (False, 0.3), (True, 0.83), (True, 1.97)], [(True, 0.52), (True, 0.49)]]
    app_ts = [[(1.53, 64, 0.05), (0.71, 0, 0.0)], [(3.07, 200, 0.11)], [(0.43, 1, 0.4), (2.51, 37, 0.2)]]
    m = tk.Manager(tk.POLICY_TACKER, simulate=True, idle_cap_ms=2.0, slice_be=True, slice_ratio=ratio,
                   reorder_rule=rule)
    qs = []
    for i, tt in enumerate(arrivals):
        sh = shapes[i % 2]
        m.submit_lc([lc_kernel(tk, tc, d) for tc, d in sh], float(tt))
        qs.append(mr.Query(i, float(tt), list(sh)))
    apps = []
    for ts in app_ts:
        ks, rk = [], []
        for T, n, fl in ts:
            if n > 1:
                ks.append(be_kernel_sliced(tk, T, n, fl))
                rk.append((True, T, n, (T - fl) / n, fl))
            else:
                ks.append(be_kernel(tk, T))
                rk.append((True, T))
        m.submit_be(ks)
        apps.append(mr.App(rk))
    r_opp = 0.6 / 0.68
    ref = mr.simulate(qs, apps, 50.0, mr.TACKER, fuse_pred, idle_cap=2.0, slice_be=True, slice_ratio=ratio,
                      opp_ratio=lambda a: r_opp, reorder_rule=rule)
    got = []
    for _ in range(100000):
        if m.stats().lc_queries_done == len(arrivals):
            break
        d = m.step(50.0)
        if d.action in (tk.DEC_FUSED, tk.DEC_ORIGINAL_LC, tk.DEC_REORDER_BE, tk.DEC_IDLE_BE):
            got.append((d.action, d.fused_app, d.fused_blocks if d.action == tk.DEC_FUSED else -1,
                        tuple(d.reorder_apps[:d.n_reorder])))
    exp = [(x.action, x.fused_app, x.blocks if x.action == mr.FUSED else -1, tuple(x.reorder))
           for x in ref["decisions"]]
    assert got == exp
    assert any(x[0] == mr.FUSED and x[2] > 0 for x in exp), "no slice was fused"
    for i in range(len(arrivals)):
        assert abs(m.latency(i) - ref["latency"][i]) < 1e-9
    assert abs(m.stats().be_work_ms - ref["be_work"]) < 1e-9
    assert m.stats().be_kernels_done == sum(ref["be_completed"])


def test_training_prefixes_spread_over_the_latency_floor(tk):
    """Calibration host logic: the two-stage model's training prefixes are picked on the measured
    BE time curve; two prefixes on the one-block latency floor (the r01 sweep's degenerate stage-1
    fits) or a clamp at the whole kernel must not give coincident points."""
    from paper_conf_hpca_zhaocczlllg22_b200.qos import training_prefixes
    full = 1000
    t_of = lambda n: 0.04 + (0.0 if n < 8 else 0.0002 * (n - 8))      # floor 40 us up to 8 blocks
    curve = [(n, t_of(n)) for n in (1, 50, 125, 250, 500, 1000)]
    for x_tc in (0.05, 0.2, 1.0):
        out = training_prefixes(lambda n: n, full, x_tc, curve, t_of)
        ns = [n for n, _ in out]
        rs = [x / x_tc for _, x in out]
        assert ns == sorted(ns) and len(set(ns)) == len(ns) >= 3, ns
        gap = 0.08 if rs[-1] > 0.6 else 0.5 * (rs[-1] - rs[0]) / 5
        for i in range(1, len(ns)):
            assert rs[i] - rs[i - 1] >= gap - 1e-9 or ns[i] == full
        assert all(abs(x - t_of(n)) < 1e-12 for n, x in out)


@pytest.mark.parametrize("rule", ["min_be", "eps"])
def test_manager_s7_direct_launch_c(tk, rule):
    """S7 (tests/golden/manager_scenarios.json, hand-computed from P:2092-2096) through the C
    manager: Thr 2.5 <= the 3 ms ready BE head -> the whole query runs direct (min_be, default);
    with the eps reading the first kernel fuses (Thr 0.5) and the second does not."""
    s = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "manager_scenarios.json")))["S7"]
    tk.tacker_model_clear()
    # tau(r) = 1 + (2/3) r  ->  Tk_fuse = Ttc + (2/3) Tcd = Ttc + 2 for the 3 ms head
    fit_pair_closed_form(tk, lambda r: 1 + s["extra"] / s["be"] * r)
    m = tk.Manager(tk.POLICY_TACKER, simulate=True,
                   direct_rule=tk.DIRECT_MIN_BE if rule == "min_be" else tk.DIRECT_EPS)
    m.submit_lc([lc_kernel(tk, True, t) for t in s["kernels"]], 0.0)
    m.submit_be([be_kernel(tk, float(s["be"]))])
    names = {tk.DEC_FUSED: "FUSED", tk.DEC_ORIGINAL_LC: "ORIGINAL_LC", tk.DEC_REORDER_BE: "REORDER_BE"}
    got, thr = [], []
    for _ in range(100):
        if m.stats().lc_queries_done == 1:
            break
        d = m.step(s["qos"])
        if d.action in names and d.query >= 0:
            got.append(names[d.action])
            thr.append(d.thr_ms)
    assert got == s[rule]["actions"]
    assert abs(m.latency(0) - s[rule]["latency"]) < 1e-9
    if rule == "eps":
        assert abs(thr[0] - s["eps"]["thr_after_first"]) < 1e-9


@pytest.mark.parametrize("policy", ["tacker", "baymax", "tacker_reverse", "tacker_older_always", "tacker_noreorder"])
def test_manager_trace_replay_sim(tk, policy):
    """The C manager's decision trace (simulated GPU) replayed through manager_ref.replay: every
    decision, Tgain and headroom recomputed from the recorded observations matches (the same
    check the GPU-mode test applies to a hardware run)."""
    from tests.trace_check import check_trace
    tk.tacker_model_clear()
    tau = lambda r: max(1 + 0.25 * r, 0.4 + 0.93 * r)
    fit_pair_closed_form(tk, tau)
    reverse = policy == "tacker_reverse"
    fit_reverse_pair_closed_form(tk, lambda r: max(1 + 0.35 * r, 0.3 + 0.97 * r))
    rng = np.random.default_rng(17)
    arrivals = np.cumsum(rng.exponential(3.3, 60))
    shapes = [[(True, 1.21), (False, 0.3), (True, 0.83), (True, 1.97)], [(True, 0.52), (True, 0.49)]]
    if reverse:
        shapes = [[(True, 1.21), (False, 1.3), (True, 0.83), (False, 0.61)], [(False, 0.92), (True, 0.49)]]
    app_ts = [[1.53, 0.71], [3.07], [0.43, 0.37, 2.51]]
    tc_apps = [[0.47, 1.12], [0.81]] if reverse else []
    older = policy in ("tacker_older_always", "tacker_noreorder")
    rules = dict(fuse_older=older, older_margin=0.7 if older else 0.0,
                 reorder_rule={"tacker_older_always": mr.REORDER_ALWAYS,
                               "tacker_noreorder": mr.REORDER_NEVER}.get(policy, mr.REORDER_UNFUSED))
    pol = tk.POLICY_BAYMAX if policy == "baymax" else tk.POLICY_TACKER
    m = tk.Manager(pol, simulate=True, idle_cap_ms=2.0, fuse_older=older, older_margin_ms=rules["older_margin"],
                   reorder_rule=rules["reorder_rule"])
    m.trace_enable(100000)
    queries = []
    for i, t in enumerate(arrivals):
        sh = shapes[i % 2]
        m.submit_lc([lc_kernel(tk, tc, d) for tc, d in sh], float(t))
        queries.append((float(t), sh))
    apps = []
    for ts in app_ts:
        m.submit_be([be_kernel(tk, d) for d in ts])
        apps.append([(mr.BE_CD, d) for d in ts])
    for ts in tc_apps:
        m.submit_be([be_kernel_tc(tk, d) for d in ts])
        apps.append([(mr.BE_TC, d) for d in ts])
    m.run(50.0, float(arrivals[-1]))
    trace, dropped = m.trace_dicts()
    assert dropped == 0 and len(trace) > 100
    n = check_trace(trace, queries, apps, 50.0, mr.BAYMAX if policy == "baymax" else mr.TACKER,
                    idle_cap=2.0, **rules)
    assert n == len(trace)
    if policy != "baymax":
        assert any(d["action"] == tk.DEC_FUSED for d in trace)
    # a corrupted decision is caught
    bad = [dict(d) for d in trace]
    i = next(j for j, d in enumerate(bad) if d["action"] in (tk.DEC_ORIGINAL_LC, tk.DEC_REORDER_BE))
    bad[i]["thr"] += 0.5
    with pytest.raises(AssertionError):
        check_trace(bad, queries, apps, 50.0, mr.BAYMAX if policy == "baymax" else mr.TACKER, idle_cap=2.0, **rules)


def test_blacklist_and_manager_never_fuses_listed_kernel(tk):
    """NEXT-1: a blacklisted BE kernel is never fused; the C manager's decisions then
    equal the reference's with that app's kernels marked never-fusable."""
    tk.tacker_blacklist_clear()
    assert not tk.tacker_blacklist("be:stencil:nz8")
    assert tk.tacker_blacklist("be:stencil:nz8", 1)
    assert tk.tacker_blacklist("be:stencil:nz8", -1)
    assert not tk.tacker_blacklist("be:stencil:nz8", 0)
    tk.tacker_model_clear()
    tau = lambda r: max(1 + 0.25 * r, 0.4 + 0.93 * r)
    fit_pair_closed_form(tk, tau)
    fuse_pred = lambda ttc, tcd: ttc * tau(tcd / ttc)
    rng = np.random.default_rng(23)
    arrivals = np.cumsum(rng.exponential(6.0, 40))
    shapes = [[(True, 1.21), (False, 0.3), (True, 0.83)], [(True, 0.52), (True, 0.49)]]
    for listed in (False, True):
        if listed:
            tk.tacker_blacklist("be:stencil:nz8", 1)     # the BE kernels' model key (stencil nz=8)
        m = tk.Manager(tk.POLICY_TACKER, simulate=True, idle_cap_ms=2.0)
        qs = []
        for i, t in enumerate(arrivals):
            m.submit_lc([lc_kernel(tk, tc, d) for tc, d in shapes[i % 2]], float(t))
            qs.append(mr.Query(i, float(t), list(shapes[i % 2])))
        m.submit_be([be_kernel(tk, 1.53), be_kernel(tk, 0.71)])
        app = mr.App([(mr.BE_OTHER if listed else mr.BE_CD, 1.53), (mr.BE_OTHER if listed else mr.BE_CD, 0.71)])
        ref = mr.simulate(qs, [app], 50.0, mr.TACKER, fuse_pred, idle_cap=2.0)
        m.run(50.0, float(arrivals[-1]))
        assert m.stats().fused_launches == sum(d.action == mr.FUSED for d in ref["decisions"])
        assert (m.stats().fused_launches == 0) == listed
    tk.tacker_blacklist_clear()
