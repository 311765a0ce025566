"""Pins for the host-side oracle: fusion index mapping (Fig. 5/6), PTB coverage (Fig. 7),
fusion budget (§V-C), predictor (§VI), manager (§VII) and metrics (Eqs. 10/11)."""
import json
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import fusion, manager_ref as mr, metrics, predictor

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ------------------------------------------------------------------ Fig. 6 worked example
def test_fig6_direct_fusion_worked_example():
    g = gold("fig6_direct_fusion.json")
    grid, block, role = fusion.direct_fusion_map(g["block_num_tc"], g["thread_num_tc"],
                                                 g["block_num_cd"], g["thread_num_cd"])
    assert (grid, block) == (g["fused_grid"], g["fused_block"])
    lo, hi = g["cd_thread_range"]
    for b in range(grid):
        for t in range(lo, hi + 1):
            assert role[b][t] == ("cd", b, t - lo)
        for t in range(lo):
            if b in g["idle_tc_blocks"]:
                assert role[b][t] is None
            else:
                assert role[b][t] == ("tc", b, t)


# ------------------------------------------------------------------ Fig. 7 PTB
@settings(max_examples=200, deadline=None)
@given(st.integers(0, 3000), st.integers(1, 400))
def test_ptb_visits_every_block_exactly_once(orig, issued):
    v = fusion.ptb_visits(orig, issued)
    flat = sorted(x for row in v for x in row)
    assert flat == list(range(orig))


def test_ptb_figure_bound_reading():
    # Fig. 7 literally uses `<=`, which would visit block `original_block_num`: reading `<`.
    assert fusion.ptb_visits(4, 3) == [[0, 3], [1], [2]]


# ------------------------------------------------------------------ §V-C budget
def test_sec5c_budget_example():
    g = gold("sec5c_budget.json")
    cap = g["smem_capacity"]
    assert g["tc_smem"] + g["cd_smem"] == g["one_to_one_block_smem"]
    assert fusion.fused_blocks_per_sm(1, g["tc_smem"], 1, g["cd_smem"], cap) == g["one_to_one_blocks_per_sm"]
    r = fusion.flexible_ratio(g["tc_blocks_needed"], g["tc_smem"], g["cd_smem"], cap)
    assert list(r) == g["flexible_ratio"]
    assert fusion.fused_blocks_per_sm(r[0], g["tc_smem"], r[1], g["cd_smem"], cap) == g["flexible_blocks_per_sm"]
    assert fusion.fused_blocks_per_sm(3, g["tc_smem"], 1, g["cd_smem"], cap) == 0   # over budget: no fusion


# ------------------------------------------------------------------ predictor
def test_ols_matches_polyfit():
    rng = np.random.default_rng(0)
    x = rng.uniform(1, 100, 20)
    y = 0.37 * x + 5.0 + rng.normal(0, 0.3, 20)
    a, b = predictor.ols(list(x), list(y))
    pa, pb = np.polyfit(x, y, 1)
    assert abs(a - pa) < 1e-12 and abs(b - pb) < 1e-10


def test_kernel_lr_exact_recovery():
    m = predictor.KernelLR()
    for blocks in (16, 32, 64, 128, 256, 512):
        m.add(blocks, 0.002 * blocks + 0.011)
    a, b = m.fit()
    assert abs(a - 0.002) < 1e-15 and abs(b - 0.011) < 1e-13
    assert abs(m.predict(1000) - 2.011) < 1e-12


def closed_form_tau(r, r_o=0.8, tau_o=1.25):
    # Eqs. 3-6 reading: stage 1 linear from tau(0)=1 to (r_o, tau_o); stage 2 slope 1 after r_o
    return 1 + (tau_o - 1) * r / r_o if r <= r_o else tau_o + (r - r_o)


def test_two_stage_recovers_closed_form():
    m = predictor.TwoStage()
    xtc = 3.0
    for r in predictor.TRAIN_RATIOS:
        m.add(xtc, r * xtc, xtc * closed_form_tau(r))
    m.fit()
    assert abs(m.inflection() - 0.8) < 1e-12
    assert abs(m.l2[1] - 1.0) < 1e-12   # slope 1 after the inflection
    for r in np.linspace(0.01, 3, 40):
        for x in (0.5, 3.0, 11.0):      # linear in X_tc at fixed r (Fig. 11)
            assert abs(m.predict(x, r * x) - x * closed_form_tau(r)) < 1e-10


def test_two_stage_online_refit():
    m = predictor.TwoStage()
    for r in predictor.TRAIN_RATIOS:
        m.add(1.0, r, closed_form_tau(r))
    m.fit()
    assert not m.observe(1.0, 0.5, closed_form_tau(0.5) * 1.05)      # 5 % error: keep
    assert m.observe(1.0, 0.5, closed_form_tau(0.5) * 1.3)           # 30 % error: refit
    assert len(m.samples) == 5


# ------------------------------------------------------------------ manager
def heads_and_pred(spec):
    heads = [(a, tcd, True) for a, tcd, _ in spec["heads"]]
    tf = {a: f for a, _, f in spec["heads"]}
    return heads, (lambda a: tf[a])


@pytest.mark.parametrize("sid", ["S1", "S2", "S3", "S4", "S6", "S3_reorder_always", "S6_reorder_always"])
def test_manager_scenarios(sid):
    s = gold("manager_scenarios.json")[sid]
    heads, fp = heads_and_pred(s)
    rule = mr.REORDER_ALWAYS if sid.endswith("_reorder_always") else mr.REORDER_UNFUSED
    fused, reorder, thr, gain = mr.decide(s["ttc"], True, s["thr"], heads, mr.TACKER, fp, reorder_rule=rule)
    assert fused == s["fused"]
    assert reorder == s["reorder"]
    assert abs(thr - s["thr_after"]) < 1e-12
    if "gain" in s:
        assert abs(gain - s["gain"]) < 1e-12


def test_manager_baymax_never_fuses():
    s = gold("manager_scenarios.json")["S1"]
    heads, fp = heads_and_pred(s)
    fused, reorder, thr, _ = mr.decide(s["ttc"], True, s["thr"], heads, mr.BAYMAX, fp)
    assert fused == -1 and reorder == [0] and thr == 37


@pytest.mark.parametrize("rule", ["min_be", "eps"])
def test_manager_s7_direct_launch(rule):
    """S7 (golden, hand-computed): Thr close to 0 -> every kernel of the query launched directly."""
    s = gold("manager_scenarios.json")["S7"]
    q = mr.Query(0, 0.0, [(True, t) for t in s["kernels"]])
    app = mr.App([(True, float(s["be"]))])
    fp = lambda ttc, tcd: ttc + s["extra"]
    res = mr.simulate([q], [app], s["qos"], mr.TACKER, fp,
                      direct_rule=mr.DIRECT_MIN_BE if rule == "min_be" else mr.DIRECT_EPS)
    names = {mr.FUSED: "FUSED", mr.ORIGINAL_LC: "ORIGINAL_LC", mr.REORDER_BE: "REORDER_BE"}
    lc_dec = [d for d in res["decisions"] if d.lc is not None]
    assert [names[d.action] for d in lc_dec] == s[rule]["actions"]
    assert res["latency"][0] == s[rule]["latency"]
    if rule == "eps":
        assert abs(lc_dec[0].thr - s["eps"]["thr_after_first"]) < 1e-12
        assert lc_dec[0].reorder == []


def test_manager_eq9_headroom_two_queries():
    s = gold("manager_scenarios.json")["S5"]
    # earlier query (12 ms remaining) still active when Q (Tori_solo 10) is issued
    q_old = mr.Query(0, 0.0, [(True, 12.0)])
    q_new = mr.Query(1, 0.0, [(True, 5.0), (True, 5.0)])
    res = mr.simulate([q_old, q_new], [], s["qos"], mr.TACKER, lambda a, b: None)
    # q_new issues at t=12 after q_old; Tqueue = 12 so Thr = 50 - 12 - 10 - 0 = 28 (== S5)
    assert res["latency"] == {0: 12.0, 1: 22.0}
    q_new2 = mr.Query(1, 0.0, [(True, 5.0), (True, 5.0)])
    thr = s["qos"] - s["tqueue"] - s["tori_solo"] - sum(s["earlier_remaining"])
    assert thr == s["thr"] and q_new2.remaining() == 10.0


def test_manager_fig13_schedule():
    # Fig. 13: Q = [TC1, CD1, ..., TCn]; BE task 0 = [CD1, CD2]: Q-TC1 fuses with
    # a BE CD kernel, later Q-CD kernels are followed by reordered BE kernels while headroom lasts.
    q = mr.Query(0, 0.0, [(True, 2.0), (False, 1.0), (True, 2.0)])
    apps = [mr.App([(True, 3.0), (True, 3.0)])]
    fp = lambda ttc, tcd: 4.0 if ttc == 2.0 else None
    res = mr.simulate([q], apps, 50.0, mr.TACKER, fp)
    kinds = [e[0] for e in res["timeline"]]
    assert kinds[0] == "fused"                   # FUSE1 = Q-TC1 + B-CD
    assert "be" in kinds[1:]                     # a reordered BE kernel follows
    assert res["latency"][0] <= 50.0


def test_manager_qos_holds_and_tacker_beats_baymax():
    rng = np.random.default_rng(3)
    arrivals = np.cumsum(rng.exponential(20.0, 200))
    mk = lambda: [mr.Query(i, float(t), [(True, 1.5), (False, 0.5)] * 4) for i, t in enumerate(arrivals)]
    apps = lambda: [mr.App([(True, 2.0)]), mr.App([(True, 3.0), (True, 1.0)])]
    fp = lambda ttc, tcd: max(ttc, tcd) + 0.2 * min(ttc, tcd)
    out = {}
    for pol in (mr.BAYMAX, mr.TACKER):
        a = apps()
        res = mr.simulate(mk(), a, 50.0, pol, fp, idle_cap=5.0)
        assert max(res["latency"].values()) <= 50.0 + 1e-9
        out[pol] = sum(x.completed for x in a) / res["t"]
    assert out[mr.TACKER] > out[mr.BAYMAX]


def test_manager_slice_to_opportune_ratio():
    """Reading 13, hand-computed: TC kernel 2 ms; BE head 10 ms = 100 blocks,
    X_cd(n) = 0.1 n; tau(r) = max(1 + 0.1 r, 0.5 + r) -> r* = 0.5/0.9 = 5/9 (Fig. 10 inflection).
    Slice n = ceil(r* 2 / 0.1) = ceil(11.1) = 12 blocks: Tcd = 1.2, Tk_fuse = 2 tau(0.6) = 2.2,
    Tgain = 1.2 - 0.2 = 1.0 (Eq. 8 holds), Thr 48 -> 47.8; the query ends at 2.2 and the idle GPU
    then runs the other 88 blocks (X_cd(88) = 8.8 ms, ending at 11.0) before a second query
    arrives at 20 (one 1 ms CUDA-core kernel, behind which the app's next 30 ms kernel is
    reordered).  Whole-kernel fusion has the same Tgain (Tk_fuse = 2 tau(5) = 11, Tgain =
    10 - 9 = 1) but costs 9 ms of headroom and an 11 ms query."""
    tau = lambda r: max(1 + 0.1 * r, 0.5 + r)
    fp = lambda ttc, tcd: ttc * tau(tcd / ttc)
    for sliced, lat, thr_after, blocks in ((True, 2.2, 47.8, 12), (False, 11.0, 39.0, -1)):
        qs = [mr.Query(0, 0.0, [(True, 2.0)]), mr.Query(1, 20.0, [(False, 1.0)])]
        app = mr.App([(True, 10.0, 100, 0.1, 0.0), (True, 30.0)])
        res = mr.simulate(qs, [app], 50.0, mr.TACKER, fp, slice_be=sliced, opp_ratio=lambda a: 5 / 9,
                          idle_cap=9.0)
        d0 = res["decisions"][0]
        assert d0.action == mr.FUSED and d0.blocks == blocks
        assert abs(d0.gain - 1.0) < 1e-12 and abs(d0.thr - thr_after) < 1e-12
        assert abs(res["latency"][0] - lat) < 1e-12
        if sliced:
            d1 = res["decisions"][1]
            assert d1.action == mr.IDLE_BE and d1.reorder == [0]
            assert [e for e in res["timeline"] if e[0] == "be"][0][4:] == (2.2, 2.2 + 8.8)
        # both kernels complete (the 30 ms one is reordered behind query 1): 10 + 30 ms of work
        assert abs(res["be_work"] - 40.0) < 1e-12 and res["be_completed"] == [2]


def test_manager_reverse_fusion_scenarios():
    """NEXT-2, hand-computed (Thr 40 as in S1-S7): LC CUDA-core kernel 2 ms, BE tensor-core head
    3 ms, Tk_fuse 4 -> Eq. 8 holds (5 > 4, 4 - 2 = 2 < 40): FUSED, Tgain 3 - 2 = 1, Thr 38.
    Tk_fuse 5 -> not admitted (strict >): the head is reordered (3 < 40), Thr 37.  A CUDA-core
    head never pairs with a CUDA-core LC kernel, nor a tensor-core head with a tensor-core one."""
    fp = lambda a: {0: 4.0, 1: 4.5}[a]
    fused, reorder, thr, gain, rev = mr.decide(2.0, False, 40.0, [(0, 3.0, mr.BE_TC)], mr.TACKER, fp,
                                               with_reverse_flag=True)
    assert (fused, reorder, rev) == (0, [], True) and thr == 38.0 and gain == 1.0
    fused, reorder, thr, _ = mr.decide(2.0, False, 40.0, [(0, 3.0, mr.BE_TC)], mr.TACKER, lambda a: 5.0)
    assert (fused, reorder, thr) == (-1, [0], 37.0)
    # two tensor-core heads: gains 1 (3 ms, 4.0) and 3 - 2.5 = 0.5 (3 ms, 4.5): the first wins;
    # paper rule: nothing reordered after a fused launch (Thr 38); reading 6: head 1 too (Thr 35)
    heads2 = [(0, 3.0, mr.BE_TC), (1, 3.0, mr.BE_TC)]
    fused, reorder, thr, gain = mr.decide(2.0, False, 40.0, heads2, mr.TACKER, fp)
    assert fused == 0 and gain == 1.0 and reorder == [] and thr == 38.0
    fused, reorder, thr, gain = mr.decide(2.0, False, 40.0, heads2, mr.TACKER, fp, reorder_rule=mr.REORDER_ALWAYS)
    assert fused == 0 and gain == 1.0 and reorder == [1] and thr == 35.0
    assert mr.decide(2.0, False, 40.0, [(0, 3.0, mr.BE_CD)], mr.TACKER, lambda a: 1.0)[0] == -1
    assert mr.decide(2.0, True, 40.0, [(0, 3.0, mr.BE_TC)], mr.TACKER, lambda a: 1.0)[0] == -1
    assert mr.decide(2.0, False, 40.0, [(0, 3.0, mr.BE_TC)], mr.TACKER, fp, reverse=False)[0] == -1
    assert mr.decide(2.0, False, 40.0, [(0, 3.0, mr.BE_TC)], mr.BAYMAX, fp)[0] == -1
    # in a run: TC kernel (1 ms, no CUDA-core head to fuse) with the 3 ms tensor-core head
    # reordered behind it (Thr 47); the CUDA-core kernel then fuses with the app's next
    # tensor-core kernel (Tk_fuse 4): latency 1 + 3 + 4 = 8, two BE kernels (6 ms of work)
    q = mr.Query(0, 0.0, [(True, 1.0), (False, 2.0)])
    app = mr.App([(mr.BE_TC, 3.0)])
    res = mr.simulate([q], [app], 50.0, mr.TACKER, lambda ttc, tcd: None, rfuse_pred=lambda xtc, xcd: 4.0)
    d0, d1 = res["decisions"][:2]
    assert d0.action == mr.REORDER_BE and d0.reorder == [0] and abs(d0.thr - 44.0) < 1e-12
    assert d1.action == mr.FUSED and d1.reverse and d1.fused_app == 0 and abs(d1.thr - 42.0) < 1e-12
    assert res["latency"][0] == 8.0 and res["be_completed"] == [2] and res["be_work"] == 6.0


def test_manager_fuse_older_respects_later_headroom():
    """Reading 18, hand-computed.  Q0 (arrives 0): [TC 2, TC 2]; Q1 arrives at 1: [TC 3].  BE app:
    CUDA-core kernel 4 ms, Tk_fuse = ttc + 1.5 for any pair (extra 1.5, gain 2.5).
    At t=0 Q0 is alone (newest): Thr0 = 50 - 4 = 46, fused (Thr0 44.5), ends at 3.5.  At 3.5 Q1
    has arrived, so Q0 is no longer the newest: paper rule -> Q0's second kernel runs plain;
    fuse_older -> Thr_eff = min(44.5, 50 - (3.5 - 1) - (2 + 3)) = 42.5 -> fused again, and Q1
    still has 50 - 2.5 - 3 - 3.5 (extra) >= 0 left."""
    fp = lambda ttc, tcd: ttc + 1.5
    for older, n_fused in ((False, 1), (True, 2)):
        qs = [mr.Query(0, 0.0, [(True, 2.0), (True, 2.0)]), mr.Query(1, 1.0, [(True, 3.0)])]
        apps = [mr.App([(True, 4.0)])]
        res = mr.simulate(qs, apps, 50.0, mr.TACKER, fp, fuse_older=older)
        q0 = [d for d in res["decisions"] if d.lc and d.lc[0] == 0]
        assert sum(d.action == mr.FUSED for d in q0) == n_fused
        if older:
            assert abs(q0[1].thr - (44.5 - 1.5)) < 1e-12   # Q0's own headroom pays the extra
    # a later query with no headroom left blocks the older query's fusion
    qs = [mr.Query(0, 0.0, [(True, 2.0), (True, 2.0)]), mr.Query(1, 1.0, [(True, 47.0)])]
    res = mr.simulate(qs, [mr.App([(True, 4.0)])], 50.0, mr.TACKER, fp, fuse_older=True)
    q0 = [d for d in res["decisions"] if d.lc and d.lc[0] == 0]
    assert q0[0].action == mr.FUSED and q0[1].action != mr.FUSED


# ------------------------------------------------------------------ metrics
def test_overlap_rate_bounds():
    assert metrics.overlap_rate(1.0, 1.0, 1.0) == 0.5      # perfect overlap
    assert metrics.overlap_rate(1.0, 1.0, 2.0) == 0.0      # sequential
    assert metrics.throughput_improvement(118.6, 100.0) == pytest.approx(0.186)


def test_rel_err_uses_abs_sum():
    assert metrics.max_rel_err([1e-3], [0.0], [1.0]) == pytest.approx(1e-3)
    assert metrics.max_rel_err([2.0], [1.0]) == 1.0


def test_two_stage_refit_keeps_two_samples_per_stage():
    """Reading 5: the iterative re-split at r* never leaves a stage one sample.  Pin:
    the samples of a measured pair (BERT O-projection GEMM x cutcp, ws 24; r = X_cd / X_tc,
    tau = T_fused / X_tc) whose two stages are nearly parallel: r* lands beyond all but the last
    sample, and the old rule re-split to {5 | 1} samples, fitting a flat stage 2 (slope 0) through the
    single point -- every prediction below r = 17 became that point's tau (errors up to 3.7x on the
    pair's held-out prefixes).  Kept at the median split, both stages have slope ~1."""
    r = [1.529, 2.027, 3.333, 4.558, 8.204, 16.31]
    tau = [2.471, 3.288, 4.258, 5.623, 8.747, 17.416]
    m = predictor.TwoStage()
    for x, y in zip(r, tau):
        m.add(1.0, x, y)
    (a1, b1), (a2, b2) = m.fit()
    assert b2 > 0.5 and b1 > 0.5                     # neither stage flat
    for x, y in ((3.456, 4.383), (8.581, 8.787), (11.902, 12.80), (15.312, 17.09)):   # held-out prefixes
        assert abs(m.tau(x) - y) / y < 0.12, (x, m.tau(x), y)


def test_manager_idle_round_robin():
    """Idle GPU (B200 reading, DESIGN.md §2 reading 6): BE heads launched round robin over the apps
    from the one after the last idle launch -- a 5 ms app 0 does not starve a 1 ms app 1."""
    apps = [mr.App([(True, 5.0)]), mr.App([(True, 1.0)])]
    q = mr.Query(0, 13.0, [(True, 1.0)])
    res = mr.simulate([q], apps, 50.0, mr.TACKER, lambda a, b: None, idle_cap=10.0)
    idle = [d.reorder[0] for d in res["decisions"] if d.action == mr.IDLE_BE]
    assert idle[:4] == [0, 1, 0, 1]
    # 0..5 app 0, 5..6 app 1, 6..11 app 0, 11..12 app 1, 12..17 app 0 -> the query (13) waits to 17
    assert res["latency"][0] == 17.0 - 13.0 + 1.0


def test_two_stage_inverted_slopes_fall_back_to_one_lr():
    # DESIGN.md reading 5: samples of a concave curve (steep, then slope 1) give stage slopes in
    # the wrong order for Fig. 10's co-run -> CD-solo shape; the model must be the single LR over
    # all samples (pinned against numpy.polyfit), not max() of the two lines
    import numpy as np
    from oracle import predictor as op
    rs = [0.2, 0.4, 0.6, 0.8, 1.5, 2.5, 4.0, 6.0]
    taus = [1 + 2.0 * r if r < 1 else 3.0 + (r - 1.0) for r in rs]
    m = op.TwoStage()
    for r, t in zip(rs, taus):
        m.add(1.0, r, t)
    (a1, b1), (a2, b2) = m.fit()
    b, a = np.polyfit(rs, taus, 1)
    assert (a1, b1) == (a2, b2)
    assert abs(b1 - b) < 1e-12 and abs(a1 - a) < 1e-12
    assert m.inflection() is None
    for r in (0.3, 1.0, 5.0):
        assert abs(m.tau(r) - (a + b * r)) < 1e-12
    # a convex curve keeps its two stages (b1 < b2)
    m2 = op.TwoStage()
    for r in rs:
        m2.add(1.0, r, max(1 + 0.3 * r, 0.55 + r))
    (c1, d1), (c2, d2) = m2.fit()
    assert d1 < d2 and abs(d2 - 1.0) < 1e-9

