"""GPU: NEXT-2 reverse fusion (LC CUDA-core kernel + BE tensor-core kernel) through the
C ABI -- the fused kernel against the oracle and bit-identical to the original launches, and a
short managed run whose reverse-fused queries produce the same bytes as standalone queries."""
import numpy as np
import pytest
import torch

import synth
from oracle import lc as olc
from oracle.metrics import max_rel_err

pytestmark = pytest.mark.gpu

from tests.gpu_helpers import dev, host, t  # noqa: E402


@pytest.fixture(scope="module")
def tk():
    from paper_conf_hpca_zhaocczlllg22_b200 import tacker
    assert torch.cuda.is_available()
    return tacker


def test_reverse_fused_im2col_with_be_gemm(tk):
    # LC CUDA-core part: conv1's explicit im2col (b2, ragged last block); BE tensor-core part: a
    # training-like fp16 GEMM
    cs = synth.ConvShape("conv1", 2, 64, 60, 8, 64, 7, 7, 2, 3)
    x, _, _ = synth.conv_inputs(cs, seed=4, real_c=3)
    M, _, K = cs.gemm_mnk
    Kpad = ((K + 63) // 64) * 64
    dx = t(x)
    cols0 = torch.zeros(M, Kpad, dtype=torch.float16, device=dev())
    cols1 = torch.zeros_like(cols0)
    A, B = synth.lc_gemm_inputs(512, 384, 1024, seed=5)
    dA, dB = t(A), t(B)
    D0 = torch.zeros(512, 384, device=dev())
    D1 = torch.zeros_like(D0)
    tk.tacker_launch_original(tk.lc_gemm(dA, dB, D0), tk.be_im2col(dx, cols0, 7, 7, 2, 3, Kpad))
    f = tk.tacker_fuse(tk.lc_gemm(dA, dB, D1), tk.be_im2col(dx, cols1, 7, 7, 2, 3, Kpad), 16)
    f.launch()
    assert host(cols1).tobytes() == host(cols0).tobytes()
    assert host(D1).tobytes() == host(D0).tobytes()
    assert np.array_equal(host(cols1), olc.im2col(x, 7, 7, 2, 3, Kpad))
    ref, S = olc.lc_gemm(A, B)
    assert max_rel_err(host(D1), ref, S) <= 1e-2


def test_managed_reverse_fusion_outputs_match_standalone(tk):
    from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv
    # LC service = ResNet-50 conv1 at batch 32 (im2col on the CUDA cores + GEMM) and the next conv;
    # BE queue = one tensor-core training GEMM app (tools/reverse_pair.py: this pair overlaps)
    convs = synth.resnet50_convs(32)[:2]
    svc = sv.resnet50_service(32, convs=convs, conv1_im2col=True)
    app = sv.gemm_train_app(4096, 4096, 4096, n=1)
    # reference bytes: one standalone query
    for k in svc.kernels:
        tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd)
    ref = host(svc.outputs[-1]).tobytes()
    run = qos.QosRun(svc, [app], warp_split=16)
    run.calibrate(reps=3, pair_reps=3)
    assert any("be:im2col" in k for k in run.pairs), run.pairs.keys()
    run.measure_service(n=20)
    pk = next(k for k in run.pairs if "be:im2col" in k)
    t_be, t_lc = run.t_be[(0, 0)], run.t_lc[0]
    gain = t_be - (tk.tacker_pair_predict(pk, t_be, t_lc) - t_lc)     # Eq. 8's Tgain for this pair
    svc.outputs[-1].zero_()
    res = run.run(tk.POLICY_TACKER, 40, load=0.8)
    assert res["qos_met"]
    # the manager fuses exactly when the calibrated model predicts a gain (measured on this box)
    assert (res["reverse_fused"] > 0) == (gain > 0), (gain, res["reverse_fused"])
    assert host(svc.outputs[-1]).tobytes() == ref
    # the GPU reverse-fused launch path, whatever this box measured: a model with a sure gain
    tk.tacker_model_clear()
    tk.tacker_blacklist_clear()
    for r in (0.1, 0.2, 1.8, 1.9):
        tk.tacker_pair_add_sample(pk, 1.0, r, max(1.0, r) + 0.05)
    tk.tacker_pair_fit(pk)
    svc.outputs[-1].zero_()
    res = run.run(tk.POLICY_TACKER, 40, load=0.8)
    assert res["reverse_fused"] > 0, res
    assert host(svc.outputs[-1]).tobytes() == ref


@pytest.mark.parametrize("variant", [dict(fuse_older=True), dict(fuse_older=True, slice_be=True, reorder_rule=2)])
def test_managed_runs_keep_lc_outputs_and_qos(tk, variant):
    """GPU-mode managed runs with reading 18 (older queries fuse) and with PTB slices and no
    reorder: every LC query's output bytes equal a standalone query's, QoS holds, kernels fused."""
    from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv
    convs = [c for c in synth.resnet50_convs(8) if c.name in ("layer1.0.conv1", "layer1.0.conv2", "layer1.0.conv3")]
    svc = sv.resnet50_service(8, convs=convs)
    st, mq = sv.stencil_app(512, 512, 64), sv.mriq_app(64, 1024, 1024)   # >= 10 us: fusable kernels
    tk.tacker_launch_original(None, mq.kernels[0].desc)
    for k in svc.kernels:
        tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd)
    ref = host(svc.outputs[-1]).tobytes()
    tk.tacker_model_clear()
    run = qos.QosRun(svc, [st, mq], warp_split=16)
    run.calibrate(reps=3, pair_reps=3)
    run.measure_service(n=20)
    assert run.pairs, "no fusable pair calibrated"
    # the launch paths under test must run whatever this box measured (the NEXT-1 selection may
    # have kept a BE kernel out of fusion): every >= 10 us BE kernel fused at 16 warps, with a pair
    # model of sure gain (tau = max(1 + 0.1 r, 0.5 + r), opportune ratio 5/9), none blacklisted
    tk.tacker_model_clear()
    tk.tacker_blacklist_clear()
    for a, app in enumerate([st, mq]):
        for j, bk in enumerate(app.kernels):
            if run.t_be[(a, j)] < 0.01:
                continue
            run.ws_of[(a, j)] = 16
            for k in svc.kernels:
                pk = tk.tacker_fuse(k.lc, bk.desc, 16).keys()[2]
                for r in (0.1, 0.2, 1.8, 1.9):
                    tk.tacker_pair_add_sample(pk, 1.0, r, max(1.0 + 0.1 * r, 0.5 + r))
                tk.tacker_pair_fit(pk)
    svc.outputs[-1].zero_()
    res = run.run(tk.POLICY_TACKER, 60, load=0.8, max_inflight=8, **variant)
    brief = {k: res[k] for k in ("fused", "reordered", "idle_be", "be_kernels", "lc_p99_ms", "class_launches")}
    assert res["qos_met"], brief
    assert res["fused"] > 0, (brief, run.ws_of, run.lr_be, list(run.pairs))
    assert host(svc.outputs[-1]).tobytes() == ref


@pytest.mark.parametrize("rules", [dict(), dict(fuse_older=True, reorder_rule=1), dict(fuse_older=True)])
def test_gpu_manager_trace_replays_through_reference(tk, rules):
    """a GPU-mode managed run (steady-state window protocol of the bench) records
    its decision trace; oracle/manager_ref.replay recomputes every decision, Tgain and headroom
    from the recorded observations (clock, active queries, online Tk_fuse) and must agree."""
    from oracle import manager_ref as mr
    from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv
    from tests.trace_check import check_trace
    convs = [c for c in synth.resnet50_convs(8) if c.name in ("layer1.0.conv1", "layer1.0.conv2", "layer1.0.conv3")]
    svc = sv.resnet50_service(8, convs=convs)
    st, mq = sv.stencil_app(512, 512, 64), sv.mriq_app(64, 1024, 1024)
    tk.tacker_launch_original(None, mq.kernels[0].desc)
    tk.tacker_model_clear()
    run = qos.QosRun(svc, [st, mq], warp_split=16)
    run.calibrate(reps=3, pair_reps=3)
    run.measure_service(n=20)
    res = run.run_window(tk.POLICY_TACKER, window_ms=60.0, warm_ms=20.0, tail_ms=20.0, load=0.8, max_inflight=8,
                         trace=True, **rules)
    assert res["trace_dropped"] == 0 and len(res["trace"]) > 50
    queries, apps = run.replay_inputs(res["arrivals"])
    cap = run.idle_cap()
    ref_rules = dict(fuse_older=rules.get("fuse_older", False), older_margin=0.3 * run.qos,
                     reorder_rule=rules.get("reorder_rule", mr.REORDER_UNFUSED))
    n = check_trace(res["trace"], queries, apps, run.qos, mr.TACKER, idle_cap=cap if cap > 0 else None, **ref_rules)
    assert n == len(res["trace"])
    assert res["qos_met"], res


def test_select_fusion_through_c_abi(tk):
    """NEXT-1: tacker_select_fusion times every fused candidate and the sequential pair on the GPU;
    the returned split is the fastest (or 0 = sequential, which blacklists the BE kernel)."""
    from paper_conf_hpca_zhaocczlllg22_b200 import services as sv
    cs = next(c for c in synth.resnet50_convs(8) if c.name == "layer2.1.conv2")
    svc = sv.resnet50_service(8, convs=[cs])
    mq = sv.mriq_app(64, 1024, 1024)
    tk.tacker_launch_original(None, mq.kernels[0].desc)
    tk.tacker_blacklist_clear()
    best, best_ms, seq_ms, cand = tk.tacker_select_fusion(svc.kernels[0].lc, mq.kernels[1].desc, (24, 16, 8, 4), 3)
    assert seq_ms > 0 and cand, (best, cand)
    assert best_ms == min([seq_ms] + list(cand.values()))
    key = tk.tacker_fuse(svc.kernels[0].lc, mq.kernels[1].desc, 4).keys()[1]
    assert tk.tacker_blacklist(key) == (best == 0)
    if best:
        assert cand[best] == best_ms
    tk.tacker_blacklist_clear()
