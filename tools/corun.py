"""Co-running baselines vs fusion (NEXT-4; the paper's Fig. 20 / Eq. 11): for LC
conv x BE kernel pairs, the standalone times T_TC and T_CD, the sequential pair, the two kernels
on two streams (original kernels, the hardware scheduler interleaving CTAs) and the fused kernel,
each timed back to back (`reps` pairs between two events).  Overlap rate (Eq. 11) =
(T_TC + T_CD - T_corun) / (T_TC + T_CD).  One JSON line per pair.

  python tools/corun.py [--batch 1] [--convs layer1.0.conv2,layer3.0.conv2,layer4.2.conv2] [--ws 24]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200.qos import overlap_rate  # noqa: E402


def timed(fn, reps=10, rounds=5):
    fn()
    torch.cuda.synchronize()
    out = []
    for _ in range(rounds):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        e1.synchronize()
        out.append(e0.elapsed_time(e1) * 1e3 / reps)
    return statistics.median(out)


def be_roof_us(spec):
    """BE kernel time at its roofline: max(F / P_fp32, S / P_mufu, B / BW); peaks from
    MEASURED_PEAKS.json (HBM) and the guide's unit counts at the max SM clock (FP32 128 lanes,
    MUFU 16 lanes per SM per clock, 148 SMs)."""
    pk = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    f = pk.get("sm_max_mhz", 1965.0) * 1e6
    p_fp32, p_mufu, bw = 148 * 128 * 2 * f, 148 * 16 * f, pk["hbm_gbs"] * 1e9
    return 1e6 * max(spec.flops / p_fp32, spec.mufu / p_mufu, spec.bytes / bw)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=1)
    ap.add_argument("--convs", default="layer1.0.conv2,layer3.0.conv2,layer4.2.conv2")
    ap.add_argument("--be", default="stencil,mriq")
    ap.add_argument("--ws", type=int, default=24)
    ap.add_argument("--overlap", type=int, default=2, help="tacker_set_launch_overlap mode (0, 1, 2; library default 2)")
    args = ap.parse_args()
    tk.tacker_set_launch_overlap(args.overlap)
    svc = sv.resnet50_service(args.batch)
    st, mq = sv.stencil_app(512, 512, 64), sv.mriq_app(64, 2048, 1024)
    fh, cp, ff, tp = sv.mrifhd_app(64, 2048, 1024), sv.cp_app(), sv.fft_app(), sv.tpacf_app()
    tk.tacker_launch_original(None, mq.kernels[0].desc)
    tk.tacker_launch_original(None, fh.kernels[0].desc)
    bes = {"stencil": st.kernels[0], "mriq": mq.kernels[1], "mrifhd": fh.kernels[1], "cp": cp.kernels[0],
           "fft": ff.kernels[0], "tpacf": tp.kernels[1]}
    ks = {k.name: k for k in svc.kernels}
    s_lc, s_be = torch.cuda.Stream(), torch.cuda.Stream()
    cur = torch.cuda.current_stream()

    def streams(k, b):
        s_lc.wait_stream(cur)
        s_be.wait_stream(cur)
        tk.tacker_launch_original(k.lc, None, stream=s_lc)
        tk.tacker_launch_original(None, b.desc, stream=s_be)
        cur.wait_stream(s_lc)
        cur.wait_stream(s_be)

    for cn in args.convs.split(","):
        k = ks[cn]
        for bn in args.be.split(","):
            b = bes[bn]
            f = tk.tacker_fuse(k.lc, b.desc, args.ws)
            t_tc = timed(lambda: tk.tacker_launch_original(k.lc, None))
            t_cd = timed(lambda: tk.tacker_launch_original(None, b.desc))
            t_seq = timed(lambda: tk.tacker_launch_original(k.lc, b.desc))
            t_st = timed(lambda: streams(k, b))
            t_f = timed(lambda: f.launch())
            print(json.dumps({"overlap": args.overlap, "batch": args.batch, "conv": cn, "be": bn, "ws": args.ws, "t_tc_us": t_tc, "t_cd_us": t_cd,
                              "sequential_us": t_seq, "two_streams_us": t_st, "fused_us": t_f,
                              "overlap_eq11": {"sequential": overlap_rate(t_tc, t_cd, t_seq),
                                               "two_streams": overlap_rate(t_tc, t_cd, t_st),
                                               "fused": overlap_rate(t_tc, t_cd, t_f)},
                              "ideal_max_us": max(t_tc, t_cd),
                              "be_roofline_us": be_roof_us(b), "be_roofline_frac_standalone": be_roof_us(b) / t_cd,
                              "be_bound": b.bound}), flush=True)


if __name__ == "__main__":
    main()
