"""Config-1 perf twin (Table I): an 8192^3 fp16 tensor-core GEMM
(LC) fused with a Parboil-style fp32 sgemm (BE) sized so that its standalone time is r x the
GEMM's, r in {0.25, 0.5, 1, 2, 4}.  Per r: standalone T_TC and T_CD, the fused time, the sequential
sum, Eq. 11 overlap, and the fused time against the overlap roofline max(F_TC / P_tensor,
F_CD / P_fma) (measured peaks: MEASURED_PEAKS.json bf16 = fp16 rate, profiles/peaks.json FFMA) and
against the measured-solo ideal max(T_TC, T_CD).  One JSON line per r.

  python tools/config1_twin.py [--ws 16] [--ratios 0.25,0.5,1,2,4]"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk  # noqa: E402


def timeit(fn, reps=7):
    s = torch.cuda.current_stream()
    fn()
    out = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        out.append(e0.elapsed_time(e1))
    return statistics.median(out)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ws", type=int, default=16)
    ap.add_argument("--ratios", default="0.25,0.5,1,2,4")
    args = ap.parse_args()
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"bf16_tflops": 1653.7}
    micro = json.load(open(os.path.join(ROOT, "profiles", "peaks.json")))
    p_tc, p_fma = peaks["bf16_tflops"] * 1e12, micro["ffma_tflops"] * 1e12
    M = N = K = 8192
    A, B = synth.lc_gemm_inputs(M, N, K, seed=0)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    D = torch.empty(M, N, device="cuda")
    lc = tk.lc_gemm(dA, dB, D)
    t_tc = timeit(lambda: tk.tacker_launch_original(lc, None))
    f_tc = 2.0 * M * N * K
    SM = SN = 4096
    kmax = 16384
    SA, SB = synth.sgemm_inputs(SM, SN, kmax, seed=1)
    sA, sB = torch.from_numpy(SA).cuda(), torch.from_numpy(SB).cuda()
    Cm = torch.empty(SM, SN, device="cuda")
    t1 = timeit(lambda: tk.tacker_launch_original(None, tk.be_sgemm(sA[:, :1024].contiguous(), sB[:1024].contiguous(), Cm)))
    for r in (float(x) for x in args.ratios.split(",")):
        k = max(4, min(kmax, int(round(1024 * r * t_tc / t1 / 4)) * 4))
        a, b = sA[:, :k].contiguous(), sB[:k].contiguous()
        sg = tk.be_sgemm(a, b, Cm)
        t_cd = timeit(lambda: tk.tacker_launch_original(None, sg))
        f = tk.tacker_fuse(lc, sg, args.ws)
        t_f = timeit(lambda: f.launch())
        f_cd = 2.0 * SM * SN * k
        roof = max(f_tc / p_tc, f_cd / p_fma) * 1e3
        seq = t_tc + t_cd
        print(json.dumps({"r_target": r, "r_measured": t_cd / t_tc, "sgemm_k": k, "warp_split": args.ws,
                          "t_tc_ms": t_tc, "t_cd_ms": t_cd, "fused_ms": t_f, "sequential_ms": seq,
                          "speedup_vs_sequential": seq / t_f, "overlap_eq11": (seq - t_f) / seq,
                          "overlap_roofline_ms": roof, "overlap_roofline_frac": roof / t_f,
                          "solo_ideal_ms": max(t_tc, t_cd), "solo_ideal_frac": max(t_tc, t_cd) / t_f}), flush=True)


if __name__ == "__main__":
    main()
