"""Table I analogue (§III-B): Kt = tensor-core GEMM, Kc = register-only FMA kernel of
equal standalone duration; Bench-A = Kt || Kc in one fused kernel, normalised to Kt
(paper: 1.03 on an RTX 2080Ti).  Also GEMM || sgemm at the config-1-perf twin size.
Prints one JSON line.  Usage: python tools/table1.py [M N K] [warp_split]"""
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
    M, N, K = (int(x) for x in sys.argv[1:4]) if len(sys.argv) >= 4 else (8192, 8192, 8192)
    ws = int(sys.argv[4]) if len(sys.argv) >= 5 else 24
    A, B = synth.lc_gemm_inputs(M, N, K, seed=0)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    D = torch.empty(M, N, device="cuda")
    lc = tk.lc_gemm(dA, dB, D)
    t_kt = timeit(lambda: tk.tacker_launch_original(lc, None))
    flops = 2.0 * M * N * K
    sms = tk.tacker_device_sm_count()
    nthr = sms * ws * 32
    out = torch.empty(nthr, device="cuda")
    # calibrate Kc to Kt's standalone duration
    it0 = 20000
    t0 = timeit(lambda: tk.tacker_launch_original(None, tk.be_fma_burn(out, it0)))
    iters = max(100, int(it0 * t_kt / t0))
    kc = tk.be_fma_burn(out, iters)
    t_kc = timeit(lambda: tk.tacker_launch_original(None, kc))
    f = tk.tacker_fuse(lc, kc, ws)
    t_a = timeit(lambda: f.launch())
    res = {"gemm": [M, N, K], "warp_split": ws, "t_kt_ms": t_kt, "kt_tflops": flops / t_kt / 1e9,
           "t_kc_ms": t_kc, "kc_iters": iters, "kc_tflops": 2.0 * 4 * iters * nthr / t_kc / 1e9,
           "t_bench_a_ms": t_a, "bench_a_norm": t_a / t_kt, "seq_norm": (t_kt + t_kc) / t_kt,
           "paper_bench_a_norm": 1.03, "fused_info": {"bn": f.info().lc_tile_n, "stages": f.info().lc_stages,
                                                      "regs": f.info().regs_per_thread}}
    # GEMM || sgemm (BE sized for r ~ 1 by the sgemm original time)
    SA, SB = synth.sgemm_inputs(4096, 4096, 1024, seed=1)
    sA, sB = torch.from_numpy(SA).cuda(), torch.from_numpy(SB).cuda()
    Cm = torch.empty(4096, 4096, device="cuda")
    sg = tk.be_sgemm(sA, sB, Cm)
    t_sg = timeit(lambda: tk.tacker_launch_original(None, sg))
    f2 = tk.tacker_fuse(lc, sg, 16)
    t_f2 = timeit(lambda: f2.launch())
    res.update({"t_sgemm_ms": t_sg, "sgemm_tflops": 2.0 * 4096 * 4096 * 1024 / t_sg / 1e9, "t_gemm_sgemm_fused_ms": t_f2,
                "gemm_sgemm_seq_over_fused": (t_kt + t_sg) / t_f2,
                "gemm_sgemm_roof_ms": max(t_kt, t_sg), "gemm_sgemm_roof_frac": max(t_kt, t_sg) / t_f2})
    print(json.dumps(res))


if __name__ == "__main__":
    main()
