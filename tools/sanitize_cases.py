"""Small fused / LC-only / BE-only launches of every kind, for compute-sanitizer runs
(synccheck: named-barrier / warp-sync misuse; racecheck: shared-memory hazards; memcheck: out-of-
bounds and misaligned accesses).  Each case is checked against its original launch (bytes).
  compute-sanitizer --tool synccheck python tools/sanitize_cases.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk  # noqa: E402
from tests.gpu_helpers import be_case, host, t  # noqa: E402

KINDS = ["BE_SGEMM", "BE_STENCIL", "BE_MRIQ_Q", "BE_LBM", "BE_SPMV_JDS", "BE_HISTO", "BE_FMA_BURN", "BE_CUTCP",
         "BE_MRIFHD_RHOPHI", "BE_MRIFHD_FH", "BE_CP", "BE_FFT", "BE_TPACF"]


def main():
    A, B = synth.lc_gemm_inputs(256, 256, 256, seed=1)
    dA, dB = t(A), t(B)
    bad = 0
    for kind in KINDS:
        c = be_case(getattr(tk, kind), seed=2)
        D0, D1 = torch.zeros(256, 256, device="cuda"), torch.zeros(256, 256, device="cuda")
        c["reset"]()
        tk.tacker_launch_original(tk.lc_gemm(dA, dB, D0), c["desc"])
        orig = [host(o).copy() for o in c["outs"]]
        c["reset"]()
        tk.tacker_fuse(tk.lc_gemm(dA, dB, D1), c["desc"], 8).launch()
        same = all(a.tobytes() == host(b).tobytes() for a, b in zip(orig, c["outs"])) and torch.equal(D0, D1)
        bad += not same
        print(kind, "fused == original" if same else "MISMATCH", flush=True)
    # LC-only modes: halo conv (TMA store), im2col conv, 1x1 (GEMM view), split-K, halo + residual
    for name, cs, kw in [("halo", synth.ConvShape("h", 1, 14, 14, 64, 64, 3, 3, 1, 1), {}),
                         ("im2col s2", synth.ConvShape("s2", 1, 14, 14, 64, 64, 3, 3, 2, 1), {}),
                         ("1x1", synth.ConvShape("p", 1, 14, 14, 64, 128, 1, 1, 1, 0), {}),
                         ("split-K", synth.ConvShape("k", 1, 7, 7, 512, 128, 3, 3, 1, 1), {}),
                         ("halo residual", synth.ConvShape("r", 1, 14, 14, 64, 64, 3, 3, 1, 1), {"res": True})]:
        x, w, b = synth.conv_inputs(cs, seed=3)
        out = torch.zeros(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device="cuda")
        res = t(np.ones((cs.n, cs.p, cs.q, cs.k), np.float16)) if kw.get("res") else None
        lc = tk.lc_conv(t(x), t(w), out, cs.stride, cs.pad, bias=t(b), relu=True, residual=res)
        tk.tacker_launch_original(lc, None)
        torch.cuda.synchronize()
        print("LC", name, "mode", tk.tacker_fuse(lc, None, 0).info().lc_mode, "ok", flush=True)
    print("MISMATCHES", bad)


if __name__ == "__main__":
    main()
