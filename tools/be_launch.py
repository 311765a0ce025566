"""Launch selected bench BE kernels (original and fused with a small LC GEMM) a few times, for
ncu captures.  Usage: python tools/be_launch.py stencil,mriq [reps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def main():
    kinds = sys.argv[1].split(",") if len(sys.argv) > 1 else ["stencil", "mriq"]
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    A, B = synth.lc_gemm_inputs(256, 128, 256, seed=0)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    D = torch.empty(256, 128, device="cuda")
    lc = tk.lc_gemm(dA, dB, D)
    keep = []
    for k in kinds:
        if k == "stencil":
            app = sv.stencil_app()
            d = app.kernels[0].desc
        elif k == "mriq":
            app = sv.mriq_app()
            tk.tacker_launch_original(None, app.kernels[0].desc)
            d = app.kernels[1].desc
        elif k == "sgemm":
            app = sv.sgemm_app(2048, 2048, 2048)
            d = app.kernels[0].desc
        elif k == "mrifhd":
            app = sv.mrifhd_app()
            tk.tacker_launch_original(None, app.kernels[0].desc)
            d = app.kernels[1].desc
        elif k in ("cp", "fft", "tpacf", "lbm", "spmv", "histo", "cutcp"):
            app = getattr(sv, k + "_app")()
            d = app.kernels[-1].desc
        else:
            raise ValueError(k)
        keep.append(app)
        f = tk.tacker_fuse(lc, d, 24 if k not in ("sgemm", "fft", "tpacf") else 16)
        for _ in range(reps):
            tk.tacker_launch_original(None, d)
        for _ in range(reps):
            f.launch()
    torch.cuda.synchronize()
    print("ok")


if __name__ == "__main__":
    main()
