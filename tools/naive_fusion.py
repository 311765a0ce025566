"""NEXT-4 naive-fusion baseline (the paper's Fig. 3: an LC tensor-core kernel fused 1:1
with Parboil kernels runs ~2x slower than its parts because of resource contention).  The B200
analogue of "1:1" is one BE virtual block per fused CTA (warp_split 4, no tuning); it is timed
against the tuned split (the fastest of 8..24 warps that fits the budget, NEXT-1), the sequential
original pair and the two kernels alone.  One JSON line per BE kernel.

  python tools/naive_fusion.py [--conv layer3.0.conv2] [--be stencil,mriq,...]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402
from tools.corun import timed  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--conv", default="layer3.0.conv2")
    ap.add_argument("--be", default="sgemm,stencil,mriq,mrifhd,cp,cutcp,lbm,spmv,histo,fft,tpacf")
    args = ap.parse_args()
    svc = sv.resnet50_service(1)
    lc = next(k for k in svc.kernels if k.name == args.conv).lc
    apps = {"sgemm": lambda: sv.sgemm_app(1024, 1024, 1024), "stencil": sv.stencil_app, "mriq": sv.mriq_app,
            "mrifhd": sv.mrifhd_app, "cp": sv.cp_app, "cutcp": sv.cutcp_app, "lbm": sv.lbm_app, "spmv": sv.spmv_app,
            "histo": lambda: sv.histo_app(1 << 24), "fft": sv.fft_app, "tpacf": lambda: sv.tpacf_app(8192)}
    t_tc = timed(lambda: tk.tacker_launch_original(lc, None))
    for name in args.be.split(","):
        app = apps[name]()
        for k in app.kernels[:-1]:          # set-up kernels (phiMag, RhoPhi, binning) run once
            if not k.is_tc:
                tk.tacker_launch_original(None, k.desc)
        d = app.kernels[-1].desc
        t_cd = timed(lambda: tk.tacker_launch_original(None, d))
        t_seq = timed(lambda: tk.tacker_launch_original(lc, d))
        res = {}
        for ws in (4, 8, 12, 16, 20, 24):
            try:
                f = tk.tacker_fuse(lc, d, ws)
            except tk.TackerError:
                continue
            res[ws] = timed(lambda: f.launch())
        best = min(res, key=res.get)
        print(json.dumps({"conv": args.conv, "be": name, "t_tc_us": t_tc, "t_cd_us": t_cd, "sequential_us": t_seq,
                          "naive_1to1_us": res.get(4), "tuned_us": res[best], "tuned_ws": best,
                          "naive_over_sequential": res[4] / t_seq if 4 in res else None,
                          "tuned_over_sequential": res[best] / t_seq, "all_ws_us": res}), flush=True)


if __name__ == "__main__":
    main()
