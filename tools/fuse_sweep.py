"""Fused-kernel efficiency sweep: for each bench BE kernel (stencil sweep, mri-q Q chunk) and a
set of ResNet-50 b1 convs, the standalone LC and BE times, the fused time per warp split, the
overlap ideal max(LC, BE) and the sequential sum.  Prints one JSON line per (conv, BE, ws).

  python tools/fuse_sweep.py [--convs 0,10,30,50] [--ws 8,16,24] [--be stencil,mriq]
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


def timeit(fn, reps=20):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--convs", default="0,5,20,40,52")
    ap.add_argument("--ws", default="8,16,24")
    ap.add_argument("--be", default="stencil,mriq")
    ap.add_argument("--batch", type=int, default=1, help="ResNet-50 batch of the LC convs")
    args = ap.parse_args()
    svc = sv.resnet50_service(args.batch)
    tcs = [k for k in svc.kernels if k.is_tc]
    bes = {}
    for b in args.be.split(","):
        if b == "stencil":
            app = sv.stencil_app(512, 512, 64)
            bes[b] = (app, app.kernels[0].desc)
        elif b == "mriq":
            app = sv.mriq_app(64, 2048, 1024)
            tk.tacker_launch_original(None, app.kernels[0].desc)
            bes[b] = (app, app.kernels[1].desc)
        elif b == "sgemm":
            app = sv.sgemm_app(2048, 2048, 2048)
            bes[b] = (app, app.kernels[0].desc)
        elif b in ("fft", "lbm", "cp", "mrifhd", "tpacf"):
            app = {"fft": sv.fft_app, "lbm": sv.lbm_app, "cp": sv.cp_app, "mrifhd": sv.mrifhd_app,
                   "tpacf": sv.tpacf_app}[b]()
            sv.prime_apps([app])
            k0 = next(k for k in app.kernels if k.name not in ("mrifhd.rhophi",))
            bes[b] = (app, k0.desc)
    for ci in [int(c) for c in args.convs.split(",")]:
        k = tcs[ci]
        t_lc = timeit(lambda: tk.tacker_launch_original(k.lc, None))
        for name, (app, d) in bes.items():
            t_be = timeit(lambda: tk.tacker_launch_original(None, d))
            for ws in [int(w) for w in args.ws.split(",")]:
                try:
                    f = tk.tacker_fuse(k.lc, d, ws)
                except tk.TackerError as e:
                    print(json.dumps({"conv": ci, "be": name, "ws": ws, "err": str(e)}))
                    continue
                t_f = timeit(f.launch)
                print(json.dumps({"conv": ci, "shape": k.name, "be": name, "ws": ws, "regs": f.info().regs_per_thread, "lc_us": round(t_lc, 2),
                                  "be_us": round(t_be, 2), "fused_us": round(t_f, 2),
                                  "seq_us": round(t_lc + t_be, 2), "ideal_us": round(max(t_lc, t_be), 2),
                                  "frac_of_ideal": round(max(t_lc, t_be) / t_f, 3),
                                  "gain_us": round(t_lc + t_be - t_f, 2)}), flush=True)


if __name__ == "__main__":
    main()
