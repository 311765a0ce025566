"""PTB-slice sweep (reading 13): for ResNet-50 b1 convs x bench BE kernels, the LC kernel alone,
BE slices of n original blocks alone, and the fused launch of the LC kernel with that slice, each
timed back to back on one stream (the manager's regime: `reps` launches between two events).
Prints one JSON line per (conv, BE kernel): X_tc and, per n, X_cd(n), T_fused(n), the sequential
sum and the overlap ratio max(X_tc, X_cd) / T_fused.

  python tools/slice_sweep.py [--convs 0,5,20,40,52] [--be stencil,mriq] [--ws 24]
"""
import argparse
import ctypes
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def stream_time(fn, reps=20, rounds=5):
    """Median over `rounds` of (time of `reps` back-to-back calls) / reps, in microseconds."""
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


def slice_desc(desc, off, n):
    d = tk.BeDesc()
    ctypes.memmove(ctypes.addressof(d), ctypes.addressof(desc), ctypes.sizeof(d))
    d.block_offset, d.orig_blocks = off, n
    return d


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--convs", default="0,5,20,40,52")
    ap.add_argument("--be", default="stencil,mriq")
    ap.add_argument("--ws", type=int, default=24)
    ap.add_argument("--fracs", default="0.01,0.02,0.05,0.1,0.2,0.35,0.5,1.0")
    args = ap.parse_args()
    svc = sv.resnet50_service(1)
    apps = {"stencil": sv.stencil_app(512, 512, 64), "mriq": sv.mriq_app(64, 2048, 1024)}
    tk.tacker_launch_original(None, apps["mriq"].kernels[0].desc)
    bes = {"stencil": apps["stencil"].kernels[0], "mriq": apps["mriq"].kernels[1]}
    tc = [k for k in svc.kernels if k.is_tc]
    for ci in [int(x) for x in args.convs.split(",")]:
        k = tc[ci]
        x_tc = stream_time(lambda: tk.tacker_launch_original(k.lc, None))
        for name in args.be.split(","):
            bk = bes[name]
            N = tk.tacker_be_num_blocks(bk.desc)
            f = tk.tacker_fuse(k.lc, bk.desc, args.ws)
            rows = []
            for fr in [float(x) for x in args.fracs.split(",")]:
                n = max(1, int(round(fr * N)))
                d = slice_desc(bk.desc, 0, n)
                x_cd = stream_time(lambda: tk.tacker_launch_original(None, d))
                t_f = stream_time(lambda: f.launch_slice(0, n))
                rows.append({"n": n, "x_cd_us": x_cd, "t_fused_us": t_f, "seq_us": x_tc + x_cd,
                             "r": x_cd / x_tc, "tau": t_f / x_tc, "overlap": max(x_tc, x_cd) / t_f,
                             "gain_us": x_tc + x_cd - t_f})
            print(json.dumps({"conv": k.name, "conv_index": ci, "be": name, "ws": args.ws, "x_tc_us": x_tc,
                              "blocks": N, "lc_tiles": f.info().lc_tiles, "rows": rows}), flush=True)


if __name__ == "__main__":
    main()
