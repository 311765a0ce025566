"""LC query latency: one ResNet-50 (or VGG-16) query's kernels launched back to back on one
stream, with programmatic dependent launch on and off (CUDA events around the query, median of
`reps`).  Prints one JSON line.

  python tools/lc_chain.py [--service resnet50|vgg16] [--batch 1] [--reps 20]
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


def query(svc):
    for k in svc.kernels:
        tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd)


def timed(fn, reps):
    fn()
    torch.cuda.synchronize()
    out = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        out.append(e0.elapsed_time(e1))
    return statistics.median(out)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--service", default="resnet50")
    ap.add_argument("--batch", type=int, default=1)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--autotune", action="store_true", help="measured LC tile width per conv (services.autotune_tile_n)")
    ap.add_argument("--chain-autotune", action="store_true", help="then refine the widths on the query chain")
    args = ap.parse_args()
    svc = sv.resnet50_service(args.batch) if args.service == "resnet50" else sv.vgg16_service(args.batch)
    if args.autotune:
        sv.autotune_tile_n(svc)
    if args.chain_autotune:
        sv.chain_autotune_tile_n(svc)
    res = {"service": svc.name, "kernels": len(svc.kernels), "autotune": bool(args.autotune)}
    for on in (False, True):
        tk.tacker_set_launch_overlap(on)
        res["overlap" if on else "serial"] = {"query_ms": timed(lambda: query(svc), args.reps)}
    per = []
    tk.tacker_set_launch_overlap(2)
    for k in svc.kernels:
        f = (lambda k=k: tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd))
        us = timed(lambda: [f() for _ in range(8)], 5) * 1e3 / 8     # back to back
        row = {"name": k.name, "us": us, "flops": k.flops, "bytes": k.bytes,
               "roof_us": max(k.flops / 1637.3e12, k.bytes / 6.4821e12) * 1e6}
        if k.is_tc:
            i = tk.tacker_fuse(k.lc, None, 0).info()
            row.update(tiles=i.lc_tiles, splits=i.lc_splits, bn=i.lc_tile_n, grid=i.grid,
                       tflops=k.flops / us / 1e6)
        per.append(row)
    res["per_kernel"] = per
    print(json.dumps(res))


if __name__ == "__main__":
    main()
