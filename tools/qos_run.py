"""QoS-managed co-location (BASELINE configs 2/4): LC service + BE queue under the Tacker and the
Baymax policy on the same Poisson trace.  Prints one JSON line.

  python tools/qos_run.py [--service resnet50|vgg16] [--batch 1] [--queries 400] [--load 0.8]
                          [--be stencil,mriq] [--ws 24]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk  # noqa: E402


def build_apps(names):
    apps = []
    for n in names:
        if n == "stencil":
            apps.append(sv.stencil_app(512, 512, 64))
        elif n == "mriq":
            apps.append(sv.mriq_app(64, 2048, 1024))
        elif n == "sgemm":
            apps.append(sv.sgemm_app(2048, 2048, 2048))
        elif n == "lbm":
            apps.append(sv.lbm_app())
        elif n == "cutcp":
            apps.append(sv.cutcp_app())
        elif n == "spmv":
            apps.append(sv.spmv_app())
        elif n == "histo":
            apps.append(sv.histo_app())
        elif n == "bfs":
            apps.append(sv.bfs_app())
        elif n in ("mrifhd", "cp", "fft", "tpacf"):
            apps.append(getattr(sv, n + "_app")())
        else:
            raise ValueError(n)
    return apps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--service", default="resnet50")
    ap.add_argument("--batch", type=int, default=1)
    ap.add_argument("--queries", type=int, default=400)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--load", type=float, default=0.8)
    ap.add_argument("--be", default="stencil,mriq")
    ap.add_argument("--ws", type=int, default=24)
    ap.add_argument("--qos", type=float, default=50.0)
    ap.add_argument("--io", action="store_true", help="each query copies its input H2D and result D2H")
    ap.add_argument("--inflight", type=int, default=4)
    ap.add_argument("--variants", default="baymax,tacker,tacker_slice,tacker_slice_literal")
    ap.add_argument("--slice-ratio", type=float, default=0.0, help="fixed slice load ratio (0: opportune r*)")
    ap.add_argument("--autotune", action="store_true", help="measured LC tile width per conv (as the bench)")
    args = ap.parse_args()
    svc = sv.resnet50_service(args.batch) if args.service == "resnet50" else sv.vgg16_service(args.batch)
    if args.autotune:
        sv.autotune_tile_n(svc)
    apps = build_apps(args.be.split(","))
    tk.tacker_model_clear()
    q = qos.QosRun(svc, apps, warp_split=args.ws, qos_ms=args.qos)
    if args.io:
        q.with_io()
    q.calibrate()
    q.measure_service(max_inflight=args.inflight)
    res = {}
    variants = {"baymax": (tk.POLICY_BAYMAX, {}), "tacker": (tk.POLICY_TACKER, {}),
                "tacker_slice": (tk.POLICY_TACKER, {"slice_be": True}),
                "tacker_slice_literal": (tk.POLICY_TACKER, {"slice_be": True}),
                "tacker_older": (tk.POLICY_TACKER, {"fuse_older": True}),   # reading 18 (the bench headline)
                "baymax_older": (tk.POLICY_BAYMAX, {"fuse_older": True})}   # Baymax with the same queueing rule
    for name in args.variants.split(","):
        pol, kw = variants[name]
        if args.slice_ratio > 0 and kw.get("slice_be"):
            kw = dict(kw, slice_ratio=args.slice_ratio)
        res[name] = q.run(pol, args.queries, load=args.load, warmup=args.warmup, max_inflight=args.inflight, **kw)
    for name in res:
        if name != "baymax" and "baymax" in res:
            res[name]["improvement_eq10"] = res[name]["be_kernels_per_s"] / res["baymax"]["be_kernels_per_s"] - 1.0
            res[name]["improvement_eq10_normalised"] = res[name]["be_norm_thpt"] / res["baymax"]["be_norm_thpt"] - 1.0
    res["slice_lr"] = {f"{a}.{j}": v for (a, j), v in q.lr_be.items()}
    res["pairs_fitted"] = len(q.pairs)
    res["pair_pred_err"] = ({"max": max(q.pair_err), "mean": sum(q.pair_err) / len(q.pair_err), "n": len(q.pair_err)}
                            if q.pair_err else None)
    res["config"] = {"service": svc.name, "be": args.be, "queries": args.queries, "load": args.load, "qos_ms": args.qos}
    print(json.dumps(res))


if __name__ == "__main__":
    main()
