"""Per-kernel time of selected LC convs (b32, back to back, CUDA events), for the diagnostic
variants TACKER_LC_DBG selects: run once per flag value (the flag is read at plan time).
  TACKER_LC_DBG=<f> python tools/lc_breakdown.py [--bn 0] name ...   -> one JSON line"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("names", nargs="+")
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--bn", type=int, default=0)
    args = ap.parse_args()
    convs = [c for c in __import__("synth").resnet50_convs(args.batch) if c.name in args.names]
    svc = sv.resnet50_service(args.batch, convs=convs)
    out = {"dbg": int(os.environ.get("TACKER_LC_DBG", "0"))}
    for k in svc.kernels:
        if not k.is_tc:
            continue
        if args.bn:
            k.lc.tile_n = args.bn
        us = qos._time(lambda: tk.tacker_launch_original(k.lc, None), 10) * 1e3
        out[k.name] = round(us, 2)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
