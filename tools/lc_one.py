"""Launch named LC kernels of a ResNet-50 / VGG-16 service (LC only) `reps` times each, for ncu
captures of one kernel class:  python tools/lc_one.py [--batch 32] [--bn 0] [--reps 3] name [name ...]"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("names", nargs="+")
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--bn", type=int, default=0, help="tile width (0: autotuned)")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--service", default="resnet50")
    args = ap.parse_args()
    svc = sv.resnet50_service(args.batch) if args.service == "resnet50" else sv.vgg16_service(args.batch)
    ks = {k.name: k for k in svc.kernels}
    if args.bn:
        for n in args.names:
            ks[n].lc.tile_n = args.bn
    else:
        sv.autotune_tile_n(svc)
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_push("target")     # ncu --nvtx --nvtx-include "target/" selects these launches
    for n in args.names:
        k = ks[n]
        for _ in range(args.reps):
            tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd)
    torch.cuda.nvtx.range_pop()
    torch.cuda.synchronize()
    print("ok")


if __name__ == "__main__":
    main()
