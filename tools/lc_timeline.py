"""Per-role timeline of one LC conv launch (TACKER_LC_DBG must include bit 3, set before import):
clock64 stamps of the producer / MMA / epilogue per work unit on a few CTAs (a -DTK_LC_DIAG=1 build via
TACKER_LIB: production kernels carry no diagnostics), as cycles from the
first producer stamp.   TACKER_LC_DBG=8 python tools/lc_timeline.py --bn 64 layer1.0.conv2"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("name")
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--bn", type=int, default=0)
    ap.add_argument("--ctas", default="0,1,73,147")
    args = ap.parse_args()
    convs = [c for c in synth.resnet50_convs(args.batch) if c.name == args.name]
    svc = sv.resnet50_service(args.batch, convs=convs)
    k = [k for k in svc.kernels if k.is_tc][0]
    if args.bn:
        k.lc.tile_n = args.bn
    for _ in range(3):
        tk.tacker_launch_original(k.lc, None)
    torch.cuda.synchronize()
    ts = tk.tacker_debug_lc_timestamps().astype(np.int64)
    names = ["prod", "mma0", "mma1", "epi0", "epi1"]
    for c in [int(x) for x in args.ctas.split(",")]:
        t0 = ts[c, 0, 0]
        print(f"CTA {c}:")
        for e in range(5):
            row = [int(x - t0) if x else -1 for x in ts[c, e]]
            print(f"  {names[e]:5s}", " ".join(f"{v:7d}" for v in row[:10]))


if __name__ == "__main__":
    main()
