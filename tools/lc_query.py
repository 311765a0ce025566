"""Launch the LC kernels of one ResNet-50 query (original launches, no BE) `reps` times, for ncu
captures of the bench's dominant kernel class.  Usage: python tools/lc_query.py [batch] [reps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def main():
    batch = int(sys.argv[1]) if len(sys.argv) > 1 else 1
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
    svc = sv.resnet50_service(batch)
    for _ in range(reps):
        for k in svc.kernels:
            tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd)
    torch.cuda.synchronize()
    print("ok", len(svc.kernels))


if __name__ == "__main__":
    main()
