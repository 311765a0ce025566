"""Launch the LC kernels of one ResNet-50 query (original launches, no BE) `reps` times, for ncu
captures of the bench's dominant kernel class (tile widths autotuned as in the bench when the third
argument is 1).  Usage: python tools/lc_query.py [batch] [reps] [autotune]"""
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
    if len(sys.argv) > 3 and sys.argv[3] == "1":
        sv.autotune_tile_n(svc)
    for k in svc.kernels:   # warm-up query (plans, tensor maps) outside the NVTX range
        tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd)
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_push("query")   # ncu --nvtx --nvtx-include "query/"
    for _ in range(reps):
        for k in svc.kernels:
            tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd)
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_pop()
    print("ok", len(svc.kernels))


if __name__ == "__main__":
    main()
