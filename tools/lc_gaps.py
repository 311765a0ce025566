"""Kernel-boundary cost of an LC query: per launch %globaltimer stamps (TACKER_LC_DBG=16, set
before import) of one ResNet-50 query's convs launched back to back; prints per kernel the gap
from the previous kernel's last CTA exit to this kernel's CTA-0 entry, prologue, dependency-wait
release, first stage landed, and its own span.

  (the stamps are compiled in only with -DTK_LC_GT=1: python -m paper_conf_hpca_zhaocczlllg22_b200.build
   --out variants/lib_gt.so -DTK_LC_GT=1, then TACKER_LIB=variants/lib_gt.so)
  TACKER_LC_DBG=16 python tools/lc_gaps.py [--batch 32] [--overlap 2]"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--overlap", type=int, default=2)
    args = ap.parse_args()
    svc = sv.resnet50_service(args.batch)
    sv.autotune_tile_n(svc)
    tk.tacker_set_launch_overlap(args.overlap)
    ks = [k for k in svc.kernels if k.is_tc]
    for _ in range(3):
        for k in ks:
            tk.tacker_launch_original(k.lc, None)
    torch.cuda.synchronize()
    tk.tacker_debug_lc_globaltimer()
    for k in ks:
        tk.tacker_launch_original(k.lc, None)
    g, n = tk.tacker_debug_lc_globaltimer()
    rows = []
    for i, k in enumerate(ks):
        e0, pro, dep, first, emin, epi, ex = (int(x) for x in g[i, :7])
        emin = (~emin) & ((1 << 64) - 1) if emin else e0
        prev_exit = int(g[i - 1, 6]) if i else e0
        rows.append({"name": k.name, "gap_prev_exit_to_entry_ns": e0 - prev_exit,
                     "entry_spread_ns": e0 - emin, "prologue_ns": pro - e0, "dep_wait_ns": dep - e0,
                     "first_stage_ns": first - e0, "epi_end_ns": epi - e0, "span_ns": ex - e0})
    tot = {key: sum(r[key] for r in rows) for key in rows[0] if key != "name"}
    print(json.dumps({"launches": n, "kernels": rows, "sum": tot, "query_ns": int(g[len(ks) - 1, 6]) - int(g[0, 0])}))


if __name__ == "__main__":
    main()
