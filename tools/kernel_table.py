"""Per-kernel diagnostic: original LC / original BE / fused durations for the bench's fused-step
pairs (CUDA events, L2 flushed before each measurement).  Prints a table and one JSON line.
Usage: python tools/kernel_table.py [warp_split]"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def timeit(fn, reps=5, flush=None):
    s = torch.cuda.current_stream()
    out = []
    for _ in range(reps):
        if flush:
            flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        out.append(e0.elapsed_time(e1))
    return statistics.median(out)


def main():
    ws = int(sys.argv[1]) if len(sys.argv) > 1 else 24
    svc = sv.resnet50_service(1, 2022)
    stencil, mriq = sv.stencil_app(), sv.mriq_app()
    tk.tacker_launch_original(None, mriq.kernels[0].desc)
    step = bench.FusedStep(svc, stencil, mriq, ws)
    buf = torch.empty(64 * 1024 * 1024, device="cuda")
    flush = lambda: buf.fill_(1.0)
    rows = []
    for k, be, f in step.plan:
        if f is None:
            continue
        t_lc = timeit(lambda: tk.tacker_launch_original(k.lc, None), flush=flush)
        t_be = timeit(lambda: tk.tacker_launch_original(None, be.desc), flush=flush)
        t_f = timeit(lambda: f.launch(), flush=flush)
        i = f.info()
        rows.append(dict(lc=k.name, be=be.name, t_lc=t_lc, t_be=t_be, t_fused=t_f, seq=t_lc + t_be,
                         gain=(t_lc + t_be) / t_f, tiles=i.lc_tiles, bn=i.lc_tile_n, stages=i.lc_stages,
                         regs=i.regs_per_thread, smem=i.smem_bytes, be_warps=i.be_warps))
    for r in rows:
        print(f"{r['lc']:28s} {r['be']:14s} lc {r['t_lc']*1e3:7.1f}us be {r['t_be']*1e3:7.1f}us "
              f"fused {r['t_fused']*1e3:7.1f}us seq/fused {r['gain']:.2f} tiles {r['tiles']} bn {r['bn']} "
              f"st {r['stages']} regs {r['regs']} bew {r['be_warps']}")
    print(json.dumps({"warp_split": ws, "rows": rows}))


if __name__ == "__main__":
    main()
