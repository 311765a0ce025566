"""NEXT-2 reverse fusion, kernel level: LC CUDA-core kernel (ResNet-50 conv1 im2col at batch B)
with a BE tensor-core GEMM -- standalone, sequential, two streams and fused at several CUDA-core
warp splits (Eq. 11 overlap).  One JSON line per (GEMM, warp split).

  python tools/reverse_pair.py [--batch 32] [--gemm 4096,4096,4096]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200.qos import overlap_rate  # noqa: E402
from tools.corun import timed  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--gemm", default="4096,4096,4096;2048,2048,2048;8192,4096,1024")
    ap.add_argument("--ws", default="8,16,24")
    args = ap.parse_args()
    svc = sv.resnet50_service(args.batch, convs=synth.resnet50_convs(args.batch)[:1], conv1_im2col=True)
    cd = svc.kernels[0].cd
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    cur = torch.cuda.current_stream()
    for g in args.gemm.split(";"):
        M, N, K = (int(v) for v in g.split(","))
        app = sv.gemm_train_app(M, N, K, n=1)
        tc = app.kernels[0].desc

        def streams():
            s1.wait_stream(cur)
            s2.wait_stream(cur)
            tk.tacker_launch_original(tc, None, stream=s1)
            tk.tacker_launch_original(None, cd, stream=s2)
            cur.wait_stream(s1)
            cur.wait_stream(s2)

        t_tc = timed(lambda: tk.tacker_launch_original(tc, None))
        t_cd = timed(lambda: tk.tacker_launch_original(None, cd))
        t_seq = timed(lambda: tk.tacker_launch_original(tc, cd))
        t_st = timed(streams)
        for ws in (int(w) for w in args.ws.split(",")):
            try:
                f = tk.tacker_fuse(tc, cd, ws)
            except tk.TackerError as e:
                print(json.dumps({"gemm": [M, N, K], "ws": ws, "error": str(e)}))
                continue
            t_f = timed(lambda: f.launch())
            print(json.dumps({"batch": args.batch, "gemm": [M, N, K], "ws": ws, "t_gemm_us": t_tc, "t_im2col_us": t_cd,
                              "sequential_us": t_seq, "two_streams_us": t_st, "fused_us": t_f,
                              "overlap_eq11_fused": overlap_rate(t_tc, t_cd, t_f),
                              "overlap_eq11_two_streams": overlap_rate(t_tc, t_cd, t_st)}), flush=True)


if __name__ == "__main__":
    main()
