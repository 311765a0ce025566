"""fft BE kernel alone (original launch) against its HBM roofline (16 bytes per
complex point, read + write): median of back-to-back launches between CUDA events,.

  python tools/fft_bench.py [--batch 16384] [--n 1024]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk  # noqa: E402

sys.path.insert(0, os.path.join(ROOT, "tools"))
from corun import timed  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=1 << 14)
    ap.add_argument("--n", type=int, default=1024)
    a = ap.parse_args()
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    bw = peaks["hbm_gbs"]
    x = torch.from_numpy(synth.fft_inputs(a.batch, a.n, 0)).cuda()
    y = torch.zeros_like(x)
    tw = torch.zeros(a.n, 2, device="cuda")
    tk.tacker_launch_original(None, tk.be_fft_twiddle(tw, a.n))
    d = tk.be_fft(x, y, tw)
    us = timed(lambda: tk.tacker_launch_original(None, d), reps=20)
    roof_us = 16.0 * a.batch * a.n / (bw * 1e9) * 1e6
    print(json.dumps({"kernel": "fft", "batch": a.batch, "n": a.n, "us": us, "hbm_roofline_us": roof_us,
                      "frac": roof_us / us, "peak_gbps": bw}))


if __name__ == "__main__":
    main()
