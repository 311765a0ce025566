"""Standalone time of every BE kernel of the Table II queue (back-to-back launches, CUDA events)
against its roofline (profiles/peaks.json + MEASURED_PEAKS.json).  Prints one JSON line."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk  # noqa: E402


def main():
    names = sys.argv[1].split(",") if len(sys.argv) > 1 else sv.TABLE2_BE
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"hbm_gbs": 6543.7}
    micro = json.load(open(os.path.join(ROOT, "profiles", "peaks.json")))
    bw, p_mufu, p_fma = peaks["hbm_gbs"] * 1e9, micro["mufu_sincos_tops"] * 1e12, micro["ffma_tflops"] * 1e12
    apps = sv.be_apps(names)
    sv.prime_apps(apps)
    out = {}
    for a in apps:
        for k in a.kernels:
            ms = qos._time(lambda: tk.tacker_launch_original(None, k.desc), 10)
            roof = max(k.bytes / bw, k.mufu / p_mufu if k.mufu else 0.0, k.flops / p_fma if k.bound == "fma" else 0.0)
            out[k.name] = {"ms": round(ms, 4), "roofline_ms": round(roof * 1e3, 4), "frac": round(roof * 1e3 / ms, 3),
                           "bound": k.bound}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
