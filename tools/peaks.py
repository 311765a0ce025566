"""Measure this box's roofline peaks (SURVEY §8(d) "Peaks"): FP32 FFMA, MUFU sin/cos and rsqrt,
fp16 tcgen05 MMA (M=128, N=256) and an HBM copy, with the SM clock sampled by nvidia-smi during the
run; writes profiles/peaks.json (read by bench.py as the FFMA / MUFU peaks).

  python tools/peaks.py [--out profiles/peaks.json]"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MICRO = os.path.join(ROOT, "tools", "micro")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "peaks.json"))
    args = ap.parse_args()
    exe = os.path.join(MICRO, "peaks_bench")
    if not os.path.exists(exe):
        subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17",
                               "-I", os.path.join(ROOT, "paper_conf_hpca_zhaocczlllg22_b200", "csrc", "kernels"),
                               "-I", os.path.join(ROOT, "include"), "-o", exe, exe + ".cu"])
    lines = []
    proc = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active",
                             "--format=csv,noheader,nounits", "-lms", "50"], stdout=subprocess.PIPE, text=True)
    threading.Thread(target=lambda: [lines.append(l) for l in proc.stdout], daemon=True).start()
    time.sleep(0.3)
    out = subprocess.check_output([exe], text=True)
    proc.terminate()
    res = json.loads(out.strip().splitlines()[-1])
    sm = [float(l.split(",")[0]) for l in lines if l.count(",") >= 3]
    res["sm_mhz_median"] = statistics.median(sm) if sm else None
    res["sm_mhz_max"] = max(sm) if sm else None
    res["how"] = ("tools/micro/peaks_bench.cu: FFMA = 8 independent fma.rn chains per thread (148x8 CTAs x 256); "
                  "MUFU = sin.approx + cos.approx (4 chains) and rsqrt.approx (8 chains); tcgen05 = one elected "
                  "thread per SM issuing M=128 N=256 K=16 kind::f16 MMAs from resident SW128 operands; HBM = float4 "
                  "copy of 1 GiB (read + write bytes); best of 5-10 launches, CUDA events")
    res["when"] = time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime())
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
