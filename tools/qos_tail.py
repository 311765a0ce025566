"""Diagnose LC tail latency in a long steady-state window: one arm (Baymax paper rule by default)
on the bench's workload; prints the latency percentiles, the violations' time clustering and the
decision mix around the worst query (from the manager trace)."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--queries", type=int, default=10000)
    ap.add_argument("--policy", default="baymax")
    ap.add_argument("--load", type=float, default=0.8)
    ap.add_argument("--inflight", type=int, default=16)
    ap.add_argument("--be", default="table2")
    args = ap.parse_args()
    svc = sv.resnet50_service(32)
    sv.autotune_tile_n(svc)
    apps = sv.be_apps(sv.TABLE2_BE if args.be == "table2" else args.be.split(","))
    sv.prime_apps(apps)
    tk.tacker_model_clear()
    q = qos.QosRun(svc, apps, warp_split=24)
    q.calibrate()
    q.measure_service(max_inflight=args.inflight)
    pol = tk.POLICY_BAYMAX if args.policy.startswith("baymax") else tk.POLICY_TACKER
    rules = {"fuse_older": True} if args.policy.endswith("older") else {}
    win = args.queries * q.service_ms / args.load
    r = q.run_window(pol, win, 500.0, load=args.load, max_inflight=args.inflight, trace=True, **rules)
    lat = r.pop("trace"), None
    trace = lat[0]
    arr = np.array(r.pop("arrivals"))
    print(json.dumps({k: r[k] for k in ("lc_p50_ms", "lc_p99_ms", "violations", "queries", "be_kernels_per_s",
                                          "be_norm_thpt", "fused", "reordered", "idle_be")}))
    print("service_ms", q.service_ms, "t_be", {f"{a}:{j}": round(v, 3) for (a, j), v in q.t_be.items()})
    # per-query latency from the trace: the decision times of each query's kernels
    first = {}
    last = {}
    for d in trace:
        if d["query"] >= 0:
            first.setdefault(d["query"], d["t"])
            last[d["query"]] = d["t"]
    qs = sorted(last)
    waits = np.array([first[i] - arr[i] for i in qs])
    spans = np.array([last[i] - first[i] for i in qs])
    print("queue wait (issue of first kernel - arrival) p50/p99/max", np.percentile(waits, [50, 99, 100]))
    print("issue span (first to last kernel issue) p50/p99/max", np.percentile(spans, [50, 99, 100]))
    worst = qs[int(np.argmax(waits))]
    t0, t1 = arr[worst] - 60, first[worst]
    kinds = {}
    busy_be = 0.0
    for d in trace:
        if t0 <= d["t"] <= t1:
            kinds[d["action"]] = kinds.get(d["action"], 0) + 1
    arrivals_in = int(((arr >= t0) & (arr <= t1)).sum())
    print("worst query", worst, "wait", first[worst] - arr[worst], "decisions in the 60 ms before it", kinds,
          "arrivals in that span", arrivals_in)


if __name__ == "__main__":
    main()
