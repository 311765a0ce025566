"""Host cost of the native manager loop: an LC service alone (no BE queue), queries spaced far
apart, under the Baymax policy.  Compares the managed query latency with the sum of standalone
kernel times and with a plain back-to-back launch of the same kernels, and reports the host
wall-clock per decision.  Prints one JSON line.

  python tools/manager_overhead.py [--service resnet50] [--batch 1] [--queries 200]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--service", default="resnet50")
    ap.add_argument("--batch", type=int, default=1)
    ap.add_argument("--queries", type=int, default=200)
    args = ap.parse_args()
    svc = sv.resnet50_service(args.batch) if args.service == "resnet50" else sv.vgg16_service(args.batch)
    q = qos.QosRun(svc, [], qos_ms=50.0)
    q.calibrate()
    solo = q.query_solo_ms()
    stream = torch.cuda.current_stream()

    # back-to-back launches of the query's kernels through the C ABI, no manager
    def plain():
        for is_tc, d in q._kernel_list():
            if is_tc:
                tk.tacker_launch_original(d, None)
            else:
                tk.tacker_launch_original(None, d)
    plain()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    t0 = time.perf_counter()
    for _ in range(20):
        plain()
    t_host_plain = (time.perf_counter() - t0) / 20
    e1.record(stream)
    e1.synchronize()
    t_plain = e0.elapsed_time(e1) / 20

    m = tk.Manager(tk.POLICY_BAYMAX, stream=stream, simulate=False, max_inflight=4)
    kernels = q.lc_kernels()
    gap = 4.0 * solo
    base = m.stats().now_ms + 2.0
    qids = [m.submit_lc(kernels, base + i * gap) for i in range(args.queries)]
    t0 = time.perf_counter()
    m.run(50.0, base + args.queries * gap)
    wall = time.perf_counter() - t0
    lat = np.array([m.latency(i) for i in qids])
    st = m.stats()
    print(json.dumps({
        "service": f"{args.service}_b{args.batch}", "kernels_per_query": len(kernels),
        "query_solo_ms": solo, "plain_launch_ms": t_plain, "plain_host_ms_per_query": t_host_plain * 1e3,
        "managed_lat_p50_ms": float(np.median(lat)), "managed_lat_p99_ms": float(np.percentile(lat, 99)),
        "managed_overhead_p50_ms": float(np.median(lat)) - solo,
        "class_ms": {n: float(st.class_ms[c]) for c, n in enumerate(("lc_tc", "lc_cd", "fused", "be"))},
        "class_launches": {n: int(st.class_launches[c]) for c, n in enumerate(("lc_tc", "lc_cd", "fused", "be"))},
        "host_ms_per_query": {"poll": st.host_poll_ms / args.queries, "launch_and_events": st.host_launch_ms / args.queries,
                              "step_total": st.host_decide_ms / args.queries, "steps": st.host_steps / args.queries},
        "saturated_service_ms": q.measure_service(200),
        "wall_s": wall}))


if __name__ == "__main__":
    main()
