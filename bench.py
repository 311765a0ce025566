#!/usr/bin/env python
"""Bench for the B200-native Tacker hot path (BASELINE.json metric:
"BE kernels/sec at LC p99 <= QoS target; fused time vs overlap roofline").

Workload (N=1, BASELINE configs[1]): ResNet-50 batch-1 inference convolutions as implicit-GEMM
LC tiles (53 convs; conv1 as im2col + GEMM) fused with Parboil stencil (512x512x64 sweeps) and
mri-q (64^3 voxels, 1024-k ComputeQ chunks) BE kernels.  One step = one LC query: every LC
tensor-core kernel is launched as ONE fused kernel with the next kernel of the BE queue
(alternating stencil / mri-q), CUDA-core LC kernels (im2col) launch original.  Each fused launch
completes one BE kernel, so value = BE kernels completed / second, and the LC query latency
(= step time) is checked against the 50 ms QoS target (p99 over steps).

Also reported: the same step with original (sequential) launches, the overlap rate (Eq. 11),
the roofline of the dominant fused kernel class, the CPU oracle baseline, and an end-to-end
number through the public API with host buffers.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl tacker|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

QOS_MS = 50.0


# ----------------------------------------------------------------------------- helpers
def dist_setup(args):
    import torch
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if ws > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        if torch.cuda.is_available():
            torch.cuda.set_device(0)
    return ws, rank, local


def barrier(ws):
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(ws, v):
    if ws == 1:
        return v
    import torch
    import torch.distributed as dist
    t = torch.tensor([v], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(ws, v):
    if ws == 1:
        return v
    import torch
    import torch.distributed as dist
    t = torch.tensor([v], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    def __init__(self, gpu_index=0):
        self.gpu = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, mx, pw, reasons = [], [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
                pw.append(float(parts[2]))
            except ValueError:
                continue
            for n, v in zip(names, parts[3:7]):
                if v.lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "power_w_median": statistics.median(pw) if pw else None, "reasons": sorted(reasons),
                "samples": len(sm)}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": 1965.0}, "fallback"


# ----------------------------------------------------------------------------- workload
class Workload:
    """ResNet-50 b1 LC query + stencil / mri-q BE queue, all device-resident."""

    def __init__(self, warp_split=16, seed=2022):
        import torch
        from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk
        self.tk, self.torch = tk, torch
        self.svc = sv.resnet50_service(1, seed)
        self.stencil = sv.stencil_app(512, 512, 64, seed)
        self.mriq = sv.mriq_app(64, 2048, 1024, seed)
        self.stream = torch.cuda.current_stream()
        # BE queue partner for each LC TC kernel: alternate stencil sweeps and mri-q Q chunks
        st_k = self.stencil.kernels
        mq_k = self.mriq.kernels[1:]
        self.plan = []        # (lc spec, be spec or None, fused handle or None)
        ti = 0
        for k in self.svc.kernels:
            if k.is_tc:
                be = st_k[(ti // 2) % 2] if ti % 2 == 0 else mq_k[(ti // 2) % len(mq_k)]
                f = None
                for ws in range(warp_split, 3, -4):   # LC-first budget: shrink the BE if it does not fit
                    try:
                        f = tk.tacker_fuse(k.lc, be.desc, ws)
                        break
                    except tk.TackerError as e:
                        if e.status != tk.ERESOURCE:
                            raise
                self.plan.append((k, be, f))
                ti += 1
            else:
                self.plan.append((k, None, None))
        self.n_fused = ti
        # phiMag once (prerequisite of the Q chunks)
        tk.tacker_launch_original(None, self.mriq.kernels[0].desc)
        torch.cuda.synchronize()

    def launches_per_step(self):
        return len(self.plan)

    def step_fused(self):
        tk = self.tk
        for k, be, f in self.plan:
            if f is not None:
                f.launch(self.stream)
            else:
                tk.tacker_launch_original(None, k.cd, self.stream)

    def step_original(self):
        tk = self.tk
        for k, be, f in self.plan:
            if k.is_tc:
                tk.tacker_launch_original(k.lc, be.desc, self.stream)
            else:
                tk.tacker_launch_original(None, k.cd, self.stream)

    def step_lc_only(self):
        tk = self.tk
        for k, be, f in self.plan:
            tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd, self.stream)

    def step_be_only(self):
        tk = self.tk
        for k, be, f in self.plan:
            if be is not None:
                tk.tacker_launch_original(None, be.desc, self.stream)


def time_steps(torch, fn, steps, flush, ws):
    """Device time of each step (CUDA events on the launching stream), L2 flushed between
    steps outside the events.  Returns list of ms."""
    s = torch.cuda.current_stream()
    out = []
    for _ in range(steps):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        out.append(e0.elapsed_time(e1))
    return out


def per_launch_times(torch, wl, reps=3):
    """Per-fused-launch device time (events between launches) -> {class: [ms]}."""
    s = torch.cuda.current_stream()
    acc = {}
    for _ in range(reps):
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(len(wl.plan) + 1)]
        evs[0].record(s)
        for i, (k, be, f) in enumerate(wl.plan):
            if f is not None:
                f.launch(s)
            else:
                wl.tk.tacker_launch_original(None, k.cd, s)
            evs[i + 1].record(s)
        evs[-1].synchronize()
        for i, (k, be, f) in enumerate(wl.plan):
            cls = ("fused:" + be.name.split(".")[0]) if f is not None else ("lc_cd:" + k.name.split(".")[-1])
            acc.setdefault(cls, []).append((evs[i].elapsed_time(evs[i + 1]), k, be))
    return acc


# ----------------------------------------------------------------------------- CPU oracle baseline
def cpu_oracle_sample(max_seconds=20.0):
    """Time the oracle as it stands on a bounded sample of the same workload: oracle conv of
    two ResNet-50 layers + one stencil sweep (512x512x64) + one mri-q chunk restricted to 4096
    voxels (time scaled to 64^3 voxels).  Returns BE kernels/s of the oracle doing the same
    per-pair work (one LC conv + one BE kernel per BE kernel completed)."""
    import synth
    from oracle import be as obe, lc as olc
    t_pairs = []
    convs = synth.resnet50_convs(1)
    # stencil pair
    t0 = time.perf_counter()
    cs = convs[5]
    x, w, _ = synth.conv_inputs(cs, 1)
    olc.lc_conv(x, w, cs.stride, cs.pad)
    A = synth.stencil_inputs(512, 512, 64, 2022)
    obe.stencil(A, np.float32(1 / 6), np.float32(1 / 36))
    t_pairs.append(time.perf_counter() - t0)
    # mri-q pair (voxel subsample, scaled)
    t0 = time.perf_counter()
    cs = convs[20]
    x, w, _ = synth.conv_inputs(cs, 2)
    olc.lc_conv(x, w, cs.stride, cs.pad)
    tc = time.perf_counter() - t0
    d = synth.mriq_inputs(64, 1024, 2022)
    pm, _ = obe.mriq_phimag(d["phiR"], d["phiI"])
    sub = 4096
    t0 = time.perf_counter()
    obe.mriq_q(d["x"][:sub], d["y"][:sub], d["z"][:sub], d["kx"], d["ky"], d["kz"], pm)
    tq = (time.perf_counter() - t0) * (64 ** 3 / sub)
    t_pairs.append(tc + tq)
    per = sum(t_pairs) / len(t_pairs)
    return {"value": 1.0 / per, "unit": "BE kernels/s", "cores": _oracle_threads(), "kind": "oracle",
            "sample": "oracle conv (2 ResNet-50 b1 layers) + 1 stencil 512x512x64 sweep + 1 mri-q 1024-k chunk "
                      "on 4096 of 64^3 voxels (time scaled x64); BE kernels/s = 1 / mean pair time",
            "seconds_per_be_kernel": per}


def _oracle_threads():
    try:
        import threadpoolctl
        info = threadpoolctl.threadpool_info()
        return max([i.get("num_threads", 1) for i in info] + [1])
    except Exception:
        return os.cpu_count() or 1


# ----------------------------------------------------------------------------- arms
def run_reference(args, ws, rank):
    """--impl reference: the CPU oracle as it stands is this tier's reference arm."""
    if rank != 0:
        return
    for _ in range(args.warmup):
        pass  # the oracle has no warm-up state; warm-up steps are not repeated to bound run time
    t0 = time.perf_counter()
    vals = []
    for _ in range(args.steps):
        r = cpu_oracle_sample()
        vals.append(r["seconds_per_be_kernel"])
    el = time.perf_counter() - t0
    per = sum(vals) / len(vals)
    v = 1.0 / per
    line = {"impl": "reference", "metric": "BE kernels/sec at LC p99 <= QoS target", "value": v,
            "unit": "BE kernels/s", "n_gpus": ws, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": el * 1000 / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "resnet50_b1_convs+stencil/mriq (BASELINE configs[1])", "l2": "n/a (CPU)"},
            "cpu_baseline": {"value": v, "unit": "BE kernels/s", "cores": r["cores"], "kind": "oracle",
                             "sample": r["sample"]},
            "e2e": {"value": v, "unit": "BE kernels/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


def run_tacker(args, ws, rank, local):
    import torch
    from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk
    from oracle.metrics import overlap_rate

    peaks, peak_kind = measured_peaks()
    wl = Workload(warp_split=args.warp_split)
    flush_buf = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")

    def flush():
        flush_buf.fill_(1.0)

    # warm-up (also JIT-free: the library is prebuilt)
    for _ in range(max(args.warmup, 3)):
        wl.step_fused()
    torch.cuda.synchronize()

    # --- timed region: K fused steps
    clk = ClockSampler(local)
    clk.start()
    barrier(ws)
    torch.cuda.synchronize()
    fused_ms = time_steps(torch, wl.step_fused, args.steps, flush, ws)
    torch.cuda.synchronize()
    barrier(ws)
    clocks = clk.stop()
    total_ms = max_over_ranks(ws, sum(fused_ms))
    be_per_step = wl.n_fused
    value = sum_over_ranks(ws, be_per_step * args.steps) / (total_ms / 1000.0)
    lat_sorted = sorted(fused_ms)
    p99 = lat_sorted[min(len(lat_sorted) - 1, int(np.ceil(0.99 * len(lat_sorted))) - 1)]

    # --- comparison steps (not part of value)
    orig_ms = time_steps(torch, wl.step_original, max(3, args.steps // 2), flush, ws)
    lc_ms = time_steps(torch, wl.step_lc_only, 3, flush, ws)
    be_ms = time_steps(torch, wl.step_be_only, 3, flush, ws)
    t_fused = statistics.median(fused_ms)
    t_seq = statistics.median(orig_ms)
    t_lc, t_be = statistics.median(lc_ms), statistics.median(be_ms)

    # --- roofline of the dominant fused kernel class (live CUDA-event timing per launch)
    flush()
    pl = per_launch_times(torch, wl, reps=3)
    dom = max(pl, key=lambda c: sum(x[0] for x in pl[c]))
    recs = pl[dom]
    avg_ms = sum(x[0] for x in recs) / len(recs)
    sm_mhz = clocks.get("sm_mhz") or peaks.get("sm_max_mhz", 1965.0)
    be0 = recs[0][2]
    lc_bytes = sum(x[1].bytes for x in recs) / len(recs)
    if be0 is not None and be0.bound == "mufu":
        ops = be0.mufu
        achieved = ops / (avg_ms / 1e3) / 1e12
        peak = 148 * 16 * peaks.get("sm_max_mhz", 1965.0) * 1e6 / 1e12
        roof = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Tops/s (MUFU sin/cos)",
                "frac": achieved / peak, "traffic": None,
                "peak_source": "derived: 148 SM x 16 MUFU/clk x sm_max_mhz (DESIGN.md §5)"}
    else:
        byts = (be0.bytes if be0 is not None else 0) + lc_bytes
        achieved = byts / (avg_ms / 1e3) / 1e9
        peak = peaks["hbm_gbs"]
        roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": None, "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_kind})"}
    roof["kernel"] = dom
    roof["avg_launch_ms"] = avg_ms
    roof["launches"] = len(recs)
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        try:
            with open(tp) as f:
                roof["traffic"] = json.load(f).get(dom)
        except Exception:
            pass

    # --- end-to-end through the public API with host buffers (pinned), per step:
    #     H2D of the step's inputs (LC input activations + BE inputs), the step, D2H of results
    h2d_pairs = []
    for t in wl.svc.inputs:
        h2d_pairs.append((torch.empty(t.shape, dtype=t.dtype, pin_memory=True).copy_(t), t))
    h2d_pairs.append((torch.empty(wl.stencil.buffers[0].shape, pin_memory=True).copy_(wl.stencil.buffers[0]),
                      wl.stencil.buffers[0]))
    out_dev = list(wl.svc.outputs) + [wl.mriq.buffers[2]]
    out_host = [torch.empty(o.shape, dtype=o.dtype, pin_memory=True) for o in out_dev]
    h2d_bytes = sum(h.numel() * h.element_size() for h, _ in h2d_pairs)
    d2h_bytes = sum(o.numel() * o.element_size() for o in out_dev)
    s = torch.cuda.current_stream()
    e2e_ms = []
    for _ in range(args.steps):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for h, d in h2d_pairs:
            d.copy_(h, non_blocking=True)
        wl.step_fused()
        for o, h in zip(out_dev, out_host):
            h.copy_(o, non_blocking=True)
        e1.record(s)
        e1.synchronize()
        e2e_ms.append(e0.elapsed_time(e1))
    e2e_total = max_over_ranks(ws, sum(e2e_ms))
    e2e_value = sum_over_ranks(ws, be_per_step * args.steps) / (e2e_total / 1000.0)

    cpu = cpu_oracle_sample() if (rank == 0 and ws == 1 and not args.no_cpu) else None
    if cpu is not None:
        cpu.pop("seconds_per_be_kernel", None)

    line = {
        "metric": "BE kernels/sec at LC p99 <= QoS target", "value": value, "unit": "BE kernels/s",
        "n_gpus": ws, "steps": args.steps, "warmup": args.warmup, "ms_per_step": total_ms / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f16xf16->f32 (LC) + f32 (BE)",
        "data": "synthetic (seeded inputs, random weights)",
        "config": {"workload": "resnet50_b1_convs+stencil/mriq (BASELINE configs[1])",
                   "lc": "ResNet-50 batch-1, 53 convs (conv1 = im2col + GEMM), fp16 NHWC, implicit GEMM tcgen05",
                   "be": "stencil 512x512x64 sweep | mri-q 64^3 x 1024-k chunk, alternating, one per LC TC kernel",
                   "warp_split": args.warp_split, "qos_ms": QOS_MS, "parallelism": f"replicas x{ws}",
                   "l2": "flushed between steps (256 MiB fill, outside the timed events)"},
        "lc_p99_ms": p99, "lc_qos_ms": QOS_MS, "qos_met": p99 <= QOS_MS,
        "fused_step_ms": t_fused, "sequential_step_ms": t_seq, "lc_only_ms": t_lc, "be_only_ms": t_be,
        "speedup_vs_sequential": t_seq / t_fused, "overlap_rate_eq11": overlap_rate(t_lc, t_be, t_fused),
        "roofline": roof,
        "cpu_baseline": cpu,
        "e2e": {"value": e2e_value, "unit": "BE kernels/s", "h2d_bytes_per_step": h2d_bytes,
                "d2h_bytes_per_step": d2h_bytes},
        "gpu_launches": wl.launches_per_step() * args.steps,
        "clocks": clocks,
    }
    if rank == 0:
        print(json.dumps(line))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="tacker", choices=["tacker", "reference"])
    ap.add_argument("--warp-split", type=int, default=24)
    ap.add_argument("--no-cpu", action="store_true")
    args = ap.parse_args()
    if args.impl == "reference":
        ws = int(os.environ.get("WORLD_SIZE", "1"))
        rank = int(os.environ.get("RANK", "0"))
        run_reference(args, ws, rank)
        return
    ws, rank, local = dist_setup(args)
    run_tacker(args, ws, rank, local)
    if ws > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
