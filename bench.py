#!/usr/bin/env python
"""Bench for the B200-native Tacker hot path (BASELINE.json metric:
"BE kernels/sec at LC p99 <= QoS target; fused time vs overlap roofline").

Workload (N=1): BASELINE configs[3] (SURVEY config 4), QoS-managed co-location -- ResNet-50 at
the paper's batch 32 (Table II) as the LC service (53 convs as implicit-GEMM tcgen05
kernels, split-K where few tiles; conv1 = im2col + GEMM) with a BE queue of two Parboil
applications, stencil (512x512x64 sweeps) and mri-q (64^3 voxels, 2048 k in two 1024-k chunks).

* Headline (`value`): the QoS-managed run.  One step = one LC query; queries arrive as a
  Poisson process at 80 % of the peak LC load (peak = the manager's LC-only
  service rate, measured), the native manager (tacker_manager_run, Tacker policy) launches
  fused / original / reordered kernels from each query's headroom under a 50 ms QoS target
  (with B200 reading 18: an older query may fuse within the headroom of every later query, minus
  a 15 ms guard; the paper-literal newest-query-only rule is reported as `tacker_paper`).
  value = BE kernels completed per second over the K timed queries (CUDA events on the manager
  stream), with the queries' p99 latency checked against the target.  The same trace under the
  Baymax policy (fusion off) gives Eq. 10; a PTB-sliced Tacker run (reading 13) is reported too.
* `e2e`: the same managed run through the public API where every query also moves its input
  images host->device and its result device->host (pinned host memory, UVA copy kernels inside
  the managed stream).
* `roofline`: the dominant launch class of the timed run (LC convs: achieved vs tensor / HBM
  peak).  `fused_step` + `roofline_fused`: BASELINE configs[1] -- every LC tensor-core kernel of a
  ResNet-50 batch-1 query fused with the next BE kernel (fused time vs overlap roofline and vs
  the sequential original launches); `config1_resnet50_b1` = the managed protocol at batch 1.
* `cpu_baseline`: the CPU oracle on a bounded sample.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--batch 32] [--impl tacker|reference]
"""
from __future__ import annotations

import argparse
import json
import math
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
# Manager options of the headline Tacker run: B200 reading 18 -- an older query may
# fuse / reorder within the headroom of every later active query, minus a 0.3 x QoS guard (qos.py).
# The paper-literal rule (only the newest query fuses) is reported as tacker_paper.
HEADLINE = {"fuse_older": True}
LOAD = 0.8
METRIC = "BE kernels/sec at LC p99 <= QoS target"
WORKLOAD = "resnet50_b{b} LC + stencil/mriq BE queue, QoS 50 ms (BASELINE configs[3])"


# ----------------------------------------------------------------------------- helpers
_BACKEND = "nccl"


def dist_setup(simulate=False):
    """One process per GPU (replicas: no data-path collective).  The process group only carries
    the barrier and the max/sum reductions of the timing; --simulate uses gloo on CPU."""
    global _BACKEND
    import torch
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    _BACKEND = "gloo" if simulate else "nccl"
    if ws > 1:
        import torch.distributed as dist
        if simulate:
            dist.init_process_group("gloo")
        else:
            torch.cuda.set_device(local)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    elif not simulate and torch.cuda.is_available():
        torch.cuda.set_device(0)
    return ws, rank, local


def barrier(ws):
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()


def reduce_ranks(ws, v, op="max"):
    if ws == 1:
        return v
    import torch
    import torch.distributed as dist
    t = torch.tensor([v], dtype=torch.float64, device="cpu" if _BACKEND == "gloo" else "cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
    return float(t.item())


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    def __init__(self, gpu_index=0):
        self.gpu, self.proc, self.lines = gpu_index, None, []

    def start(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            threading.Thread(target=self._read, daemon=True).start()
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
            return json.load(f), "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": 1965.0}, "fallback"


# ----------------------------------------------------------------------------- kernel-level step
class FusedStep:
    """Every LC tensor-core kernel of one query fused with the next BE kernel (alternating a
    stencil sweep and a mri-q Q chunk); CUDA-core LC kernels (im2col) launch original."""

    def __init__(self, svc, stencil, mriq, warp_split):
        from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk
        self.tk, self.svc = tk, svc
        st_k, mq_k = stencil.kernels, mriq.kernels[1:]
        self.plan = []
        ti = 0
        for k in svc.kernels:
            if not k.is_tc:
                self.plan.append((k, None, None))
                continue
            be = st_k[(ti // 2) % 2] if ti % 2 == 0 else mq_k[(ti // 2) % len(mq_k)]
            f = None
            for ws in range(warp_split, 3, -4):    # LC-first budget: shrink the BE if needed
                try:
                    f = tk.tacker_fuse(k.lc, be.desc, ws)
                    break
                except tk.TackerError as e:
                    if e.status != tk.ERESOURCE:
                        raise
            self.plan.append((k, be, f))
            ti += 1
        self.n_fused = ti

    def fused(self):
        for k, be, f in self.plan:
            if f is not None:
                f.launch()
            else:
                self.tk.tacker_launch_original(None, k.cd)

    def original(self):
        for k, be, f in self.plan:
            self.tk.tacker_launch_original(k.lc if k.is_tc else None, be.desc if be is not None else k.cd)

    def lc_only(self):
        for k, be, f in self.plan:
            self.tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd)

    def be_only(self):
        for k, be, f in self.plan:
            if be is not None:
                self.tk.tacker_launch_original(None, be.desc)

    def two_streams(self):
        """Co-running baseline (NEXT-4, the paper's Stream co-location of Fig. 20): the LC
        kernels in order on one stream, the BE kernels in order on another, original kernels,
        the hardware scheduler interleaving their CTAs; joined back into the current stream."""
        import torch
        cur = torch.cuda.current_stream()
        if not hasattr(self, "_streams"):
            self._streams = (torch.cuda.Stream(), torch.cuda.Stream())
        s_lc, s_be = self._streams
        s_lc.wait_stream(cur)
        s_be.wait_stream(cur)
        for k, be, f in self.plan:
            self.tk.tacker_launch_original(k.lc if k.is_tc else None, None if k.is_tc else k.cd, stream=s_lc)
            if be is not None:
                self.tk.tacker_launch_original(None, be.desc, stream=s_be)
        cur.wait_stream(s_lc)
        cur.wait_stream(s_be)


def time_steps(torch, fn, steps, flush):
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


def per_launch_times(torch, step, reps=3):
    """Per-fused-launch device time (events between launches on the launching stream)."""
    s = torch.cuda.current_stream()
    acc = {}
    for _ in range(reps):
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(len(step.plan) + 1)]
        evs[0].record(s)
        for i, (k, be, f) in enumerate(step.plan):
            if f is not None:
                f.launch()
            else:
                step.tk.tacker_launch_original(None, k.cd)
            evs[i + 1].record(s)
        evs[-1].synchronize()
        for i, (k, be, f) in enumerate(step.plan):
            cls = ("fused:" + be.name.split(".")[0]) if f is not None else ("lc_cd:" + k.name.split(".")[-1])
            acc.setdefault(cls, []).append((evs[i].elapsed_time(evs[i + 1]), k, be))
    return acc


def kernel_level(torch, step, flush, peaks, peak_kind, clocks, steps):
    from paper_conf_hpca_zhaocczlllg22_b200.qos import overlap_rate   # Eq. 11
    fused_ms = time_steps(torch, step.fused, steps, flush)
    orig_ms = time_steps(torch, step.original, max(3, steps // 2), flush)
    lc_ms = time_steps(torch, step.lc_only, 3, flush)
    be_ms = time_steps(torch, step.be_only, 3, flush)
    st_ms = time_steps(torch, step.two_streams, max(3, steps // 2), flush)
    t_f, t_s = statistics.median(fused_ms), statistics.median(orig_ms)
    t_lc, t_be = statistics.median(lc_ms), statistics.median(be_ms)
    t_st = statistics.median(st_ms)
    flush()
    pl = per_launch_times(torch, step)
    dom = max(pl, key=lambda c: sum(x[0] for x in pl[c]))
    recs = pl[dom]
    avg_ms = sum(x[0] for x in recs) / len(recs)
    be0 = recs[0][2]
    lc_bytes = sum(x[1].bytes for x in recs) / len(recs)
    if be0 is not None and be0.bound == "mufu":
        achieved = be0.mufu / (avg_ms / 1e3) / 1e12
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
    roof.update(kernel=dom, avg_launch_ms=avg_ms, launches=len(recs), stream="launching stream (torch current)")
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            roof["traffic"] = json.load(f).get(dom)
    # BASELINE's overlap roofline per fused launch: max(F_LC / P_tensor, BE at its roofline,
    # (B_LC + B_BE) / BW), summed over the step (CUDA-core LC kernels at their HBM time)
    p_tensor = peaks["bf16_tflops"] * 1e12          # fp16 runs at the bf16 rate
    bw = peaks["hbm_gbs"] * 1e9
    p_mufu = 148 * 16 * peaks.get("sm_max_mhz", 1965.0) * 1e6
    t_roof = 0.0
    for k, be, f in step.plan:
        if f is None:
            t_roof += k.bytes / bw
            continue
        t_be_roof = be.mufu / p_mufu if be.bound == "mufu" else be.bytes / bw
        t_roof += max(k.flops / p_tensor, t_be_roof, (k.bytes + be.bytes) / bw)
    fs = {"fused_step_ms": t_f, "sequential_step_ms": t_s, "lc_only_ms": t_lc, "be_only_ms": t_be,
          "speedup_vs_sequential": t_s / t_f, "overlap_rate_eq11": overlap_rate(t_lc, t_be, t_f),
          "two_streams_step_ms": t_st, "overlap_rate_eq11_two_streams": overlap_rate(t_lc, t_be, t_st),
          "overlap_roofline_ms": t_roof * 1e3, "overlap_roofline_frac": t_roof * 1e3 / t_f,
          "be_kernels_per_s": step.n_fused / (t_f / 1e3), "launches_per_step": len(step.plan)}
    # LC convolutions alone against the tensor peak (batch 1: latency-bound, few tiles)
    lc_flops = sum(k.flops for k, _, _ in step.plan if k.is_tc)
    fs["lc_only_tflops"] = lc_flops / (t_lc / 1e3) / 1e12
    fs["lc_only_tensor_frac"] = fs["lc_only_tflops"] * 1e12 / p_tensor
    return fs, roof


# ----------------------------------------------------------------------------- CPU oracle baseline
def cpu_oracle_sample(small=False, batch=32):
    """The oracle as it stands on a bounded sample of the same workload: oracle conv of two
    ResNet-50 layers on one image (time x batch: the conv is linear in the batch) + one stencil
    sweep (512x512x64, or an 8-plane slab scaled x8 when small) + one mri-q 1024-k chunk on 4096
    (small: 256) of the 64^3 voxels, time scaled to the full kernel.  Returns BE kernels/s =
    1 / mean (LC conv + BE kernel) pair time."""
    import synth
    from oracle import be as obe, lc as olc
    convs = synth.resnet50_convs(1)
    t_pairs = []
    nz, zscale = (10, 64 / 8) if small else (64, 1.0)
    t0 = time.perf_counter()
    cs = convs[5]
    x, w, _ = synth.conv_inputs(cs, 1)
    olc.lc_conv(x, w, cs.stride, cs.pad)
    tc = (time.perf_counter() - t0) * batch
    A = synth.stencil_inputs(512, 512, nz, 2022)
    t0 = time.perf_counter()
    obe.stencil(A, np.float32(1 / 6), np.float32(1 / 36))
    t_pairs.append(tc + (time.perf_counter() - t0) * zscale)
    t0 = time.perf_counter()
    cs = convs[20]
    x, w, _ = synth.conv_inputs(cs, 2)
    olc.lc_conv(x, w, cs.stride, cs.pad)
    tc = (time.perf_counter() - t0) * batch
    d = synth.mriq_inputs(64, 1024, 2022)
    pm, _ = obe.mriq_phimag(d["phiR"], d["phiI"])
    sub = 256 if small else 4096
    t0 = time.perf_counter()
    obe.mriq_q(d["x"][:sub], d["y"][:sub], d["z"][:sub], d["kx"], d["ky"], d["kz"], pm)
    t_pairs.append(tc + (time.perf_counter() - t0) * (64 ** 3 / sub))
    per = sum(t_pairs) / len(t_pairs)
    desc = (f"oracle conv (2 ResNet-50 layers, 1 image, time x{batch}) + 1 stencil 512x512x64 sweep ({'8-plane slab x8' if small else 'full'})"
            f" + 1 mri-q 1024-k chunk on {sub} of 64^3 voxels (time scaled x{64 ** 3 // sub}); "
            "BE kernels/s = 1 / mean pair time")
    return {"value": 1.0 / per, "unit": "BE kernels/s", "cores": _oracle_threads(), "kind": "oracle",
            "sample": desc, "seconds_per_be_kernel": per}


def _oracle_threads():
    try:
        import threadpoolctl
        return max([i.get("num_threads", 1) for i in threadpoolctl.threadpool_info()] + [1])
    except Exception:
        return os.cpu_count() or 1


# ----------------------------------------------------------------------------- arms
def run_reference(args, ws, rank):
    """--impl reference: the CPU oracle as it stands is this tier's reference arm."""
    if rank != 0:
        return
    for _ in range(min(args.warmup, 3)):    # untimed warm-up steps (bounded)
        cpu_oracle_sample(small=True, batch=args.batch)
    # bounded: each step is a small sample (~0.3 s); at most 120 s of steps
    t0 = time.perf_counter()
    vals, r = [], None
    for _ in range(args.steps):
        r = cpu_oracle_sample(small=True, batch=args.batch)
        vals.append(r["seconds_per_be_kernel"])
        if time.perf_counter() - t0 > 120.0:
            break
    el = time.perf_counter() - t0
    v = 1.0 / (sum(vals) / len(vals))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "BE kernels/s", "n_gpus": ws,
            "steps": len(vals), "warmup": args.warmup, "ms_per_step": el * 1000 / len(vals),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": WORKLOAD.format(b=args.batch), "l2": "n/a (CPU)"},
            "cpu_baseline": {"value": v, "unit": "BE kernels/s", "cores": r["cores"], "kind": "oracle",
                             "sample": "per step: " + r["sample"]},
            "e2e": {"value": v, "unit": "BE kernels/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


def managed_runs(q, tk, steps, seed, inflight, variants=("tacker", "baymax", "tacker_slice")):
    """The same Poisson trace under each policy (the headline Tacker run first, timed by the
    caller's window); returns {variant: result}."""
    out = {}
    kw = {"tacker": (tk.POLICY_TACKER, dict(HEADLINE)), "baymax": (tk.POLICY_BAYMAX, {}),
          "tacker_paper": (tk.POLICY_TACKER, {}),
          "baymax_older": (tk.POLICY_BAYMAX, dict(HEADLINE)),
          "tacker_fuse_first": (tk.POLICY_TACKER, dict(HEADLINE, reorder_only_unfused=True)),
          "tacker_slice_ff": (tk.POLICY_TACKER, dict(HEADLINE, slice_be=True, reorder_only_unfused=True)),
          "tacker_slice_noreorder": (tk.POLICY_TACKER, dict(HEADLINE, slice_be=True, reorder_only_unfused=2)),
          "tacker_slice": (tk.POLICY_TACKER, dict(HEADLINE, slice_be=True)),
          "tacker_no_reverse": (tk.POLICY_TACKER, dict(HEADLINE, reverse_fusion=False))}
    for v in variants:
        pol, extra = kw[v]
        out[v] = q.run(pol, steps, load=LOAD, seed=seed, max_inflight=inflight, **extra)
    return out


def lc_class_roofline(q, peaks, peak_kind, svc):
    """Roofline of the LC tensor-core kernels (the dominant launch class of the managed run):
    per kernel the algorithmic flops (2 NPQ K CRS) and bytes (x, w, out once), timed back to back
    with CUDA events on the launching stream (QosRun.calibrate).  The bound is the one that gives
    the larger roofline time summed over the query."""
    off = 1 if getattr(q, "io", None) else 0
    tc = [(k, q.t_lc[i + off]) for i, k in enumerate(svc.kernels) if k.is_tc]
    p_t, bw = peaks["bf16_tflops"] * 1e12, peaks["hbm_gbs"] * 1e9
    fl = sum(k.flops for k, _ in tc)
    by = sum(k.bytes for k, _ in tc)
    t_ms = sum(t for _, t in tc)
    t_roof = sum(max(k.flops / p_t, k.bytes / bw) for k, _ in tc)
    n = len(tc)
    if fl / p_t >= by / bw:
        ach = fl / n / (t_ms / n / 1e3) / 1e12
        roof = {"bound": "tensor", "achieved": ach, "peak": peaks["bf16_tflops"], "unit": "TFLOP/s",
                "frac": ach / peaks["bf16_tflops"], "per_launch_work": "mean 2*NPQ*K*CRS of the TC convs",
                "peak_source": f"MEASURED_PEAKS.json bf16_tflops burst ({peak_kind}); fp16 = bf16 rate"}
    else:
        ach = by / n / (t_ms / n / 1e3) / 1e9
        roof = {"bound": "hbm", "achieved": ach, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": ach / peaks["hbm_gbs"], "per_launch_work": "mean 2*(NHWC + KRSC + NPQK) bytes of the TC convs",
                "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_kind})"}
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp) and svc.name == "resnet50_b32":
        with open(tp) as f:
            traffic = json.load(f).get("lc_tc")
    roof.update(traffic=traffic, kernel=f"LC tensor-core convs of {svc.name} (implicit GEMM tcgen05, split-K where few tiles)",
                avg_launch_ms=t_ms / n, launches_per_query=n,
                per_kernel_roofline_frac=t_roof * 1e3 / t_ms,
                stream="launching stream, back-to-back launches (CUDA events)")
    return roof


def run_tacker(args, ws, rank, local):
    import torch
    from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk

    peaks, peak_kind = measured_peaks()
    seed = 2022 + rank
    svc = sv.resnet50_service(args.batch, seed)
    sv.autotune_tile_n(svc)                                      # LC tile width per conv, measured
    stencil = sv.stencil_app(512, 512, 64, seed)
    mriq = sv.mriq_app(64, 2048, 1024, seed)
    tk.tacker_launch_original(None, mriq.kernels[0].desc)       # phiMag ready for the Q chunks
    flush_buf = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")

    def flush():
        flush_buf.fill_(1.0)

    # ---- calibration (predictor, §VI-C) and the peak LC load -- untimed
    tk.tacker_model_clear()
    q = qos.QosRun(svc, [stencil, mriq], warp_split=args.warp_split, qos_ms=QOS_MS)
    q.calibrate()
    q.measure_service(max_inflight=args.inflight)
    # ---- warm-up queries (untimed)
    q.run(tk.POLICY_TACKER, max(args.warmup, 3), load=LOAD, seed=1000 + rank, max_inflight=args.inflight, **HEADLINE)
    torch.cuda.synchronize()

    # ---- timed region: K queries under the Tacker policy
    clk = ClockSampler(local)
    clk.start()
    barrier(ws)
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_push("timed")      # ncu --nvtx --nvtx-include "timed/" selects these launches
    res = q.run(tk.POLICY_TACKER, args.steps, load=LOAD, seed=2000 + rank, max_inflight=args.inflight, **HEADLINE)
    torch.cuda.nvtx.range_pop()
    torch.cuda.synchronize()
    barrier(ws)
    clocks = clk.stop()
    elapsed_ms = reduce_ranks(ws, res["elapsed_ms"], "max")
    be_total = reduce_ranks(ws, res["be_kernels"], "sum")
    value = be_total / (elapsed_ms / 1e3)
    p99 = reduce_ranks(ws, res["lc_p99_ms"], "max")

    # ---- Baymax (Eq. 10) and PTB-sliced Tacker on the same trace
    other = managed_runs(q, tk, args.steps, 2000 + rank, args.inflight,
                         ("baymax", "tacker_slice", "tacker_paper", "baymax_older", "tacker_fuse_first",
                          "tacker_slice_ff", "tacker_slice_noreorder"))
    bay, slc, old, bay18 = other["baymax"], other["tacker_slice"], other["tacker_paper"], other["baymax_older"]

    # ---- e2e: the same managed run, each query with its H2D input + D2H result
    qi = qos.QosRun(svc, [stencil, mriq], warp_split=args.warp_split, qos_ms=QOS_MS).with_io()
    qi.pairs, qi.ws_of, qi.t_be, qi.lr_be = q.pairs, q.ws_of, q.t_be, q.lr_be
    qi.t_lc = []
    for is_tc, d in qi._kernel_list():
        qi.t_lc.append(qos._time(lambda: tk.tacker_launch_original(d, None) if is_tc
                                  else tk.tacker_launch_original(None, d), 5))
    qi.measure_service(max_inflight=args.inflight)
    e2e = qi.run(tk.POLICY_TACKER, args.steps, load=LOAD, seed=2000 + rank, max_inflight=args.inflight, **HEADLINE)
    e2e_value = reduce_ranks(ws, e2e["be_kernels"], "sum") / (reduce_ranks(ws, e2e["elapsed_ms"], "max") / 1e3)

    # ---- NEXT-2 reverse fusion side run: the same service with a tensor-core training BE app added
    #      (Table II's DNN-training BE jobs); conv1's im2col (an LC CUDA-core kernel) may now fuse
    #      with a BE GEMM.  The b32 calibration is reused; only the new pairs are fitted.
    reverse = None
    if not args.no_extra:
        train = sv.gemm_train_app(4096, 4096, 4096, n=2, seed=seed + 3)
        qr = qos.QosRun(svc, [stencil, mriq], warp_split=args.warp_split, qos_ms=QOS_MS)
        qr.t_lc, qr.t_be, qr.pairs, qr.ws_of, qr.lr_be = q.t_lc, dict(q.t_be), dict(q.pairs), q.ws_of, q.lr_be
        qr.service_ms = q.service_ms
        qr.add_tc_apps([train])
        rr = managed_runs(qr, tk, args.steps, 2000 + rank, args.inflight, ("tacker", "tacker_no_reverse", "baymax"))
        reverse = {"workload": "resnet50_b%d LC + stencil / mri-q / train-GEMM (2 x 4096^3 fp16) BE queue" % args.batch,
                   "train_gemm_ms": [qr.t_be[(2, j)] for j in range(len(train.kernels))],
                   "im2col_ms": qr.t_lc[0], "pairs": {}}
        for j, bk in enumerate(train.kernels):
            f = tk.tacker_fuse(bk.desc, svc.kernels[0].cd, qr.REV_WS)
            pk = f.keys()[2]
            reverse["pairs"][pk] = {"fused_ms": qos._time(lambda: f.launch(), 5),
                                    "predicted_ms": tk.tacker_pair_predict(pk, qr.t_be[(2, j)], qr.t_lc[0]),
                                    "in_model": pk in qr.pairs}
        for v, r in rr.items():
            reverse[v] = {k: r[k] for k in ("be_kernels_per_s", "be_norm_thpt", "lc_p99_ms", "qos_met", "fused",
                                            "reverse_fused", "reordered")}
        for v in ("tacker", "tacker_no_reverse"):
            reverse[v]["improvement_vs_baymax_eq10_normalised"] = rr[v]["be_norm_thpt"] / rr["baymax"]["be_norm_thpt"] - 1

    # ---- roofline of the dominant launch class of the timed run (class shares from the manager's
    #      sampled CUDA events on its stream)
    cms, cn = res["class_ms"], res["class_launches"]
    tot_ms = sum(cms.values()) or 1.0
    shares = {c: {"ms": cms[c], "launches": cn[c], "share": cms[c] / tot_ms} for c in cms}
    dom = max(cms, key=cms.get)

    # ---- BASELINE configs[1]: ResNet-50 batch-1 convs fused with stencil / mri-q -- the kernel-
    #      level fused step (fused time vs overlap roofline) and the same managed protocol
    svc1 = sv.resnet50_service(1, seed)
    sv.autotune_tile_n(svc1)
    step = FusedStep(svc1, stencil, mriq, args.warp_split)
    for _ in range(3):
        step.fused()
    torch.cuda.synchronize()
    fstep, roof_fused = kernel_level(torch, step, flush, peaks, peak_kind, clocks, max(5, min(args.steps, 20)))
    b1 = None
    if not args.no_extra:
        tk.tacker_model_clear()
        q1 = qos.QosRun(svc1, [stencil, mriq], warp_split=args.warp_split, qos_ms=QOS_MS)
        q1.calibrate()
        q1.measure_service(max_inflight=args.inflight)
        q1.run(tk.POLICY_TACKER, 20, load=LOAD, seed=1000 + rank, max_inflight=args.inflight, **HEADLINE)
        r1 = managed_runs(q1, tk, 1000, 3000 + rank, args.inflight, ("tacker", "baymax", "tacker_slice", "tacker_paper"))
        b1 = {"workload": "resnet50_b1 LC + stencil/mriq BE queue, QoS 50 ms (BASELINE configs[1], config-4 protocol)",
              "queries": 1000, "service_ms": q1.service_ms, "lc_roofline": lc_class_roofline(q1, peaks, peak_kind, svc1)}
        for v, r in r1.items():
            b1[v] = {k: r[k] for k in ("be_kernels_per_s", "be_norm_thpt", "lc_p50_ms", "lc_p99_ms", "qos_met",
                                        "fused", "reordered", "idle_be")}
        for v in ("tacker", "tacker_slice", "tacker_paper"):
            b1[v]["improvement_vs_baymax_eq10"] = r1[v]["be_kernels_per_s"] / r1["baymax"]["be_kernels_per_s"] - 1
            b1[v]["improvement_vs_baymax_eq10_normalised"] = r1[v]["be_norm_thpt"] / r1["baymax"]["be_norm_thpt"] - 1

    if dom in ("lc_tc", "lc_cd"):
        roof = lc_class_roofline(q, peaks, peak_kind, svc)
    else:
        roof = dict(roof_fused)
    roof["class_shares"] = shares

    cpu = cpu_oracle_sample(batch=args.batch) if (rank == 0 and ws == 1 and not args.no_cpu) else None
    if cpu is not None:
        cpu.pop("seconds_per_be_kernel", None)

    line = {
        "metric": METRIC, "value": value, "unit": "BE kernels/s", "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": elapsed_ms / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f16xf16->f32 (LC tcgen05) + f32 (BE CUDA cores)",
        "data": "synthetic (seeded inputs, random weights)",
        "config": {"workload": WORKLOAD.format(b=args.batch),
                   "lc": f"ResNet-50 batch-{args.batch} (Table II), 53 convs, fp16 NHWC, implicit GEMM tcgen05",
                   "be": "stencil 512x512x64 sweeps | mri-q 64^3 x (phiMag + 2 x 1024-k chunks)",
                   "arrivals": f"Poisson at {LOAD:.0%} of the peak rate (the manager's LC-only service rate)",
                   "qos_ms": QOS_MS, "policy": "tacker (+ reading 18: older queries fuse within later queries' headroom - 15 ms)", "warp_split": args.warp_split, "max_inflight": args.inflight,
                   "step": "one LC query", "parallelism": f"replicas x{ws}",
                   "l2": "inputs larger than L2 (stencil 2 x 64 MiB ping-pong + activations and weights > 1 GB)"},
        "lc_p99_ms": p99, "lc_p50_ms": res["lc_p50_ms"], "lc_qos_ms": QOS_MS, "qos_met": p99 <= QOS_MS,
        "lambda_per_s": res["lambda_per_s"], "service_ms": q.service_ms, "query_solo_ms": q.query_solo_ms(),
        "fused_launches": res["fused"], "reordered_be": res["reordered"],
        "idle_be": res["idle_be"], "model_refits": res["model_refits"],
        "baymax": {"value": bay["be_kernels_per_s"], "lc_p99_ms": bay["lc_p99_ms"], "qos_met": bay["qos_met"],
                   "be_norm_thpt": bay["be_norm_thpt"]},
        "improvement_vs_baymax_eq10": res["be_kernels_per_s"] / bay["be_kernels_per_s"] - 1.0,
        # BE work in standalone-kernel milliseconds per wall millisecond (app-length independent)
        "be_norm_thpt": res["be_norm_thpt"],
        "improvement_vs_baymax_eq10_normalised": res["be_norm_thpt"] / bay["be_norm_thpt"] - 1.0,
        "tacker_slice": {"value": slc["be_kernels_per_s"], "be_norm_thpt": slc["be_norm_thpt"],
                         "lc_p99_ms": slc["lc_p99_ms"], "fused": slc["fused"],
                         "improvement_vs_baymax_eq10_normalised": slc["be_norm_thpt"] / bay["be_norm_thpt"] - 1.0},
        # Baymax with the same reading-18 queueing rule (older queries reorder within later
        # queries' headroom): Eq. 10 against it isolates what fusion adds
        "baymax_same_rule": {"value": bay18["be_kernels_per_s"], "be_norm_thpt": bay18["be_norm_thpt"],
                             "lc_p99_ms": bay18["lc_p99_ms"], "qos_met": bay18["qos_met"]},
        "improvement_vs_baymax_same_rule_eq10": res["be_kernels_per_s"] / bay18["be_kernels_per_s"] - 1.0,
        # reorder only after LC kernels that were not fused (the literal P:2035 rule) on top of reading 18
        "tacker_fuse_first": {k: other["tacker_fuse_first"][k] for k in ("be_kernels_per_s", "be_norm_thpt", "lc_p99_ms",
                                                                         "qos_met", "fused", "reordered")},
        "tacker_slice_ff": {k: other["tacker_slice_ff"][k] for k in ("be_kernels_per_s", "be_norm_thpt", "lc_p99_ms",
                                                                     "qos_met", "fused", "reordered")},
        "tacker_slice_noreorder": {k: other["tacker_slice_noreorder"][k] for k in ("be_kernels_per_s", "be_norm_thpt",
                                                                                   "lc_p99_ms", "qos_met", "fused",
                                                                                   "reordered", "idle_be")},
        "improvement_vs_baymax_same_rule_eq10_normalised": res["be_norm_thpt"] / bay18["be_norm_thpt"] - 1.0,
        # the paper-literal manager rule: only the newest query fuses / reorders
        "tacker_paper": {"value": old["be_kernels_per_s"], "be_norm_thpt": old["be_norm_thpt"],
                         "lc_p99_ms": old["lc_p99_ms"], "qos_met": old["qos_met"], "fused": old["fused"],
                         "improvement_vs_baymax_eq10": old["be_kernels_per_s"] / bay["be_kernels_per_s"] - 1.0,
                         "improvement_vs_baymax_eq10_normalised": old["be_norm_thpt"] / bay["be_norm_thpt"] - 1.0},
        "reverse_fusion": reverse,
        "fused_pred_err_mean": res["fused_pred_err_mean"],
        "pair_pred_err_mean": statistics.mean(q.pair_err) if q.pair_err else None,
        "roofline": roof,
        "roofline_fused": roof_fused,
        "fused_step": fstep,
        "cpu_baseline": cpu,
        "e2e": {"value": e2e_value, "unit": "BE kernels/s", "h2d_bytes_per_step": qi.h2d_bytes,
                "d2h_bytes_per_step": qi.d2h_bytes, "lc_p99_ms": e2e["lc_p99_ms"],
                "how": "each query copies its input image H2D and its result D2H from/to pinned host memory "
                       "(UVA copy kernels on the manager stream) inside the timed managed run"},
        # counted by the manager: every LC kernel of every query (fused or original) plus the
        # reordered and idle-time BE launches
        "gpu_launches": int(sum(res["class_launches"].values())),
        "clocks": clocks,
        "config1_resnet50_b1": b1,
    }
    if rank == 0:
        print(json.dumps(line))


def run_simulated(args, ws, rank):
    """--simulate: the same managed run on the manager's simulated GPU (kernels take their
    predicted time; no CUDA), for CPU tests of the multi-rank path (gloo).  Kernel durations are
    a fixed table shaped like the B200 measurements of the ResNet-50 b1 / stencil / mri-q run."""
    from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk
    tk.tacker_model_clear()
    fake = 0x10000
    lc = tk.LcDesc(kind=tk.LC_GEMM_F16, M=1024, N=256, K=256, A=fake, B=fake, D=fake)
    ks = [tk.LcKernel(is_tc=1, t_pred_ms=0.010 + 0.0005 * (i % 7), lc=lc) for i in range(53)]
    st = tk.BeDesc(kind=tk.BE_STENCIL)
    st.p.stencil = tk.BeStencil(512, 512, 64, 1 / 6, 1 / 36, fake, fake)
    key = f"pair:lc:gemm:N256:K256:bn128:f32|be:stencil:nz64|ws{args.warp_split}"
    for r in (0.1, 0.2, 1.8, 1.9):      # tau(r) = max(1 + 0.3 r, 0.45 + 0.95 r)
        tk.tacker_pair_add_sample(key, 1.0, r, max(1 + 0.3 * r, 0.45 + 0.95 * r))
    tk.tacker_pair_fit(key)
    apps = [[tk.BeKernel(is_cd=1, t_pred_ms=0.035, be=st, warp_split=args.warp_split)] * 2,
            [tk.BeKernel(is_cd=1, t_pred_ms=0.147, be=st, warp_split=args.warp_split)] * 2]
    rng = np.random.default_rng(2000 + rank)
    solo = sum(k.t_pred_ms for k in ks)
    gaps = rng.exponential(solo / LOAD, args.steps)
    out = {}
    for pol in (tk.POLICY_BAYMAX, tk.POLICY_TACKER):
        m = tk.Manager(pol, simulate=True, idle_cap_ms=0.5 * (QOS_MS - solo))
        for a in apps:
            m.submit_be(a)
        arr = np.cumsum(gaps)
        q = [m.submit_lc(ks, float(t)) for t in arr]
        barrier(ws)
        m.run(QOS_MS, float(arr[-1]))
        s = m.stats()
        lat = np.sort([m.latency(i) for i in q])
        out[pol] = (s.be_kernels_done, s.now_ms, float(lat[min(len(lat) - 1, int(math.ceil(0.99 * len(lat))) - 1)]))
    be, el, p99 = out[tk.POLICY_TACKER]
    elapsed = reduce_ranks(ws, el, "max")
    value = reduce_ranks(ws, be, "sum") / (elapsed / 1e3)
    bay = reduce_ranks(ws, out[tk.POLICY_BAYMAX][0], "sum") / (reduce_ranks(ws, out[tk.POLICY_BAYMAX][1], "max") / 1e3)
    line = {"metric": METRIC, "value": value, "unit": "BE kernels/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": elapsed / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "n/a (simulated GPU)", "data": "synthetic",
            "config": {"workload": WORKLOAD.format(b=1) + " [simulated durations]", "parallelism": f"replicas x{ws}"},
            "lc_p99_ms": reduce_ranks(ws, p99, "max"), "baymax": {"value": bay},
            "improvement_vs_baymax_eq10": value / bay - 1.0, "simulated": True}
    if rank == 0:
        print(json.dumps(line))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300, help="timed LC queries")
    ap.add_argument("--batch", type=int, default=32, help="LC batch (Table II: ResNet-50 at 32)")
    ap.add_argument("--inflight", type=int, default=16, help="manager: launches in flight on its stream")
    ap.add_argument("--warmup", type=int, default=20, help="untimed warm-up LC queries")
    ap.add_argument("--impl", default="tacker", choices=["tacker", "reference"])
    ap.add_argument("--warp-split", type=int, default=24)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-extra", action="store_true", help="skip the ResNet-50 b1 (configs[1]) managed side run")
    ap.add_argument("--simulate", action="store_true", help="CPU-only: manager on its simulated GPU (gloo)")
    ap.add_argument("--overlap", type=int, default=None,
                    help="programmatic dependent launch mode (tacker_set_launch_overlap: 0, 1, 2)")
    args = ap.parse_args()
    if args.impl == "reference":
        run_reference(args, int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")))
        return
    ws, rank, local = dist_setup(simulate=args.simulate)
    if args.simulate:
        run_simulated(args, ws, rank)
    else:
        if args.overlap is not None:
            from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk
            tk.tacker_set_launch_overlap(args.overlap)
        run_tacker(args, ws, rank, local)
    if ws > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
