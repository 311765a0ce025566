#!/usr/bin/env python
"""Bench for the B200-native Tacker hot path (BASELINE.json metric:
"BE kernels/sec at LC p99 <= QoS target; fused time vs overlap roofline").

Workload (N=1): BASELINE configs[3] (SURVEY config 4), QoS-managed co-location -- ResNet-50 at
the paper's batch 32 (Table II) as the LC service (53 convs as implicit-GEMM tcgen05
kernels, split-K where few tiles; conv1 = im2col + GEMM) with the paper's mixed BE queue (Table II
P:2021-2023: mri-q, fft, mri-fhd, cutcp, cp, sgemm, lbm, tpacf; each app resubmitted forever).

Protocol:
* lambda_peak = the largest LC arrival rate whose LC-only p99 meets the 50 ms QoS target
  (bisection on LC-only windowed runs); arrivals are Poisson at 0.8 lambda_peak.
* A STEP is a fixed block of STEP_QUERIES (100) LC queries' worth of arrivals (100 / lambda ms
  of the trace).  One continuous Poisson run per arm: W warm-up steps, then the timed window of
  exactly K steps, then a tail (1.5 x QoS of arrivals while the window's last queries finish),
  then drain.  The window is bracketed by a stream sync + barrier and CUDA events on the manager
  stream; the ramp-up and drain are outside it, so `value` does not depend on K.
* value = BE kernels issued inside the window / its device time (sum over replicas / max time);
  lc_p99 over every query that arrived inside the window (nearest rank) with a bootstrap 95 % CI.
* Arms on the same trace: `tacker` (the headline; its rules are named in config.policy),
  `baymax` (fusion off, the paper's queueing rule), `baymax_same_rule` (fusion off, the headline's
  queueing rule: Eq. 10 against it isolates what fusion adds), `tacker_paper` (every rule as the
  paper states it).  Each of tacker / baymax_same_rule runs `--seeds` trace seeds.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--seeds S] [--impl tacker|reference]
  --gpus N (no torchrun): N replica processes, one per GPU (CUDA_VISIBLE_DEVICES=i), no NCCL;
  under torchrun the replicas coordinate over gloo (CPU), never NCCL.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

QOS_MS = 50.0
LOAD = 0.8                    # x lambda_peak
STEP_QUERIES = 100            # LC queries per step
METRIC = "BE kernels/sec at LC p99 <= QoS target"
WORKLOAD = "resnet50_b{b} LC + Table II mixed BE queue ({be}), QoS 50 ms (BASELINE configs[3])"
# Manager rules of the headline Tacker arm: the paper's reorder rule and direct rule
# plus B200 reading 18 (older queries may fuse / reorder within the headroom of
# every later active query, minus a 0.3 x QoS guard).  `tacker_paper` drops reading 18.
HEADLINE = {"fuse_older": True}


# ----------------------------------------------------------------------------- replicas (no NCCL)
class Comm:
    """Coordination of replica processes, never a data-path collective: a single
    process, gloo on CPU (under torchrun), or files (bench.py --gpus N spawns the replicas)."""

    def __init__(self):
        self.ws = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        self.local = int(os.environ.get("LOCAL_RANK", "0"))
        self.dir = os.environ.get("TACKER_REPLICA_DIR")
        self.mode = "single" if self.ws == 1 else ("files" if self.dir else "gloo")
        self._n = 0
        if self.mode == "gloo":
            import torch.distributed as dist
            dist.init_process_group("gloo")

    def reduce(self, v, op="max"):
        if self.mode == "single":
            return v
        if self.mode == "gloo":
            import torch
            import torch.distributed as dist
            t = torch.tensor([float(v)], dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
            return float(t.item())
        self._n += 1
        path = os.path.join(self.dir, f"c{self._n}.r{self.rank}")
        with open(path + ".tmp", "w") as f:
            json.dump(float(v), f)
        os.replace(path + ".tmp", path)
        vals, t0 = [], time.time()
        for r in range(self.ws):
            p = os.path.join(self.dir, f"c{self._n}.r{r}")
            while not os.path.exists(p):
                if time.time() - t0 > 3600:
                    raise TimeoutError(f"replica {r} never reached sync point {self._n}")
                time.sleep(0.002)
            with open(p) as f:
                vals.append(json.load(f))
        return max(vals) if op == "max" else sum(vals)

    def barrier(self):
        self.reduce(0.0)

    def close(self):
        if self.mode == "gloo":
            import torch.distributed as dist
            dist.destroy_process_group()


def spawn_replicas(n):
    """bench.py --gpus N without torchrun: N replica processes, replica i pinned to GPU i
    (CUDA_VISIBLE_DEVICES), own seeds (rank), coordinating through files; rank 0 prints the line."""
    d = tempfile.mkdtemp(prefix="tacker_replicas_")
    procs = []
    for i in range(n):
        env = dict(os.environ, WORLD_SIZE=str(n), RANK=str(i), LOCAL_RANK="0", TACKER_REPLICA_DIR=d)
        if "--simulate" not in sys.argv:
            env["CUDA_VISIBLE_DEVICES"] = str(i)
        procs.append(subprocess.Popen([sys.executable, os.path.abspath(__file__)] + sys.argv[1:], env=env))
    rc = 0
    for p in procs:
        rc = max(rc, p.wait())
    sys.exit(rc)


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
    """MEASURED_PEAKS.json (driver-written: HBM, bf16 burst / sustained) plus this repo's own
    micro-benchmark peaks (profiles/peaks.json: FFMA, MUFU, fp16 GEMM) when present."""
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            peaks, kind = json.load(f), "measured"
    else:
        peaks, kind = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": 1965.0}, "fallback"
    q = os.path.join(ROOT, "profiles", "peaks.json")
    if os.path.exists(q):
        with open(q) as f:
            peaks["micro"] = json.load(f)
    return peaks, kind


# ----------------------------------------------------------------------------- kernel-level step
class FusedStep:
    """BASELINE configs[1]: every LC tensor-core kernel of one ResNet-50 batch-1 query fused with
    the next BE kernel (alternating a stencil sweep and a mri-q Q chunk); CUDA-core LC kernels
    (im2col) launch original."""

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
        kernels in order on one stream, the BE kernels in order on another, original kernels."""
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


def kernel_level(torch, step, flush, peaks, steps):
    """configs[1] fused step vs the BASELINE overlap roofline and vs sequential / two streams."""
    from paper_conf_hpca_zhaocczlllg22_b200.qos import overlap_rate   # Eq. 11
    fused_ms = time_steps(torch, step.fused, steps, flush)
    orig_ms = time_steps(torch, step.original, max(3, steps // 2), flush)
    lc_ms = time_steps(torch, step.lc_only, 3, flush)
    be_ms = time_steps(torch, step.be_only, 3, flush)
    st_ms = time_steps(torch, step.two_streams, max(3, steps // 2), flush)
    t_f, t_s = statistics.median(fused_ms), statistics.median(orig_ms)
    t_lc, t_be = statistics.median(lc_ms), statistics.median(be_ms)
    t_st = statistics.median(st_ms)
    p_tensor = peaks["bf16_tflops"] * 1e12          # fp16 runs at the bf16 rate
    bw = peaks["hbm_gbs"] * 1e9
    p_mufu = mufu_peak(peaks)[0] * 1e12
    t_roof = 0.0
    for k, be, f in step.plan:
        if f is None:
            t_roof += k.bytes / bw
            continue
        t_be_roof = be.mufu / p_mufu if be.bound == "mufu" else be.bytes / bw
        t_roof += max(k.flops / p_tensor, t_be_roof, (k.bytes + be.bytes) / bw)
    return {"workload": "resnet50_b1 TC convs each fused with the next stencil sweep / mri-q chunk (BASELINE configs[1])",
            "fused_step_ms": t_f, "sequential_step_ms": t_s, "lc_only_ms": t_lc, "be_only_ms": t_be,
            "speedup_vs_sequential": t_s / t_f, "overlap_rate_eq11": overlap_rate(t_lc, t_be, t_f),
            "two_streams_step_ms": t_st, "overlap_rate_eq11_two_streams": overlap_rate(t_lc, t_be, t_st),
            "overlap_roofline_ms": t_roof * 1e3, "overlap_roofline_frac": t_roof * 1e3 / t_f,
            "launches_per_step": len(step.plan), "l2": "256 MiB fill before every step"}


def mufu_peak(peaks):
    """(Tops/s, source) of the MUFU sin/cos pipe: the repo's micro-benchmark if measured, else
    148 SMs x 16 /clk x sm_max_mhz (the guide's unit count)."""
    m = peaks.get("micro", {}).get("mufu_sincos_tops")
    if m:
        return m, "measured: profiles/peaks.json (tools/peaks.py MUFU sin+cos micro-benchmark)"
    return 148 * 16 * peaks.get("sm_max_mhz", 1965.0) * 1e6 / 1e12, "derived: 148 SM x 16 MUFU/clk x sm_max_mhz"


# ----------------------------------------------------------------------------- rooflines
def lc_class_roofline(q, peaks, peak_kind, svc, traffic_key=None):
    """The LC tensor-core convs of the timed run: per kernel the algorithmic flops (2 NPQ K CRS)
    and bytes (x, w, out once), timed back to back with CUDA events on the launching stream
    (QosRun.calibrate).  The bound is the one that gives the larger roofline time summed over
    the query."""
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
    roof["traffic"] = _traffic(traffic_key or f"lc_tc:{svc.name}")
    roof.update(kernel=f"LC tensor-core convs of {svc.name} (implicit GEMM tcgen05, split-K where few tiles)",
                avg_launch_ms=t_ms / n, launches_per_query=n, algorithmic_flops_per_launch=fl / n,
                algorithmic_bytes_per_launch=by / n,
                per_kernel_roofline_frac=t_roof * 1e3 / t_ms,
                stream="launching stream, back-to-back launches (CUDA events)")
    return roof


def _traffic(key):
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            return json.load(f).get(key)
    return None


def be_class_roofline(q, peaks, apps):
    """BE kernels of the timed run (original launches): per kernel its roofline time at its own
    bound (HBM bytes / BW, FP32 flops / P_fp32, MUFU ops / P_mufu) against its measured
    back-to-back time; aggregated as sum(T_roof) / sum(T_meas) over one cycle of every app."""
    bw = peaks["hbm_gbs"] * 1e9
    p_mufu = mufu_peak(peaks)[0] * 1e12
    p_fma = peaks.get("micro", {}).get("ffma_tflops", 148 * 128 * 2 * peaks.get("sm_max_mhz", 1965.0) * 1e6 / 1e12) * 1e12
    rows, t_roof, t_meas = [], 0.0, 0.0
    for a, app in enumerate(apps):
        for j, bk in enumerate(app.kernels):
            t = q.t_be[(a, j)]
            r = max(bk.bytes / bw, bk.mufu / p_mufu if bk.mufu else 0.0, bk.flops / p_fma if bk.bound == "fma" else 0.0)
            rows.append({"kernel": bk.name, "ms": t, "roofline_ms": r * 1e3, "frac": r * 1e3 / t if t else None,
                         "bound": bk.bound})
            t_roof += r * 1e3
            t_meas += t
    return {"frac": t_roof / t_meas if t_meas else None, "kernels": rows}


# ----------------------------------------------------------------------------- CPU oracle baseline
def cpu_oracle_sample(small=False, batch=32, be="table2"):
    """The oracle as it stands on a bounded sample of the same workload: the oracle conv of two
    ResNet-50 layers on one image (time x batch: the conv is linear in the batch) paired with each
    BE kernel of the queue, every BE kernel computed on a bounded part of its problem and its time
    scaled to the whole kernel (the oracle's cost is linear in the part).  Table II queue: mri-q
    and mri-fhd chunks on 256 of the 64^3 voxels (x1024), fft on 16 of the 16384 transforms
    (x1024), cutcp on 512 of the 96^3 lattice points (x1728), cp on a 32x32 corner of the 512^2
    slice (x256), sgemm on 64 of the 2048 rows (x32), lbm on a 120x120x10 slab (x15), tpacf DR on
    1024 x 1024 of the 16384^2 pairs (x256); small = half of each part (scale x2).  Returns BE
    kernels/s = 1 / mean (conv + BE kernel) time."""
    import synth
    from oracle import be as obe, lc as olc
    convs = synth.resnet50_convs(1)
    t0 = time.perf_counter()
    for i in (5, 20):
        cs = convs[i]
        x, w, _ = synth.conv_inputs(cs, i)
        olc.lc_conv(x, w, cs.stride, cs.pad)
    t_conv = (time.perf_counter() - t0) / 2 * batch
    f = 2 if small else 1
    times = {}

    def timed(name, fn, scale):
        t = time.perf_counter()
        fn()
        times[name] = (time.perf_counter() - t) * scale

    if be == "table2":
        d = synth.mriq_inputs(64, 1024, 2022)
        n = 256 // f
        pm, _ = obe.mriq_phimag(d["phiR"], d["phiI"])
        timed("mriq.q", lambda: obe.mriq_q(d["x"][:n], d["y"][:n], d["z"][:n], d["kx"], d["ky"], d["kz"], pm),
              64 ** 3 / n)
        dd = synth.mrifhd_inputs(64, 1024, 2022)
        rr, ri, _, _ = obe.mrifhd_rhophi(dd["phiR"], dd["phiI"], dd["dR"], dd["dI"])
        timed("mrifhd.fh", lambda: obe.mrifhd_fh(dd["x"][:n], dd["y"][:n], dd["z"][:n], dd["kx"], dd["ky"], dd["kz"],
                                                 rr, ri), 64 ** 3 / n)
        xf = synth.fft_inputs(16 // f, 1024, 2022)
        timed("fft", lambda: obe.fft(xf), 16384 / (16 // f))
        cu = synth.cutcp_inputs(48.0, 2022)
        pts = np.random.default_rng(0).integers(0, cu["nx"] ** 3, size=512 // f)
        timed("cutcp", lambda: obe.cutcp(cu["atoms"], cu["nx"], cu["nx"], cu["nx"], cu["h"], points=pts),
              cu["nx"] ** 3 / (512 // f))
        at, z = synth.cp_inputs(4000, 512, 512, 0.1, 2022)
        m = 32 // f
        timed("cp", lambda: obe.cp(at, m, m, 0.1, z), 512 * 512 / (m * m))
        A, B = synth.sgemm_inputs(2048, 2048, 2048, 2022)
        timed("sgemm", lambda: obe.sgemm(A[:64 // f], B), 2048 / (64 // f))
        src, fl = synth.lbm_inputs(120, 120, 10 // f, 2022)
        timed("lbm", lambda: obe.lbm_step(src, fl, src.copy()), 150 / (10 // f))
        a = synth.tpacf_inputs(1024 // f, 2022)
        b = synth.tpacf_inputs(1024 // f, 2023, "uniform")
        e = synth.tpacf_edges()
        timed("tpacf", lambda: obe.tpacf(a, b, e, False), (16384 / (1024 // f)) ** 2)
        desc = ("oracle conv (2 ResNet-50 layers, 1 image, time x%d) paired with each Table II BE kernel on a bounded "
                "part, time scaled to the whole kernel (%s)" % (batch, "; ".join(f"{k} {v:.3g} s" for k, v in times.items())))
    else:
        A = synth.stencil_inputs(512, 512, 10 if small else 64, 2022)
        timed("stencil", lambda: obe.stencil(A, np.float32(1 / 6), np.float32(1 / 36)), 64 / 8 if small else 1.0)
        d = synth.mriq_inputs(64, 1024, 2022)
        pm, _ = obe.mriq_phimag(d["phiR"], d["phiI"])
        n = 256 if small else 4096
        timed("mriq.q", lambda: obe.mriq_q(d["x"][:n], d["y"][:n], d["z"][:n], d["kx"], d["ky"], d["kz"], pm),
              64 ** 3 / n)
        desc = "oracle conv (2 ResNet-50 layers, 1 image, time x%d) + stencil sweep + mri-q chunk, scaled" % batch
    per = t_conv + sum(times.values()) / len(times)
    return {"value": 1.0 / per, "unit": "BE kernels/s", "cores": _oracle_threads(), "kind": "oracle",
            "sample": desc + "; BE kernels/s = 1 / mean (conv + BE kernel) time", "seconds_per_be_kernel": per}


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
    for _ in range(min(args.warmup, 1)):    # untimed warm-up step (bounded)
        cpu_oracle_sample(small=True, batch=args.batch, be=args.be)
    t0 = time.perf_counter()
    vals, r = [], None
    for _ in range(args.steps):
        r = cpu_oracle_sample(small=True, batch=args.batch, be=args.be)
        vals.append(r["seconds_per_be_kernel"])
        if time.perf_counter() - t0 > 120.0:
            break
    el = time.perf_counter() - t0
    v = 1.0 / (sum(vals) / len(vals))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "BE kernels/s", "n_gpus": ws,
            "steps": len(vals), "warmup": args.warmup, "ms_per_step": el * 1000 / len(vals),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": WORKLOAD.format(b=args.batch, be=args.be), "l2": "n/a (CPU)"},
            "cpu_baseline": {"value": v, "unit": "BE kernels/s", "cores": r["cores"], "kind": "oracle",
                             "sample": "per step: " + r["sample"]},
            "e2e": {"value": v, "unit": "BE kernels/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


ARMS = {   # name -> (policy, manager rules); the rules of each arm are also named in its result
    "tacker": ("T", dict(HEADLINE)),
    "baymax": ("B", {}),
    "baymax_same_rule": ("B", dict(HEADLINE)),
    "tacker_paper": ("T", {}),
    "tacker_reorder_always": ("T", dict(HEADLINE, reorder_rule=1)),
}
KEEP = ("be_kernels_per_s", "be_norm_thpt", "lc_p50_ms", "lc_p99_ms", "lc_p99_ci95_ms", "qos_met", "violations",
        "queries", "fused", "reordered", "idle_be", "rules", "elapsed_ms")


def arm_result(q, tk, name, window_ms, warm_ms, load, seed, inflight, sync=None):
    pol, rules = ARMS[name]
    return q.run_window(tk.POLICY_TACKER if pol == "T" else tk.POLICY_BAYMAX, window_ms, warm_ms, load=load,
                        seed=seed, max_inflight=inflight, sync=sync, **rules)


def calibrated_run(qos, tk, svc, apps, args, comm, peak_steps=50):
    q = qos.QosRun(svc, apps, warp_split=args.warp_split, qos_ms=QOS_MS)
    q.calibrate()
    q.measure_service(max_inflight=args.inflight)
    # lambda_peak by bisection on LC-only runs of peak_steps x 100 queries' worth each
    q.find_peak_load(window_ms=peak_steps * STEP_QUERIES * q.service_ms, max_inflight=args.inflight)
    return q


def side_runs(q, tk, arms, steps, rank, inflight, seeds=(0,)):
    """The same protocol on other arms / seeds (not the timed headline)."""
    load = LOAD * q.peak_load
    win = steps * STEP_QUERIES * q.service_ms / load
    warm = 5 * STEP_QUERIES * q.service_ms / load
    out = {}
    for a in arms:
        rs = [arm_result(q, tk, a, win, warm, load, 2000 + 100 * s + rank, inflight) for s in seeds]
        out[a] = {k: rs[0][k] for k in KEEP if k in rs[0]}
        if len(rs) > 1:
            out[a]["seeds"] = [{k: r[k] for k in ("be_kernels_per_s", "be_norm_thpt", "lc_p99_ms")} for r in rs]
            out[a]["be_norm_thpt_mean"] = statistics.mean(r["be_norm_thpt"] for r in rs)
            out[a]["be_kernels_per_s_mean"] = statistics.mean(r["be_kernels_per_s"] for r in rs)
    return out


def eq10(a, b, key):
    return a[key] / b[key] - 1.0 if a and b and b.get(key) else None


def run_tacker(args, comm):
    import torch
    from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk

    if torch.cuda.is_available():
        torch.cuda.set_device(comm.local)
    ws, rank = comm.ws, comm.rank
    peaks, peak_kind = measured_peaks()
    seed = 2022 + rank
    svc = sv.resnet50_service(args.batch, seed)
    sv.autotune_tile_n(svc)                                      # LC tile width per conv, measured
    chain_tune = sv.chain_autotune_tile_n(svc)                   # ... refined on the query chain
    names = sv.TABLE2_BE if args.be == "table2" else tuple(args.be.split(","))
    apps = sv.be_apps(names, seed)
    sv.prime_apps(apps)
    flush_buf = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")

    def flush():
        flush_buf.fill_(1.0)

    # ---- calibration (predictor, §VI-C), service rate and lambda_peak -- untimed
    tk.tacker_model_clear()
    q = calibrated_run(qos, tk, svc, apps, args, comm)
    load = LOAD * q.peak_load
    step_ms = STEP_QUERIES * q.service_ms / load          # one step = 100 queries' worth of arrivals
    window_ms, warm_ms = args.steps * step_ms, max(args.warmup, 3) * step_ms

    # ---- timed region: the steady-state window of the headline arm
    clk = ClockSampler(comm.local)
    clk.start()
    comm.barrier()
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_push("timed")
    res = arm_result(q, tk, "tacker", window_ms, warm_ms, load, 2000 + rank, args.inflight, sync=comm.barrier)
    torch.cuda.nvtx.range_pop()
    torch.cuda.synchronize()
    comm.barrier()
    clocks = clk.stop()
    elapsed_ms = comm.reduce(res["elapsed_ms"], "max")
    be_total = comm.reduce(res["be_kernels"], "sum")
    value = be_total / (elapsed_ms / 1e3)
    p99 = comm.reduce(res["lc_p99_ms"], "max")
    norm = comm.reduce(res["be_work_ms"], "sum") / elapsed_ms

    # ---- the other arms on the same trace; tacker / baymax_same_rule over --seeds seeds
    seeds = tuple(range(args.seeds))
    other = side_runs(q, tk, ("baymax", "baymax_same_rule", "tacker_paper", "tacker_reorder_always"), args.steps,
                      rank, args.inflight)
    if args.seeds > 1:
        more = side_runs(q, tk, ("tacker", "baymax_same_rule"), args.steps, rank, args.inflight, seeds)
        other["tacker_seeds"] = more["tacker"]
        other["baymax_same_rule_seeds"] = more["baymax_same_rule"]
    bay, same, paper = other["baymax"], other["baymax_same_rule"], other["tacker_paper"]

    # ---- e2e: the same windowed run, each query with its H2D input + D2H result
    qi = qos.QosRun(svc, apps, warp_split=args.warp_split, qos_ms=QOS_MS).with_io()
    qi.pairs, qi.ws_of, qi.t_be, qi.lr_be = q.pairs, q.ws_of, q.t_be, q.lr_be
    qi.t_lc = []
    for is_tc, d in qi._kernel_list():
        qi.t_lc.append(qos._time(lambda: tk.tacker_launch_original(d, None) if is_tc
                                  else tk.tacker_launch_original(None, d), 5))
    qi.measure_service(max_inflight=args.inflight)
    qi.peak_load = q.peak_load
    load_io = LOAD * qi.peak_load
    e2e = arm_result(qi, tk, "tacker", args.steps * STEP_QUERIES * qi.service_ms / load_io,
                     max(args.warmup, 3) * STEP_QUERIES * qi.service_ms / load_io, load_io, 2000 + rank, args.inflight)
    e2e_value = comm.reduce(e2e["be_kernels"], "sum") / (comm.reduce(e2e["elapsed_ms"], "max") / 1e3)

    # ---- roofline of the dominant launch class of the timed window
    cms, cn = res["class_ms"], res["class_launches"]
    tot_ms = sum(cms.values()) or 1.0
    shares = {c: {"ms": cms[c], "launches": cn[c], "share": cms[c] / tot_ms} for c in cms}
    dom = max(cms, key=cms.get)
    if dom in ("lc_tc", "lc_cd"):
        roof = lc_class_roofline(q, peaks, peak_kind, svc)
    else:
        roof = lc_class_roofline(q, peaks, peak_kind, svc)
        roof["note"] = f"dominant class of the window is {dom}; the LC convs are reported (BE: be_roofline)"
    roof["class_shares"] = shares
    be_roof = be_class_roofline(q, peaks, apps)

    extra = {}
    if not args.no_extra:
        extra = side_workloads(args, comm, peaks, flush, tk, qos, sv, torch)

    cpu = cpu_oracle_sample(batch=args.batch, be=args.be) if (rank == 0 and ws == 1 and not args.no_cpu) else None
    if cpu is not None:
        cpu.pop("seconds_per_be_kernel", None)

    tk_line = {k: res[k] for k in KEEP if k in res}
    line = {
        "metric": METRIC, "value": value, "unit": "BE kernels/s", "n_gpus": ws, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": elapsed_ms / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f16xf16->f32 (LC tcgen05) + f32 (BE CUDA cores)",
        "data": "synthetic (seeded inputs, random weights)",
        "config": {"workload": WORKLOAD.format(b=args.batch, be=",".join(names)),
                   "lc": f"ResNet-50 batch-{args.batch} (Table II), 53 convs, fp16 NHWC, implicit GEMM tcgen05, "
                         f"tile widths measured per kernel then on the query chain "
                         f"({chain_tune['before_ms']:.3f} -> {chain_tune['after_ms']:.3f} ms per query, "
                         f"{len(chain_tune['changed'])} changed)",
                   "be": " | ".join(a.name for a in apps),
                   "arrivals": f"Poisson at {LOAD:.0%} of lambda_peak (LC-only p99 <= QoS, bisection) = "
                               f"{load:.3f} x the LC-only service rate",
                   "step": f"{STEP_QUERIES} LC queries' worth of arrivals ({step_ms:.1f} ms); timed window = "
                           f"{args.steps} steps inside one continuous run after {max(args.warmup, 3)} warm-up steps, "
                           "followed by a 1.5 x QoS tail",
                   "qos_ms": QOS_MS, "policy": res["rules"], "warp_split": args.warp_split,
                   "max_inflight": args.inflight, "parallelism": f"replicas x{ws} ({comm.mode}, no NCCL)",
                   "l2": "inputs larger than L2 (activations > 1 GB, BE working sets 8-340 MB)"},
        "be_norm_thpt": norm,
        "lc_p99_ms": p99, "lc_p99_ci95_ms": res["lc_p99_ci95_ms"], "lc_p50_ms": res["lc_p50_ms"],
        "lc_qos_ms": QOS_MS, "qos_met": p99 <= QOS_MS, "queries_in_window": res["queries"],
        "violations": res["violations"],
        "lambda_peak_load": q.peak_load, "lambda_per_s": res["lambda_per_s"], "service_ms": q.service_ms,
        "query_solo_ms": q.query_solo_ms(),
        "fused_launches": res["fused"], "reordered_be": res["reordered"], "idle_be": res["idle_be"],
        "model_refits": res["model_refits"], "fused_pred_err_mean": res["fused_pred_err_mean"],
        "pair_pred_err_mean": statistics.mean(q.pair_err) if q.pair_err else None,
        # NEXT-1 selection per BE kernel (tacker_select_fusion): best warp split, 0 = sequential won
        # (blacklisted, never fused)
        "fusion_selection": {k: v["best_ws"] for k, v in getattr(q, "selection", {}).items()},
        # Eq. 10 on normalised BE throughput (app-length independent) and on kernels/s
        "improvement_vs_baymax_same_rule_eq10_normalised": eq10(res, same, "be_norm_thpt"),
        "improvement_vs_baymax_same_rule_eq10": eq10(res, same, "be_kernels_per_s"),
        "improvement_vs_baymax_eq10_normalised": eq10(res, bay, "be_norm_thpt"),
        "improvement_vs_baymax_eq10": eq10(res, bay, "be_kernels_per_s"),
        "tacker_paper_vs_baymax_eq10_normalised": eq10(paper, bay, "be_norm_thpt"),
        "arms": dict(other, tacker=tk_line),
        "roofline": roof,
        "be_roofline": be_roof,
        "cpu_baseline": cpu,
        "e2e": {"value": e2e_value, "unit": "BE kernels/s", "h2d_bytes_per_step": qi.h2d_bytes * STEP_QUERIES,
                "d2h_bytes_per_step": qi.d2h_bytes * STEP_QUERIES, "lc_p99_ms": e2e["lc_p99_ms"],
                "be_norm_thpt": e2e["be_norm_thpt"],
                "how": "the same windowed run where each query copies its input image H2D and its result D2H "
                       "from/to pinned host memory (UVA copy kernels on the manager stream)"},
        # counted by the manager: every LC kernel of every query (fused or original) plus the
        # reordered and idle-time BE launches inside the window
        "gpu_launches": int(sum(res["class_launches"].values())),
        "clocks": clocks,
    }
    line.update(extra)
    if rank == 0:
        print(json.dumps(line))


def side_workloads(args, comm, peaks, flush, tk, qos, sv, torch):
    """Beside the headline: VGG-16 b24 with the same mixed queue, ResNet-50 b32 with the round-1
    stencil / mri-q queue, and BASELINE configs[1] (ResNet-50 b1) as a managed run and as the
    kernel-level fused step (fused time vs the overlap roofline)."""
    out = {}
    rank = comm.rank
    steps = max(5, min(args.steps, 30))
    seed = 2022 + rank
    names = sv.TABLE2_BE if args.be == "table2" else tuple(args.be.split(","))
    # VGG-16 batch 24 (Table II) + the mixed queue
    tk.tacker_model_clear()
    vgg = sv.vgg16_service(24, seed)
    sv.autotune_tile_n(vgg)
    apps = sv.be_apps(names, seed)
    sv.prime_apps(apps)
    qv = calibrated_run(qos, tk, vgg, apps, args, comm, peak_steps=20)
    r = side_runs(qv, tk, ("tacker", "baymax", "baymax_same_rule", "tacker_paper"), steps, rank, args.inflight)
    out["vgg16_b24"] = dict(workload="vgg16_b24 LC + Table II mixed BE queue, QoS 50 ms (BASELINE configs[3])",
                            service_ms=qv.service_ms, lambda_peak_load=qv.peak_load, steps=steps, **r,
                            improvement_vs_baymax_same_rule_eq10_normalised=eq10(r["tacker"], r["baymax_same_rule"], "be_norm_thpt"),
                            tacker_paper_vs_baymax_eq10_normalised=eq10(r["tacker_paper"], r["baymax"], "be_norm_thpt"))
    del vgg, apps, qv
    torch.cuda.empty_cache()
    # ResNet-50 b32 + stencil / mri-q (round-1 queue) and b1 (configs[1])
    st, mq = sv.be_apps(("stencil", "mriq"), seed)
    sv.prime_apps([mq])
    for b in (32, 1):
        tk.tacker_model_clear()
        svc = sv.resnet50_service(b, seed)
        sv.autotune_tile_n(svc)
        qb = calibrated_run(qos, tk, svc, [st, mq], args, comm, peak_steps=20)
        r = side_runs(qb, tk, ("tacker", "baymax", "baymax_same_rule", "tacker_paper"), steps, rank, args.inflight)
        out[f"resnet50_b{b}_stencil_mriq"] = dict(
            workload=f"resnet50_b{b} LC + stencil/mriq BE queue, QoS 50 ms" + (" (BASELINE configs[1])" if b == 1 else ""),
            service_ms=qb.service_ms, lambda_peak_load=qb.peak_load, steps=steps, **r,
            lc_roofline=lc_class_roofline(qb, {**peaks}, "measured", svc),
            improvement_vs_baymax_same_rule_eq10_normalised=eq10(r["tacker"], r["baymax_same_rule"], "be_norm_thpt"),
            tacker_paper_vs_baymax_eq10_normalised=eq10(r["tacker_paper"], r["baymax"], "be_norm_thpt"))
        if b == 1:
            step = FusedStep(svc, st, mq, args.warp_split)
            for _ in range(3):
                step.fused()
            torch.cuda.synchronize()
            out["fused_step"] = kernel_level(torch, step, flush, peaks, 20)
        del svc, qb
        torch.cuda.empty_cache()
    return out


def run_simulated(args, comm):
    """--simulate: the same windowed protocol on the manager's simulated GPU (kernels take their
    predicted time; no CUDA), for CPU tests of the replica path.  Kernel durations are a fixed
    table shaped like the B200 measurements of the ResNet-50 b1 / stencil / mri-q run."""
    from paper_conf_hpca_zhaocczlllg22_b200 import qos, tacker as tk
    ws, rank = comm.ws, comm.rank
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
    solo = sum(k.t_pred_ms for k in ks)
    lam = LOAD / solo
    step_ms = STEP_QUERIES / lam
    w0, w1 = max(args.warmup, 3) * step_ms, (max(args.warmup, 3) + args.steps) * step_ms
    out = {}
    for pol in (tk.POLICY_BAYMAX, tk.POLICY_TACKER):
        rng = np.random.default_rng(2000 + rank)
        m = tk.Manager(pol, simulate=True, idle_cap_ms=0.5 * (QOS_MS - solo), **HEADLINE)
        for a in apps:
            m.submit_be(a)
        arr, t = [], 0.0
        while t < w1 + 1.5 * QOS_MS:
            t += rng.exponential(1.0 / lam)
            arr.append(t)
        qids = [m.submit_lc(ks, float(a)) for a in arr]
        m.run_until(QOS_MS, w0)
        s0 = m.stats()
        m.run_until(QOS_MS, w1)
        s1 = m.stats()
        m.run(QOS_MS, float(arr[-1]))
        lat = [m.latency(i) for i, a in zip(qids, arr) if w0 <= a < w1]
        out[pol] = (s1.be_kernels_done - s0.be_kernels_done, s1.now_ms - s0.now_ms,
                    qos.latency_stats(lat, QOS_MS)["lc_p99_ms"])
    be, el, p99 = out[tk.POLICY_TACKER]
    comm.barrier()
    elapsed = comm.reduce(el, "max")
    value = comm.reduce(be, "sum") / (elapsed / 1e3)
    bay = comm.reduce(out[tk.POLICY_BAYMAX][0], "sum") / (comm.reduce(out[tk.POLICY_BAYMAX][1], "max") / 1e3)
    line = {"metric": METRIC, "value": value, "unit": "BE kernels/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": elapsed / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "n/a (simulated GPU)", "data": "synthetic",
            "config": {"workload": "resnet50_b1-like LC + stencil-like BE [simulated durations]",
                       "parallelism": f"replicas x{ws} ({comm.mode}, no NCCL)"},
            "lc_p99_ms": comm.reduce(p99, "max"), "baymax": {"value": bay},
            "improvement_vs_baymax_eq10": value / bay - 1.0, "simulated": True}
    if comm.rank == 0:
        print(json.dumps(line))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100, help=f"timed steps ({STEP_QUERIES} LC queries each)")
    ap.add_argument("--warmup", type=int, default=5, help="untimed warm-up steps (same continuous run)")
    ap.add_argument("--seeds", type=int, default=3, help="trace seeds for the tacker / baymax_same_rule arms")
    ap.add_argument("--batch", type=int, default=32, help="LC batch (Table II: ResNet-50 at 32)")
    ap.add_argument("--be", default="table2", help="BE queue: table2 (Table II mixed queue) or app names")
    ap.add_argument("--inflight", type=int, default=16, help="manager: launches in flight on its stream")
    ap.add_argument("--impl", default="tacker", choices=["tacker", "reference"])
    ap.add_argument("--warp-split", type=int, default=24)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-extra", action="store_true", help="skip the side workloads (VGG-16, stencil/mri-q, b1)")
    ap.add_argument("--simulate", action="store_true", help="CPU-only: manager on its simulated GPU")
    ap.add_argument("--overlap", type=int, default=None,
                    help="programmatic dependent launch mode (tacker_set_launch_overlap: 0, 1, 2)")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        spawn_replicas(args.gpus)
    if args.impl == "reference":
        run_reference(args, int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")))
        return
    comm = Comm()
    try:
        if args.simulate:
            run_simulated(args, comm)
        else:
            if args.overlap is not None:
                from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk
                tk.tacker_set_launch_overlap(args.overlap)
            run_tacker(args, comm)
    finally:
        comm.close()


if __name__ == "__main__":
    main()
