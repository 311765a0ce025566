"""QoS-managed co-location run (a12; BASELINE configs 2/4/5; paper §VIII-B).

LC queries of a service (ResNet-50 / VGG-16 / ...) arrive as a Poisson process at a fraction of
the service's peak rate; a BE queue of Parboil-style applications fills the rest of the GPU; the
native manager (tacker_manager_run) decides fused / original / reorder per LC kernel from each
query's QoS headroom (§VII).  Before the run, the predictor is calibrated the paper's way
(§VI-C): standalone durations of every LC and BE kernel (history), and per (LC kernel class, BE
kernel class, warp split) a two-stage model from fused runs at the training load ratios
{0.1, 0.2, 1.8, 1.9}, the BE sized through its PTB block prefix.

Reported: BE kernels/s, LC latency p50/p99 vs the QoS target, fused / reordered / idle BE
counts; the same trace under the Baymax policy (fusion disabled) gives the Eq. 10 improvement.
"""
from __future__ import annotations

import math
import statistics

import numpy as np
import torch

from . import tacker as tk


CLASSES = ("lc_tc", "lc_cd", "fused", "be")


def _rules_name(policy, rules):
    """Which manager rules a run used, by name (DESIGN.md §2 readings)."""
    rr = rules.get("reorder_rule", tk.REORDER_UNFUSED)
    parts = ["reorder: " + {tk.REORDER_UNFUSED: "only after an unfused LC kernel (P:2035)",
                            tk.REORDER_ALWAYS: "after every LC kernel (reading 6)",
                            tk.REORDER_NEVER: "never"}[rr]]
    parts.append("older queries fuse/reorder within later queries' headroom (reading 18)" if rules.get("fuse_older")
                 else "only the newest query fuses/reorders (P:2058-2072)")
    if rules.get("slice_be"):
        parts.append("PTB slices at r* (reading 13)")
    parts.append("direct when Thr <= " + ("eps" if rules.get("direct_rule") == tk.DIRECT_EPS
                                           else "the shortest ready BE head (P:2092-2096, c15)"))
    return ("Tacker" if policy == tk.POLICY_TACKER else "Baymax (fusion off)") + "; " + "; ".join(parts)


def latency_stats(lat, qos, boot=1000, seed=0):
    """p50 / p99 (nearest rank) of query latencies, with a bootstrap 95 % CI of p99."""
    lat = np.sort(np.asarray(lat, dtype=np.float64))
    n = len(lat)
    if n == 0:
        return {"lc_p50_ms": None, "lc_p99_ms": None, "lc_p99_ci95_ms": None, "lc_max_ms": None,
                "qos_met": False, "violations": 0}
    k = min(n - 1, int(math.ceil(0.99 * n)) - 1)
    rng = np.random.default_rng(seed)
    bs = np.sort(lat[rng.integers(0, n, size=(boot, n))], axis=1)[:, k]
    return {"lc_p50_ms": float(np.median(lat)), "lc_p99_ms": float(lat[k]),
            "lc_p99_ci95_ms": [float(np.percentile(bs, 2.5)), float(np.percentile(bs, 97.5))],
            "lc_mean_ms": float(lat.mean()), "lc_max_ms": float(lat[-1]),
            "qos_met": bool(lat[k] <= qos), "violations": int((lat > qos).sum())}


def overlap_rate(t_tc, t_cd, t_corun):
    """Eq. 11: (T_TC + T_CD - T_corun) / (T_TC + T_CD) -- 0 for sequential
    execution, 0.5 for perfect overlap of equal parts."""
    return (t_tc + t_cd - t_corun) / (t_tc + t_cd)


def _prefix(desc, n):
    """Copy of a BE descriptor restricted to its first n original blocks (PTB, Fig. 7)."""
    import ctypes
    d = tk.BeDesc()
    ctypes.memmove(ctypes.addressof(d), ctypes.addressof(desc), ctypes.sizeof(d))
    d.orig_blocks = n
    return d


def _time(fn, reps=10, stream=None, inner=8):
    """Device time per launch in a pipelined stream (the manager's regime): median over `reps`
    rounds of `inner` back-to-back launches between two events, divided by `inner`.  A single
    launch between two events would add the host's launch latency (Python here) to a 10 us
    kernel."""
    s = stream or torch.cuda.current_stream()
    fn()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(inner):
            fn()
        e1.record(s)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) / inner)
    return statistics.median(ts)


# Training ratios of the two-stage model: the paper's {0.1, 0.2, 1.8, 1.9} with the
# middle of the range sampled too (0.6, 1.0: the PTB slices the manager fuses sit near r* ~ 1) and
# the last point at the whole kernel (training_prefixes) -- DESIGN.md §2 reading 5.
TRAIN_RATIOS = (0.1, 0.2, 0.6, 1.0, 1.8, 1.9)


def _interp_n(curve, t_target, full):
    """Smallest block count whose standalone time reaches t_target, by linear interpolation of the
    measured (blocks, ms) curve (the BE time is not linear near its one-block latency floor)."""
    pts = sorted(curve)
    if t_target <= pts[0][1]:
        return pts[0][0]
    for (n0, t0), (n1, t1) in zip(pts, pts[1:]):
        if t0 <= t_target <= t1:
            return min(full, max(1, int(round(n0 + (n1 - n0) * (t_target - t0) / max(t1 - t0, 1e-9)))))
    return full


def training_prefixes(prefix, full, x_tc, curve, time_fn, ratios=TRAIN_RATIOS, min_gap=0.08,
                      stage2_to_full=True):
    """BE block prefixes for the two-stage model's training ratios, realised on the MEASURED BE
    time: each target r gives the block count whose interpolated standalone time is r X_tc.
    Below the one-block floor the targets shift up (as the sweep does); stage2_to_full: the last
    sample is the whole kernel (the ratio the manager predicts for whole-kernel fusion); targets
    beyond what the whole kernel reaches fold onto it.  Consecutive samples are kept at least
    min_gap apart in measured r (prefixes on the latency floor, or a clamp, would otherwise give
    coincident points); if fewer than three targets are reachable the samples spread evenly over
    [lowest target, r_full].
    prefix(n) -> descriptor, time_fn(desc) -> ms, curve = [(blocks, ms)] incl. 1 and full.
    Returns [(n, x_cd)] (fewer than len(ratios) when the kernel has fewer distinct prefixes)."""
    pts = sorted(curve)
    r_floor, r_full = pts[0][1] / x_tc, pts[-1][1] / x_tc
    shift = max(0.0, 1.25 * r_floor - ratios[0])
    tr = [r + shift for r in ratios]
    if stage2_to_full and r_full > tr[-2] + min_gap:
        tr[-1] = r_full
    if sum(1 for r in tr if r < r_full) < 3:
        lo = min(tr[0], r_full)
        tr = [lo + (r_full - lo) * i / (len(ratios) - 1) for i in range(len(ratios))]
        min_gap = min(min_gap, 0.5 * (r_full - lo) / (len(ratios) - 1))
    out = []
    for r in tr:
        n = _interp_n(pts, r * x_tc, full) if r < r_full else full
        if out and n <= out[-1][0]:
            if out[-1][0] >= full:
                break                    # fewer distinct samples than targets
            n = min(full, out[-1][0] + 1)
        x = time_fn(prefix(n))
        while out and (x - out[-1][1]) / x_tc < min_gap and n < full:
            n = min(full, max(n + 1, int(n * 1.5)))
            x = time_fn(prefix(n))
        if out and n == out[-1][0]:
            break
        out.append((n, x))
    return out


class QosRun:
    def __init__(self, svc, apps, warp_split=24, qos_ms=50.0):
        self.svc, self.apps, self.ws, self.qos = svc, apps, warp_split, qos_ms
        self.t_lc = []           # standalone ms per LC kernel
        self.t_be = {}           # (app index, kernel index) -> ms
        self.pairs = {}          # pair key -> fitted coefficients
        self.ws_of = {}          # (app, kernel) -> warp split that fits the budget
        self.pair_err = []       # |pred - meas| / meas of the fused model on the real pairs
        self.lr_be = {}          # (app, kernel) -> (n_blocks, t_block_ms, t_floor_ms): slice LR
        self.curve_be = {}       # (app, kernel) -> [(blocks, ms)] measured prefixes incl. 1 block

    # ------------------------------------------------------------------ calibration (§VI-C)
    def with_io(self):
        """End-to-end queries: each query first copies its input image from pinned host memory
        to the device and ends by copying its result back, both as LC CUDA-core kernels through
        UVA (TACKER_BE_COPY), so the transfers sit inside the managed, timed run."""
        x, y = self.svc.inputs[0], self.svc.outputs[-1]
        self.h_in = torch.empty(x.shape, dtype=x.dtype, pin_memory=True).copy_(x)
        self.h_out = torch.empty(y.shape, dtype=y.dtype, pin_memory=True)
        self.io = (tk.be_copy(self.h_in, x), tk.be_copy(y, self.h_out))
        self.h2d_bytes = x.numel() * x.element_size()
        self.d2h_bytes = y.numel() * y.element_size()
        return self

    def _kernel_list(self):
        ks = [(k.is_tc, k.lc if k.is_tc else k.cd) for k in self.svc.kernels]
        if getattr(self, "io", None):
            ks = [(False, self.io[0])] + ks + [(False, self.io[1])]
        return ks

    def calibrate(self, reps=8, pair_reps=5):
        for is_tc, d in self._kernel_list():
            if is_tc:
                self.t_lc.append(_time(lambda: tk.tacker_launch_original(d, None), reps))
            else:
                self.t_lc.append(_time(lambda: tk.tacker_launch_original(None, d), reps))
        for a, app in enumerate(self.apps):
            for j, bk in enumerate(app.kernels):
                if bk.is_tc:       # NEXT-2: tensor-core BE kernel (never sliced)
                    self.t_be[(a, j)] = _time(lambda: tk.tacker_launch_original(bk.desc, None), reps)
                    continue
                self.t_be[(a, j)] = _time(lambda: tk.tacker_launch_original(None, bk.desc), reps)
                if self.t_be[(a, j)] >= 0.01 and bk.desc.kind != tk.BE_JDS_SCAN:
                    self.lr_be[(a, j)] = self._fit_slice_lr(a, j, bk, reps)
        # NEXT-1 through the C ABI: per BE kernel, every fused candidate
        # (warp split) with a representative LC kernel and the sequential pair are timed; the fastest
        # split is kept, and a BE kernel for which sequential wins is blacklisted (never fused)
        tcs = [k for k in self.svc.kernels if k.is_tc]
        tk.tacker_blacklist_clear()
        self.selection = {}
        for a, app in enumerate(self.apps):
            for j, bk in enumerate(app.kernels):
                if self.t_be[(a, j)] < 0.01 or bk.is_tc:
                    continue
                best, best_ms, seq_ms, cand = tk.tacker_select_fusion(
                    tcs[len(tcs) // 2].lc, bk.desc, splits=tuple(range(self.ws, 3, -4)), reps=3)
                self.selection[bk.name] = {"best_ws": best, "best_ms": best_ms, "seq_ms": seq_ms, "fused_ms": cand}
                if best > 0:
                    self.ws_of[(a, j)] = best
        # two-stage models per (LC class, BE class, ws), trained on block prefixes
        off = 1 if getattr(self, "io", None) else 0      # t_lc index of svc.kernels[0]
        refit = set()
        for i0, k in enumerate(self.svc.kernels):
            i = i0 + off
            if not k.is_tc:
                continue
            for a, app in enumerate(self.apps):
                for j, bk in enumerate(app.kernels):
                    if self.t_be[(a, j)] < 0.01 or bk.is_tc:   # < 10 us (phiMag, binning, bfs levels): reorder only
                        continue
                    if (a, j) not in self.ws_of:
                        continue
                    ws = self.ws_of[(a, j)]       # the manager fuses this BE kernel at one split
                    try:
                        f = tk.tacker_fuse(k.lc, bk.desc, ws)
                    except tk.TackerError as e:
                        if e.status not in (tk.ERESOURCE, tk.EUNSUPPORTED):   # budget / per-kind warp cap
                            raise
                        continue                  # no model -> the manager never fuses this pair
                    pkey = f.keys()[2]
                    if pkey not in self.pairs:
                        self.pairs[pkey] = self._fit_pair(k, bk, ws, self.t_lc[i], pkey, pair_reps)
                    if self.pairs[pkey] is None:
                        continue
                    # accuracy of the 4-point model on the actual whole-kernel pair, then that
                    # co-run joins the pair's history (the paper trains on historical data and
                    # refits from co-running data)
                    t_meas = _time(lambda: f.launch(), 3)
                    t_pred = tk.tacker_pair_predict(pkey, self.t_lc[i], self.t_be[(a, j)])
                    self.pair_err.append(abs(t_pred - t_meas) / t_meas)
                    tk.tacker_pair_add_sample(pkey, self.t_lc[i], self.t_be[(a, j)], t_meas)
                    refit.add(pkey)
        self._calibrate_reverse(range(len(self.apps)), pair_reps, refit)
        for pkey in refit:
            self.pairs[pkey] = tk.tacker_pair_fit(pkey)

    def _calibrate_reverse(self, app_ids, pair_reps, refit):
        """NEXT-2 reverse pairs: every LC CUDA-core kernel (the fused kernel's CUDA-core part) with
        every tensor-core kernel of the BE apps `app_ids` (its tcgen05 part), at REV_WS warps."""
        for i, (is_tc, d) in enumerate(self._kernel_list()):
            if is_tc or self.t_lc[i] < 0.01 or d.kind == tk.BE_COPY:
                continue
            for a in app_ids:
                for j, bk in enumerate(self.apps[a].kernels):
                    if not bk.is_tc:
                        continue
                    try:
                        f = tk.tacker_fuse(bk.desc, d, self.REV_WS)
                    except tk.TackerError as e:
                        if e.status not in (tk.ERESOURCE, tk.EUNSUPPORTED):
                            raise
                        continue
                    pkey = f.keys()[2]
                    if pkey not in self.pairs:
                        self.pairs[pkey] = self._fit_pair_rev(bk.desc, d, self.t_be[(a, j)], self.t_lc[i], pkey,
                                                              pair_reps)
                    t_meas = _time(lambda: f.launch(), 3)
                    t_pred = tk.tacker_pair_predict(pkey, self.t_be[(a, j)], self.t_lc[i])
                    self.pair_err.append(abs(t_pred - t_meas) / t_meas)
                    tk.tacker_pair_add_sample(pkey, self.t_be[(a, j)], self.t_lc[i], t_meas)
                    refit.add(pkey)

    def add_tc_apps(self, apps, reps=8, pair_reps=5):
        """Append tensor-core BE apps (NEXT-2) to a calibrated run: time their kernels and fit the
        reverse pairs with the LC CUDA-core kernels (the existing calibration is kept)."""
        first = len(self.apps)
        self.apps = list(self.apps) + list(apps)
        for a in range(first, len(self.apps)):
            for j, bk in enumerate(self.apps[a].kernels):
                assert bk.is_tc, "add_tc_apps takes tensor-core BE apps only"
                self.t_be[(a, j)] = _time(lambda: tk.tacker_launch_original(bk.desc, None), reps)
        refit = set()
        self._calibrate_reverse(range(first, len(self.apps)), pair_reps, refit)
        for pkey in refit:
            self.pairs[pkey] = tk.tacker_pair_fit(pkey)
        return self

    REV_WS = 24    # CUDA-core warps of a reverse-fused LC kernel (tools/reverse_pair.py: im2col needs 24)

    def _fit_pair_rev(self, tc, cd, x_tc, x_cd, pkey, reps):
        """Reverse pair (NEXT-2) at the training ratios r = X_cd / X_tc in {0.1, 0.2, 1.8, 1.9}
        (P:1852-1858): below the whole pair's ratio the CUDA-core kernel runs a PTB block prefix
        (Fig. 7); above it the tensor-core GEMM runs a prefix of its rows (fewer M tiles)."""
        import ctypes
        full = tk.tacker_be_num_blocks(cd)
        r_full = x_cd / x_tc
        for r in (0.1, 0.2, 1.8, 1.9):
            if r <= r_full:
                n = min(max(int(round(full * r / r_full)), 1), full)
                c, t = _prefix(cd, n), tc
            else:
                t = tk.LcDesc()
                ctypes.memmove(ctypes.addressof(t), ctypes.addressof(tc), ctypes.sizeof(t))
                t.M = max(128, int(round(tc.M * r_full / r / 128)) * 128)
                c = cd
            f = tk.tacker_fuse(t, c, self.REV_WS)
            t_f = _time(lambda: f.launch(), reps)
            xt = _time(lambda: tk.tacker_launch_original(t, None), reps)
            xc = _time(lambda: tk.tacker_launch_original(None, c), reps)
            tk.tacker_pair_add_sample(pkey, xt, xc, t_f)
        return tk.tacker_pair_fit(pkey)

    def _fit_slice_lr(self, a, j, bk, reps):
        """Per-kernel LR over PTB slices (§VI-C): standalone time of the first n
        original blocks, X_cd(n) = t_floor + t_block n, OLS over n in {N/16, N/8, N/4, N/2, N}
        (the regime a fused slice runs in; one block alone sits on the latency floor)."""
        full = tk.tacker_be_num_blocks(bk.desc)
        key = f"be:slice:app{a}:k{j}"
        ns = sorted({max(1, full // d) for d in (16, 8, 4, 2, 1)})
        curve = []
        for n in ns:
            d = _prefix(bk.desc, n)
            t = self.t_be[(a, j)] if n == full else _time(lambda: tk.tacker_launch_original(None, d), reps)
            tk.tacker_model_add_sample(key, n, t)
            curve.append((n, t))
        if ns[0] > 1:     # the one-block floor (not an LR sample: the LR covers the slice regime)
            d1 = _prefix(bk.desc, 1)
            curve.append((1, _time(lambda: tk.tacker_launch_original(None, d1), reps)))
        self.curve_be[(a, j)] = sorted(curve)
        slope, icpt = tk.tacker_model_fit(key)
        return (full, max(slope, 0.0), max(icpt, 0.0))

    def _fit_pair(self, k, bk, ws, x_tc, pkey, reps):
        """Two-stage model of (LC kernel k, BE kernel bk, ws) from fused runs at the training ratios
        (P:1852-1858), the BE sized by PTB prefixes picked on its measured time curve
        (training_prefixes)."""
        full = tk.tacker_be_num_blocks(bk.desc)
        prefix = lambda n: _prefix(bk.desc, n)
        aj = next(((a_, j_) for (a_, j_) in self.t_be if self.apps[a_].kernels[j_] is bk), None)
        curve = self.curve_be.get(aj)
        if not curve:
            curve = [(1, _time(lambda: tk.tacker_launch_original(None, prefix(1)), reps)), (full, self.t_be_of(bk))]
        time_fn = lambda d: _time(lambda: tk.tacker_launch_original(None, d), reps)
        samples = training_prefixes(prefix, full, x_tc, curve, time_fn)
        if len(samples) < 2:
            return None           # too few distinct prefixes (a tiny kernel): no model, never fused
        for n, x_cd in samples:
            d = prefix(n)
            f = tk.tacker_fuse(k.lc, d, ws)
            t_f = _time(lambda: f.launch(), reps)
            tk.tacker_pair_add_sample(pkey, x_tc, x_cd, t_f)
        return tk.tacker_pair_fit(pkey)

    def t_be_of(self, bk):
        for a, app in enumerate(self.apps):
            for j, b in enumerate(app.kernels):
                if b is bk:
                    return self.t_be[(a, j)]
        raise KeyError(bk.name)

    # ------------------------------------------------------------------ structs for the manager
    def lc_kernels(self):
        out = []
        for (is_tc, d), t in zip(self._kernel_list(), self.t_lc):
            lk = tk.LcKernel(is_tc=1 if is_tc else 0, t_pred_ms=t, warp_split=0 if is_tc else self.REV_WS)
            if is_tc:
                lk.lc = d
            else:
                lk.cd = d
            out.append(lk)
        return out

    def be_apps(self):
        out = []
        for a, app in enumerate(self.apps):
            ks = []
            for j, bk in enumerate(app.kernels):
                if bk.is_tc:
                    ks.append(tk.BeKernel(is_cd=0, is_tc=1, t_pred_ms=self.t_be[(a, j)], tc=bk.desc))
                    continue
                n, tb, tf = self.lr_be.get((a, j), (0, 0.0, 0.0))
                ks.append(tk.BeKernel(is_cd=1, t_pred_ms=self.t_be[(a, j)], be=bk.desc,
                                      warp_split=self.ws_of.get((a, j), self.ws),
                                      n_blocks=n, t_block_ms=tb, t_floor_ms=tf))
            out.append(ks)
        return out

    def replay_inputs(self, arrivals):
        """(queries, apps) in the form tests/trace_check.check_trace takes: the predicted times the
        manager was given (every query of a run has the same kernels)."""
        ks = [(bool(k.is_tc), k.t_pred_ms) for k in self.lc_kernels()]
        queries = [(float(a), list(ks)) for a in arrivals]
        apps = [[(2 if b.is_tc else (1 if b.is_cd else 0), b.t_pred_ms) for b in app] for app in self.be_apps()]
        return queries, apps

    def idle_cap(self):
        return max(0.5 * (self.qos - self.query_solo_ms()), 0.0)

    def query_solo_ms(self):
        return sum(self.t_lc)

    def measure_service(self, n=200, max_inflight=4):
        """Peak LC load: the manager's service rate for LC-only queries -- n
        queries all arriving at once, run back to back through the manager (no BE apps); with a
        50 ms target and ~1 ms queries the QoS-safe peak rate is this service rate.  Returns and
        stores the mean service time per query (ms)."""
        stream = torch.cuda.current_stream()
        torch.cuda.synchronize()
        m = tk.Manager(tk.POLICY_BAYMAX, stream=stream, simulate=False, max_inflight=max_inflight)
        kernels = self.lc_kernels()
        t0 = m.stats().now_ms + 1.0
        for _ in range(n):
            m.submit_lc(kernels, t0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        m.run(self.qos, t0)
        e1.record(stream)
        e1.synchronize()
        self.service_ms = e0.elapsed_time(e1) / n
        return self.service_ms

    # ------------------------------------------------------------------ steady-state window
    def _manager(self, policy, stream, max_inflight, idle_cap_ms, slice_be=False, slice_ratio=0.0,
                 reorder_rule=tk.REORDER_UNFUSED, reverse_fusion=True, fuse_older=False, older_margin_ms=None,
                 direct_rule=tk.DIRECT_MIN_BE, lc_only=False):
        cap = idle_cap_ms if idle_cap_ms is not None else 0.5 * (self.qos - self.query_solo_ms())
        m = tk.Manager(policy, stream=stream, simulate=False, idle_cap_ms=max(cap, 0.0), max_inflight=max_inflight,
                       slice_be=slice_be, slice_ratio=slice_ratio, reorder_rule=reorder_rule,
                       reverse_fusion=reverse_fusion, fuse_older=fuse_older,
                       older_margin_ms=0.3 * self.qos if older_margin_ms is None else older_margin_ms,
                       direct_rule=direct_rule)
        if not lc_only:
            for ks in self.be_apps():
                m.submit_be(ks)
        return m

    def find_peak_load(self, window_ms, warm_ms=200.0, lo=0.5, hi=1.0, iters=5, seed=4242, max_inflight=4):
        """lambda_peak ("the peak load that meets QoS"): bisection on the load
        fraction of the LC-only service rate (1 / service_ms) with LC-only windowed runs (no BE
        apps), criterion p99 <= QoS.  Rates above the service rate are not sustainable, so the
        search is capped at it.  Returns (peak load fraction, [(load, p99)])."""
        hist = []

        def ok(load):
            r = self.run_window(tk.POLICY_BAYMAX, window_ms, warm_ms, load=load, seed=seed,
                                max_inflight=max_inflight, lc_only=True)
            hist.append((load, r["lc_p99_ms"]))
            return r["qos_met"]

        if ok(hi):
            self.peak_load = hi
            return hi, hist
        for _ in range(iters):
            mid = 0.5 * (lo + hi)
            if ok(mid):
                lo = mid
            else:
                hi = mid
        self.peak_load = lo
        return lo, hist

    def run_window(self, policy, window_ms, warm_ms, tail_ms=None, load=0.8, seed=1000, max_inflight=4,
                   idle_cap_ms=None, sync=None, trace=False, lc_only=False, **rules):
        """Steady-state measurement: ONE continuous Poisson run of
        warm_ms + window_ms + tail_ms at `load` x the peak rate; the manager runs natively up to
        the window start (tacker_manager_run_until: no drain, no sync), the window is bracketed by
        CUDA events on the manager stream (after a stream sync and `sync()`, e.g. a barrier, at its
        start and end), then the run continues through the tail (arrivals keep coming while the
        window's last queries finish) and drains.  Reported over the window only: BE kernels and
        BE work issued inside it / its device time, and the latency of every query that ARRIVED
        inside it (p50 / p99 nearest rank, bootstrap 95 % CI of p99).  The ramp-up and drain are
        outside the window, so the result does not depend on the run length."""
        stream = torch.cuda.current_stream()
        torch.cuda.synchronize()
        tail_ms = self.qos * 1.5 if tail_ms is None else tail_ms
        lam = load / getattr(self, "service_ms", self.query_solo_ms())     # queries per ms
        rng = np.random.default_rng(seed)
        m = self._manager(policy, stream, max_inflight, idle_cap_ms, lc_only=lc_only, **rules)
        if trace:
            m.trace_enable(4_000_000)
        kernels = self.lc_kernels()
        m.prepare(kernels)
        # the whole trace is submitted (one C call) before its first arrival: offsets first, then
        # t0 a few ms after the submission finishes
        span = warm_ms + window_ms + tail_ms
        offs, t = [], 0.0
        while True:
            t += rng.exponential(1.0 / lam)
            if t >= span:
                break
            offs.append(t)
        t0 = m.stats().now_ms + 20.0 + 1e-3 * len(offs)
        w0, w1 = t0 + warm_ms, t0 + warm_ms + window_ms
        arr = [t0 + o for o in offs]
        qids = m.submit_lc_batch(kernels, arr)
        if m.stats().now_ms > t0:
            raise RuntimeError("query submission overran the trace start")
        m.run_until(self.qos, w0)
        torch.cuda.synchronize()
        if sync:
            sync()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0 = m.stats()
        e0.record(stream)
        m.run_until(self.qos, w1)
        e1.record(stream)
        s1 = m.stats()
        torch.cuda.synchronize()
        if sync:
            sync()
        m.run(self.qos, float(arr[-1]) if arr else w1)
        gpu_ms = e0.elapsed_time(e1)
        inwin = [q for q, a in zip(qids, arr) if w0 <= a < w1]
        lat = np.array([m.latency(q) for q in inwin])
        st = m.stats()
        d = lambda f: getattr(s1, f) - getattr(s0, f)
        be = d("be_kernels_done")
        out = {"policy": "tacker" if policy == tk.POLICY_TACKER else "baymax", "rules": _rules_name(policy, rules),
               "queries": int(len(lat)), "lambda_per_s": lam * 1e3, "load": load,
               "window_ms": window_ms, "warm_ms": warm_ms, "tail_ms": tail_ms, "elapsed_ms": gpu_ms,
               "be_kernels": int(be), "be_kernels_per_s": be / (gpu_ms / 1e3),
               "be_work_ms": d("be_work_ms"), "be_norm_thpt": d("be_work_ms") / gpu_ms,
               "fused": int(d("fused_launches")), "reverse_fused": int(d("reverse_fused")),
               "reordered": int(d("reordered_be")), "idle_be": int(d("idle_be")),
               "model_refits": int(st.model_refits),
               "fused_pred_err_mean": st.pred_err_sum / st.pred_err_n if st.pred_err_n else None,
               "class_ms": {n: float(s1.class_ms[c] - s0.class_ms[c]) for c, n in enumerate(CLASSES)},
               "class_launches": {n: int(s1.class_launches[c] - s0.class_launches[c]) for c, n in enumerate(CLASSES)},
               "qos_ms": self.qos, "query_solo_ms": self.query_solo_ms(),
               "service_ms": getattr(self, "service_ms", None), "max_inflight": max_inflight,
               "host_decide_us_per_step": (st.host_decide_ms * 1e3 / st.host_steps) if st.host_steps else None}
        out.update(latency_stats(lat, self.qos))
        if trace:
            out["trace"], out["trace_dropped"] = m.trace_dicts()
            out["arrivals"] = list(arr)
        return out

    # ------------------------------------------------------------------ one managed run
    def run(self, policy, n_queries, load=0.8, seed=1000, warmup=0, max_inflight=4, idle_cap_ms=None,
            slice_be=False, slice_ratio=0.0, reorder_rule=tk.REORDER_UNFUSED, reverse_fusion=True, fuse_older=False,
            older_margin_ms=None, direct_rule=tk.DIRECT_MIN_BE):
        """Poisson arrivals at `load` x the service's peak rate (1 / standalone query time; the
        paper's 80 % of the peak QoS-safe load).  Returns a result dict."""
        stream = torch.cuda.current_stream()
        torch.cuda.synchronize()
        # peak rate = the measured LC-only service rate through the manager (measure_service), else
        # 1 / the standalone query time
        lam = load / getattr(self, "service_ms", self.query_solo_ms())     # queries per ms
        rng = np.random.default_rng(seed)
        gaps = rng.exponential(1.0 / lam, n_queries + warmup)
        cap = idle_cap_ms if idle_cap_ms is not None else 0.5 * (self.qos - self.query_solo_ms())
        m = tk.Manager(policy, stream=stream, simulate=False, idle_cap_ms=max(cap, 0.0), max_inflight=max_inflight,
                       slice_be=slice_be, slice_ratio=slice_ratio, reorder_rule=reorder_rule,
                       reverse_fusion=reverse_fusion, fuse_older=fuse_older,
                       older_margin_ms=0.3 * self.qos if older_margin_ms is None else older_margin_ms,
                       direct_rule=direct_rule)
        for ks in self.be_apps():
            m.submit_be(ks)
        kernels = self.lc_kernels()
        m.prepare(kernels)                          # fused handles built before arrivals are fixed
        t0 = m.stats().now_ms + 20.0 + 1e-3 * len(gaps)
        arr = t0 + np.cumsum(gaps)
        qids = m.submit_lc_batch(kernels, arr)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        m.run(self.qos, float(arr[-1]))
        e1.record(stream)
        e1.synchronize()
        st = m.stats()
        lat = np.array([m.latency(q) for q in qids[warmup:]])
        gpu_ms = e0.elapsed_time(e1)
        lat_sorted = np.sort(lat)
        p99 = float(lat_sorted[min(len(lat) - 1, int(math.ceil(0.99 * len(lat))) - 1)])
        return {"policy": "tacker" if policy == tk.POLICY_TACKER else "baymax", "slice_be": bool(slice_be),
                "reorder_rule": int(reorder_rule), "queries": int(len(lat)),
                "lambda_per_s": lam * 1e3, "load": load, "elapsed_ms": gpu_ms,
                "be_kernels": int(st.be_kernels_done), "be_kernels_per_s": st.be_kernels_done / (gpu_ms / 1e3),
                # normalised BE throughput: standalone-milliseconds of BE work per wall millisecond
                "be_work_ms": st.be_work_ms, "be_norm_thpt": st.be_work_ms / gpu_ms,
                "fused": int(st.fused_launches), "reverse_fused": int(st.reverse_fused),
                "reordered": int(st.reordered_be), "idle_be": int(st.idle_be),
                "model_refits": int(st.model_refits),
                "fused_pred_err_mean": st.pred_err_sum / st.pred_err_n if st.pred_err_n else None,
                "class_ms": {n: float(st.class_ms[c]) for c, n in enumerate(("lc_tc", "lc_cd", "fused", "be"))},
                "class_launches": {n: int(st.class_launches[c]) for c, n in enumerate(("lc_tc", "lc_cd", "fused", "be"))},
                "lc_p50_ms": float(np.median(lat)), "lc_p99_ms": p99, "lc_max_ms": float(lat.max()),
                "qos_ms": self.qos, "qos_met": bool(p99 <= self.qos), "query_solo_ms": self.query_solo_ms(),
                "service_ms": getattr(self, "service_ms", None), "max_inflight": max_inflight}
