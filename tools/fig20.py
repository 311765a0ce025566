"""Fig. 20 analogue (Eq. 11): an LC tensor-core kernel and a BE CUDA-core kernel
of balanced solo times (T_TC ~ T_CD) run (a) sequentially, (b) fused (Tacker), (c) co-running on two
streams (the paper's Stream co-location), (d) co-running in two green contexts that partition the
SMs (the B200 substitute for the paper's MPS co-location; several LC/BE SM splits, best kept).
Overlap = Eq. 11 (T_TC + T_CD - T_corun) / (T_TC + T_CD).  Prints one JSON line per pair.

  python tools/fig20.py [--pairs conv:mriq,conv:stencil,conv:sgemm,conv:cp]"""
import argparse
import ctypes
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200.qos import overlap_rate  # noqa: E402


def green_streams(n_lc):
    """Two green contexts splitting the device's SMs into >= n_lc SMs for the LC and the rest for
    the BE; returns (lc stream, be stream, (lc SMs, be SMs), contexts)."""
    from cuda.bindings import driver as d
    d.cuInit(0)
    _, dev = d.cuDeviceGet(0)
    _, res = d.cuDeviceGetDevResource(dev, d.CUdevResourceType.CU_DEV_RESOURCE_TYPE_SM)
    err, groups, n, rem = d.cuDevSmResourceSplitByCount(1, res, 0, n_lc)
    assert err == d.CUresult.CUDA_SUCCESS, err
    out = []
    for r in (groups[0], rem):
        _, desc = d.cuDevResourceGenerateDesc([r], 1)
        _, g = d.cuGreenCtxCreate(desc, dev, d.CUgreenCtxCreate_flags.CU_GREEN_CTX_DEFAULT_STREAM)
        _, s = d.cuGreenCtxStreamCreate(g, d.CUstream_flags.CU_STREAM_NON_BLOCKING, 0)
        out.append((g, s, r.sm.smCount))
    return out[0][1], out[1][1], (out[0][2], out[1][2]), out


def timed(fn, reps=20, streams=()):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        for s in streams:   # join side streams into the current one
            ev = torch.cuda.Event()
            ev.record(s)
            torch.cuda.current_stream().wait_event(ev)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--pairs", default="conv:mriq,conv:stencil,conv:sgemm,conv:cp,conv:fft")
    ap.add_argument("--ws", type=int, default=24)
    args = ap.parse_args()
    apps = {n: sv.be_apps([n])[0] for n in ("mriq", "stencil", "sgemm", "cp", "fft")}
    sv.prime_apps(list(apps.values()))
    N = K = 4096
    B = torch.randn(N, K, device="cuda").half()
    for pair in args.pairs.split(","):
        be_name = pair.split(":")[1]
        bk = [k for k in apps[be_name].kernels if k.name not in ("mriq.phimag",)][0]
        t_be = qos._time(lambda: tk.tacker_launch_original(None, bk.desc), 10)
        # balance (Fig. 20 compares pairs of equal solo time): an fp16 GEMM [M, 4096] x [4096, 4096]^T
        # as the LC tensor-core kernel with M sized so that T_TC ~ T_CD, fused 1:1 with the whole BE kernel
        M = 1024
        for _ in range(3):
            A = torch.randn(M, K, device="cuda").half()
            D = torch.empty(M, N, device="cuda", dtype=torch.float16)
            lc = tk.lc_gemm(A, B, D, b_const=True)
            t_g = qos._time(lambda: tk.tacker_launch_original(lc, None), 5)
            M = max(128, int(round(M * t_be / t_g / 128)) * 128)
        A = torch.randn(M, K, device="cuda").half()
        D = torch.empty(M, N, device="cuda", dtype=torch.float16)
        lc = tk.lc_gemm(A, B, D, b_const=True)
        lc_chain = lambda s=None: tk.tacker_launch_original(lc, None, stream=s)
        reps = M
        t_tc = timed(lambda: lc_chain())
        t_cd = timed(lambda: tk.tacker_launch_original(None, bk.desc))
        seq = timed(lambda: (lc_chain(), tk.tacker_launch_original(None, bk.desc)))
        fs = []
        for ws in range(args.ws, 3, -4):   # the widest split the BE kind and the budget allow
            try:
                fs.append(tk.tacker_fuse(lc, bk.desc, ws))
                break
            except tk.TackerError as e:
                if e.status not in (tk.EUNSUPPORTED, tk.ERESOURCE):
                    raise
        fused = timed(lambda: [f.launch() for f in fs])
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

        def two_streams():
            s1.wait_stream(torch.cuda.current_stream())
            s2.wait_stream(torch.cuda.current_stream())
            lc_chain(s1)
            tk.tacker_launch_original(None, bk.desc, stream=s2)
        streams = timed(two_streams, streams=(s1, s2))
        green = {}
        for n_lc in (32, 64, 96, 112):
            try:
                g1, g2, split, keep = green_streams(n_lc)
            except Exception as e:   # noqa: BLE001
                green[n_lc] = f"unavailable: {e}"
                continue
            gs1, gs2 = int(g1), int(g2)
            ext = [torch.cuda.ExternalStream(gs1), torch.cuda.ExternalStream(gs2)]

            def green_run():
                for s in ext:
                    s.wait_stream(torch.cuda.current_stream())
                lc_chain(gs1)
                tk.tacker_launch_original(None, bk.desc, stream=gs2)
            green[f"{split[0]}/{split[1]}"] = timed(green_run, streams=ext)
        best_green = min((v for v in green.values() if isinstance(v, float)), default=None)
        row = {"pair": f"gemm {M}x4096x4096 fp16 | {bk.name}", "warp_split": fs[0].info().be_warps, "T_TC_ms": t_tc, "T_CD_ms": t_cd, "sequential_ms": seq,
               "fused_ms": fused, "two_streams_ms": streams, "green_ctx_ms": green,
               "overlap_eq11": {"fused": overlap_rate(t_tc, t_cd, fused),
                                "two_streams": overlap_rate(t_tc, t_cd, streams),
                                "green_ctx_best": overlap_rate(t_tc, t_cd, best_green) if best_green else None,
                                "sequential": overlap_rate(t_tc, t_cd, seq)}}
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
