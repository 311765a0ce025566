"""Which (LC kernel, BE kernel) pairs can Eq. 8 fuse at all?  After the bench's calibration
(ResNet-50 batch B service, stencil / mri-q BE queue), for every TC kernel x BE kernel: is a pair
model fitted, the predicted gain of whole-kernel fusion, and of a PTB slice at the pair's
opportune ratio.  One JSON line.   python tools/fusion_gains.py [--batch 32]"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=32)
    args = ap.parse_args()
    svc = sv.resnet50_service(args.batch)
    st, mq = sv.stencil_app(512, 512, 64), sv.mriq_app(64, 2048, 1024)
    tk.tacker_launch_original(None, mq.kernels[0].desc)
    tk.tacker_model_clear()
    q = qos.QosRun(svc, [st, mq], warp_split=24)
    q.calibrate()
    rows = []
    for i, k in enumerate(svc.kernels):
        if not k.is_tc:
            continue
        ttc = q.t_lc[i]
        for a, app in enumerate(q.apps):
            for j, bk in enumerate(app.kernels):
                ws = q.ws_of.get((a, j))
                if ws is None:
                    continue
                try:
                    pk = tk.tacker_fuse(k.lc, bk.desc, ws).keys()[2]
                except tk.TackerError as e:
                    rows.append({"lc": k.name, "be": bk.name, "model": False, "why": str(e)[:40]})
                    continue
                if q.pairs.get(pk) is None:
                    rows.append({"lc": k.name, "be": bk.name, "model": False})
                    continue
                tbe = q.t_be[(a, j)]
                tf = tk.tacker_pair_predict(pk, ttc, tbe)
                row = {"lc": k.name, "be": bk.name, "model": True, "t_lc": ttc, "t_be": tbe, "t_fuse": tf,
                       "gain_whole": tbe - (tf - ttc)}
                lr = q.lr_be.get((a, j))
                if lr:
                    n_full, tb, t0 = lr
                    n = max(1, int((ttc - t0) / tb)) if tb > 0 else n_full     # slice ~ as long as the LC kernel
                    xs = t0 + tb * n
                    tfs = tk.tacker_pair_predict(pk, ttc, xs)
                    row.update(slice_blocks=n, t_slice=xs, t_fuse_slice=tfs, gain_slice=xs - (tfs - ttc))
                rows.append(row)
    ok = [r for r in rows if r["model"]]
    summary = {"pairs": len(rows), "with_model": len(ok),
               "gain_whole_pos": sum(1 for r in ok if r["gain_whole"] > 0),
               "gain_slice_pos": sum(1 for r in ok if r.get("gain_slice", -1) > 0),
               "mean_gain_whole_ms": sum(r["gain_whole"] for r in ok) / max(1, len(ok)),
               "mean_gain_slice_ms": sum(r.get("gain_slice", 0) for r in ok) / max(1, len(ok))}
    print(json.dumps({"summary": summary, "rows": rows}))


if __name__ == "__main__":
    main()
