import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
from paper_conf_hpca_zhaocczlllg22_b200 import qos, services as sv, tacker as tk
convs = [c for c in synth.resnet50_convs(8) if c.name in ("layer1.0.conv1", "layer1.0.conv2", "layer1.0.conv3")]
svc = sv.resnet50_service(8, convs=convs)
st, mq = sv.stencil_app(512, 512, 64), sv.mriq_app(64, 1024, 1024)
tk.tacker_launch_original(None, mq.kernels[0].desc)
tk.tacker_model_clear()
run = qos.QosRun(svc, [st, mq], warp_split=16)
run.calibrate(reps=3, pair_reps=3)
run.measure_service(n=20)
print("lr", run.lr_be, "ws", run.ws_of, "sel", run.selection)
tk.tacker_model_clear(); tk.tacker_blacklist_clear()
for pk in run.pairs:
    for r in (0.1, 0.2, 1.8, 1.9):
        tk.tacker_pair_add_sample(pk, 1.0, r, max(1.0 + 0.1 * r, 0.5 + r))
    print(pk, tk.tacker_pair_fit(pk))
res = run.run_window(tk.POLICY_TACKER, 30.0, 5.0, load=0.8, max_inflight=8, trace=True, fuse_older=True, slice_be=True, reorder_rule=2)
print({k: res[k] for k in ("fused", "reordered", "idle_be", "be_kernels")})
print("first 40 actions", [(d["action"], d["query"], d["reorder"]) for d in res["trace"][:40]])
n = 0
for d in res["trace"]:
    if d["query"] >= 0:
        print(d["t"], d["query"], d["lc_index"], d["action"], d["ready"], d["tk_fuse"], round(d["thr"], 3), d["direct"])
        n += 1
        if n > 12: break
print([k.t_pred_ms for k in run.lc_kernels()], [[b.t_pred_ms, b.n_blocks, b.t_floor_ms, b.t_block_ms, b.warp_split] for app in run.be_apps() for b in app])
for k in run.lc_kernels():
    for b in run.be_apps()[1]:
        try:
            f = tk.tacker_fuse(k.lc, b.be, 16)
            ks = f.keys()
            print(ks[2], "blacklisted", tk.tacker_blacklist(ks[1]), "pred", tk.tacker_pair_predict(ks[2], k.t_pred_ms, 0.01) if ks[2] in run.pairs else None)
        except tk.TackerError as e:
            print("fuse err", e)
m = tk.Manager(tk.POLICY_TACKER, simulate=True, idle_cap_ms=20.0, slice_be=True, reorder_rule=2, fuse_older=True, older_margin_ms=15.0)
m.trace_enable(100000)
for ks in run.be_apps():
    m.submit_be(ks)
m.submit_lc_batch(run.lc_kernels(), [0.5 + 0.3 * i for i in range(20)])
m.run(50.0, 7.0)
tr, _ = m.trace_dicts()
print("SIM", m.stats().fused_launches, [(d["action"], d["query"], d["reorder"], d["tk_fuse"]) for d in tr[:30]])
