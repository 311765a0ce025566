"""Replay of a recorded manager trace through the discrete-event reference:
shared by the CPU (simulated GPU) and the GPU-mode tests."""
from oracle import manager_ref as mr

_ACT = {0: mr.FUSED, 1: mr.ORIGINAL_LC, 2: mr.REORDER_BE, 3: mr.IDLE_BE}


def check_trace(trace, queries, apps, qos, policy, **rules):
    """trace: Manager.trace_dicts()[0]; queries: [(arrival, [(is_tc, T)])] by query id; apps: [[(kind, T)]]
    (kind as manager_ref.App).  Asserts every decision (action, query kernel, fused app, reorder
    list, Tgain, headroom after) equals the reference's; returns the number of decisions."""
    qs = [mr.Query(i, a, list(ks)) for i, (a, ks) in enumerate(queries)]
    ap = [mr.App(list(ks)) for ks in apps]
    ref = mr.replay(trace, qs, ap, qos, policy, **rules)
    assert len(ref) == len(trace)
    for i, (r, g) in enumerate(zip(ref, trace)):
        got = (_ACT[g["action"]], (g["query"], g["lc_index"]) if g["query"] >= 0 else None, g["fused_app"],
               g["reorder"], bool(g["reverse"]))
        exp = (r.action, r.lc, r.fused_app, r.reorder, bool(r.reverse))
        assert got == exp, (i, g, r)
        if r.action != mr.IDLE_BE and (r.action == mr.FUSED or r.lc is not None):
            assert abs(g["thr"] - r.thr) <= 1e-9 * max(1.0, abs(r.thr)), (i, g["thr"], r.thr)
        if r.action == mr.FUSED:
            assert abs(g["gain"] - r.gain) <= 1e-9 * max(1.0, abs(r.gain)), (i, g["gain"], r.gain)
    return len(ref)
