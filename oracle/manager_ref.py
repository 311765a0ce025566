"""Discrete-event reference of Tacker's QoS-aware kernel manager (§VII).
Test infrastructure only.

Rules, in the paper's order:
  * Eq. 7: T_Q = T_queue + T_lc + T_fuse + T_be <= T_qos.
  * Eq. 9: when the first kernel of the newest query Q is issued,
        Thr = T_qos - T_queue - T_ori_solo(Q) - sum_i T_lc_i
    over the remaining predicted GPU time of earlier still-active queries.
    T_queue = time Q waited between arrival and the issue of its first kernel (reading).
  * Only the newest query fuses or reorders; earlier queries' kernels launch directly
    (P:2058-2072).  Thr "close to 0" -> launch directly: reading Thr <= direct_eps.
  * Eq. 8: for the current TC kernel (Ttc) and each ready BE head kernel (Tcd) with a
    fused prediction Tk_fuse: admissible iff Ttc + Tcd > Tk_fuse and Tk_fuse - Ttc < Thr.
    Pick the max Tgain = Tcd - (Tk_fuse - Ttc); ties -> lowest app index.
    Then Thr -= Tk_fuse - Ttc.
  * Reorder: after the LC kernel (fused or not), launch the other ready BE heads
    (app index order) whose Ttmp < Thr, Thr -= Ttmp.  Reading: the text applies
    reorder when no fusion is possible; Tacker is described as using "both adaptive kernel
    fusion and kernel reorder", so reordering also follows a fused launch and
    Tacker never reorders less than Baymax.
  * Only the head kernel of each BE app is a candidate; the next kernel of an app
    becomes ready when the previous one completes.
  * Baymax mode = the same manager with fusion disabled ("static scheduling").
  * Idle GPU (no active LC query; the paper is silent): launch one ready BE head whose
    duration <= idle_cap, round robin over apps.
"""
from __future__ import annotations

from dataclasses import dataclass, field

TACKER, BAYMAX = 0, 1
FUSED, ORIGINAL_LC, REORDER_BE, IDLE_BE, NOTHING = 0, 1, 2, 3, 4


@dataclass
class Decision:
    action: int
    lc: tuple | None = None       # (query id, kernel index)
    fused_app: int = -1
    reorder: list = field(default_factory=list)   # app ids launched after the LC kernel
    thr: float = 0.0
    gain: float = 0.0


def decide(ttc, lc_is_tc, thr, heads, policy, fuse_pred, allow=True):
    """Pure decision for one LC kernel.

    heads: list of (app, Tcd, be_is_cd) for READY BE head kernels, in app order.
    fuse_pred(app) -> Tk_fuse or None.  Returns (fused_app, reorder_apps, thr, gain)."""
    fused, gain_best, tf_best = -1, None, None
    if allow and policy == TACKER and lc_is_tc:
        for app, tcd, be_cd in heads:
            if not be_cd:
                continue
            tf = fuse_pred(app)
            if tf is None:
                continue
            if ttc + tcd > tf and tf - ttc < thr:
                gain = tcd - (tf - ttc)
                if gain_best is None or gain > gain_best:
                    fused, gain_best, tf_best = app, gain, tf
    reorder = []
    if fused >= 0:
        thr -= tf_best - ttc
    if allow:
        for app, tcd, _ in heads:
            if app == fused:
                continue
            if tcd < thr:
                reorder.append(app)
                thr -= tcd
    return fused, reorder, thr, (gain_best or 0.0)


@dataclass
class Query:
    qid: int
    arrival: float
    kernels: list          # [(is_tc, T_pred)]
    pos: int = 0
    thr: float | None = None
    direct: bool = False
    issue: float | None = None
    done_at: float | None = None

    def remaining(self):
        return sum(t for _, t in self.kernels[self.pos:])


@dataclass
class App:
    kernels: list          # [(is_cd, T_pred)], cycled forever
    pos: int = 0
    ready_at: float = 0.0
    completed: int = 0

    def head(self):
        return self.kernels[self.pos % len(self.kernels)]


def simulate(queries, apps, qos, policy, fuse_pred, direct_eps=0.0, idle_cap=None, t_end=None):
    """Serial single-stream GPU whose kernels take exactly their predicted time.

    fuse_pred(lc_T, be_T) -> Tk_fuse or None.  The manager acts whenever the stream drains.
    Returns dict(latency per query, be_completed, timeline, decisions)."""
    t = 0.0
    active: list[Query] = []
    pending = sorted(queries, key=lambda q: q.arrival)
    timeline, decisions = [], []
    qi = 0
    while True:
        while qi < len(pending) and pending[qi].arrival <= t:
            active.append(pending[qi])
            qi += 1
        active = [q for q in active if q.pos < len(q.kernels)]
        if not active and qi >= len(pending):
            break
        if t_end is not None and t >= t_end:
            break
        heads = [(a, app.head()[1], app.head()[0]) for a, app in enumerate(apps) if app.ready_at <= t]
        if active:
            q = active[0]
            newest = active[-1]
            if q.issue is None:
                q.issue = t
                if q is newest:
                    earlier = sum(o.remaining() for o in active[:-1])
                    q.thr = qos - (t - q.arrival) - q.remaining() - earlier
                    q.direct = q.thr <= direct_eps
            is_tc, ttc = q.kernels[q.pos]
            allow = (q is newest) and not q.direct and q.thr is not None
            thr = q.thr if q.thr is not None else 0.0
            fused, reorder, thr2, gain = decide(
                ttc, is_tc, thr, heads, policy,
                lambda a: fuse_pred(ttc, apps[a].head()[1]), allow)
            if allow:
                q.thr = thr2
            start = t
            if fused >= 0:
                dur = fuse_pred(ttc, apps[fused].head()[1])
                timeline.append(("fused", q.qid, q.pos, fused, start, start + dur))
                apps[fused].pos += 1
                apps[fused].completed += 1
                apps[fused].ready_at = start + dur
                decisions.append(Decision(FUSED, (q.qid, q.pos), fused, list(reorder), q.thr, gain))
            else:
                dur = ttc
                timeline.append(("lc", q.qid, q.pos, -1, start, start + dur))
                decisions.append(Decision(REORDER_BE if reorder else ORIGINAL_LC, (q.qid, q.pos), -1,
                                          list(reorder), thr2 if allow else thr))
            t = start + dur
            q.pos += 1
            if q.pos == len(q.kernels):
                q.done_at = t
            for a in reorder:
                d = apps[a].head()[1]
                timeline.append(("be", -1, -1, a, t, t + d))
                apps[a].pos += 1
                apps[a].completed += 1
                t += d
                apps[a].ready_at = t
        else:
            nxt = pending[qi].arrival if qi < len(pending) else None
            cands = [(a, d) for a, d, _ in heads if idle_cap is None or d <= idle_cap]
            if cands:
                a, d = cands[0]
                timeline.append(("be", -1, -1, a, t, t + d))
                decisions.append(Decision(IDLE_BE, None, -1, [a], 0.0))
                apps[a].pos += 1
                apps[a].completed += 1
                t += d
                apps[a].ready_at = t
            else:
                future = [app.ready_at for app in apps if app.ready_at > t]
                cand = [x for x in ([nxt] if nxt is not None else []) + future]
                if not cand:
                    break
                t = min(cand)
    lat = {q.qid: (q.done_at - q.arrival) for q in queries if q.done_at is not None}
    return dict(latency=lat, be_completed=[a.completed for a in apps], timeline=timeline,
                decisions=decisions, t=t)
