"""Discrete-event reference of Tacker's QoS-aware kernel manager (§VII).
Test infrastructure only.

Rules, in the paper's order:
  * Eq. 7: T_Q = T_queue + T_lc + T_fuse + T_be <= T_qos.
  * Eq. 9: when the first kernel of the newest query Q is issued,
        Thr = T_qos - T_queue - T_ori_solo(Q) - sum_i T_lc_i
    over the remaining predicted GPU time of earlier still-active queries.
    T_queue = time Q waited between arrival and the issue of its first kernel (reading).
  * Only the newest query fuses or reorders; earlier queries' kernels launch directly
    (P:2058-2072).  "If the Thr of the new query is close to 0, Tacker directly launches all the
    kernels to the GPU".  Reading (direct_rule DIRECT_MIN_BE, the
    default): close to 0 = Thr <= max(direct_eps, the smallest predicted time of a ready BE head)
    at the query's first issue, i.e. not even the shortest ready BE kernel fits; DIRECT_EPS: Thr <=
    direct_eps only.  A direct query's kernels are all launched plain (no fusion, no reorder).
  * Eq. 8: for the current TC kernel (Ttc) and each ready BE head kernel (Tcd) with a
    fused prediction Tk_fuse: admissible iff Ttc + Tcd > Tk_fuse and Tk_fuse - Ttc < Thr.
    Pick the max Tgain = Tcd - (Tk_fuse - Ttc); ties -> lowest app index.
    Then Thr -= Tk_fuse - Ttc.
  * Reorder (literal, the default reorder_rule REORDER_UNFUSED): "If all the ready
    BE kernels may not be fused with the current kernel of Q", launch the ready BE heads (app
    index order) whose Ttmp < Thr, Thr -= Ttmp; after a fused launch nothing is reordered.
    REORDER_ALWAYS (B200 reading 6, a named option): reorder after every LC kernel,
    fused or not ("both adaptive kernel fusion and kernel reorder").
    REORDER_NEVER: BE work runs fused or on an idle GPU only.
  * Only the head kernel of each BE app is a candidate; the next kernel of an app
    becomes ready when the previous one completes.
  * Baymax mode = the same manager with fusion disabled ("static scheduling").
  * Idle GPU (no active LC query; the paper is silent): launch one ready BE head whose
    duration <= idle_cap, the apps taken round robin from the one after the last idle launch.
  * PTB slicing (B200 reading 13 in DESIGN.md §2; off by default): with slice_be, the BE part of
    a fused launch is a slice of n of the head kernel's N original blocks (PTB, Fig. 7), with
    predicted standalone time X_cd(n) = t_floor + t_block * n (the kernel's LR, §VI-C
    P:1839-1851); n is the smallest block count with X_cd(n) >= r * Ttc, r = the pair's opportune
    ratio (Fig. 10) or a fixed slice_ratio, clamped to [1, remaining]; a slice that
    would take every remaining block is the whole rest.  The head kernel stays the head until
    its last block is issued; reorder and idle launches issue the whole rest, whose predicted
    time is X_cd(remaining) once a slice of it has run.  BE work = n/N of the kernel's
    standalone time per slice.
  * Reverse fusion (NEXT-2; "LC and BE kernels are not limited to a specified type",
    P:924-926; DNN-training BE apps, Table II): when the LC kernel is a CUDA-core
    kernel (T_lc) and a ready BE head is a tensor-core kernel (T_be; kind 2 below), the same
    Eq. 8 applies with the roles of the two solo times exchanged in the predictor,
    Tk_fuse = fuse_pred(x_tc = T_be, x_cd = T_lc): admissible iff T_lc + T_be > Tk_fuse and
    Tk_fuse - T_lc < Thr; Tgain = T_be - (Tk_fuse - T_lc); Thr -= Tk_fuse - T_lc.  Tensor-core
    BE kernels are never sliced.

  * fuse_older (B200 reading 18 in DESIGN.md §2; off by default): an older query (not the
    newest) also fuses / reorders, spending at most min(its own Thr, Thr_j of every later active
    query j) with Thr_j = T_qos - (t - arrival_j) - sum of the remaining predicted time of j and
    of every active query ahead of j (Eq. 9 at time t); its own Thr is then reduced by what the
    decision spent.  Eq. 9 for a query at its first issue counts only the queries ahead of it.
    older_margin lowers that bound (a guard against prediction error on the GPU).

BE kernel kinds (first tuple element of an App kernel): 1 (True) = CUDA-core kernel (fusable with
an LC tensor-core kernel), 2 = tensor-core kernel (fusable with an LC CUDA-core kernel), 0 (False)
= never fused (reorder / idle only).
"""
from __future__ import annotations

import math

from dataclasses import dataclass, field

TACKER, BAYMAX = 0, 1
REORDER_UNFUSED, REORDER_ALWAYS, REORDER_NEVER = 0, 1, 2      # reorder_rule
DIRECT_MIN_BE, DIRECT_EPS = 0, 1                              # direct_rule
BE_OTHER, BE_CD, BE_TC = 0, 1, 2
FUSED, ORIGINAL_LC, REORDER_BE, IDLE_BE, NOTHING = 0, 1, 2, 3, 4


@dataclass
class Decision:
    action: int
    lc: tuple | None = None       # (query id, kernel index)
    fused_app: int = -1
    reorder: list = field(default_factory=list)   # app ids launched after the LC kernel
    thr: float = 0.0
    gain: float = 0.0
    blocks: int = -1              # BE blocks of the fused launch (PTB slice), -1 = whole rest
    reverse: bool = False         # fused: LC CUDA-core kernel + BE tensor-core kernel (NEXT-2)


def decide(ttc, lc_is_tc, thr, heads, policy, fuse_pred, allow=True, fuse_tcd=None, reorder_rule=REORDER_UNFUSED,
           reverse=True, with_reverse_flag=False):
    """Pure decision for one LC kernel.

    heads: list of (app, Tcd, be_kind) for READY BE head kernels, in app order (Tcd = the
    predicted time of what is left of the head kernel; be_kind as in the module doc).
    fuse_tcd(app) -> the BE time a fused launch would carry (a PTB slice; default Tcd).
    fuse_pred(app) -> Tk_fuse or None (for a reverse pair: the model at x_tc = the BE kernel,
    x_cd = the LC kernel).  Returns (fused_app, reorder_apps, thr, gain[, reversed])."""
    fused, gain_best, tf_best, rev = -1, None, None, False
    if allow and policy == TACKER and not lc_is_tc and reverse:
        for app, tbe, kind in heads:
            if kind != BE_TC:
                continue
            tf = fuse_pred(app)
            if tf is None:
                continue
            if ttc + tbe > tf and tf - ttc < thr:                   # Eq. 8, roles exchanged
                gain = tbe - (tf - ttc)
                if gain_best is None or gain > gain_best:
                    fused, gain_best, tf_best, rev = app, gain, tf, True
    if allow and policy == TACKER and lc_is_tc:
        for app, tcd, be_cd in heads:
            if be_cd != BE_CD:
                continue
            if fuse_tcd is not None:
                tcd = fuse_tcd(app)
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
    if allow and reorder_rule != REORDER_NEVER and not (reorder_rule == REORDER_UNFUSED and fused >= 0):
        for app, tcd, _ in heads:
            if app == fused:
                continue
            if tcd < thr:
                reorder.append(app)
                thr -= tcd
    if with_reverse_flag:
        return fused, reorder, thr, (gain_best or 0.0), rev
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
    kernels: list          # [(is_cd, T_pred[, N_blocks, t_block, t_floor])], cycled forever
    pos: int = 0
    ready_at: float = 0.0
    completed: int = 0
    done: int = 0          # blocks of the head kernel already issued (PTB slices)
    work: float = 0.0      # standalone-time of the BE work issued

    def head(self):
        return self.kernels[self.pos % len(self.kernels)]

    def lr(self):
        """(N, t_block, t_floor) of the head kernel; N = 0 when it has no slicing data (and for
        tensor-core kernels, which are never sliced)."""
        h = self.head()
        return (h[2], h[3], h[4]) if len(h) >= 5 and h[0] != BE_TC else (0, 0.0, 0.0)

    def rem(self):
        """Predicted standalone time of what is left of the head kernel."""
        N, a, b = self.lr()
        return self.head()[1] if self.done == 0 else b + a * (N - self.done)

    def issue(self, n):
        """n blocks of the head kernel issued (n < 0: the whole rest, completing it)."""
        N, _, _ = self.lr()
        T = self.head()[1]
        if n >= 0 and N > 1 and self.done + n < N:
            self.work += T * n / N
            self.done += n
            return
        self.work += T if self.done == 0 else T * (N - self.done) / N
        self.done = 0
        self.pos += 1
        self.completed += 1


def slice_blocks(app, ttc, r_opp, slice_be, slice_ratio):
    """Blocks of app's head kernel for a fused launch with a TC kernel of time ttc, or -1 for
    the whole rest (reading 13)."""
    N, a, b = app.lr()
    if not (slice_be and N > 1 and a > 0):
        return -1
    rt = slice_ratio if slice_ratio > 0 else r_opp
    if rt is None:
        return -1
    R = N - app.done
    n = max(1, min(math.ceil((rt * ttc - b) / a - 1e-9), R))
    return n if n < R else -1


def _round_robin(cands, rr):
    """Idle-GPU candidates [(app, T)] in round-robin order from app rr[0] (B200 reading, the paper is
    silent on an idle GPU: no BE app starves behind a lower-numbered one)."""
    return [c for c in cands if c[0] >= rr[0]] + [c for c in cands if c[0] < rr[0]]


def _first_issue(q, active, t, qos, heads, direct_eps, direct_rule, fuse_older):
    """Eq. 9 at the first issue of q and the direct rule."""
    q.issue = t
    if q is active[-1] or fuse_older:
        earlier = sum(o.remaining() for o in active[:active.index(q)])
        q.thr = qos - (t - q.arrival) - q.remaining() - earlier
        bound = direct_eps
        if direct_rule == DIRECT_MIN_BE and heads:
            bound = max(bound, min(d for _, d, _ in heads))
        q.direct = q.thr <= bound


def _lc_decision(q, active, t, qos, heads, apps, policy, pred, tcd_of, reorder_rule, reverse, fuse_older,
                 older_margin):
    """Eq. 8 / Tgain / reorder for the current kernel of q (the oldest query with work), with the
    older-query bound of reading 18.  pred(a) -> Tk_fuse or None.  Updates q.thr; returns
    (fused, reorder, thr_after, gain, rev, allow)."""
    newest = active[-1]
    is_tc, ttc = q.kernels[q.pos]
    allow = (q is newest or fuse_older) and not q.direct and q.thr is not None
    thr = q.thr if q.thr is not None else 0.0
    thr_in = thr
    if allow and q is not newest:
        ahead = 0.0
        for j, o in enumerate(active):
            ahead += o.remaining()
            if j > active.index(q):
                thr = min(thr, qos - (t - o.arrival) - ahead)
        thr -= older_margin
    thr_eff = thr
    fused, reorder, thr2, gain, rev = decide(
        ttc, is_tc, thr, heads, policy, pred, allow, fuse_tcd=tcd_of,
        reorder_rule=reorder_rule, reverse=reverse, with_reverse_flag=True)
    if allow:
        q.thr = thr_in - (thr_eff - thr2)
    return fused, reorder, (thr2 if allow else thr), gain, rev, allow


def simulate(queries, apps, qos, policy, fuse_pred, direct_eps=0.0, idle_cap=None, t_end=None,
             slice_be=False, slice_ratio=0.0, opp_ratio=None, reorder_rule=REORDER_UNFUSED, reverse=True,
             rfuse_pred=None, fuse_older=False, older_margin=0.0, direct_rule=DIRECT_MIN_BE):
    """Serial single-stream GPU whose kernels take exactly their predicted time.

    fuse_pred(lc_T, be_T) -> Tk_fuse or None; opp_ratio(app) -> the pair's opportune ratio or
    None (slicing); rfuse_pred(x_tc = BE tensor-core T, x_cd = LC CUDA-core T) -> Tk_fuse or None
    for reverse pairs (default fuse_pred).  The manager acts whenever the stream drains.
    Returns dict(latency per query, be_completed, be_work, timeline, decisions)."""
    t = 0.0
    active: list[Query] = []
    pending = sorted(queries, key=lambda q: q.arrival)
    timeline, decisions = [], []
    qi = 0
    rr = [0]   # idle launches: round robin over the apps
    while True:
        while qi < len(pending) and pending[qi].arrival <= t:
            active.append(pending[qi])
            qi += 1
        active = [q for q in active if q.pos < len(q.kernels)]
        if not active and qi >= len(pending):
            break
        if t_end is not None and t >= t_end:
            break
        heads = [(a, app.rem(), app.head()[0]) for a, app in enumerate(apps) if app.ready_at <= t]
        if active:
            q = active[0]
            if q.issue is None:
                _first_issue(q, active, t, qos, heads, direct_eps, direct_rule, fuse_older)
            is_tc, ttc = q.kernels[q.pos]
            nblk = {a: slice_blocks(apps[a], ttc, opp_ratio(a) if opp_ratio else None, slice_be, slice_ratio)
                    for a, _, _ in heads}

            def tcd_of(a):
                n = nblk[a]
                if n < 0:
                    return apps[a].rem()
                N, sa, sb = apps[a].lr()
                return sb + sa * n

            rpred = rfuse_pred or fuse_pred
            kind_of = {a: k for a, _, k in heads}

            def pred(a):
                if not is_tc and kind_of[a] == BE_TC:
                    return rpred(apps[a].rem(), ttc)
                return fuse_pred(ttc, tcd_of(a))

            fused, reorder, thr_after, gain, rev, allow = _lc_decision(
                q, active, t, qos, heads, apps, policy, pred, tcd_of, reorder_rule, reverse, fuse_older,
                older_margin)
            start = t
            if fused >= 0:
                dur = pred(fused)
                timeline.append(("fused", q.qid, q.pos, fused, start, start + dur))
                apps[fused].issue(-1 if rev else nblk[fused])
                apps[fused].ready_at = start + dur
                decisions.append(Decision(FUSED, (q.qid, q.pos), fused, list(reorder), q.thr, gain,
                                          -1 if rev else nblk[fused], rev))
            else:
                dur = ttc
                timeline.append(("lc", q.qid, q.pos, -1, start, start + dur))
                decisions.append(Decision(REORDER_BE if reorder else ORIGINAL_LC, (q.qid, q.pos), -1,
                                          list(reorder), thr_after))
            t = start + dur
            q.pos += 1
            if q.pos == len(q.kernels):
                q.done_at = t
            for a in reorder:
                d = apps[a].rem()
                timeline.append(("be", -1, -1, a, t, t + d))
                apps[a].issue(-1)
                t += d
                apps[a].ready_at = t
        else:
            nxt = pending[qi].arrival if qi < len(pending) else None
            cands = _round_robin([(a, d) for a, d, _ in heads if idle_cap is None or d <= idle_cap], rr)
            if cands:
                a, d = cands[0]
                rr[0] = a + 1
                timeline.append(("be", -1, -1, a, t, t + d))
                decisions.append(Decision(IDLE_BE, None, -1, [a], 0.0))
                apps[a].issue(-1)
                t += d
                apps[a].ready_at = t
            else:
                future = [app.ready_at for app in apps if app.ready_at > t]
                cand = [x for x in ([nxt] if nxt is not None else []) + future]
                if not cand:
                    break
                t = min(cand)
    lat = {q.qid: (q.done_at - q.arrival) for q in queries if q.done_at is not None}
    return dict(latency=lat, be_completed=[a.completed for a in apps], be_work=sum(a.work for a in apps),
                timeline=timeline, decisions=decisions, t=t)


def replay(trace, queries, apps, qos, policy, direct_eps=0.0, idle_cap=None, reorder_rule=REORDER_UNFUSED,
           reverse=True, fuse_older=False, older_margin=0.0, direct_rule=DIRECT_MIN_BE):
    """Trace-driven reference of a GPU-mode run ("the manager is gated by the
    discrete-event reference on the recorded trace").  On the GPU the clock, the set of active
    queries, which BE heads are ready and the online-refitted fused predictions come from the
    hardware, so they are taken as observations from each trace record: (t, active query ids
    oldest first, ready app ids, {app: Tk_fuse}).
    Everything the manager DECIDES -- Eq. 9 at first issue, the direct rule, Eq. 8 admission,
    max Tgain, Thr updates, reorder, the newest-query rule, idle launches -- is recomputed here
    with the rules above and the query / app state this function tracks itself.  (On the GPU every
    BE head is ready: the manager's single stream orders an app's kernels.)  Whole-kernel fusion
    only (no PTB slices).  Returns the list of Decisions (thr = the headroom after the decision as
    the manager reports it: the effective bound of an older query under reading 18)."""
    by_id = {q.qid: q for q in queries}
    out = []
    rr = [0]
    for rec in trace:
        t, act_ids, tf, ready = rec["t"], rec["active"], rec["tk_fuse"], set(rec["ready"])
        active = [by_id[i] for i in act_ids]
        heads = [(a, app.rem(), app.head()[0]) for a, app in enumerate(apps) if a in ready]
        work = [q for q in active if q.pos < len(q.kernels)]
        if not work:
            cands = [a for a, _ in _round_robin([(a, d) for a, d, _ in heads if idle_cap is None or d <= idle_cap],
                                                rr)] if not active else []
            a = cands[0] if cands else -1
            if a >= 0:
                rr[0] = a + 1
            out.append(Decision(IDLE_BE, None, -1, [a] if a >= 0 else [], 0.0))
            if a >= 0:
                apps[a].issue(-1)
            continue
        q = work[0]
        if q.issue is None:
            _first_issue(q, active, t, qos, heads, direct_eps, direct_rule, fuse_older)
        pred = lambda a: tf.get(a)
        fused, reorder, thr_after, gain, rev, allow = _lc_decision(
            q, active, t, qos, heads, apps, policy, pred, None, reorder_rule, reverse, fuse_older, older_margin)
        if fused >= 0:
            apps[fused].issue(-1)
            out.append(Decision(FUSED, (q.qid, q.pos), fused, list(reorder), thr_after, gain, -1, rev))
        else:
            out.append(Decision(REORDER_BE if reorder else ORIGINAL_LC, (q.qid, q.pos), -1, list(reorder),
                                thr_after))
        q.pos += 1
        for a in reorder:
            apps[a].issue(-1)
    return out
