"""Duration predictor reference (§VI).  Test infrastructure only.

a9 / c13 — per-kernel LR (§VI-C): duration = a * blocks + b, blocks = the
           number of blocks in non-PTB mode (here: original BE blocks, or LC tiles), fitted
           by ordinary least squares from "a few points".
a10 / c14 — two-stage fused model (§VI-A/B, Eqs. 1-6):
           load ratio r = X_ori_cd / X_ori_tc (Eq. 1).  With X_tc fixed the fused duration is
           piecewise linear in r with an inflection at the opportune ratio (Fig. 10,
           P:1411-1447), and at fixed r it is linear in X_tc (Fig. 11).
           Reading (Eq. 6 is garbled): normalise by X_tc,
               tau(r) = T_fuse / X_tc = max(l1(r), l2(r)),  l_s(r) = a_s + b_s * r,
           each stage fitted by its own LR from samples at r in {0.1, 0.2}
           (stage 1) and {1.8, 1.9} (stage 2); the opportune ratio is the
           intersection r* = (a2 - a1) / (b1 - b2).
           Online update: when |pred - meas| / meas > 10 %, add the sample to
           the stage it falls in and refit.
"""
from __future__ import annotations

TRAIN_RATIOS = (0.1, 0.2, 1.8, 1.9)
REFIT_THRESHOLD = 0.10


def ols(xs, ys):
    """Closed-form least squares y = a*x + b. One distinct x -> slope 0 through the mean."""
    n = len(xs)
    if n == 0:
        raise ValueError("no samples")
    mx = sum(xs) / n
    my = sum(ys) / n
    sxx = sum((x - mx) ** 2 for x in xs)
    sxy = sum((x - mx) * (y - my) for x, y in zip(xs, ys))
    if sxx == 0.0:
        return 0.0, my
    a = sxy / sxx
    return a, my - a * mx


class KernelLR:
    """Per-kernel model X = a * blocks + b."""

    def __init__(self):
        self.xs, self.ys = [], []
        self.a = self.b = None

    def add(self, blocks, ms):
        self.xs.append(float(blocks))
        self.ys.append(float(ms))

    def fit(self):
        self.a, self.b = ols(self.xs, self.ys)
        return self.a, self.b

    def predict(self, blocks):
        return self.a * blocks + self.b


class TwoStage:
    """tau(r) = max(a1 + b1 r, a2 + b2 r); T_fuse = X_tc * tau(X_cd / X_tc)."""

    def __init__(self):
        self.samples = []  # (r, tau)
        self.l1 = self.l2 = None

    def add(self, x_tc, x_cd, t_fused):
        self.samples.append((x_cd / x_tc, t_fused / x_tc))

    def fit(self, split=None, iters=16):
        """split=None: the lower half of the samples (by r) starts as stage 1 (for the training
        ratios {0.1, 0.2, 1.8, 1.9}: {0.1, 0.2} vs {1.8, 1.9}); a split leaving one side empty
        falls back to that median split."""
        pts = sorted(self.samples)
        if len(pts) < 2:
            raise ValueError("need at least 2 samples")
        lo = [p for p in pts if split is not None and p[0] <= split]
        hi = [p for p in pts if split is not None and p[0] > split]
        if not lo or not hi:
            lo, hi = pts[:len(pts) // 2], pts[len(pts) // 2:]
        for _ in range(iters):
            b1, a1 = ols([p[0] for p in lo], [p[1] for p in lo])
            b2, a2 = ols([p[0] for p in hi], [p[1] for p in hi])
            self.l1, self.l2 = (a1, b1), (a2, b2)
            rs = self.inflection()
            if rs is None:
                break
            nlo = [p for p in pts if p[0] <= rs]
            nhi = [p for p in pts if p[0] > rs]
            # each stage is a line through >= 2 samples (one LR per stage): a re-split
            # leaving a stage one sample would fix no slope (OLS slope 0, a flat stage)
            if len(nlo) < 2 or len(nhi) < 2 or (nlo == lo and nhi == hi):
                break
            lo, hi = nlo, nhi
        if self.l1[1] >= self.l2[1]:
            # DESIGN.md reading 5: the two stages of Fig. 10 are co-run (slope below the CD-solo
            # stage's) then CD solo; fitted slopes in the other order describe no such
            # curve (max() would put the steeper first stage at large r), so one LR over all samples
            b, a = ols([p[0] for p in pts], [p[1] for p in pts])
            self.l1 = self.l2 = (a, b)
        return self.l1, self.l2

    def inflection(self):
        (a1, b1), (a2, b2) = self.l1, self.l2
        if b1 == b2:
            return None
        return (a2 - a1) / (b1 - b2)

    def tau(self, r):
        (a1, b1), (a2, b2) = self.l1, self.l2
        return max(a1 + b1 * r, a2 + b2 * r)

    def predict(self, x_tc, x_cd):
        return x_tc * self.tau(x_cd / x_tc)

    def observe(self, x_tc, x_cd, t_meas):
        """Online refit rule: returns True if the model was refitted."""
        pred = self.predict(x_tc, x_cd)
        if abs(pred - t_meas) / t_meas > REFIT_THRESHOLD:
            self.add(x_tc, x_cd, t_meas)
            rs = self.inflection()
            self.fit(split=rs if rs is not None and rs > 0 else None)
            return True
        return False
