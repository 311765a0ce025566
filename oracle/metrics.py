"""Metrics and the parity error measure (test infrastructure only; see oracle/__init__.py).

* rel_err: DESIGN.md §2 reading of BASELINE's "max relative error": for an output with
  exact value r = sum_t x_t and absolute sum s = sum_t |x_t|,
      e = |g - r| / max(|r|, s, 1e-30)
  which equals plain relative error when all terms are non-negative and stays meaningful
  under cancellation.
* overlap_rate: Eq. 11 (§VIII-G).
* throughput_improvement: Eq. 10 (§VIII-C); the text says "processing time"
  but the formula is only positive for throughput -> reading: throughput.
"""
from __future__ import annotations

import numpy as np


def rel_err(got, ref, abssum=None) -> np.ndarray:
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    den = np.abs(ref)
    if abssum is not None:
        den = np.maximum(den, np.asarray(abssum, np.float64))
    den = np.maximum(den, 1e-30)
    return np.abs(got - ref) / den


def max_rel_err(got, ref, abssum=None) -> float:
    e = rel_err(got, ref, abssum)
    return float(e.max()) if e.size else 0.0


def overlap_rate(t_tc: float, t_cd: float, t_corun: float) -> float:
    """Eq. 11: (T_TC + T_CD - T_corun) / (T_TC + T_CD).  Range [0, 0.5] when the fused run
    is no faster than the longer component and no slower than the sequential sum."""
    return (t_tc + t_cd - t_corun) / (t_tc + t_cd)


def throughput_improvement(thpt_tacker: float, thpt_baymax: float) -> float:
    """Eq. 10 with throughputs: (Thpt_Tacker - Thpt_Baymax) / Thpt_Baymax."""
    return (thpt_tacker - thpt_baymax) / thpt_baymax
