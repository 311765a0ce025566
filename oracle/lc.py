"""LC (tensor-core) work of the fused kernel, fp64 reference.  Test infrastructure only.

c1 — LC GEMM.  The paper's TC kernel Kt is "the Nvidia official GEMM implementation"
     (§III-B; refs [4],[11]).  Precision and layout are unstated -> reading
     (DESIGN.md §2): fp16 inputs, fp32 accumulate, K-major A [M,K] and B [N,K] ("TN"),
         D[i,j] = sum_k A[i,k] * B[j,k]
     plus an optional epilogue (bias, ReLU, residual) used by the DNN conv chains.
c2 — LC convolution as implicit GEMM (§VIII-H, P:3350-3381 converts convs to im2col+GEMM;
     the implicit form computes the same values):
         out[n,p,q,k] = sum_{c,r,s} x[n, p*st - pad + r, q*st - pad + s, c] * w[k,r,s,c]
     with x = 0 outside the image.  NHWC activations, KRSC filters.

Each function returns (exact fp64 value, absolute sum of the terms) for rel_err().
"""
from __future__ import annotations

import numpy as np


def lc_gemm(A, B, bias=None, relu=False, residual=None):
    """D = A . B^T (+ bias[j]) (+ residual[i,j]) then optional ReLU; fp64.

    A [M,K], B [N,K] (fp16 arrays are widened exactly).  A library matmul is one step.
    """
    A64 = np.asarray(A, np.float64)
    B64 = np.asarray(B, np.float64)
    D = A64 @ B64.T
    S = np.abs(A64) @ np.abs(B64).T
    if bias is not None:
        b = np.asarray(bias, np.float64)[None, :]
        D = D + b
        S = S + np.abs(b)
    if residual is not None:
        r = np.asarray(residual, np.float64)
        D = D + r
        S = S + np.abs(r)
    if relu:
        D = np.maximum(D, 0.0)
    return D, S


def lc_conv(x, w, stride: int, pad: int, bias=None, relu=False, residual=None):
    """Direct convolution, NHWC x [n,h,w,c], KRSC w [k,r,s,c] -> NHWC out [n,p,q,k], fp64.

    Written as the definition: zero-pad the image, then for each filter tap (r,s) add
    x_shifted[n,p,q,:] . w[k,r,s,:] (a library tensordot over c is one step).
    """
    x64 = np.asarray(x, np.float64)
    w64 = np.asarray(w, np.float64)
    n, h, wd, c = x64.shape
    k, r, s, c2 = w64.shape
    assert c == c2
    p = (h + 2 * pad - r) // stride + 1
    q = (wd + 2 * pad - s) // stride + 1
    xp = np.zeros((n, h + 2 * pad, wd + 2 * pad, c))
    xp[:, pad:pad + h, pad:pad + wd, :] = x64
    out = np.zeros((n, p, q, k))
    S = np.zeros((n, p, q, k))
    for rr in range(r):
        for ss in range(s):
            xs = xp[:, rr:rr + stride * (p - 1) + 1:stride, ss:ss + stride * (q - 1) + 1:stride, :]
            out += np.tensordot(xs, w64[:, rr, ss, :], axes=([3], [1]))
            S += np.tensordot(np.abs(xs), np.abs(w64[:, rr, ss, :]), axes=([3], [1]))
    if bias is not None:
        b = np.asarray(bias, np.float64)
        out = out + b
        S = S + np.abs(b)
    if residual is not None:
        rsd = np.asarray(residual, np.float64)
        out = out + rsd
        S = S + np.abs(rsd)
    if relu:
        out = np.maximum(out, 0.0)
    return out, S


def im2col(x, r, s, stride, pad, Kpad):
    """Explicit im2col of the paper's conv->GEMM lowering (cudnnIm2col, §VIII-H):
    out[m, kk] = x[n, p*st-pad+rr, q*st-pad+ss, c], m = (n*P+p)*Q+q, kk = (rr*S+ss)*C+c;
    0 outside the image and for kk >= R*S*C.  Exact copy (same dtype as x)."""
    n, h, wd, c = x.shape
    P = (h + 2 * pad - r) // stride + 1
    Q = (wd + 2 * pad - s) // stride + 1
    out = np.zeros((n * P * Q, Kpad), x.dtype)
    for ni in range(n):
        for pi in range(P):
            for qi in range(Q):
                m = (ni * P + pi) * Q + qi
                for rr in range(r):
                    hh = pi * stride - pad + rr
                    if hh < 0 or hh >= h:
                        continue
                    for ss in range(s):
                        ww = qi * stride - pad + ss
                        if ww < 0 or ww >= wd:
                            continue
                        out[m, (rr * s + ss) * c:(rr * s + ss + 1) * c] = x[ni, hh, ww, :]
    return out


def lc_conv_point(x, w, stride, pad, n, p, q, k):
    """One output element of lc_conv by explicit loops (for sampled full-size checks)."""
    _, h, wd, c = x.shape
    _, r, s, _ = w.shape
    acc = 0.0
    ab = 0.0
    for rr in range(r):
        hi = p * stride - pad + rr
        if hi < 0 or hi >= h:
            continue
        for ss in range(s):
            wi = q * stride - pad + ss
            if wi < 0 or wi >= wd:
                continue
            t = np.asarray(x[n, hi, wi, :], np.float64) * np.asarray(w[k, rr, ss, :], np.float64)
            acc += float(t.sum())
            ab += float(np.abs(t).sum())
    return acc, ab
