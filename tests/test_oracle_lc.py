"""Pins for oracle/lc.py (c1 LC GEMM, c2 implicit-GEMM conv) against things other than
itself: identity / one-hot closed forms, brute-force loops, integer exactness, and torch's
CPU conv2d as a second opinion."""
import itertools

import numpy as np
import pytest
import torch

import synth
from oracle import lc
from oracle.metrics import max_rel_err


def brute_gemm(A, B):
    M, K = A.shape
    N = B.shape[0]
    D = [[0.0] * N for _ in range(M)]
    for i in range(M):
        for j in range(N):
            s = 0.0
            for k in range(K):
                s += float(A[i, k]) * float(B[j, k])
            D[i][j] = s
    return np.array(D)


def test_gemm_identity_returns_A():
    A, B = synth.lc_gemm_inputs(40, 64, 64, seed=1, variant="identity")
    D, _ = lc.lc_gemm(A, B)
    assert np.array_equal(D, A.astype(np.float64))


def test_gemm_onehot_selects_rows_of_B():
    A, B = synth.lc_gemm_inputs(24, 40, 32, seed=2, variant="onehot")
    D, _ = lc.lc_gemm(A, B)
    cols = A.argmax(axis=1)
    assert np.array_equal(D, B.astype(np.float64)[:, cols].T)


@pytest.mark.parametrize("M,N,K", [(8, 8, 8), (16, 24, 8), (24, 16, 40), (9, 13, 16)])
def test_gemm_bruteforce_integer_exact(M, N, K):
    A, B = synth.lc_gemm_inputs(M, N, K, seed=M * 100 + N, variant="int")
    D, S = lc.lc_gemm(A, B)
    assert np.array_equal(D, brute_gemm(A, B))
    assert np.all(S >= np.abs(D))


def test_gemm_transpose_convention():
    # D[i,j] pairs row i of A with row j of B (both K-major): a transposed-operand bug fails.
    A = np.array([[1, 2], [3, 4], [5, 6]], np.float16)
    B = np.array([[1, 0], [0, 1], [1, 1], [2, -1]], np.float16)
    D, _ = lc.lc_gemm(A, B)
    assert D.shape == (3, 4)
    assert np.array_equal(D, np.array([[1, 2, 3, 0], [3, 4, 7, 2], [5, 6, 11, 4]], np.float64))


def test_gemm_epilogue_bias_relu_residual():
    A = np.array([[1.0, -2.0]], np.float16)
    B = np.array([[1.0, 1.0], [0.0, 1.0]], np.float16)
    bias = np.array([0.5, 0.25], np.float32)
    res = np.array([[1.0, 10.0]])
    D, _ = lc.lc_gemm(A, B, bias=bias, relu=True, residual=res)
    # raw: [-1, -2] + bias -> [-0.5, -1.75] + res -> [0.5, 8.25] -> relu unchanged
    assert np.array_equal(D, np.array([[0.5, 8.25]]))
    D2, _ = lc.lc_gemm(A, B, bias=bias, relu=True)
    assert np.array_equal(D2, np.array([[0.0, 0.0]]))


def brute_conv(x, w, stride, pad):
    n, h, wd, c = x.shape
    k, r, s, _ = w.shape
    p = (h + 2 * pad - r) // stride + 1
    q = (wd + 2 * pad - s) // stride + 1
    out = np.zeros((n, p, q, k))
    for ni, pi, qi, ki in itertools.product(range(n), range(p), range(q), range(k)):
        acc = 0.0
        for ri, si, ci in itertools.product(range(r), range(s), range(c)):
            hh = pi * stride - pad + ri
            ww = qi * stride - pad + si
            if 0 <= hh < h and 0 <= ww < wd:
                acc += float(x[ni, hh, ww, ci]) * float(w[ki, ri, si, ci])
        out[ni, pi, qi, ki] = acc
    return out


@pytest.mark.parametrize("h,c,k,r,stride,pad", [(5, 3, 4, 3, 1, 1), (7, 2, 3, 3, 2, 1), (6, 4, 2, 1, 2, 0),
                                                (9, 2, 2, 7, 2, 3)])
def test_conv_bruteforce_integer(h, c, k, r, stride, pad):
    cs = synth.ConvShape("t", 1, h, h, c, k, r, r, stride, pad)
    x, w, _ = synth.conv_inputs(cs, seed=h + c, variant="int")
    out, _ = lc.lc_conv(x, w, stride, pad)
    assert np.array_equal(out, brute_conv(x, w, stride, pad))


def test_conv_1x1_equals_gemm():
    cs = synth.ConvShape("t", 2, 6, 5, 16, 24, 1, 1, 1, 0)
    x, w, _ = synth.conv_inputs(cs, seed=3)
    out, _ = lc.lc_conv(x, w, 1, 0)
    D, _ = lc.lc_gemm(x.reshape(-1, 16), w.reshape(24, 16))
    assert np.allclose(out.reshape(-1, 24), D, rtol=0, atol=1e-12)


def test_conv_delta_filter_copies_channel():
    cs = synth.ConvShape("t", 1, 8, 8, 5, 5, 3, 3, 1, 1)
    x, _, _ = synth.conv_inputs(cs, seed=4)
    w = np.zeros((5, 3, 3, 5), np.float16)
    for kk in range(5):
        w[kk, 1, 1, (kk + 2) % 5] = 1.0
    out, _ = lc.lc_conv(x, w, 1, 1)
    for kk in range(5):
        assert np.array_equal(out[..., kk], x[..., (kk + 2) % 5].astype(np.float64))


def test_conv_vs_torch_second_opinion():
    cs = synth.ConvShape("t", 1, 14, 14, 8, 16, 3, 3, 2, 1)
    x, w, b = synth.conv_inputs(cs, seed=5)
    out, S = lc.lc_conv(x, w, 2, 1, bias=b, relu=True)
    xt = torch.from_numpy(x.astype(np.float64)).permute(0, 3, 1, 2)
    wt = torch.from_numpy(w.astype(np.float64)).permute(0, 3, 1, 2)
    ref = torch.relu(torch.nn.functional.conv2d(xt, wt, torch.from_numpy(b.astype(np.float64)), stride=2, padding=1))
    ref = ref.permute(0, 2, 3, 1).numpy()
    assert max_rel_err(ref, out, S) < 1e-12


def test_conv_point_matches_full():
    cs = synth.ConvShape("t", 1, 9, 9, 4, 3, 3, 3, 2, 1)
    x, w, _ = synth.conv_inputs(cs, seed=6)
    out, S = lc.lc_conv(x, w, 2, 1)
    for (p, q, k) in [(0, 0, 0), (4, 4, 2), (2, 3, 1)]:
        v, a = lc.lc_conv_point(x, w, 2, 1, 0, p, q, k)
        assert abs(v - out[0, p, q, k]) < 1e-12 and abs(a - S[0, p, q, k]) < 1e-12


def test_resnet50_table():
    convs = synth.resnet50_convs(1)
    assert len(convs) == 53
    c1 = convs[0]
    gflop = (sum(c.flops for c in convs) - c1.flops + c1.flops * 3 // 8) / 1e9
    # ~4.09 GMAC of convolutions per ResNet-50 forward at 224x224 (conv1 with its real C=3)
    assert 8.1 < gflop < 8.25
    assert len(synth.vgg16_convs(1)) == 13


def test_im2col_times_filter_is_conv():
    cs = synth.ConvShape("t", 1, 11, 11, 8, 6, 7, 7, 2, 3)
    x, w, _ = synth.conv_inputs(cs, seed=8, variant="int")
    cols = lc.im2col(x, 7, 7, 2, 3, 400)
    assert cols.shape == (cs.p * cs.q, 400) and np.all(cols[:, 392:] == 0)
    wf = np.zeros((6, 400), np.float16)
    wf[:, :392] = w.reshape(6, -1)
    D, _ = lc.lc_gemm(cols, wf)
    assert np.array_equal(D.reshape(1, cs.p, cs.q, 6), brute_conv(x, w, 2, 3))
    # corner element: padding rows/cols of the window are zero
    assert np.all(cols[0, :3 * 7 * 8] == 0)
