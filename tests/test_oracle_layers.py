"""Pins for the float64 layer oracle (oracle/layers_ref.py).

Checked against: brute-force scalar loops on tiny inputs (the textbook
definitions), an independent library (torch CPU float64 functional ops), closed
forms (identity / delta kernels, 1x1 conv == GEMM, LayerNorm moments) and the
published GELU values.
"""
import math

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from oracle import layers_ref as L

R = np.random.default_rng(0)


def _t(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.float64))


def brute_conv(x, w, stride, pad, groups):
    N, H, W, C = x.shape
    K, Rr, Ss, Cg = w.shape
    OH = (H + 2 * pad - Rr) // stride + 1
    OW = (W + 2 * pad - Ss) // stride + 1
    Kg = K // groups
    y = np.zeros((N, OH, OW, K))
    for n in range(N):
        for oh in range(OH):
            for ow in range(OW):
                for k in range(K):
                    gi = k // Kg
                    acc = 0.0
                    for r in range(Rr):
                        for s in range(Ss):
                            ih, iw = oh * stride - pad + r, ow * stride - pad + s
                            if 0 <= ih < H and 0 <= iw < W:
                                for c in range(Cg):
                                    acc += x[n, ih, iw, gi * Cg + c] * w[k, r, s, c]
                    y[n, oh, ow, k] = acc
    return y


@pytest.mark.parametrize("k,stride,pad,groups", [(3, 1, 1, 1), (3, 2, 1, 1), (1, 2, 0, 1), (7, 2, 3, 1), (3, 1, 1, 4)])
def test_conv_bruteforce(k, stride, pad, groups):
    x = R.standard_normal((1, 7, 6, 4))
    w = R.standard_normal((4, k, k, 4 // groups))
    got = L.conv2d_nhwc(x, w, stride=stride, pad=pad, groups=groups)
    assert np.allclose(got, brute_conv(x, w, stride, pad, groups), rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("k,stride,pad,groups", [(3, 1, 1, 1), (3, 2, 1, 1), (1, 1, 0, 1), (7, 2, 3, 1), (3, 1, 1, 16)])
def test_conv_vs_torch(k, stride, pad, groups):
    x = R.standard_normal((2, 12, 11, 16))
    w = R.standard_normal((32, k, k, 16 // groups))
    sc, sh = R.uniform(0.5, 1.5, 32), R.standard_normal(32)
    res = None
    ref = F.conv2d(_t(x).permute(0, 3, 1, 2), _t(w).permute(0, 3, 1, 2), stride=stride, padding=pad, groups=groups)
    ref = ref.permute(0, 2, 3, 1).numpy() * sc + sh
    res = R.standard_normal(ref.shape)
    got = L.conv2d_nhwc(x, w, sc, sh, stride, pad, groups, act="relu", residual=res)
    assert np.allclose(got, np.maximum(ref + res, 0), rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("k,stride,pad", [(3, 1, 1), (7, 2, 3)])
def test_im2col_ref_times_weights_is_conv(k, stride, pad):
    """The test-side im2col (tests/layer_check.py) pinned to the conv
    definition: im2col(x) @ w.reshape(K, -1)^T == conv2d(x, w)."""
    from tests.layer_check import im2col_ref
    x = R.standard_normal((1, 11, 9, 3))
    w = R.standard_normal((5, k, k, 3))
    cols = im2col_ref(x, k, stride, pad, 3 * k * k + 5)
    assert np.all(cols[:, 3 * k * k:] == 0)
    got = cols[:, :3 * k * k] @ w.reshape(5, -1).T
    ref = L.conv2d_nhwc(x, w, stride=stride, pad=pad).reshape(-1, 5)
    assert np.allclose(got, ref, rtol=1e-12, atol=1e-12)


def test_conv_delta_kernel_is_identity():
    x = R.standard_normal((1, 5, 5, 3))
    w = np.zeros((3, 3, 3, 3))
    for c in range(3):
        w[c, 1, 1, c] = 1.0
    assert np.array_equal(L.conv2d_nhwc(x, w, pad=1), x)


def test_conv1x1_equals_gemm():
    x = R.standard_normal((1, 4, 5, 8))
    w = R.standard_normal((6, 1, 1, 8))
    b = R.standard_normal(6)
    y = L.conv2d_nhwc(x, w, None, b, act="relu")
    g = L.gemm(x.reshape(-1, 8), w.reshape(6, 8), b, act="relu")
    assert np.allclose(y.reshape(-1, 6), g, rtol=1e-13, atol=1e-13)


def test_gemm_bruteforce_and_epilogue_order():
    x, w, b, r = R.standard_normal((3, 5)), R.standard_normal((4, 5)), R.standard_normal(4), R.standard_normal((3, 4))
    y = L.gemm(x, w, b, act="relu", residual=r)
    for i in range(3):
        for j in range(4):
            acc = sum(x[i, k] * w[j, k] for k in range(5)) + b[j] + r[i, j]
            assert math.isclose(y[i, j], max(acc, 0.0), rel_tol=1e-12, abs_tol=1e-12)


def test_activations_closed_forms():
    v = np.array([-7.0, -1.0, 0.0, 0.5, 3.0, 6.0, 9.0])
    assert np.array_equal(L.act_ref(v, "relu"), [0, 0, 0, 0.5, 3, 6, 9])
    assert np.array_equal(L.act_ref(v, "relu6"), [0, 0, 0, 0.5, 3, 6, 6])
    # GELU(x) = x * Phi(x): Phi(1) = 0.841344746..., Phi(-1) = 0.158655254...
    g = L.act_ref(np.array([1.0, -1.0, 0.0]), "gelu")
    assert np.allclose(g, [0.8413447460685429, -0.15865525393145707, 0.0], rtol=1e-14)
    assert np.allclose(L.act_ref(v, "gelu"), F.gelu(_t(v)).numpy(), rtol=1e-12, atol=1e-15)


@pytest.mark.parametrize("k,s,p", [(2, 2, 0), (3, 2, 1)])
def test_pools_vs_torch(k, s, p):
    x = R.standard_normal((1, 9, 8, 5))
    xt = _t(x).permute(0, 3, 1, 2)
    mx = F.max_pool2d(xt, k, s, p).permute(0, 2, 3, 1).numpy()
    av = F.avg_pool2d(xt, k, s, p).permute(0, 2, 3, 1).numpy()
    assert np.array_equal(L.maxpool_nhwc(x, k, s, p), mx)
    assert np.allclose(L.avgpool_nhwc(x, k, s, p), av, rtol=1e-13, atol=1e-14)
    assert np.allclose(L.global_avgpool_nhwc(x), x.mean(axis=(1, 2)))


def test_layernorm_moments_and_torch():
    x, res = R.standard_normal((6, 32)) * 3 + 1, R.standard_normal((6, 32))
    ones, zeros = np.ones(32), np.zeros(32)
    y = L.layernorm(x, ones, zeros, 1e-12, residual=res)
    assert np.allclose(y.mean(-1), 0, atol=1e-12)
    assert np.allclose((y ** 2).mean(-1), 1, atol=1e-9)
    gm, bt = R.standard_normal(32), R.standard_normal(32)
    ref = F.layer_norm(_t(x + res), (32,), _t(gm), _t(bt), 1e-12).numpy()
    assert np.allclose(L.layernorm(x, gm, bt, 1e-12, residual=res), ref, rtol=1e-11, atol=1e-12)


def test_sdpa_and_softmax():
    q, k, v = (R.standard_normal((2, 7, 8)) for _ in range(3))
    ref = F.scaled_dot_product_attention(_t(q), _t(k), _t(v)).numpy()
    assert np.allclose(L.sdpa(q, k, v), ref, rtol=1e-11, atol=1e-12)
    s = L.softmax(R.standard_normal((3, 5)))
    assert np.allclose(s.sum(-1), 1.0)
    # uniform scores -> uniform attention -> output = mean of v
    assert np.allclose(L.sdpa(np.zeros((1, 4, 8)), k[:1, :4], v[:1, :4]), np.broadcast_to(v[:1, :4].mean(1, keepdims=True), (1, 4, 8)))


def test_embedding():
    word, pos, typ = R.standard_normal((50, 16)), R.standard_normal((10, 16)), R.standard_normal((2, 16))
    ids = np.array([3, 7, 7, 0])
    gm, bt = np.ones(16), np.zeros(16)
    y = L.embedding(ids, word, pos, typ, gm, bt)
    raw = np.stack([word[i] + pos[p] + typ[0] for p, i in enumerate(ids)])
    assert np.allclose(y, L.layernorm(raw, gm, bt))


def test_max_rel_err_definition():
    ref = np.array([1.0, -2.0, 1e-9, 0.0])
    rms = math.sqrt((1 + 4 + 1e-18) / 4)
    got = ref + np.array([0.01, 0.0, 0.001, 0.0])
    assert math.isclose(L.max_rel_err(got, ref), max(0.01 / max(1.0, rms), 0.001 / rms))
