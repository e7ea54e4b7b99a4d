"""Float64 reference of the tenants' layers -- TEST INFRASTRUCTURE ONLY.

The paper writes no kernels of its own: its tenants are TVM/nnfusion inference
models and PyTorch jobs.  The build's tenants are the
configs' models (BASELINE.json configs); their layers follow
the torchvision / HF definitions, restated here as plain
float64 numpy.  Inputs are the GPU's own (bf16- or fp32-valued) tensors cast
to float64, so every comparison is per layer (errors do not compound).

Layouts: activations NHWC (or [tokens, features]); conv weights KRSC
([out, kh, kw, in/groups]); GEMM weights [N, K] (y = x W^T).

Common epilogue (reading R27 in DESIGN.md):
    y = act(acc * scale + shift + residual)
where scale/shift are the folded batch-norm (or scale = 1, shift = bias),
matching "conv3 -> BN -> + residual -> ReLU" (ResNet bottleneck) and
"act(XW^T + b)" (MLP).
"""
from __future__ import annotations

import numpy as np
from scipy.special import erf

F64 = np.float64


def act_ref(y: np.ndarray, act: str) -> np.ndarray:
    if act == "none":
        return y
    if act == "relu":
        return np.maximum(y, 0.0)
    if act == "relu6":
        return np.minimum(np.maximum(y, 0.0), 6.0)
    if act == "gelu":        # erf form (BERT)
        return 0.5 * y * (1.0 + erf(y / np.sqrt(2.0)))
    raise ValueError(act)


def epilogue(acc, scale=None, shift=None, residual=None, act="none"):
    y = np.asarray(acc, F64)
    if scale is not None:
        y = y * np.asarray(scale, F64)
    if shift is not None:
        y = y + np.asarray(shift, F64)
    if residual is not None:
        y = y + np.asarray(residual, F64)
    return act_ref(y, act)


def gemm(x, w, bias=None, act="none", residual=None, scale=None):
    """y[M,N] = act((x[M,K] @ w[N,K]^T) * scale + bias + residual)."""
    acc = np.asarray(x, F64) @ np.asarray(w, F64).T
    return epilogue(acc, scale, bias, residual, act)


def conv2d_nhwc(x, w, scale=None, shift=None, stride=1, pad=0, groups=1, act="none", residual=None):
    """2-D cross-correlation, NHWC input, KRSC weights (torch Conv2d semantics).

    y[n,oh,ow,k] = sum_{r,s,c} xpad[n, oh*stride + r, ow*stride + s, g(k)*Cg + c] * w[k,r,s,c]
    with zero padding ``pad`` on both spatial sides, then the common epilogue.
    Written as a sum over the R*S taps of (strided window) @ w[:, r, s, :]^T.
    """
    x = np.asarray(x, F64)
    w = np.asarray(w, F64)
    N, H, W, C = x.shape
    K, R, Sk, Cg = w.shape
    assert C == Cg * groups and K % groups == 0
    Kg = K // groups
    OH = (H + 2 * pad - R) // stride + 1
    OW = (W + 2 * pad - Sk) // stride + 1
    xp = np.zeros((N, H + 2 * pad, W + 2 * pad, C), F64)
    xp[:, pad:pad + H, pad:pad + W, :] = x
    y = np.zeros((N, OH, OW, K), F64)
    for gi in range(groups):
        xs = xp[..., gi * Cg:(gi + 1) * Cg]
        ws = w[gi * Kg:(gi + 1) * Kg]
        for r in range(R):
            for s in range(Sk):
                win = xs[:, r:r + stride * (OH - 1) + 1:stride, s:s + stride * (OW - 1) + 1:stride, :]
                y[..., gi * Kg:(gi + 1) * Kg] += win @ ws[:, r, s, :].T
    return epilogue(y, scale, shift, residual, act)


def maxpool_nhwc(x, k, stride, pad=0):
    """Max over k x k windows; padded positions are -inf (torch MaxPool2d)."""
    x = np.asarray(x, F64)
    N, H, W, C = x.shape
    OH = (H + 2 * pad - k) // stride + 1
    OW = (W + 2 * pad - k) // stride + 1
    xp = np.full((N, H + 2 * pad, W + 2 * pad, C), -np.inf)
    xp[:, pad:pad + H, pad:pad + W, :] = x
    y = np.full((N, OH, OW, C), -np.inf)
    for r in range(k):
        for s in range(k):
            y = np.maximum(y, xp[:, r:r + stride * (OH - 1) + 1:stride, s:s + stride * (OW - 1) + 1:stride, :])
    return y


def avgpool_nhwc(x, k, stride, pad=0):
    """Mean over k x k windows, count_include_pad=True (torch AvgPool2d default)."""
    x = np.asarray(x, F64)
    N, H, W, C = x.shape
    OH = (H + 2 * pad - k) // stride + 1
    OW = (W + 2 * pad - k) // stride + 1
    xp = np.zeros((N, H + 2 * pad, W + 2 * pad, C), F64)
    xp[:, pad:pad + H, pad:pad + W, :] = x
    y = np.zeros((N, OH, OW, C), F64)
    for r in range(k):
        for s in range(k):
            y += xp[:, r:r + stride * (OH - 1) + 1:stride, s:s + stride * (OW - 1) + 1:stride, :]
    return y / (k * k)


def global_avgpool_nhwc(x):
    """[N,H,W,C] -> [N,C] mean over H, W."""
    x = np.asarray(x, F64)
    return x.mean(axis=(1, 2))


def bn_act_nhwc(x, scale, shift, act="relu"):
    """Per-channel affine + activation (DenseNet pre-activation BN-ReLU)."""
    return epilogue(x, scale, shift, None, act)


def layernorm(x, gamma, beta, eps=1e-12, residual=None):
    """Row LayerNorm over the last dim (biased variance), after an optional
    residual add (BERT post-LN: LN(x + residual))."""
    x = np.asarray(x, F64)
    if residual is not None:
        x = x + np.asarray(residual, F64)
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps) * np.asarray(gamma, F64) + np.asarray(beta, F64)


def softmax(x, axis=-1):
    x = np.asarray(x, F64)
    z = x - x.max(axis=axis, keepdims=True)
    e = np.exp(z)
    return e / e.sum(axis=axis, keepdims=True)


def sdpa(q, k, v):
    """Scaled dot-product attention per head: softmax(q k^T / sqrt(dh)) v.
    q, k, v: [heads, L, dh]; all-ones mask."""
    q, k, v = (np.asarray(a, F64) for a in (q, k, v))
    dh = q.shape[-1]
    s = q @ np.swapaxes(k, -1, -2) / np.sqrt(float(dh))
    return softmax(s, -1) @ v


def embedding(ids, word, pos, typ, gamma, beta, eps=1e-12):
    """BERT embeddings: LN(word[ids] + pos[0:L] + type[0])."""
    ids = np.asarray(ids)
    L = ids.shape[0]
    x = np.asarray(word, F64)[ids] + np.asarray(pos, F64)[:L] + np.asarray(typ, F64)[0][None, :]
    return layernorm(x, gamma, beta, eps)


def max_rel_err(got, ref) -> float:
    """Reading R24: max_i |g_i - r_i| / max(|r_i|, rms(r))."""
    g = np.asarray(got, F64).ravel()
    r = np.asarray(ref, F64).ravel()
    if r.size == 0:
        return 0.0
    rms = float(np.sqrt(np.mean(r * r)))
    den = np.maximum(np.abs(r), rms if rms > 0 else 1e-300)
    return float(np.max(np.abs(g - r) / den))
