"""Test helper: compare one kernel's GPU output with the float64 oracle on the
kernel's own GPU input (per-layer comparison, errors do
not compound).  Test infrastructure only."""
import numpy as np

from oracle import layers_ref as L


def np64(t):
    return None if t is None else t.detach().float().cpu().numpy().astype(np.float64)


def reference(layer):
    x = np64(layer.x)
    if layer.kind == "gemm":
        return L.gemm(x, np64(layer.w), np64(layer.shift), layer.act, np64(layer.res), np64(layer.scale))
    if layer.kind == "conv":
        g = layer.geom
        return L.conv2d_nhwc(x, np64(layer.w), np64(layer.scale), np64(layer.shift), g["stride"], g["pad"],
                             g.get("groups", 1), layer.act, np64(layer.res))
    if layer.kind == "pool":
        g = layer.geom
        f = L.maxpool_nhwc if g["mode"] == "max" else L.avgpool_nhwc
        return f(x, g["k"], g["stride"], g["pad"])
    if layer.kind == "gap":
        return L.global_avgpool_nhwc(x)
    if layer.kind == "im2col":
        g = layer.geom
        return im2col_ref(x, g["k"], g["stride"], g["pad"], g["Kpad"])
    if layer.kind == "eltwise":
        return L.bn_act_nhwc(x, np64(layer.scale), np64(layer.shift), layer.act)
    if layer.kind == "layernorm":
        return L.layernorm(x, np64(layer.scale), np64(layer.shift), layer.geom["eps"], np64(layer.res))
    if layer.kind == "attention":
        H, dh = layer.geom["heads"], layer.geom["dh"]
        Lq = x.shape[0]
        q = x[:, :H * dh].reshape(Lq, H, dh).transpose(1, 0, 2)
        k = x[:, H * dh:2 * H * dh].reshape(Lq, H, dh).transpose(1, 0, 2)
        v = x[:, 2 * H * dh:].reshape(Lq, H, dh).transpose(1, 0, 2)
        return L.sdpa(q, k, v).transpose(1, 0, 2).reshape(Lq, H * dh)
    if layer.kind == "embed":
        g = layer.geom
        ids = layer.x.detach().cpu().numpy()
        return L.embedding(ids, np64(layer.w), np64(g["pos"]), np64(g["typ"]), np64(layer.scale),
                           np64(layer.shift), g["eps"])
    raise ValueError(layer.kind)


def im2col_ref(x, k, stride, pad, kpad):
    """Plain im2col: row = output pixel (raster order), column = (r*k + s)*C + c,
    zero padding outside the image and beyond k*k*C."""
    N, H, W, C = x.shape
    OH, OW = (H + 2 * pad - k) // stride + 1, (W + 2 * pad - k) // stride + 1
    xp = np.zeros((N, H + 2 * pad, W + 2 * pad, C))
    xp[:, pad:pad + H, pad:pad + W, :] = x
    out = np.zeros((N * OH * OW, kpad))
    cols = []
    for r in range(k):
        for s in range(k):
            cols.append(xp[:, r:r + stride * (OH - 1) + 1:stride, s:s + stride * (OW - 1) + 1:stride, :])
    out[:, :k * k * C] = np.concatenate(cols, axis=-1).reshape(N * OH * OW, k * k * C)
    return out


def tolerance(dtype: str) -> float:
    # north star: max relative error 1e-2 (bf16 in / fp32 accumulate), 1e-4 (fp32)
    return 1e-2 if dtype == "bf16" else 1e-4


def check_layer(layer, dtype):
    ref = reference(layer)
    got = np64(layer.y).reshape(ref.shape)
    err = L.max_rel_err(got, ref)
    return err, tolerance(dtype)
