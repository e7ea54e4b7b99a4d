"""Float64 forward passes of the configs' tenant models -- TEST INFRASTRUCTURE
ONLY (cpu_baseline and ``bench.py --impl reference``).

Architectures as torchvision defines them (VGG11 cfg A; ResNet v1.5 with the
stride on the 3x3 and BN folded to per-channel scale/shift) at batch 1,
224x224, NHWC; layer semantics from oracle/layers_ref.py.  Weights are drawn
from ``synth.tensors`` in the same order the product's model builder draws
them, so both sides see the same values (bf16 rounding aside).
"""
from __future__ import annotations

import numpy as np

from synth import tensors as syn

from . import layers_ref as L


class _Draw:
    def __init__(self, seed):
        self.g = syn.rng(seed)

    def conv(self, cin, cout, k, bn, bias):
        w = syn.weight(self.g, (cout, k, k, cin), k * k * cin).astype(np.float64)
        sc = syn.bn_scale(self.g, cout).astype(np.float64) if bn else None
        sh = (syn.bn_shift(self.g, cout) if bn else syn.bias(self.g, cout)).astype(np.float64) if (bn or bias) else None
        return w, sc, sh

    def fc(self, cin, cout):
        w = syn.weight(self.g, (cout, cin), cin).astype(np.float64)
        b = syn.bias(self.g, cout).astype(np.float64)
        return w, b


def mlp_forward(seed=1000):
    d = _Draw(seed)
    x = syn.activation(d.g, (256, 256)).astype(np.float64)
    for _ in range(3):
        w, b = d.fc(256, 256)
        x = L.gemm(x, w, b, "relu")
    return x


def cnn_forward(seed=1001):
    d = _Draw(seed)
    x = syn.activation(d.g, (1, 32, 32, 16)).astype(np.float64)
    for _ in range(2):
        w, _, b = d.conv(16, 16, 3, bn=False, bias=True)
        x = L.conv2d_nhwc(x, w, None, b, 1, 1, 1, "relu")
    return x


def vgg11_forward(seed=1000):
    d = _Draw(seed)
    x = syn.activation(d.g, (1, 224, 224, 3)).astype(np.float64)
    cin = 3
    for v in [64, "M", 128, "M", 256, 256, "M", 512, 512, "M", 512, 512, "M"]:
        if v == "M":
            x = L.maxpool_nhwc(x, 2, 2, 0)
        else:
            w, _, b = d.conv(cin, v, 3, bn=False, bias=True)
            x = L.conv2d_nhwc(x, w, None, b, 1, 1, 1, "relu")
            cin = v
    x = x.reshape(1, -1)
    for n, act in [(4096, "relu"), (4096, "relu"), (1000, "none")]:
        w, b = d.fc(x.shape[1], n)
        x = L.gemm(x, w, b, act)
    return x


def resnet_forward(depth=50, seed=1000):
    blocks = {50: [3, 4, 6, 3], 101: [3, 4, 23, 3], 152: [3, 8, 36, 3]}[depth]
    d = _Draw(seed)
    x = syn.activation(d.g, (1, 224, 224, 3)).astype(np.float64)
    w, sc, sh = d.conv(3, 64, 7, bn=True, bias=False)
    x = L.conv2d_nhwc(x, w, sc, sh, 2, 3, 1, "relu")
    x = L.maxpool_nhwc(x, 3, 2, 1)
    cin = 64
    for li, (nb, width) in enumerate(zip(blocks, [64, 128, 256, 512])):
        for bi in range(nb):
            stride = 2 if (bi == 0 and li > 0) else 1
            identity = x
            if bi == 0:
                w, sc, sh = d.conv(cin, width * 4, 1, True, False)
                identity = L.conv2d_nhwc(x, w, sc, sh, stride, 0, 1, "none")
            w, sc, sh = d.conv(cin, width, 1, True, False)
            h = L.conv2d_nhwc(x, w, sc, sh, 1, 0, 1, "relu")
            w, sc, sh = d.conv(width, width, 3, True, False)
            h = L.conv2d_nhwc(h, w, sc, sh, stride, 1, 1, "relu")
            w, sc, sh = d.conv(width, width * 4, 1, True, False)
            x = L.conv2d_nhwc(h, w, sc, sh, 1, 0, 1, "relu", residual=identity)
            cin = width * 4
    x = L.global_avgpool_nhwc(x)
    w, b = d.fc(2048, 1000)
    return L.gemm(x, w, b, "none")


def vgg_forward(cfg, seed=1000):
    d = _Draw(seed)
    x = syn.activation(d.g, (1, 224, 224, 3)).astype(np.float64)
    cin = 3
    for v in cfg:
        if v == "M":
            x = L.maxpool_nhwc(x, 2, 2, 0)
        else:
            w, _, b = d.conv(cin, v, 3, bn=False, bias=True)
            x = L.conv2d_nhwc(x, w, None, b, 1, 1, 1, "relu")
            cin = v
    x = x.reshape(1, -1)
    for n, act in [(4096, "relu"), (4096, "relu"), (1000, "none")]:
        w, b = d.fc(x.shape[1], n)
        x = L.gemm(x, w, b, act)
    return x


def _dw(d, C, k):
    w = syn.weight(d.g, (C, k, k, 1), k * k).astype(np.float64)
    return w, syn.bn_scale(d.g, C).astype(np.float64), syn.bn_shift(d.g, C).astype(np.float64)


def _affine(d, C):
    return syn.bn_scale(d.g, C).astype(np.float64), syn.bn_shift(d.g, C).astype(np.float64)


def mobilenet_v2_forward(seed=1000):
    d = _Draw(seed)
    x = syn.activation(d.g, (1, 224, 224, 3)).astype(np.float64)
    w, sc, sh = d.conv(3, 32, 3, True, False)
    x = L.conv2d_nhwc(x, w, sc, sh, 2, 1, 1, "relu6")
    cin = 32
    for t, c, n, s in [(1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2), (6, 96, 3, 1), (6, 160, 3, 2),
                       (6, 320, 1, 1)]:
        for i in range(n):
            stride = s if i == 0 else 1
            h = x
            if t != 1:
                w, sc, sh = d.conv(cin, cin * t, 1, True, False)
                h = L.conv2d_nhwc(h, w, sc, sh, 1, 0, 1, "relu6")
            C = h.shape[-1]
            w, sc, sh = _dw(d, C, 3)
            h = L.conv2d_nhwc(h, w, sc, sh, stride, 1, C, "relu6")
            w, sc, sh = d.conv(C, c, 1, True, False)
            res = x if (stride == 1 and cin == c) else None
            x = L.conv2d_nhwc(h, w, sc, sh, 1, 0, 1, "none", residual=res)
            cin = c
    w, sc, sh = d.conv(320, 1280, 1, True, False)
    x = L.conv2d_nhwc(x, w, sc, sh, 1, 0, 1, "relu6")
    x = L.global_avgpool_nhwc(x)
    w, b = d.fc(1280, 1000)
    return L.gemm(x, w, b, "none")


def bert_forward(size="base", seq=128, seed=1000):
    layers, C, H = {"base": (12, 768, 12), "large": (24, 1024, 16)}[size]
    d = _Draw(seed)
    ids = syn.token_ids(d.g, seq)
    word = 0.02 * syn.activation(d.g, (30522, C)).astype(np.float64)
    pos = 0.02 * syn.activation(d.g, (512, C)).astype(np.float64)
    typ = 0.02 * syn.activation(d.g, (2, C)).astype(np.float64)
    gm, bt = _affine(d, C)
    x = L.embedding(ids, word, pos, typ, gm, bt)
    dh = C // H
    for _ in range(layers):
        w, b = d.fc(C, 3 * C)
        qkv = L.gemm(x, w, b, "none")
        q, k, v = (qkv[:, i * C:(i + 1) * C].reshape(seq, H, dh).transpose(1, 0, 2) for i in range(3))
        ctx = L.sdpa(q, k, v).transpose(1, 0, 2).reshape(seq, C)
        w, b = d.fc(C, C)
        a = L.gemm(ctx, w, b, "none", residual=x)
        gm, bt = _affine(d, C)
        h1 = L.layernorm(a, gm, bt)
        w, b = d.fc(C, 4 * C)
        f = L.gemm(h1, w, b, "gelu")
        w, b = d.fc(4 * C, C)
        o = L.gemm(f, w, b, "none", residual=h1)
        gm, bt = _affine(d, C)
        x = L.layernorm(o, gm, bt)
    return x


def densenet121_forward(seed=1000):
    d = _Draw(seed)
    x = syn.activation(d.g, (1, 224, 224, 3)).astype(np.float64)
    w, sc, sh = d.conv(3, 64, 7, True, False)
    x = L.conv2d_nhwc(x, w, sc, sh, 2, 3, 1, "relu")
    feats = L.maxpool_nhwc(x, 3, 2, 1)
    for bi, nl in enumerate([6, 12, 24, 16]):
        for _ in range(nl):
            C = feats.shape[-1]
            sc, sh = _affine(d, C)
            t = L.bn_act_nhwc(feats, sc, sh, "relu")
            w, sc, sh = d.conv(C, 128, 1, True, False)
            h = L.conv2d_nhwc(t, w, sc, sh, 1, 0, 1, "relu")
            w, _, _ = d.conv(128, 32, 3, False, False)
            feats = np.concatenate([feats, L.conv2d_nhwc(h, w, None, None, 1, 1, 1, "none")], axis=-1)
        if bi < 3:
            C = feats.shape[-1]
            sc, sh = _affine(d, C)
            t = L.bn_act_nhwc(feats, sc, sh, "relu")
            w, _, _ = d.conv(C, C // 2, 1, False, False)
            feats = L.avgpool_nhwc(L.conv2d_nhwc(t, w, None, None, 1, 0, 1, "none"), 2, 2, 0)
    sc, sh = _affine(d, feats.shape[-1])
    x = L.global_avgpool_nhwc(L.bn_act_nhwc(feats, sc, sh, "relu"))
    w, b = d.fc(1024, 1000)
    return L.gemm(x, w, b, "none")


FORWARD = {
    "mlp": lambda seed: mlp_forward(seed),
    "cnn": lambda seed: cnn_forward(seed),
    "vgg11": lambda seed: vgg11_forward(seed),
    "resnet50": lambda seed: resnet_forward(50, seed),
    "resnet152": lambda seed: resnet_forward(152, seed),
    "vgg16": lambda seed: vgg_forward([64, 64, "M", 128, 128, "M", 256, 256, 256, "M", 512, 512, 512, "M",
                                       512, 512, 512, "M"], seed),
    "mobilenet_v2": lambda seed: mobilenet_v2_forward(seed),
    "bert_base": lambda seed: bert_forward("base", 128, seed),
    "bert_large": lambda seed: bert_forward("large", 384, seed),
    "densenet121": lambda seed: densenet121_forward(seed),
}
