"""Tenant applications of the configs as kernel sequences (batch 1).

The paper's tenants are DNN inference applications that "invoke GPU functions
at the granularity of GPU kernels".  Each builder here
allocates the application's weights and activation buffers with PyTorch
(device memory only), appends one ``bl_op`` per fused kernel to the tenant's
sequence through the C ABI, and records a ``Layer`` per kernel so tests can
compare every kernel with the oracle on the kernel's own input tensor.

Synthetic values: weights N(0, 1/fan_in), folded-BN scale
U(0.5, 1.5) and shift N(0, 0.1), inputs N(0, 1), seeds 1000 + tenant index.
Layouts: activations NHWC, conv weights KRSC, GEMM weights [N, K].
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence

import os

import numpy as np
import torch

from synth import tensors as syn

from . import capi


@dataclass
class Layer:
    kind: str                      # "gemm" | "conv" | "pool" | "gap" | "eltwise"
    x: torch.Tensor
    y: torch.Tensor
    w: Optional[torch.Tensor] = None
    scale: Optional[torch.Tensor] = None
    shift: Optional[torch.Tensor] = None
    res: Optional[torch.Tensor] = None
    act: str = "none"
    geom: Dict[str, int] = field(default_factory=dict)
    name: str = ""


@dataclass
class TenantModel:
    name: str
    quota: float
    tenant: int
    dtype: str
    layers: List[Layer] = field(default_factory=list)
    keep: List[torch.Tensor] = field(default_factory=list)
    input: Optional[torch.Tensor] = None
    output: Optional[torch.Tensor] = None


class Builder:
    def __init__(self, ctx: capi.Ctx, tenant: int, name: str, quota: float, dtype: str, seed: int,
                 device: str = "cuda"):
        self.ctx, self.dev = ctx, device
        self.tdtype = torch.bfloat16 if dtype == "bf16" else torch.float32
        self.bl_dtype = capi.BL_BF16 if dtype == "bf16" else capi.BL_F32
        self.g = syn.rng(seed)
        self.m = TenantModel(name, quota, tenant, dtype)

    # tensors -------------------------------------------------------------
    def act_buf(self, shape) -> torch.Tensor:
        t = torch.empty(shape, dtype=self.tdtype, device=self.dev)
        self.m.keep.append(t)
        return t

    def param(self, arr: np.ndarray, fp32: bool = False) -> torch.Tensor:
        t = torch.from_numpy(np.ascontiguousarray(arr)).to(self.dev)
        t = t.float() if fp32 else t.to(self.tdtype)
        self.m.keep.append(t)
        return t

    def input(self, shape) -> torch.Tensor:
        x = self.param(syn.activation(self.g, shape))
        self.m.input = x
        return x

    def _op(self, kind, act, dims, ptrs) -> capi.bl_op:
        op = capi.bl_op()
        op.kind, op.dtype, op.act = kind, self.bl_dtype, capi.ACTS[act]
        for i, v in enumerate(dims):
            op.dims[i] = int(v)
        for i, t in enumerate(ptrs):
            op.ptr[i] = t.data_ptr() if t is not None else None
        return op

    # layers --------------------------------------------------------------
    def gemm(self, x: torch.Tensor, n_out: int, act="relu", bn=False, bias=True, res=None, name=""):
        M, K = x.shape
        w = self.param(syn.weight(self.g, (n_out, K), K))
        scale = self.param(syn.bn_scale(self.g, n_out), fp32=True) if bn else None
        shift = self.param(syn.bn_shift(self.g, n_out) if bn else syn.bias(self.g, n_out), fp32=True) \
            if (bn or bias) else None
        y = self.act_buf((M, n_out))
        op = self._op(capi.BL_OP_GEMM, act, [M, n_out, K, 0, 0, 0, 0], [x, w, scale, shift, res, y])
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("gemm", x, y, w, scale, shift, res, act, {}, name))
        return y

    def conv(self, x: torch.Tensor, k_out: int, k: int, stride=1, pad=None, act="relu", bn=True, bias=False,
             res=None, name="", out=None):
        """out: optional NHWC view of a wider buffer (DenseNet concat slice) to write into."""
        N, H, W, C = x.shape
        pad = k // 2 if pad is None else pad
        w_np = syn.weight(self.g, (k_out, k, k, C), k * k * C)
        scale = self.param(syn.bn_scale(self.g, k_out), fp32=True) if bn else None
        shift = self.param(syn.bn_shift(self.g, k_out) if bn else syn.bias(self.g, k_out), fp32=True) \
            if (bn or bias) else None
        OH, OW = (H + 2 * pad - k) // stride + 1, (W + 2 * pad - k) // stride + 1
        if C < 16 and self.bl_dtype == capi.BL_BF16:
            # first layers (C = 3): explicit im2col into a zero-padded [M, Kpad]
            # matrix, then the conv is a tensor-core GEMM
            K = k * k * C
            # K padding of the im2col matrix: 32 (B200: VGG conv1 im2col 10.0 -> 7.7 us
            # vs 64, profiles/round2/im2col_kalign/); BLESS_IM2COL_KALIGN for A/B
            ka = int(os.environ.get("BLESS_IM2COL_KALIGN", "32"))
            Kpad = (K + ka - 1) // ka * ka
            cols = self.act_buf((N * OH * OW, Kpad))
            op = self._op(capi.BL_OP_IM2COL, "none", [N, H, W, C, k, k, stride, pad, Kpad], [x, cols])
            self.ctx.append_kernel(self.m.tenant, op)
            self.m.layers.append(Layer("im2col", x, cols, act="none",
                                       geom=dict(k=k, stride=stride, pad=pad, Kpad=Kpad), name=name + ".im2col"))
            wp = np.zeros((k_out, Kpad), np.float32)
            wp[:, :K] = w_np.reshape(k_out, K)
            w = self.param(wp)
            y = self.act_buf((N, OH, OW, k_out))
            y2 = y.view(N * OH * OW, k_out)
            r2 = res.view(N * OH * OW, k_out) if res is not None else None
            op = self._op(capi.BL_OP_GEMM, act, [N * OH * OW, k_out, Kpad, 0, 0, 0, 0], [cols, w, scale, shift, r2, y2])
            self.ctx.append_kernel(self.m.tenant, op)
            self.m.layers.append(Layer("gemm", cols, y2, w, scale, shift, r2, act, {}, name))
            return y
        w = self.param(w_np)
        ldy = 0
        if out is not None:
            y, ldy = out, out.stride(2)
        else:
            y = self.act_buf((N, OH, OW, k_out))
        ldx = x.stride(2) if x.stride(2) != C else 0
        op = self._op(capi.BL_OP_CONV, act, [N, H, W, C, k_out, k, k, stride, pad, 1, ldx, ldy],
                      [x, w, scale, shift, res, y])
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("conv", x, y, w, scale, shift, res, act,
                                   dict(stride=stride, pad=pad, groups=1), name))
        return y

    def pool(self, x, k, stride, pad=0, mode="max", name="", out=None):
        """out: optional NHWC view of a wider buffer (channel slice) to write into."""
        N, H, W, C = x.shape
        ldy = 0
        if mode == "gap":
            y = self.act_buf((N, C))
            md = capi.BL_POOL_GLOBAL_AVG
        else:
            OH, OW = (H + 2 * pad - k) // stride + 1, (W + 2 * pad - k) // stride + 1
            if out is not None:
                y, ldy = out, out.stride(2)
            else:
                y = self.act_buf((N, OH, OW, C))
            md = capi.BL_POOL_MAX if mode == "max" else capi.BL_POOL_AVG
        op = self._op(capi.BL_OP_POOL, "none", [N, H, W, C, k, stride, pad, md, ldy], [x, y])
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("gap" if mode == "gap" else "pool", x, y, act="none",
                                   geom=dict(k=k, stride=stride, pad=pad, mode=mode), name=name))
        return y

    def dwconv(self, x, k, stride, act="relu6", name=""):
        """Depthwise k x k conv + folded BN + act (MobileNetV2), weights [C, k, k, 1]."""
        N, H, W, C = x.shape
        pad = k // 2
        w = self.param(syn.weight(self.g, (C, k, k, 1), k * k))
        scale = self.param(syn.bn_scale(self.g, C), fp32=True)
        shift = self.param(syn.bn_shift(self.g, C), fp32=True)
        OH, OW = (H + 2 * pad - k) // stride + 1, (W + 2 * pad - k) // stride + 1
        y = self.act_buf((N, OH, OW, C))
        op = self._op(capi.BL_OP_DWCONV, act, [N, H, W, C, k, k, stride, pad], [x, w, scale, shift, None, y])
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("conv", x, y, w, scale, shift, None, act,
                                   dict(stride=stride, pad=pad, groups=C), name))
        return y

    def bn_act(self, x2d, act="relu", out=None, name=""):
        """Per-channel folded BN + act on a [rows, C] (possibly strided) view."""
        rows, C = x2d.shape
        scale = self.param(syn.bn_scale(self.g, C), fp32=True)
        shift = self.param(syn.bn_shift(self.g, C), fp32=True)
        y = out if out is not None else self.act_buf((rows, C))
        op = self._op(capi.BL_OP_ELTWISE, act, [rows, C, x2d.stride(0), y.stride(0)], [x2d, scale, shift, None, y])
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("eltwise", x2d, y, None, scale, shift, None, act, {}, name))
        return y

    def layernorm(self, x, res=None, name=""):
        rows, C = x.shape
        gamma = self.param(syn.bn_scale(self.g, C), fp32=True)
        beta = self.param(syn.bn_shift(self.g, C), fp32=True)
        y = self.act_buf((rows, C))
        op = self._op(capi.BL_OP_LAYERNORM, "none", [rows, C, 0, 0], [x, gamma, beta, res, y])
        op.fparam[0] = 1e-12
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("layernorm", x, y, None, gamma, beta, res, "none", dict(eps=1e-12), name))
        return y

    def attention(self, qkv, heads, dh, name=""):
        L = qkv.shape[0]
        o = self.act_buf((L, heads * dh))
        op = self._op(capi.BL_OP_ATTENTION, "none", [L, heads, dh, 0, 0], [qkv, o])
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("attention", qkv, o, act="none", geom=dict(heads=heads, dh=dh), name=name))
        return o

    def embedding(self, L, C, vocab=30522, max_pos=512, name="embed"):
        ids = torch.from_numpy(syn.token_ids(self.g, L)).to(self.dev)
        self.m.keep.append(ids)
        self.m.input = ids
        word = self.param(0.02 * syn.activation(self.g, (vocab, C)))
        pos = self.param(0.02 * syn.activation(self.g, (max_pos, C)))
        typ = self.param(0.02 * syn.activation(self.g, (2, C)))
        gamma = self.param(syn.bn_scale(self.g, C), fp32=True)
        beta = self.param(syn.bn_shift(self.g, C), fp32=True)
        y = self.act_buf((L, C))
        op = self._op(capi.BL_OP_EMBED, "none", [L, C, vocab], [ids, word, pos, typ, gamma, beta, y])
        op.fparam[0] = 1e-12
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("embed", ids, y, word, gamma, beta, None, "none",
                                   dict(pos=pos, typ=typ, eps=1e-12), name))
        return y

    def done(self, y) -> TenantModel:
        self.m.output = y
        return self.m


# ---------------------------------------------------------------------------- C1
def tiny_mlp(ctx, tenant, quota, dtype="fp32", seed=1000) -> TenantModel:
    """C1 tenant 0: X 256x256, 3 x (W 256x256 + b, ReLU)."""
    b = Builder(ctx, tenant, "mlp", quota, dtype, seed)
    x = b.input((256, 256))
    for i in range(3):
        x = b.gemm(x, 256, act="relu", bias=True, name=f"fc{i}")
    return b.done(x)


def tiny_cnn(ctx, tenant, quota, dtype="fp32", seed=1001) -> TenantModel:
    """C1 tenant 1: NHWC 1x32x32x16, 2 x (conv3x3 p1 16->16 + b + ReLU)."""
    b = Builder(ctx, tenant, "cnn", quota, dtype, seed)
    x = b.input((1, 32, 32, 16))
    for i in range(2):
        x = b.conv(x, 16, 3, 1, 1, act="relu", bn=False, bias=True, name=f"conv{i}")
    return b.done(x)


# ---------------------------------------------------------------------------- C2
def vgg11(ctx, tenant, quota, dtype="bf16", seed=1000) -> TenantModel:
    """torchvision vgg11 (cfg A) at 224x224, batch 1: 8 conv3x3+bias+ReLU, 5
    max-pools, 3 FC.  Adaptive avg-pool is identity at 224 (7x7 -> 7x7) and
    dropout is identity at inference.  The FC1 weight is
    defined over the NHWC flatten order."""
    b = Builder(ctx, tenant, "vgg11", quota, dtype, seed)
    x = b.input((1, 224, 224, 3))
    cfg = [64, "M", 128, "M", 256, 256, "M", 512, 512, "M", 512, 512, "M"]
    i = 0
    for v in cfg:
        if v == "M":
            x = b.pool(x, 2, 2, 0, "max", name=f"pool{i}")
        else:
            x = b.conv(x, v, 3, 1, 1, act="relu", bn=False, bias=True, name=f"conv{i}")
            i += 1
    x = x.view(1, -1)
    x = b.gemm(x, 4096, act="relu", name="fc1")
    x = b.gemm(x, 4096, act="relu", name="fc2")
    x = b.gemm(x, 1000, act="none", name="fc3")
    return b.done(x)


def resnet(ctx, tenant, quota, depth=50, dtype="bf16", seed=1000) -> TenantModel:
    """torchvision ResNet-50/152 (v1.5: stride on the 3x3), batch 1, 224x224,
    BN folded into per-channel scale/shift.  Bottleneck epilogue order:
    conv3 -> BN -> + residual -> ReLU; the downsample branch is its own conv
    kernel."""
    blocks = {50: [3, 4, 6, 3], 101: [3, 4, 23, 3], 152: [3, 8, 36, 3]}[depth]
    b = Builder(ctx, tenant, f"resnet{depth}", quota, dtype, seed)
    x = b.input((1, 224, 224, 3))
    x = b.conv(x, 64, 7, 2, 3, act="relu", name="stem")
    x = b.pool(x, 3, 2, 1, "max", name="maxpool")
    cin = 64
    for li, (nb, width) in enumerate(zip(blocks, [64, 128, 256, 512])):
        for bi in range(nb):
            stride = 2 if (bi == 0 and li > 0) else 1
            identity = x
            if bi == 0:
                identity = b.conv(x, width * 4, 1, stride, 0, act="none", name=f"l{li}b{bi}down")
            h = b.conv(x, width, 1, 1, 0, act="relu", name=f"l{li}b{bi}c1")
            h = b.conv(h, width, 3, stride, 1, act="relu", name=f"l{li}b{bi}c2")
            x = b.conv(h, width * 4, 1, 1, 0, act="relu", res=identity, name=f"l{li}b{bi}c3")
            cin = width * 4
    x = b.pool(x, 0, 1, 0, "gap", name="avgpool")
    x = b.gemm(x, 1000, act="none", name="fc")
    del cin
    return b.done(x)


VGG_CFG = {
    "vgg11": [64, "M", 128, "M", 256, 256, "M", 512, 512, "M", 512, 512, "M"],
    "vgg16": [64, 64, "M", 128, 128, "M", 256, 256, 256, "M", 512, 512, 512, "M", 512, 512, 512, "M"],
}


def vgg(ctx, tenant, quota, name="vgg16", dtype="bf16", seed=1000) -> TenantModel:
    """torchvision VGG (cfg A = vgg11, D = vgg16), as vgg11() above."""
    b = Builder(ctx, tenant, name, quota, dtype, seed)
    x = b.input((1, 224, 224, 3))
    i = 0
    for v in VGG_CFG[name]:
        if v == "M":
            x = b.pool(x, 2, 2, 0, "max", name=f"pool{i}")
        else:
            x = b.conv(x, v, 3, 1, 1, act="relu", bn=False, bias=True, name=f"conv{i}")
            i += 1
    x = x.view(1, -1)
    x = b.gemm(x, 4096, act="relu", name="fc1")
    x = b.gemm(x, 4096, act="relu", name="fc2")
    x = b.gemm(x, 1000, act="none", name="fc3")
    return b.done(x)


def mobilenet_v2(ctx, tenant, quota, dtype="bf16", seed=1000) -> TenantModel:
    """torchvision MobileNetV2 (width 1.0), batch 1, 224x224: ReLU6 everywhere
    except the linear bottleneck projections; residual when stride 1 and
    in == out channels."""
    b = Builder(ctx, tenant, "mobilenet_v2", quota, dtype, seed)
    x = b.input((1, 224, 224, 3))
    x = b.conv(x, 32, 3, 2, 1, act="relu6", name="stem")
    cin = 32
    settings = [(1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2), (6, 96, 3, 1), (6, 160, 3, 2),
                (6, 320, 1, 1)]
    bi = 0
    for t, c, n, s in settings:
        for i in range(n):
            stride = s if i == 0 else 1
            h = x
            if t != 1:
                h = b.conv(h, cin * t, 1, 1, 0, act="relu6", name=f"b{bi}.expand")
            h = b.dwconv(h, 3, stride, act="relu6", name=f"b{bi}.dw")
            res = x if (stride == 1 and cin == c) else None
            x = b.conv(h, c, 1, 1, 0, act="none", res=res, name=f"b{bi}.project")
            cin = c
            bi += 1
    x = b.conv(x, 1280, 1, 1, 0, act="relu6", name="head")
    x = b.pool(x, 0, 1, 0, "gap", name="avgpool")
    x = b.gemm(x, 1000, act="none", name="classifier")
    return b.done(x)


def bert(ctx, tenant, quota, size="base", seq=128, dtype="bf16", seed=1000) -> TenantModel:
    """HF BertModel encoder (post-LN), batch 1, all-ones mask, erf-GELU,
    LayerNorm eps 1e-12; 7 kernels per layer:
    QKV GEMM, attention, output GEMM (+ residual), LN, FFN1 (GELU), FFN2
    (+ residual), LN; plus the embedding (gather + add + LN)."""
    layers, C, H = {"base": (12, 768, 12), "large": (24, 1024, 16)}[size]
    b = Builder(ctx, tenant, f"bert_{size}", quota, dtype, seed)
    x = b.embedding(seq, C)
    for li in range(layers):
        qkv = b.gemm(x, 3 * C, act="none", bias=True, name=f"l{li}.qkv")
        ctx_ = b.attention(qkv, H, C // H, name=f"l{li}.attn")
        a = b.gemm(ctx_, C, act="none", bias=True, res=x, name=f"l{li}.out")
        h1 = b.layernorm(a, name=f"l{li}.ln1")
        f = b.gemm(h1, 4 * C, act="gelu", bias=True, name=f"l{li}.ffn1")
        o = b.gemm(f, C, act="none", bias=True, res=h1, name=f"l{li}.ffn2")
        x = b.layernorm(o, name=f"l{li}.ln2")
    return b.done(x)


def densenet121(ctx, tenant, quota, dtype="bf16", seed=1000) -> TenantModel:
    """torchvision DenseNet-121 (growth 32, bn_size 4, blocks 6/12/24/16),
    batch 1, 224x224.  Each block owns one NHWC concat buffer; a dense layer is
    BN-ReLU on the first C_i channels (strided eltwise) -> 1x1 conv with BN-ReLU
    epilogue -> 3x3 conv writing its 32 channels into the buffer slice
    (SURVEY.md §8(c) C-4)."""
    b = Builder(ctx, tenant, "densenet121", quota, dtype, seed)
    x = b.input((1, 224, 224, 3))
    x = b.conv(x, 64, 7, 2, 3, act="relu", name="conv0")
    c = 64
    hw = 56
    blocks = [6, 12, 24, 16]
    buf = b.act_buf((1, hw, hw, c + blocks[0] * 32))
    b.pool(x, 3, 2, 1, "max", name="pool0", out=buf[..., :c])
    for bi, nl in enumerate(blocks):
        for li in range(nl):
            xin = buf.view(hw * hw, -1)[:, :c]          # first c channels of the concat buffer
            t = b.bn_act(xin, "relu", name=f"b{bi}l{li}.norm1")
            t = t.view(1, hw, hw, c)
            h = b.conv(t, 128, 1, 1, 0, act="relu", bn=True, name=f"b{bi}l{li}.conv1")   # + norm2 + relu2
            b.conv(h, 32, 3, 1, 1, act="none", bn=False, bias=False, name=f"b{bi}l{li}.conv2",
                   out=buf[..., c:c + 32])
            c += 32
        if bi < len(blocks) - 1:
            t = b.bn_act(buf.view(hw * hw, -1), "relu", name=f"trans{bi}.norm")
            t = b.conv(t.view(1, hw, hw, c), c // 2, 1, 1, 0, act="none", bn=False, bias=False,
                       name=f"trans{bi}.conv")
            c = c // 2
            hw //= 2
            buf = b.act_buf((1, hw, hw, c + blocks[bi + 1] * 32))
            b.pool(t, 2, 2, 0, "avg", name=f"trans{bi}.pool", out=buf[..., :c])
    t = b.bn_act(buf.view(hw * hw, -1), "relu", name="norm5")
    x = b.pool(t.view(1, hw, hw, c), 0, 1, 0, "gap", name="avgpool")
    x = b.gemm(x, 1000, act="none", name="classifier")
    return b.done(x)


BUILDERS = {
    "mlp": tiny_mlp,
    "cnn": tiny_cnn,
    "vgg11": vgg11,
    "vgg16": lambda ctx, t, q, dtype="bf16", seed=1000: vgg(ctx, t, q, "vgg16", dtype, seed),
    "resnet50": lambda ctx, t, q, dtype="bf16", seed=1000: resnet(ctx, t, q, 50, dtype, seed),
    "resnet152": lambda ctx, t, q, dtype="bf16", seed=1000: resnet(ctx, t, q, 152, dtype, seed),
    "mobilenet_v2": mobilenet_v2,
    "bert_base": lambda ctx, t, q, dtype="bf16", seed=1000: bert(ctx, t, q, "base", 128, dtype, seed),
    "bert_large": lambda ctx, t, q, dtype="bf16", seed=1000: bert(ctx, t, q, "large", 384, dtype, seed),
    "densenet121": densenet121,
}

CONFIGS = {
    "C1": [("mlp", 1 / 3), ("cnn", 2 / 3)],
    "C2": [("vgg11", 1 / 3), ("resnet50", 2 / 3)],
    "C3": [("resnet50", 0.4), ("vgg16", 0.3), ("bert_base", 0.2), ("mobilenet_v2", 0.1)],
    "C4": [("bert_large", 0.5), ("resnet152", 0.25), ("densenet121", 0.25)],
}


def build_config(ctx: capi.Ctx, cfg: str, dtype: str, quotas: Optional[Sequence[float]] = None,
                 device: Optional[int] = None) -> List[TenantModel]:
    """Register and build the tenants of a config; ``quotas`` overrides the
    config's quota per tenant (Table 2's two-model quota sets, L295).
    ``device``: CUDA device of the tenants' memory (default: the ctx's)."""
    dev = ctx.device if device is None else device
    if dev is not None and dev >= 0 and torch.cuda.is_available():
        with torch.cuda.device(dev):
            return _build_config(ctx, cfg, dtype, quotas)
    return _build_config(ctx, cfg, dtype, quotas)


def _build_config(ctx, cfg, dtype, quotas):
    models = []
    spec = CONFIGS[cfg]
    if quotas is not None:
        if len(quotas) != len(spec):
            raise ValueError(f"{cfg} has {len(spec)} tenants, got {len(quotas)} quotas")
        spec = [(name, float(q)) for (name, _), q in zip(spec, quotas)]
    for i, (name, q) in enumerate(spec):
        t = ctx.register_tenant(q, name)
        models.append(BUILDERS[name](ctx, t, q, dtype=dtype, seed=1000 + i))
    return models
