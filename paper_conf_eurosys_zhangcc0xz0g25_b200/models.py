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
from typing import Dict, List, Optional

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
             res=None, name=""):
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
            Kpad = (K + 63) // 64 * 64
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
        y = self.act_buf((N, OH, OW, k_out))
        op = self._op(capi.BL_OP_CONV, act, [N, H, W, C, k_out, k, k, stride, pad, 1, 0, 0],
                      [x, w, scale, shift, res, y])
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("conv", x, y, w, scale, shift, res, act,
                                   dict(stride=stride, pad=pad, groups=1), name))
        return y

    def pool(self, x, k, stride, pad=0, mode="max", name=""):
        N, H, W, C = x.shape
        if mode == "gap":
            y = self.act_buf((N, C))
            md = capi.BL_POOL_GLOBAL_AVG
        else:
            OH, OW = (H + 2 * pad - k) // stride + 1, (W + 2 * pad - k) // stride + 1
            y = self.act_buf((N, OH, OW, C))
            md = capi.BL_POOL_MAX if mode == "max" else capi.BL_POOL_AVG
        op = self._op(capi.BL_OP_POOL, "none", [N, H, W, C, k, stride, pad, md], [x, y])
        self.ctx.append_kernel(self.m.tenant, op)
        self.m.layers.append(Layer("gap" if mode == "gap" else "pool", x, y, act="none",
                                   geom=dict(k=k, stride=stride, pad=pad, mode=mode), name=name))
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


BUILDERS = {
    "mlp": tiny_mlp,
    "cnn": tiny_cnn,
    "vgg11": vgg11,
    "resnet50": lambda ctx, t, q, dtype="bf16", seed=1000: resnet(ctx, t, q, 50, dtype, seed),
    "resnet152": lambda ctx, t, q, dtype="bf16", seed=1000: resnet(ctx, t, q, 152, dtype, seed),
}

CONFIGS = {
    "C1": [("mlp", 1 / 3), ("cnn", 2 / 3)],
    "C2": [("vgg11", 1 / 3), ("resnet50", 2 / 3)],
}


def build_config(ctx: capi.Ctx, cfg: str, dtype: str) -> List[TenantModel]:
    models = []
    for i, (name, q) in enumerate(CONFIGS[cfg]):
        t = ctx.register_tenant(q, name)
        models.append(BUILDERS[name](ctx, t, q, dtype=dtype, seed=1000 + i))
    return models
