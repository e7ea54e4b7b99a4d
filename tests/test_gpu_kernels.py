"""Per-kernel parity of the sm_100a tenant kernels with the float64 oracle
(bf16: max relative error <= 1e-2, fp32: <= 1e-4; reading R24), on shapes of
the configs' layers plus ragged and degenerate cases, run full-range and
SM-restricted through the C ABI."""
import numpy as np
import pytest
import torch

from tests.layer_check import check_layer

pytestmark = pytest.mark.gpu

from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi  # noqa: E402
from paper_conf_eurosys_zhangcc0xz0g25_b200.models import Builder  # noqa: E402


@pytest.fixture
def ctx():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)
    c = capi.Ctx(0)
    yield c
    c.close()


def one_layer(ctx, dtype, make):
    t = ctx.register_tenant(1.0, "k")
    b = Builder(ctx, t, "k", 1.0, dtype, seed=77)
    make(b)
    return b.m


def run_and_check(ctx, m, dtype, ranges=((0, 148), (5, 9))):
    errs = []
    for lo, hi in ranges:
        for k, layer in enumerate(m.layers):
            layer.y.fill_(float("nan"))
            ctx.run_kernel(m.tenant, k, lo, hi)
            err, tol = check_layer(layer, dtype)
            errs.append(err)
            assert err <= tol, (k, lo, hi, err, tol)
    return max(errs)


GEMMS = [(256, 256, 256, "relu"), (128, 2304, 768, "none"), (384, 1024, 1024, "gelu"), (200, 48, 72, "relu"),
         (17, 16, 16, "relu6"), (1000, 128, 64, "none"), (128, 768, 3072, "none")]


@pytest.mark.parametrize("M,N,K,act", GEMMS)
def test_tc_gemm(ctx, M, N, K, act):
    def mk(b):
        x = b.input((M, K))
        r = b.param(np.random.default_rng(1).standard_normal((M, N)).astype(np.float32)) if act == "none" else None
        b.gemm(x, N, act=act, bias=True, res=r)
    m = one_layer(ctx, "bf16", mk)
    run_and_check(ctx, m, "bf16")


@pytest.mark.parametrize("M,N,K,dtype", [(1, 4096, 25088, "bf16"), (1, 1000, 2048, "bf16"), (3, 100, 50, "bf16"),
                                         (2, 1000, 4096, "bf16"), (1, 37, 512, "bf16"), (8, 129, 96, "bf16"),
                                         (1, 4096, 4096, "fp32"), (8, 64, 1000, "fp32"),
                                         (1, 2050, 256, "bf16"), (2, 4100, 512, "bf16")])
def test_gemv(ctx, M, N, K, dtype):
    def mk(b):
        x = b.input((M, K))
        b.gemm(x, N, act="relu", bias=True)
    m = one_layer(ctx, dtype, mk)
    run_and_check(ctx, m, dtype)


@pytest.mark.parametrize("rows", ["1", "2", "4", "8"])
@pytest.mark.parametrize("M,N,K", [(1, 4096, 25088), (1, 1000, 2048), (3, 37, 4112), (8, 129, 96)])
def test_gemv_forced_rows(ctx, M, N, K, rows, monkeypatch):
    """Every GEMV tile height (rows of W per tile, stage = rows x 8192/rows k)
    is exact, including K tails shorter than a stage and N % rows != 0."""
    monkeypatch.setenv("BLESS_GEMV_ROWS", rows)

    def mk(b):
        b.gemm(b.input((M, K)), N, act="none", bias=True)
    m = one_layer(ctx, "bf16", mk)
    assert ctx.kernel_info(m.tenant, 0).family.decode() == "gemv_tma_bf16"
    run_and_check(ctx, m, "bf16")


CONVS = [  # H, W, C, K, k, stride, pad, act, residual
    (56, 56, 64, 64, 3, 1, 1, "relu", False),
    (56, 56, 64, 256, 1, 1, 0, "relu", True),
    (56, 56, 128, 128, 3, 2, 1, "relu", False),
    (56, 56, 256, 512, 1, 2, 0, "none", False),
    (14, 14, 256, 256, 3, 1, 1, "relu", False),
    (7, 7, 512, 2048, 1, 1, 0, "relu", True),
    (7, 7, 512, 512, 3, 1, 1, "relu", False),
    (32, 32, 16, 16, 3, 1, 1, "relu", False),
    (112, 112, 64, 128, 3, 1, 1, "relu", False),
    (10, 13, 32, 48, 3, 1, 1, "relu6", True),
    (224, 224, 3, 64, 3, 1, 1, "relu", False),   # C = 3 -> generic path
    (224, 224, 3, 64, 7, 2, 3, "relu", False),   # ResNet stem -> generic path
    (37, 37, 3, 24, 5, 2, 2, "relu", False),     # im2col: odd sizes, 5x5 stride 2, ragged pixel runs
    (17, 23, 4, 16, 3, 1, 1, "none", False),     # im2col: C = 4, non-square
    (224, 224, 64, 64, 3, 1, 1, "relu", False),  # VGG16 conv1_2: too wide for a halo tile (OW + 2 > 128)
]


@pytest.mark.parametrize("H,W,C,K,k,s,p,act,res", CONVS)
def test_conv_bf16(ctx, H, W, C, K, k, s, p, act, res):
    def mk(b):
        x = b.input((1, H, W, C))
        OH, OW = (H + 2 * p - k) // s + 1, (W + 2 * p - k) // s + 1
        r = b.param(np.random.default_rng(2).standard_normal((1, OH, OW, K)).astype(np.float32)) if res else None
        b.conv(x, K, k, s, p, act=act, bn=True, res=r)
    m = one_layer(ctx, "bf16", mk)
    run_and_check(ctx, m, "bf16")


@pytest.mark.parametrize("cfg", ["256,64,1", "256,32,3", "128,64,5", "64,32,2", "32,64,1", "128,128,1", "64,128,3"])
@pytest.mark.parametrize("shape", [("conv", (56, 56, 64, 256, 3, 1, 1)), ("conv", (28, 28, 128, 256, 3, 2, 1)),
                                   ("conv", (20, 27, 256, 96, 3, 1, 1)), ("conv", (9, 9, 192, 64, 1, 1, 0)),
                                   ("conv", (14, 14, 256, 512, 1, 1, 0)), ("gemm", (384, 1024, 320)),
                                   ("gemm", (200, 272, 136))])
def test_tc_forced_configs(ctx, cfg, shape, monkeypatch):
    """Every tile configuration the selector may pick (BN 32..256, BK 32/64,
    BK 128 = two 64-deep slabs per TMA box where C % 128 == 0 (3x3) or
    K % 64 == 0 (GEMM, 1x1; the K tail zero-filled), split-K) is exact on convs
    (stride 1/2, 1x1) and ragged GEMMs."""
    monkeypatch.setenv("BLESS_TC_CFG", cfg)
    kind, dims = shape

    def mk(b):
        if kind == "conv":
            H, W, C, K, k, s, p = dims
            x = b.input((1, H, W, C))
            OH, OW = (H + 2 * p - k) // s + 1, (W + 2 * p - k) // s + 1
            r = b.param(np.random.default_rng(2).standard_normal((1, OH, OW, K)).astype(np.float32))
            b.conv(x, K, k, s, p, act="relu", bn=True, res=r)
        else:
            M, N, K = dims
            b.gemm(b.input((M, K)), N, act="gelu", bias=True)
    m = one_layer(ctx, "bf16", mk)
    assert ctx.kernel_info(m.tenant, 0).family.decode().startswith("tc_")
    run_and_check(ctx, m, "bf16")


@pytest.mark.parametrize("cfg", ["64,64,1", "128,64,1", "128,64,3", "64,64,2"])
@pytest.mark.parametrize("shape", [("gemm", (384, 1024, 320)), ("gemm", (200, 272, 136)), ("gemm", (1000, 128, 64)),
                                   ("gemm", (128, 3072, 768)), ("conv", (14, 14, 256, 512, 1, 1, 0)),
                                   ("conv", (9, 9, 192, 64, 1, 1, 0))])
def test_tc_mt256(ctx, cfg, shape, monkeypatch):
    """M tiles of 256 rows (BLESS_TC_MT=256): one A box of 256 rows and two
    M = 128 tcgen05.mma per K step into two TMEM accumulators sharing the B
    tile; ragged M (384, 200, 81 pixels), K tails, split-K over 256-row tiles
    (workspace sub-tiles), residual + GELU/ReLU epilogue."""
    monkeypatch.setenv("BLESS_TC_MT", "256")
    monkeypatch.setenv("BLESS_TC_CFG", cfg)
    kind, dims = shape

    def mk(b):
        if kind == "conv":
            H, W, C, K, k, s_, p_ = dims
            x = b.input((1, H, W, C))
            r = b.param(np.random.default_rng(2).standard_normal((1, H, W, K)).astype(np.float32))
            b.conv(x, K, k, s_, p_, act="relu", bn=True, res=r)
        else:
            M, N, K = dims
            r = b.param(np.random.default_rng(2).standard_normal((M, N)).astype(np.float32))
            b.gemm(b.input((M, K)), N, act="gelu", bias=True, res=r)
    m = one_layer(ctx, "bf16", mk)
    assert ctx.kernel_info(m.tenant, 0).family.decode().startswith("tc_")
    run_and_check(ctx, m, "bf16")


@pytest.mark.parametrize("cfg", ["32,64,1", "64,64,1", "128,64,1", "64,64,3", "32,64,4"])
@pytest.mark.parametrize("dims", [(56, 56, 64, 256), (28, 28, 128, 256), (14, 14, 256, 256), (7, 7, 512, 512),
                                  (20, 27, 256, 96), (112, 112, 64, 128), (13, 11, 64, 48), (56, 56, 256, 64)])
@pytest.mark.parametrize("geom", ["tight", "pow2", "tight_na1"])
def test_tc_halo_conv(ctx, cfg, dims, geom, monkeypatch):
    """Halo implicit-GEMM 3x3 conv (mode 3): one TMA box of the tile's
    (BH + 2) x BW input halo per 64-channel chunk, each tap's A operand read
    from it at row offset r*BW + s.  Tile width BW = OW + 2 ("tight": BH*BW <
    128, rows past BH*BW masked in the epilogue, two halo stages where they
    fit) or the power-of-two width; one halo stage forced.  Exact vs the oracle
    for square, ragged and 112-wide maps, every BN, split-K over channel
    chunks, with residual + ReLU epilogue."""
    monkeypatch.setenv("BLESS_TC_HALO", "1")
    monkeypatch.setenv("BLESS_TC_CFG", cfg)
    if geom == "pow2":
        monkeypatch.setenv("BLESS_TC_HALO_POW2", "1")
    if geom == "tight_na1":
        monkeypatch.setenv("BLESS_TC_HALO_NA", "1")
    H, W, C, K = dims

    def mk(b):
        x = b.input((1, H, W, C))
        r = b.param(np.random.default_rng(2).standard_normal((1, H, W, K)).astype(np.float32))
        b.conv(x, K, 3, 1, 1, act="relu", bn=True, res=r)
    m = one_layer(ctx, "bf16", mk)
    assert ctx.kernel_info(m.tenant, 0).family.decode() == "tc_conv_bf16"
    run_and_check(ctx, m, "bf16")


@pytest.mark.parametrize("H,W,C,k,s,p,mode", [(112, 112, 64, 3, 2, 1, "max"), (224, 224, 64, 2, 2, 0, "max"),
                                              (9, 8, 5, 3, 2, 1, "avg"), (7, 7, 2048, 0, 1, 0, "gap")])
@pytest.mark.parametrize("dtype", ["bf16", "fp32"])
def test_pool(ctx, H, W, C, k, s, p, mode, dtype):
    def mk(b):
        x = b.input((1, H, W, C))
        b.pool(x, k, s, p, mode)
    m = one_layer(ctx, dtype, mk)
    run_and_check(ctx, m, dtype)


@pytest.mark.parametrize("L,H", [(128, 12), (384, 16), (256, 4), (96, 2)])
@pytest.mark.parametrize("path", ["tc", "simt"])
def test_attention(ctx, L, H, path, monkeypatch):
    """SDPA per head (all-ones mask): tcgen05 path for L % 128 == 0, L <= 384;
    CUDA-core path otherwise or when forced."""
    if path == "simt":
        monkeypatch.setenv("BLESS_ATTN_SIMT", "1")
    else:
        monkeypatch.delenv("BLESS_ATTN_SIMT", raising=False)

    def mk(b):
        qkv = b.input((L, 3 * H * 64))
        b.attention(qkv, H, 64)
    m = one_layer(ctx, "bf16", mk)
    fam = ctx.kernel_info(m.tenant, 0).family.decode()
    assert fam == ("attention_tc_bf16" if path == "tc" and L % 128 == 0 else "attention_bf16"), fam
    run_and_check(ctx, m, "bf16")


@pytest.mark.parametrize("rows,C,res", [(128, 768, False), (384, 1024, True), (7, 256, True)])
def test_layernorm(ctx, rows, C, res):
    def mk(b):
        x = b.input((rows, C))
        r = b.param(np.random.default_rng(3).standard_normal((rows, C)).astype(np.float32)) if res else None
        b.layernorm(x, res=r)
    m = one_layer(ctx, "bf16", mk)
    run_and_check(ctx, m, "bf16")


@pytest.mark.parametrize("H,C,stride", [(112, 32, 1), (56, 144, 2), (7, 960, 1)])
def test_dwconv(ctx, H, C, stride):
    def mk(b):
        x = b.input((1, H, H, C))
        b.dwconv(x, 3, stride)
    m = one_layer(ctx, "bf16", mk)
    run_and_check(ctx, m, "bf16")


def test_tc_kernel_uses_only_its_sms(ctx):
    """A tensor-core conv launched on logical SMs [40, 44) processes tiles
    only there (launch log mask), via the engine's STATIC policy."""
    c = capi.Ctx(0, policy="STATIC")
    t0 = c.register_tenant(0.03, "a")      # 148 * 0.03 = 4.44 -> 4 SMs
    b = Builder(c, t0, "a", 0.03, "bf16", seed=5)
    x = b.input((1, 56, 56, 64))
    b.conv(x, 64, 3, 1, 1)
    c.profile_tenant(t0, reps=2)
    c.start()
    base = capi.now_ns()
    for i in range(3):
        c.submit(t0, base + i)
    c.drain(int(20e9))
    c.stop()
    q, _, _ = c.tenant_info(t0)
    for r in c.launches():
        bits = [w * 32 + i for w in range(8) for i in range(32) if r.sm_mask[w] >> i & 1]
        assert bits and all(0 <= x < q for x in bits) and r.fallback == 0
    err, tol = check_layer(b.m.layers[0], "bf16")
    assert err <= tol
    c.close()
