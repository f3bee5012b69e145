"""T3/T4 on the GPU: each catalog kernel on small single-layer graphs (several
tiles, ragged tails, every epilogue / split-K / operand-layout path) against the
oracle, through the C ABI; identity / delta filters bit-exact; reused-kernel
output bitwise equal to a dedicated stand-alone launch of the same kernel."""
import math

import numpy as np
import pytest
import torch

from oracle import ops as O
from paper_conf_dac_huangdxz25_b200 import pask as P
from workloads.models import _Builder, bf16_round, make_input

from .gpu_harness import TOL, rel_err, run_model, teacher_forced_errors

pytestmark = pytest.mark.gpu


def _check_spec(spec, seed=0, solutions=None):
    x = make_input(spec, seed)
    dm, ctx, plan = run_model(spec, x, solutions=solutions)
    errs = teacher_forced_errors(dm, spec, x)
    ctx.close()
    bad = [e for e in errs if not e[2] <= TOL]
    assert not bad, errs
    return dm, plan


def conv_spec(c, k, hw, r, stride=1, pad=0, dil=1, act="relu", res=False, groups=1, seed=3,
              hw2=None):
    b = _Builder("conv", seed)
    x = b.input((1, c, hw, hw2 or hw), "f32")
    t = b.layout(x, c_pad=max(8, (c + 7) // 8 * 8))
    rr = None
    if res:
        # residual of the right shape from a preceding 1x1 conv
        tmp = b.conv(t, k, r, stride, pad, dil, groups=1, act="none")
        rr = tmp
    y = b.conv(t, k, r, stride, pad, dil, groups=groups, act=act, res=rr)
    b.outputs = [y]
    return b.spec()


CONV_CASES = [
    # (C, K, HW, R, stride, pad, dil, act, res)   comment
    (8, 16, 32, 3, 1, 1, 1, "relu", False),        # bn 16, 8 M tiles
    (16, 32, 17, 3, 2, 1, 1, "relu6", False),      # bn 32, ragged M, stride 2
    (8, 48, 23, 7, 2, 3, 1, "none", False),        # bn 48, 7x7 s2 p3 (stem-like)
    (64, 64, 14, 3, 1, 2, 2, "relu", False),       # dilation 2
    (64, 256, 56, 1, 1, 0, 1, "relu", True),       # 1x1 TMA A path, residual TMA
    (256, 128, 28, 1, 2, 0, 1, "none", False),     # 1x1 stride 2 -> TMA im2col path
    (512, 512, 7, 3, 1, 1, 1, "relu", True),       # M = 49, cluster split-K 8
    (1024, 256, 14, 1, 1, 0, 1, "relu", False),    # split-K 2..8 on a 1x1
    (128, 1000, 9, 3, 1, 1, 1, "gelu", True),      # N tail 1000 % 64, GELU epilogue
    (40, 24, 19, 5, 1, 2, 1, "tanh", False),       # C % 64 != 0 taps, tanh epilogue
    (24, 64, 15, 3, 2, 1, 2, "relu", True),        # narrow-C gather, dilation + stride, residual
    (96, 64, 10, 3, 1, 1, 1, "relu6", False),      # C = 1.5 x 64 chunks: gather
]


@pytest.mark.parametrize("case", CONV_CASES, ids=[str(c) for c in CONV_CASES])
def test_conv_cases(case):
    c, k, hw, r, s, p, d, act, res = case
    _check_spec(conv_spec(c, k, hw, r, s, p, d, act, res))


_GATHER_CHILD = r"""
import sys
sys.path.insert(0, sys.argv[1])
from tests.test_gpu_kernels import CONV_CASES, _check_spec, conv_spec
for i in (0, 2, 3, 9, 10):
    _check_spec(conv_spec(*CONV_CASES[i]))
print("gather ok")
"""


def test_conv_gather_fallback():
    """The cp.async implicit-im2col gather, forced for every non-plain conv with
    PASK_NO_IM2COL (the 64-channel TMA im2col cases then take it too).  The
    runtime reads its switches once per process (tuning.h), so the cases run in
    a child process started with the switch set."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", _GATHER_CHILD, root], env={**os.environ, "PASK_NO_IM2COL": "1"},
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0 and "gather ok" in r.stdout, r.stderr[-3000:]


# Stem fold (D16): convs fed by the layout node over few channels are
# re-expressed as R2 x 1 convs over a 64-channel regrouped input (TMA im2col).
# (C, K, H, W, R, stride, pad, batch, act, res)
# (the fold needs W % 4 == 0: 16 B input loads)
STEM_FOLD_CASES = [
    (3, 64, 37, 36, 7, 2, 3, 1, "relu", False),    # ResNet-50 stem geometry, odd H, ragged M
    (3, 48, 29, 44, 7, 2, 3, 1, "none", True),     # non-square, N tail, residual (two folded-input convs)
    (4, 32, 20, 20, 5, 2, 2, 1, "relu6", False),   # R = 5 not a multiple of the stride
    (2, 16, 40, 32, 5, 3, 2, 1, "relu", False),    # stride 3: three rows per folded row
    (3, 64, 224, 224, 7, 2, 3, 2, "relu", False),  # the stem at batch 2: persistent tiles
]


@pytest.mark.parametrize("case", STEM_FOLD_CASES, ids=[str(c) for c in STEM_FOLD_CASES])
def test_stem_fold(case):
    c, k, h, w, r, st, pd, n, act, res = case
    b = _Builder("fold", 12)
    x = b.input((n, c, h, w), "f32")
    t = b.layout(x)
    rr = b.conv(t, k, r, st, pd, act="none") if res else None
    y = b.conv(t, k, r, st, pd, act=act, res=rr)
    b.outputs = [y]
    spec = b.spec()
    from paper_conf_dac_huangdxz25_b200.model import DeviceModel
    assert DeviceModel(spec, alloc=False).ws_bytes > 0, "fold not taken"
    xin = make_input(spec, 0)
    dm, ctx, _ = run_model(spec, xin)
    errs = teacher_forced_errors(dm, spec, xin)
    ctx.close()
    assert all(e <= TOL for _, _, e in errs), errs
    # the workspace holds exactly the folded input and regrouped weights of the
    # first conv reading the layout output (D16), restated from the
    # formula in tests/stem_fold_ref.py: bit-exact (bf16 copies, zeros)
    from .stem_fold_ref import fold_geometry, fold_input, fold_weights

    def bits(a):
        return (np.asarray(a, np.float64).astype(np.float32).view(np.uint32) >> 16).astype(np.uint16)

    conv = next(L for L in spec["layers"] if L["op"] == "conv")
    _, q, r2, t_rows = fold_geometry(h, w, c, r, r, (st, st), (pd, pd))
    ws = dm.ws.cpu().numpy()
    ybytes = n * t_rows * q * 64 * 2
    y_ws = ws[:ybytes].view(np.uint16).reshape(n, t_rows, q, 64)
    y_exp = bits(fold_input(O.bf16_rne(np.asarray(xin, np.float64)), r, r, (st, st), (pd, pd)).transpose(0, 2, 3, 1))
    np.testing.assert_array_equal(y_ws, y_exp)
    woff = (ybytes + 255) // 256 * 256
    w_ws = ws[woff:woff + k * r2 * 64 * 2].view(np.uint16).reshape(k, r2, 64)
    w_exp = bits(fold_weights(np.asarray(conv["w"], np.float64), (st, st))[..., 0].transpose(0, 2, 1))
    np.testing.assert_array_equal(w_ws, w_exp)


_NOFOLD_CHILD = r"""
import sys
sys.path.insert(0, sys.argv[1])
from tests.test_gpu_kernels import STEM_FOLD_CASES, _check_spec
from tests.gpu_harness import TOL, run_model, teacher_forced_errors
from workloads import build_model
from paper_conf_dac_huangdxz25_b200.model import DeviceModel
spec, x = build_model("resnet50")
assert DeviceModel(spec, alloc=False).ws_bytes == 0
dm, ctx, plan = run_model(spec, x)
errs = teacher_forced_errors(dm, spec, x)
ctx.close()
assert max(e for _, _, e in errs) <= TOL, errs
print("nofold ok")
"""


def test_resnet50_stem_unfolded():
    """PASK_STEM_FOLD=0: ResNet-50 with its stem on the cp.async gather path."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", _NOFOLD_CHILD, root], env={**os.environ, "PASK_STEM_FOLD": "0"},
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0 and "nofold ok" in r.stdout, r.stderr[-3000:]


@pytest.mark.parametrize("s,hw", [(1, 56), (2, 56), (1, 7), (2, 15)])
def test_depthwise(s, hw):
    for c in (32, 144, 960):
        _check_spec(conv_spec(c, c, hw, 3, s, 1, 1, "relu6", False, groups=c))


def test_conv_delta_filter_bit_exact():
    """3x3 delta filter (w[k,k,1,1] = 1), pad 1, no bias: output == input bits."""
    b = _Builder("delta", 5)
    x = b.input((1, 64, 20, 20), "f32")
    t = b.layout(x)
    y = b.conv(t, 64, 3, 1, 1, act="none", bias=False)
    spec = b.spec()
    w = np.zeros((64, 64, 3, 3), np.float32)
    for i in range(64):
        w[i, i, 1, 1] = 1.0
    spec["layers"][1]["w"] = w
    b.outputs = [y]
    xin = make_input(spec, 1)
    dm, ctx, _ = run_model(spec, xin)
    np.testing.assert_array_equal(dm.read_raw(y), dm.read_raw(t))
    ctx.close()


def test_conv_1x1_identity_bit_exact():
    b = _Builder("eye", 5)
    x = b.input((1, 128, 9, 11), "f32")
    t = b.layout(x)
    y = b.conv(t, 128, 1, 1, 0, act="none", bias=False)
    spec = b.spec()
    spec["layers"][1]["w"] = np.eye(128, dtype=np.float32)[:, :, None, None]
    b.outputs = [y]
    dm, ctx, _ = run_model(spec, make_input(spec, 2))
    np.testing.assert_array_equal(dm.read_raw(y), dm.read_raw(t))
    ctx.close()


def linear_spec(m, kin, nout, act="none", res=False, rows=None, seed=4):
    b = _Builder("lin", seed)
    x = b.input((m, kin), "bf16")
    rr = b.linear(x, nout, act="none") if res else None
    y = b.linear(x, nout, act=act, res=rr, rows=rows)
    b.outputs = [y]
    return b.spec()


@pytest.mark.parametrize("m,kin,nout,act,res,rows", [
    (1, 2048, 1000, "none", False, None),   # FC GEMV shape, N tail
    (1, 16384, 10, "none", False, None),    # unaligned N = 10 (direct-store path)
    (128, 768, 2304, "none", False, None),  # QKV
    (128, 3072, 768, "none", True, None),   # FFN2 + residual, split-K
    (128, 768, 3072, "gelu", False, None),  # FFN1 + GELU
    (128, 768, 768, "tanh", False, 1),      # pooler: first row only
    (200, 96, 40, "relu", True, None),      # ragged M, bn 48
    (8, 8192, 64, "relu", True, None),      # 16-CTA split-K cluster (M <= 64, 128 k-blocks),
                                            # N % 16 == 0: direct epilogue with residual, rows_per 8
    (64, 16384, 32, "none", True, None),    # 16-way split, a full 64-row A box, residual
])
def test_linear_cases(m, kin, nout, act, res, rows):
    spec = linear_spec(m, kin, nout, act, res, rows)
    _check_spec(spec)
    if m <= 8:   # s* there is the GEMV solution (D12): also run the tcgen05 GEMM on it
        _check_spec(spec, solutions={i: P.K_GEMM for i in range(len(spec["layers"]))})


@pytest.mark.parametrize("m,kin,nout,act,res,rows", [
    (1, 2048, 1000, "none", False, None),   # ResNet-50 FC: 4 columns per CTA, 2 K slices
    (1, 1280, 1000, "none", False, None),   # MobileNetV2 FC
    (1, 16384, 10, "none", False, None),    # tiny CNN FC: 10 CTAs of 32 warps, 32 K slices
    (128, 768, 768, "tanh", False, 1),      # BERT pooler (rows = 1)
    (8, 512, 33, "gelu", True, None),       # 8 rows, N tail, GELU, residual
    (3, 64, 300, "relu", True, None),       # K = 64: 8 vectors, most lanes idle
    (2, 40960, 3, "relu6", False, None),    # K slices of 160 vectors: past the 4 preloaded per lane
])
def test_gemv_cases(m, kin, nout, act, res, rows):
    """PASK_K_GEMV (D12) vs the fp64 linear definition: every layer with
    <= 8 rows is bound to it (s*), the rest to pask_gemm."""
    spec = linear_spec(m, kin, nout, act, res, rows)
    dm, plan = _check_spec(spec)
    for (i, want, bound, how, lk), L in zip(plan, spec["layers"]):
        rows_i = L["rows"] if L["rows"] is not None else m
        assert want == (P.K_GEMV if rows_i <= 8 else P.K_GEMM)


def test_attention_batched_gemm():
    """QK^T (both operands K-major, batched over heads) and PV (V MN-major)."""
    b = _Builder("attn", 6)
    s, heads, dh = 128, 4, 64
    x = b.input((s, heads * dh), "bf16")
    qkv = b.linear(x, 3 * heads * dh, w_std=0.05, b_std=0.02)
    sc = b.qk(qkv, heads, dh)
    pr = b.softmax(sc, 1 / math.sqrt(dh))
    ctx = b.pv(pr, qkv, heads, dh)
    b.outputs = [ctx]
    _check_spec(b.spec())


@pytest.mark.parametrize("s,heads", [(128, 12), (128, 1), (64, 2), (100, 3), (200, 4), (256, 2), (16, 1),
                                     (1, 1), (77, 5)])
def test_fused_attention(s, heads):
    """pask_attention (QK^T -> softmax -> PV in one tcgen05 kernel) vs the fp64
    attention definition, including sequence tails that are not multiples of the
    64-key block / 128-query tile."""
    b = _Builder("fattn", 8)
    dh = 64
    x = b.input((s, heads * dh), "bf16")
    qkv = b.linear(x, 3 * heads * dh, w_std=0.08, b_std=0.02)
    ctx = b.attention(qkv, heads, dh, 1 / math.sqrt(dh))
    b.outputs = [ctx]
    dm, plan = _check_spec(b.spec())
    assert plan[-1][2] == P.K_ATTENTION


@pytest.mark.parametrize("kind", ["max3s2p1", "max2s2", "avg3s1p1", "avg_global", "max_global"])
def test_pool(kind):
    b = _Builder("pool", 7)
    x = b.input((1, 16, 15, 13), "f32")
    t = b.layout(x)
    t = b.conv(t, 64, 1, act="none")
    if kind == "max3s2p1":
        y = b.pool(t, "max", 3, 2, 1)
    elif kind == "max2s2":
        y = b.pool(t, "max", 2, 2, 0)
    elif kind == "avg3s1p1":
        y = b.pool(t, "avg", 3, 1, 1, count_include_pad=False)
    elif kind == "avg_global":
        y = b.pool(t, "avg", "global")
    else:
        y = b.pool(t, "max", "global")
    b.outputs = [y]
    _check_spec(b.spec())


@pytest.mark.parametrize("cols,sigma", [(10, 1.0), (128, 4.0), (1000, 1.0), (1000, 4.0), (77, 2.0)])
def test_softmax_rows(cols, sigma):
    b = _Builder("sm", 8)
    x = b.input((37, cols), "bf16")
    y = b.softmax(x, 0.5)
    b.outputs = [y]
    spec = b.spec()
    xin = bf16_round(make_input(spec, 3) * sigma)
    dm, ctx, _ = run_model(spec, xin)
    ref = O.softmax(xin.astype(np.float64), 0.5)
    assert rel_err(dm.read(y), ref) <= TOL
    ctx.close()


@pytest.mark.parametrize("cols", [768, 64, 4096])
def test_layernorm_rows(cols):
    b = _Builder("ln", 9)
    x = b.input((50, cols), "bf16")
    y = b.layernorm(x, 1e-12)
    b.outputs = [y]
    _check_spec(b.spec())


def test_reused_kernel_bitwise_equals_dedicated_launch():
    """T4: a 1x1 conv whose s* is conv_1x1 runs on the reused
    igemm kernel inside the model; the same kernel launched stand-alone on the
    same input (fresh buffers) gives the same bits, and the dedicated conv_1x1
    kernel gives the same bits as well (identical tiling and K order)."""
    b = _Builder("reuse", 10)
    x = b.input((1, 64, 28, 28), "f32")
    t = b.layout(x)
    t = b.conv(t, 64, 3, 1, 1, act="relu")       # loads igemm
    y = b.conv(t, 256, 1, 1, 0, act="relu")      # s* = conv_1x1 -> reuses igemm
    b.outputs = [y]
    spec = b.spec()
    xin = make_input(spec, 0)
    dm, ctx, plan = run_model(spec, xin)
    assert plan[2][2] == P.K_CONV_IGEMM and plan[2][3] == 1     # reused
    in_bits = dm.read(spec["layers"][2]["inputs"][0])
    out_bits = dm.read_raw(y)
    ctx.close()
    # stand-alone: a 1-node graph (input bf16 values fed via an identity layout is not
    # possible, so feed the layer input as the fp32 model input of a layout + conv pair)
    b2 = _Builder("solo", 10)
    x2 = b2.input((1, 64, 28, 28), "f32")
    t2 = b2.layout(x2)
    y2 = b2.conv(t2, 256, 1, 1, 0, act="relu")
    b2.outputs = [y2]
    spec2 = b2.spec()
    spec2["layers"][1]["w"] = spec["layers"][2]["w"]
    spec2["layers"][1]["b"] = spec["layers"][2]["b"]
    for sol in (P.K_CONV_IGEMM, P.K_CONV_1X1):
        dm2, ctx2, plan2 = run_model(spec2, in_bits.astype(np.float32), solutions={1: sol})
        assert plan2[1][2] == sol
        np.testing.assert_array_equal(dm2.read_raw(y2), out_bits)
        ctx2.close()


def test_errors_fail_loudly():
    """No fallback: an inapplicable forced solution is PASK_EUNSUPPORTED."""
    spec = conv_spec(16, 32, 8, 3, 1, 1)
    from paper_conf_dac_huangdxz25_b200.model import DeviceModel
    dm = DeviceModel(spec, solutions={1: P.K_CONV_1X1})    # 3x3 on the 1x1 kernel
    ctx = P.Context(0)
    with pytest.raises(P.PaskError) as ei:
        ctx.load_model(dm.graph)
    assert ei.value.code == P.EUNSUPPORTED
    assert "not applicable" in str(ei.value)
    ctx.close()
    torch.cuda.synchronize()


@pytest.mark.parametrize("c,k,hw,r,res", [(64, 128, 160, 3, True), (8, 64, 224, 7, False), (128, 256, 144, 1, True)])
def test_persistent_tiles_bitwise(c, k, hw, r, res):
    """pask_conv_igemm_pt (s* for N*P*Q > 148 x 128 rows): <= 148 CTAs loop over
    the tiles with a double-buffered TMEM accumulator, staging tiles and a store
    agent.  Each tile is computed with the same K order as the one-tile-per-CTA
    kernel, so the outputs are bitwise equal; both within tolerance of the oracle."""
    spec = conv_spec(c, k, hw, r, 1, r // 2, 1, "relu", res)
    conv_li = len(spec["layers"]) - 1
    xin = make_input(spec, 0)
    dm, ctx, plan = run_model(spec, xin)
    assert plan[conv_li][1] == P.K_CONV_IGEMM_PT and plan[conv_li][2] == P.K_CONV_IGEMM_PT
    errs = teacher_forced_errors(dm, spec, xin)
    assert max(e for _, _, e in errs) <= TOL, errs
    out_pt = dm.read_raw(spec["outputs"][0])
    ctx.close()
    sols = {li: P.K_CONV_IGEMM for li, L in enumerate(spec["layers"]) if L["op"] == "conv"}
    dm2, ctx2, plan2 = run_model(spec, xin, solutions=sols)
    assert plan2[conv_li][2] == P.K_CONV_IGEMM
    np.testing.assert_array_equal(dm2.read_raw(spec["outputs"][0]), out_pt)
    ctx2.close()
