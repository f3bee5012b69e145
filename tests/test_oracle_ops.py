"""T0: pin the oracle operators to things other than themselves.

Pins: hand-computed worked examples (tests/golden/), closed forms, brute-force
im2col + matmul, identity/delta filters, linearity, and independent library
routines (torch float64 functional ops).
"""
import math

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from oracle import ops

RNG = np.random.default_rng(1234)


# ---------------------------------------------------------------- conv
def test_conv_worked_examples(golden):
    g = golden("conv_worked_examples.json")
    for case in g["cases"]:
        x = np.array(case["x"], float)[None, None]
        w = np.array(case["w"], float)[None, None]
        s, p, d = case["stride"], case["pad"], case["dil"]
        y = ops.conv2d(x, w, None, (s, s), (p, p), (d, d))[0, 0]
        np.testing.assert_array_equal(y, np.array(case["y"], float))


def _im2col_conv(x, w, b, stride, pad, dil, groups):
    """Brute force: explicit im2col matrix (nested loops) @ reshaped weights."""
    n, c, h, wd = x.shape
    k, cg, r, s = w.shape
    p = (h + 2 * pad[0] - dil[0] * (r - 1) - 1) // stride[0] + 1
    q = (wd + 2 * pad[1] - dil[1] * (s - 1) - 1) // stride[1] + 1
    kg = k // groups
    out = np.zeros((n, k, p, q))
    for g in range(groups):
        cols = np.zeros((n * p * q, cg * r * s))
        for nn in range(n):
            for pp in range(p):
                for qq in range(q):
                    row = (nn * p + pp) * q + qq
                    col = 0
                    for cc in range(cg):
                        for rr in range(r):
                            for ss in range(s):
                                ih = pp * stride[0] - pad[0] + rr * dil[0]
                                iw = qq * stride[1] - pad[1] + ss * dil[1]
                                if 0 <= ih < h and 0 <= iw < wd:
                                    cols[row, col] = x[nn, g * cg + cc, ih, iw]
                                col += 1
        wm = w[g * kg:(g + 1) * kg].reshape(kg, -1)
        res = cols @ wm.T
        out[:, g * kg:(g + 1) * kg] = res.reshape(n, p, q, kg).transpose(0, 3, 1, 2)
    if b is not None:
        out += b[None, :, None, None]
    return out


@pytest.mark.parametrize("r", [1, 3, 7])
@pytest.mark.parametrize("stride", [1, 2])
@pytest.mark.parametrize("pad", [0, 1, 3])
@pytest.mark.parametrize("dil", [1, 2])
@pytest.mark.parametrize("grouped", [False, True])
def test_conv_vs_bruteforce_im2col(r, stride, pad, dil, grouped):
    c, k = 4, 6
    h = 9
    if h + 2 * pad - dil * (r - 1) - 1 < 0:
        pytest.skip("empty output")
    groups = 2 if grouped else 1
    x = RNG.standard_normal((1, c, h, h - 1))
    if (h - 1) + 2 * pad - dil * (r - 1) - 1 < 0:
        pytest.skip("empty output")
    w = RNG.standard_normal((k, c // groups, r, r))
    b = RNG.standard_normal(k)
    y = ops.conv2d(x, w, b, (stride, stride), (pad, pad), (dil, dil), groups)
    yb = _im2col_conv(x, w, b, (stride, stride), (pad, pad), (dil, dil), groups)
    np.testing.assert_allclose(y, yb, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("stride,pad,dil", [(1, 1, 1), (2, 1, 1), (1, 2, 2), (2, 0, 1)])
def test_depthwise_vs_bruteforce_and_grouped(stride, pad, dil):
    c = 8
    x = RNG.standard_normal((1, c, 7, 6))
    w = RNG.standard_normal((c, 1, 3, 3))
    b = RNG.standard_normal(c)
    y = ops.conv2d_depthwise(x, w, b, (stride, stride), (pad, pad), (dil, dil))
    yb = _im2col_conv(x, w, b, (stride, stride), (pad, pad), (dil, dil), c)
    np.testing.assert_allclose(y, yb, rtol=1e-12, atol=1e-12)
    # the generic grouped path agrees too
    yg = ops.conv2d(x, w, b, (stride, stride), (pad, pad), (dil, dil), c)
    np.testing.assert_allclose(y, yg, rtol=1e-12, atol=1e-12)


def test_conv_delta_and_identity_filters():
    x = RNG.standard_normal((1, 8, 6, 5))
    delta = np.zeros((8, 8, 3, 3))
    for c in range(8):
        delta[c, c, 1, 1] = 1.0
    np.testing.assert_array_equal(ops.conv2d(x, delta, None, (1, 1), (1, 1)), x)
    eye = np.eye(8)[:, :, None, None]
    np.testing.assert_array_equal(ops.conv2d(x, eye), x)


def test_conv_linearity():
    x = RNG.standard_normal((1, 4, 8, 8))
    y = RNG.standard_normal((1, 4, 8, 8))
    w = RNG.standard_normal((5, 4, 3, 3))
    a, bb = 0.7, -1.3
    lhs = ops.conv2d(a * x + bb * y, w, None, (2, 2), (1, 1))
    rhs = a * ops.conv2d(x, w, None, (2, 2), (1, 1)) + bb * ops.conv2d(y, w, None, (2, 2), (1, 1))
    np.testing.assert_allclose(lhs, rhs, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(ops.conv2d(x, 3.0 * w), 3.0 * ops.conv2d(x, w), rtol=1e-12)


@pytest.mark.parametrize("groups", [1, 2, 8])
def test_conv_vs_torch_f64(groups):
    x = RNG.standard_normal((2, 8, 11, 9))
    w = RNG.standard_normal((16, 8 // groups, 3, 3))
    b = RNG.standard_normal(16)
    for s, p, d in [(1, 1, 1), (2, 1, 1), (2, 2, 2), (1, 0, 1)]:
        y = ops.conv2d(x, w, b, (s, s), (p, p), (d, d), groups)
        yt = F.conv2d(torch.from_numpy(x), torch.from_numpy(w), torch.from_numpy(b), s, p, d,
                      groups).numpy()
        np.testing.assert_allclose(y, yt, rtol=1e-10, atol=1e-10)


def test_conv_layer_epilogue_order():
    """act is applied after bias + residual (ReLU(conv + b + res))."""
    x = RNG.standard_normal((1, 4, 5, 5))
    w = RNG.standard_normal((4, 4, 1, 1))
    b = RNG.standard_normal(4)
    res = RNG.standard_normal((1, 4, 5, 5))
    y = ops.conv_layer(x, w, b, (1, 1), (0, 0), (1, 1), 1, "relu", res)
    ref = np.maximum(np.einsum("nchw,kc->nkhw", x, w[:, :, 0, 0]) + b[None, :, None, None]
                     + res, 0)
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------- pooling
def _pool_x(name):
    if name == "arange16":
        return np.arange(16, dtype=float).reshape(1, 1, 4, 4)
    return -np.arange(1, 17, dtype=float).reshape(1, 1, 4, 4)


def test_pool_worked_examples(golden):
    g = golden("pool_worked_examples.json")
    c = g["max_3x3_s2_p1"]
    np.testing.assert_array_equal(ops.max_pool2d(_pool_x(c["x"]), (3, 3), (2, 2), (1, 1))[0, 0],
                                  c["y"])
    c = g["max_3x3_s2_p1_neg"]
    np.testing.assert_array_equal(ops.max_pool2d(_pool_x(c["x"]), (3, 3), (2, 2), (1, 1))[0, 0],
                                  c["y"])
    c = g["avg_3x3_s2_p1_include_pad"]
    np.testing.assert_allclose(ops.avg_pool2d(_pool_x(c["x"]), (3, 3), (2, 2), (1, 1), True)[0, 0],
                               c["y"], rtol=1e-15)
    c = g["avg_3x3_s2_p1_exclude_pad"]
    np.testing.assert_allclose(ops.avg_pool2d(_pool_x(c["x"]), (3, 3), (2, 2), (1, 1), False)[0, 0],
                               c["y"], rtol=1e-15)
    c = g["global_avg"]
    assert ops.global_avg_pool(_pool_x(c["x"]))[0, 0, 0, 0] == c["y"]


@pytest.mark.parametrize("k,s,p", [(2, 2, 0), (3, 2, 1), (3, 1, 1), (5, 3, 2)])
def test_pool_vs_torch_f64(k, s, p):
    x = RNG.standard_normal((1, 8, 13, 11))
    xt = torch.from_numpy(x)
    np.testing.assert_array_equal(ops.max_pool2d(x, (k, k), (s, s), (p, p)),
                                  F.max_pool2d(xt, k, s, p).numpy())
    for cip in (True, False):
        np.testing.assert_allclose(ops.avg_pool2d(x, (k, k), (s, s), (p, p), cip),
                                   F.avg_pool2d(xt, k, s, p, count_include_pad=cip).numpy(),
                                   rtol=1e-12, atol=1e-14)
    np.testing.assert_allclose(ops.global_avg_pool(x), F.adaptive_avg_pool2d(xt, 1).numpy(),
                               rtol=1e-12)


# ---------------------------------------------------------------- gemm
def test_gemm_vs_explicit_sums():
    a = RNG.standard_normal((5, 7))
    b = RNG.standard_normal((3, 7))
    bias = RNG.standard_normal(3)
    y = ops.linear(a, b, bias)
    ref = np.array([[sum(a[i, k] * b[j, k] for k in range(7)) + bias[j] for j in range(3)]
                    for i in range(5)])
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)
    y2 = ops.gemm(a, b.T, bias, res=np.ones((5, 3)), trans_b=False, act="relu")
    np.testing.assert_allclose(y2, np.maximum(ref + 1, 0), rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------- elementwise
def test_elementwise_closed_forms(golden):
    g = golden("elementwise_closed_forms.json")
    np.testing.assert_allclose(ops.softmax(np.array([[1.0, 2.0, 3.0]]))[0], g["softmax_123"],
                               rtol=1e-14)
    np.testing.assert_allclose(ops.layernorm(np.array([[1.0, 2.0, 3.0, 4.0]]), np.ones(4),
                                             np.zeros(4), 0.0)[0], g["layernorm_1234"], rtol=1e-14)
    np.testing.assert_allclose(ops.gelu_erf(np.array(g["gelu_x"])), g["gelu_y"], rtol=1e-14,
                               atol=1e-16)
    np.testing.assert_array_equal(ops.relu6(np.array(g["relu6_x"])), g["relu6_y"])
    np.testing.assert_array_equal(ops.relu(np.array([-2.0, 0.0, 3.5])), [0.0, 0.0, 3.5])
    assert ops.tanh(np.array([0.5]))[0] == pytest.approx(math.tanh(0.5), rel=1e-15)


def test_softmax_invariants_and_torch():
    for n in (10, 128, 1000):
        for sigma in (1.0, 4.0):
            x = RNG.standard_normal((6, n)) * sigma
            y = ops.softmax(x, 0.125)
            np.testing.assert_allclose(y.sum(-1), 1.0, rtol=1e-13)
            np.testing.assert_allclose(ops.softmax(x + 3.0, 1.0), ops.softmax(x, 1.0), rtol=1e-12)
            np.testing.assert_allclose(y, F.softmax(torch.from_numpy(x) * 0.125, -1).numpy(),
                                       rtol=1e-12)
    np.testing.assert_allclose(ops.softmax(np.zeros((1, 7))), 1.0 / 7.0, rtol=1e-15)


def test_layernorm_invariants_and_torch():
    x = RNG.standard_normal((5, 768)) * 3 + 1
    y = ops.layernorm(x, np.ones(768), np.zeros(768), 0.0)
    np.testing.assert_allclose(y.mean(-1), 0.0, atol=1e-13)
    np.testing.assert_allclose(y.var(-1), 1.0, rtol=1e-12)
    g = RNG.uniform(0.5, 1.5, 768)
    b = RNG.standard_normal(768)
    np.testing.assert_allclose(
        ops.layernorm(x, g, b, 1e-12),
        F.layer_norm(torch.from_numpy(x), (768,), torch.from_numpy(g), torch.from_numpy(b),
                     1e-12).numpy(), rtol=1e-11, atol=1e-12)


def test_gelu_vs_torch():
    x = np.linspace(-6, 6, 1001)
    np.testing.assert_allclose(ops.gelu_erf(x), F.gelu(torch.from_numpy(x)).numpy(), rtol=1e-13,
                               atol=1e-15)


# ---------------------------------------------------------------- layout / bf16
def test_bf16_rne_vs_torch_cast():
    x = np.concatenate([RNG.standard_normal(100000) * 10.0 ** RNG.integers(-8, 8, 100000),
                        [1.0 + 2 ** -8, 1.0 + 3 * 2 ** -8, -1.0 - 2 ** -8, 0.0, -0.0]])
    ref = torch.from_numpy(x.astype(np.float32)).to(torch.bfloat16).to(torch.float64).numpy()
    np.testing.assert_array_equal(ops.bf16_rne(x), ref)
    # ties to even: 1 + 2^-8 is halfway between 1 and 1 + 2^-7 -> 1
    assert ops.bf16_rne(np.array([1.0 + 2 ** -8]))[0] == 1.0
    assert ops.bf16_rne(np.array([1.0 + 3 * 2 ** -8]))[0] == 1.0 + 2 ** -6


def test_layout_nchw_to_nhwc():
    x = RNG.standard_normal((1, 3, 4, 5))
    y = ops.layout_nchw_to_nhwc(x, 8)
    assert y.shape == (1, 4, 5, 8)
    np.testing.assert_array_equal(y[..., 3:], 0.0)
    np.testing.assert_array_equal(y[0, 2, 3, 1], ops.bf16_rne(x[0, 1, 2, 3]))


# ---------------------------------------------------------------- attention
def test_attention_pieces_vs_torch():
    s, heads, dh = 16, 4, 8
    qkv = RNG.standard_normal((s, 3 * heads * dh))
    sc = ops.attn_qk(qkv, heads, dh)
    t = torch.from_numpy(qkv).view(s, 3, heads, dh).permute(1, 2, 0, 3)  # [3, h, s, d]
    np.testing.assert_allclose(sc, (t[0] @ t[1].transpose(-1, -2)).numpy(), rtol=1e-12)
    pr = ops.softmax(sc, 1 / math.sqrt(dh))
    ctx = ops.attn_pv(pr, qkv, heads, dh)
    ref = (torch.from_numpy(pr) @ t[2]).permute(1, 0, 2).reshape(s, heads * dh).numpy()
    np.testing.assert_allclose(ctx, ref, rtol=1e-12)
    # cross-check against torch's fused attention in float64
    sdpa = F.scaled_dot_product_attention(t[0][None], t[1][None], t[2][None])[0]
    np.testing.assert_allclose(ctx, sdpa.permute(1, 0, 2).reshape(s, -1).numpy(), rtol=1e-10)


# ---------------------------------------------------------------- fused attention
def test_attention_vs_torch_sdpa_fp64():
    """ops.attention against torch's scaled_dot_product_attention (an independent
    library routine) in float64, several heads, S not a multiple of 16."""
    rng = np.random.default_rng(11)
    s, heads, dh = 37, 3, 64
    qkv = rng.normal(size=(s, 3 * heads * dh))
    scale = 1.0 / 8.0
    got = ops.attention(qkv, heads, dh, scale)
    t = torch.from_numpy(qkv).view(s, 3, heads, dh).permute(1, 2, 0, 3)  # [3][h][s][d]
    ref = torch.nn.functional.scaled_dot_product_attention(t[0], t[1], t[2], scale=scale)
    ref = ref.permute(1, 0, 2).reshape(s, heads * dh).numpy()
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)


def test_attention_closed_forms():
    """Q = 0: every key gets weight 1/S, output row = mean of V; one-hot
    dominant key: output = that key's V row; equals the qk -> softmax -> pv chain."""
    rng = np.random.default_rng(12)
    s, heads, dh = 20, 2, 64
    qkv = rng.normal(size=(s, 3 * heads * dh))
    hid = heads * dh
    q0 = qkv.copy()
    q0[:, :hid] = 0.0
    out = ops.attention(q0, heads, dh, 0.125)
    np.testing.assert_allclose(out, np.broadcast_to(q0[:, 2 * hid:].mean(axis=0), out.shape), atol=1e-12)
    big = qkv.copy()
    big[:, :hid] = 0.0
    big[:, hid:2 * hid] = 0.0
    big[:, 0] = 1.0                 # head 0 query component 0
    big[5, hid] = 1e4               # key 5 of head 0 dominates
    out = ops.attention(big, heads, dh, 1.0)
    np.testing.assert_allclose(out[:, :dh], np.broadcast_to(big[5, 2 * hid:2 * hid + dh], (s, dh)), atol=1e-9)
    chain = ops.attn_pv(ops.softmax(ops.attn_qk(qkv, heads, dh), 0.125), qkv, heads, dh)
    np.testing.assert_allclose(ops.attention(qkv, heads, dh, 0.125), chain, rtol=1e-12, atol=1e-12)
