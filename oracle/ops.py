"""Oracle operators: plain, slow, obviously-correct float64 definitions.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
module.  It shares no code with the CUDA path (``paper_conf_dac_huangdxz25_b200``).

The paper fixes no operator arithmetic of its own: PASK reuses already-loaded
kernels *without changing results* -- "To ensure successful executions and
correct results of DNN inference, the primitive library should only return
applicable solutions" (§II-B) -- over the ONNX "canonical
operators" exported "from PyTorch under the default configuration"
(PAPER.md:67, :172).  So each oracle function is the plain definition of the
canonical operator, in float64, in NCHW / row-major
logical layout.  All functions take and return numpy float64 arrays.
"""
from __future__ import annotations

import math

import numpy as np


def _f64(x):
    return np.asarray(x, dtype=np.float64)


# ---------------------------------------------------------------------------
# activations ("activation primitives")
# ---------------------------------------------------------------------------
def relu(x):
    return np.maximum(_f64(x), 0.0)


def relu6(x):
    return np.minimum(np.maximum(_f64(x), 0.0), 6.0)


def gelu_erf(x):
    """GELU, exact erf form: 0.5 x (1 + erf(x / sqrt 2))  (HF BERT "gelu", R13)."""
    x = _f64(x)
    erf = np.vectorize(math.erf, otypes=[np.float64])
    return 0.5 * x * (1.0 + erf(x / math.sqrt(2.0)))


def tanh(x):
    return np.tanh(_f64(x))


ACTS = {"none": lambda x: _f64(x), "relu": relu, "relu6": relu6, "gelu": gelu_erf,
        "tanh": tanh}


def activation(x, kind):
    return ACTS[kind](x)


# ---------------------------------------------------------------------------
# convolution (the DirectConv / ImplicitGEMM patterns
# of PAPER.md:83 all compute this same cross-correlation)
# ---------------------------------------------------------------------------
def conv_out_size(h, r, stride, pad, dil):
    """P = floor((H + 2p - d(R-1) - 1) / s) + 1."""
    return (h + 2 * pad - dil * (r - 1) - 1) // stride + 1


def conv2d(x, w, b=None, stride=(1, 1), pad=(0, 0), dil=(1, 1), groups=1):
    """out[n,k,p,q] = b[k] + sum_{c in grp(k), r, s} x[n, c, p*sh - ph + r*dh, q*sw - pw + s*dw]
                                                       * w[k, c - g(k)*C/G, r, s]
    Cross-correlation (no filter flip); out-of-range x reads are 0.
    Evaluated as a loop over filter taps (r, s) with one channel contraction per
    tap (fp64, any summation order is exact enough)."""
    x = _f64(x)
    w = _f64(w)
    n, c, h, wd = x.shape
    k, cg, r, s = w.shape
    assert c == cg * groups and k % groups == 0
    kg = k // groups
    p = conv_out_size(h, r, stride[0], pad[0], dil[0])
    q = conv_out_size(wd, s, stride[1], pad[1], dil[1])
    out = np.zeros((n, k, p, q), dtype=np.float64)
    # zero-padded copy: xp[.., ih + ph, iw + pw] = x[.., ih, iw]; zeros elsewhere
    xp = np.zeros((n, c, h + 2 * pad[0], wd + 2 * pad[1]), dtype=np.float64)
    xp[:, :, pad[0]:pad[0] + h, pad[1]:pad[1] + wd] = x
    for rr in range(r):
        h0 = rr * dil[0]                       # = (p*sh - ph + r*dh) + ph at p = 0
        for ss in range(s):
            w0 = ss * dil[1]
            # input tap [n, c, p, q] = x[n, c, p*sh - ph + rr*dh, q*sw - pw + ss*dw]
            tap = xp[:, :, h0:h0 + stride[0] * (p - 1) + 1:stride[0],
                     w0:w0 + stride[1] * (q - 1) + 1:stride[1]]
            for g in range(groups):
                xs = tap[:, g * cg:(g + 1) * cg]                 # [n, cg, p, q]
                ws = w[g * kg:(g + 1) * kg, :, rr, ss]            # [kg, cg]
                out[:, g * kg:(g + 1) * kg] += np.einsum("ncpq,kc->nkpq", xs, ws)
    if b is not None:
        out += _f64(b)[None, :, None, None]
    return out


def conv2d_depthwise(x, w, b=None, stride=(1, 1), pad=(0, 0), dil=(1, 1)):
    """Depthwise special case G = C = K: per-channel multiply-add over taps."""
    x = _f64(x)
    w = _f64(w)
    n, c, h, wd = x.shape
    k, one, r, s = w.shape
    assert k == c and one == 1
    p = conv_out_size(h, r, stride[0], pad[0], dil[0])
    q = conv_out_size(wd, s, stride[1], pad[1], dil[1])
    out = np.zeros((n, c, p, q), dtype=np.float64)
    for pp in range(p):
        for qq in range(q):
            for rr in range(r):
                ih = pp * stride[0] - pad[0] + rr * dil[0]
                if ih < 0 or ih >= h:
                    continue
                for ss in range(s):
                    iw = qq * stride[1] - pad[1] + ss * dil[1]
                    if iw < 0 or iw >= wd:
                        continue
                    out[:, :, pp, qq] += x[:, :, ih, iw] * w[None, :, 0, rr, ss]
    if b is not None:
        out += _f64(b)[None, :, None, None]
    return out


def conv_layer(x, w, b, stride, pad, dil, groups, act="none", res=None):
    """Conv + fused epilogue: y = act(conv(x) + b + res)."""
    c = x.shape[1]
    if groups == c and w.shape[0] == c and groups > 1:
        y = conv2d_depthwise(x, w, b, stride, pad, dil)
    else:
        y = conv2d(x, w, b, stride, pad, dil, groups)
    if res is not None:
        y = y + _f64(res)
    return activation(y, act)


# ---------------------------------------------------------------------------
# pooling ("pooling primitives")
# ---------------------------------------------------------------------------
def max_pool2d(x, kernel, stride, pad):
    """max over the window; padded cells are -inf (never 0)."""
    x = _f64(x)
    n, c, h, w = x.shape
    kh, kw = kernel
    p = (h + 2 * pad[0] - kh) // stride[0] + 1
    q = (w + 2 * pad[1] - kw) // stride[1] + 1
    xp = np.full((n, c, h + 2 * pad[0], w + 2 * pad[1]), -np.inf)
    xp[:, :, pad[0]:pad[0] + h, pad[1]:pad[1] + w] = x
    out = np.full((n, c, p, q), -np.inf)
    for i in range(kh):
        for j in range(kw):
            out = np.maximum(out, xp[:, :, i:i + stride[0] * p:stride[0],
                                      j:j + stride[1] * q:stride[1]])
    return out


def avg_pool2d(x, kernel, stride, pad, count_include_pad=True):
    """sum over the window / (window size, or number of in-range cells)."""
    x = _f64(x)
    n, c, h, w = x.shape
    kh, kw = kernel
    p = (h + 2 * pad[0] - kh) // stride[0] + 1
    q = (w + 2 * pad[1] - kw) // stride[1] + 1
    xp = np.zeros((n, c, h + 2 * pad[0], w + 2 * pad[1]))
    xp[:, :, pad[0]:pad[0] + h, pad[1]:pad[1] + w] = x
    ones = np.zeros((h + 2 * pad[0], w + 2 * pad[1]))
    ones[pad[0]:pad[0] + h, pad[1]:pad[1] + w] = 1.0
    out = np.zeros((n, c, p, q))
    cnt = np.zeros((p, q))
    for i in range(kh):
        for j in range(kw):
            out += xp[:, :, i:i + stride[0] * p:stride[0], j:j + stride[1] * q:stride[1]]
            cnt += ones[i:i + stride[0] * p:stride[0], j:j + stride[1] * q:stride[1]]
    if count_include_pad:
        return out / float(kh * kw)
    return out / cnt[None, None]


def global_avg_pool(x):
    """mean over H*W."""
    x = _f64(x)
    return x.mean(axis=(2, 3), keepdims=True)


# ---------------------------------------------------------------------------
# GEMM / linear (PAPER.md:238 GEMM extension)
# ---------------------------------------------------------------------------
def gemm(a, b, bias=None, res=None, trans_b=False, act="none"):
    """C = act(A @ op(B) + bias + res), op(B) = B or B^T."""
    a = _f64(a)
    b = _f64(b)
    c = a @ (b.T if trans_b else b)
    if bias is not None:
        c = c + _f64(bias)
    if res is not None:
        c = c + _f64(res)
    return activation(c, act)


def linear(x, w, b=None, act="none", res=None):
    """y = act(x W^T + b + res) -- ONNX Gemm(transB=1) / torch Linear."""
    return gemm(x, w, b, res, trans_b=True, act=act)


# ---------------------------------------------------------------------------
# softmax / LayerNorm
# ---------------------------------------------------------------------------
def softmax(x, scale=1.0):
    """y_j = exp(s x_j - m) / sum_k exp(s x_k - m), m = max_k s x_k, over the last axis."""
    z = _f64(x) * scale
    m = z.max(axis=-1, keepdims=True)
    e = np.exp(z - m)
    return e / e.sum(axis=-1, keepdims=True)


def layernorm(x, gamma, beta, eps):
    """mu = mean, var = mean((x-mu)^2) (biased), y = (x-mu)/sqrt(var+eps)*gamma + beta."""
    x = _f64(x)
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps) * _f64(gamma) + _f64(beta)


# ---------------------------------------------------------------------------
# attention pieces of the BERT config
# ---------------------------------------------------------------------------
def attn_qk(qkv, heads, head_dim):
    """scores[h] = Q_h K_h^T, Q_h = qkv[:, 64h:64h+64], K_h = qkv[:, H+64h : H+64h+64]."""
    qkv = _f64(qkv)
    hid = heads * head_dim
    out = np.empty((heads, qkv.shape[0], qkv.shape[0]))
    for h in range(heads):
        q = qkv[:, h * head_dim:(h + 1) * head_dim]
        k = qkv[:, hid + h * head_dim:hid + (h + 1) * head_dim]
        out[h] = q @ k.T
    return out


def attn_pv(probs, qkv, heads, head_dim):
    """ctx[:, 64h + d] = sum_j P_h[:, j] V_h[j, d], V_h = qkv[:, 2H+64h : 2H+64h+64]."""
    probs = _f64(probs)
    qkv = _f64(qkv)
    hid = heads * head_dim
    out = np.empty((qkv.shape[0], hid))
    for h in range(heads):
        v = qkv[:, 2 * hid + h * head_dim:2 * hid + (h + 1) * head_dim]
        out[:, h * head_dim:(h + 1) * head_dim] = probs[h] @ v
    return out


def attention(qkv, heads, head_dim, scale):
    """Multi-head scaled dot-product attention without mask, the definition
    Attention(Q, K, V) = softmax(scale * Q K^T) V per head (Vaswani et al. 2017,
    eq. 1; BERT self-attention), over packed rows qkv = [Q | K | V], head h at
    columns h*head_dim of each third.  Written out directly (fp64), not through
    attn_qk / softmax / attn_pv."""
    qkv = _f64(qkv)
    hid = heads * head_dim
    out = np.empty((qkv.shape[0], hid))
    for h in range(heads):
        cols = slice(h * head_dim, (h + 1) * head_dim)
        q = qkv[:, :hid][:, cols]
        k = qkv[:, hid:2 * hid][:, cols]
        v = qkv[:, 2 * hid:][:, cols]
        z = scale * (q @ k.T)
        e = np.exp(z - z.max(axis=1, keepdims=True))
        out[:, cols] = (e / e.sum(axis=1, keepdims=True)) @ v
    return out


# ---------------------------------------------------------------------------
# input layout (PAPER.md:73 footnote 2 layout kernels)
# ---------------------------------------------------------------------------
def bf16_rne(x):
    """Round float64 values to bfloat16 (round-to-nearest-even), returned as float64.
    Written out bitwise on the float32 representation (values are finite)."""
    f = np.asarray(x, dtype=np.float64).astype(np.float32)
    u = f.view(np.uint32).astype(np.uint64)
    lsb = (u >> 16) & 1
    u = (u + 0x7FFF + lsb) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32).astype(np.float64)


def layout_nchw_to_nhwc(x, c_pad):
    """NCHW fp32 -> NHWC bf16 with channels zero-padded to c_pad.  Returns the
    NHWC array (float64 holding bf16 values)."""
    x = _f64(x)
    n, c, h, w = x.shape
    out = np.zeros((n, h, w, c_pad))
    out[..., :c] = bf16_rne(x).transpose(0, 2, 3, 1)
    return out
