"""Model specs (lowered layer sequences) and seeded synthetic weights/inputs.

A *spec* is the lowered model PASK takes as input (§III, Fig. 5:
"PASK receives the lowered model (a sequence of n solutions) as input").  It is
plain data::

    {"name": str,
     "inputs":  [(tensor_name, logical_shape, dtype)],
     "outputs": [tensor_name, ...],
     "tensors": {tensor_name: logical_shape},      # NCHW for images, [rows, cols] for 2-D
     "layers":  [layer_dict, ...]}                 # in execution order

Layer dicts (logical semantics are PyTorch/ONNX):

* ``layout``    in -> out; NCHW fp32 image to the device layout (C zero-padded to ``c_pad``)
* ``conv``      w [K, C/groups, R, S], b [K] | None, stride, pad, dil, groups, act, res
* ``pool``      mode "max"|"avg", kernel (kh, kw) | "global", stride, pad, count_include_pad
* ``linear``    y = act(x @ w.T + b + res); w [N, K]; ``rows`` = use only the first rows;
                ``flatten`` = "nchw" when x is a 4-D activation flattened in NCHW order
* ``softmax``   over the last dim of (scale * x)
* ``layernorm`` over the last dim; gamma, beta, eps
* ``qk``        scores[h] = Q_h K_h^T from a fused [S, 3H] QKV tensor (Q|K|V column blocks)
* ``pv``        ctx[:, 64h+d] = P_h V_h  (head-concatenated context)

Weights are float32 arrays whose values are exactly representable in bf16
(rounded once, RNE) -- the values the GPU receives.
Biases, LayerNorm gamma/beta stay float32.

Weight recipe: He-normal conv/linear weights, std
sqrt(2/fan_in) (sqrt(1/fan_in) for layers without a following ReLU), the last
conv of each residual branch scaled by 0.3 so activations stay O(1) across the
residual stack; biases N(0, 0.05^2).  BERT follows HF init: W ~ N(0, 0.02^2),
biases N(0, 0.02^2), LN gamma ~ U(0.5, 1.5), beta ~ N(0, 0.02^2).  This is
"random-init weights of that architecture" (BatchNorm already folded into the
conv weight and bias, the MIGraphX lowering PAPER.md:67 performs offline).
"""
from __future__ import annotations

import math

import numpy as np
import torch


def bf16_round(x) -> np.ndarray:
    """Round float values to the nearest bf16 (RNE) and return them as float32."""
    t = torch.as_tensor(np.asarray(x, dtype=np.float32))
    return t.to(torch.bfloat16).to(torch.float32).numpy()


class _Gen:
    def __init__(self, seed: int):
        self.g = torch.Generator().manual_seed(seed)

    def normal(self, shape, std=1.0):
        return (torch.randn(*shape, generator=self.g, dtype=torch.float32) * std).numpy()

    def uniform(self, shape, lo, hi):
        return (torch.rand(*shape, generator=self.g, dtype=torch.float32) * (hi - lo) + lo).numpy()


class _Builder:
    def __init__(self, name, seed_weights):
        self.name = name
        self.gen = _Gen(seed_weights)
        self.layers = []
        self.tensors = {}
        self.inputs = []
        self.outputs = []
        self._n = 0

    def tensor(self, shape, name=None):
        if name is None:
            name = f"t{self._n}"
            self._n += 1
        self.tensors[name] = tuple(int(s) for s in shape)
        return name

    def input(self, shape, dtype):
        n = self.tensor(shape, "input")
        self.inputs.append((n, tuple(shape), dtype))
        return n

    def shape(self, t):
        return self.tensors[t]

    # -- layers ---------------------------------------------------------
    def layout(self, x, c_pad=None):
        n, c, h, w = self.shape(x)
        if c_pad is None:
            c_pad = max(8, (c + 7) // 8 * 8)
        y = self.tensor((n, c, h, w))
        self.layers.append(dict(op="layout", name=f"layout{len(self.layers)}", inputs=[x], out=y,
                                c_pad=c_pad))
        return y

    def conv(self, x, k, r, stride=1, pad=0, dil=1, groups=1, act="none", res=None,
             gain=1.0, bias=True):
        n, c, h, w = self.shape(x)
        fan_in = (c // groups) * r * r
        std = gain * math.sqrt((2.0 if act in ("relu", "relu6") else 1.0) / fan_in)
        wt = bf16_round(self.gen.normal((k, c // groups, r, r), std))
        b = self.gen.normal((k,), 0.05) if bias else None
        p = (h + 2 * pad - dil * (r - 1) - 1) // stride + 1
        q = (w + 2 * pad - dil * (r - 1) - 1) // stride + 1
        y = self.tensor((n, k, p, q))
        self.layers.append(dict(op="conv", name=f"conv{len(self.layers)}", inputs=[x], out=y,
                                w=wt, b=b, stride=(stride, stride), pad=(pad, pad),
                                dil=(dil, dil), groups=groups, act=act, res=res))
        return y

    def pool(self, x, mode, kernel, stride=1, pad=0, count_include_pad=True):
        n, c, h, w = self.shape(x)
        if kernel == "global":
            y = self.tensor((n, c, 1, 1))
            ks, st, pd = (h, w), (1, 1), (0, 0)
        else:
            p = (h + 2 * pad - kernel) // stride + 1
            q = (w + 2 * pad - kernel) // stride + 1
            y = self.tensor((n, c, p, q))
            ks, st, pd = (kernel, kernel), (stride, stride), (pad, pad)
        self.layers.append(dict(op="pool", name=f"pool{len(self.layers)}", inputs=[x], out=y,
                                mode=mode, kernel=ks, stride=st, pad=pd,
                                global_=(kernel == "global"),
                                count_include_pad=count_include_pad))
        return y

    def linear(self, x, nout, act="none", res=None, w_std=None, b_std=0.05, rows=None,
               flatten=None):
        shp = self.shape(x)
        if flatten == "nchw" or len(shp) == 4:
            kin = int(np.prod(shp[1:]))
            m = shp[0]
            flatten = "nchw"
        else:
            m, kin = shp
        if rows is not None:
            m = rows
        std = w_std if w_std is not None else math.sqrt(
            (2.0 if act == "relu" else 1.0) / kin)
        wt = bf16_round(self.gen.normal((nout, kin), std))
        b = self.gen.normal((nout,), b_std) if b_std is not None else None
        y = self.tensor((m, nout))
        self.layers.append(dict(op="linear", name=f"linear{len(self.layers)}", inputs=[x],
                                out=y, w=wt, b=b, act=act, res=res, rows=rows, flatten=flatten))
        return y

    def softmax(self, x, scale=1.0):
        y = self.tensor(self.shape(x))
        self.layers.append(dict(op="softmax", name=f"softmax{len(self.layers)}", inputs=[x],
                                out=y, scale=float(scale)))
        return y

    def layernorm(self, x, eps, gamma_range=(0.5, 1.5), beta_std=0.02):
        rows, cols = self.shape(x)
        gamma = self.gen.uniform((cols,), *gamma_range)
        beta = self.gen.normal((cols,), beta_std)
        y = self.tensor((rows, cols))
        self.layers.append(dict(op="layernorm", name=f"ln{len(self.layers)}", inputs=[x],
                                out=y, gamma=gamma, beta=beta, eps=float(eps)))
        return y

    def qk(self, qkv, heads, head_dim):
        s, _ = self.shape(qkv)
        y = self.tensor((heads, s, s))
        self.layers.append(dict(op="qk", name=f"qk{len(self.layers)}", inputs=[qkv], out=y,
                                heads=heads, head_dim=head_dim))
        return y

    def pv(self, probs, qkv, heads, head_dim):
        s, _ = self.shape(qkv)
        y = self.tensor((s, heads * head_dim))
        self.layers.append(dict(op="pv", name=f"pv{len(self.layers)}", inputs=[probs, qkv],
                                out=y, heads=heads, head_dim=head_dim))
        return y

    def attention(self, qkv, heads, head_dim, scale):
        """Fused multi-head attention over the packed QKV rows (the qk -> softmax ->
        pv composition as one layer)."""
        s, _ = self.shape(qkv)
        y = self.tensor((s, heads * head_dim))
        self.layers.append(dict(op="attention", name=f"attn{len(self.layers)}", inputs=[qkv],
                                out=y, heads=heads, head_dim=head_dim, scale=float(scale)))
        return y

    def spec(self):
        return dict(name=self.name, inputs=self.inputs, outputs=self.outputs,
                    tensors=self.tensors, layers=self.layers)


# ---------------------------------------------------------------------------
# C1 tiny CNN (BASELINE.json configs[0])
# ---------------------------------------------------------------------------
def tiny_cnn(seed_weights=1, hw=32, batch=1):
    b = _Builder("tiny_cnn", seed_weights)
    x = b.input((batch, 3, hw, hw), "f32")
    t = b.layout(x)
    t = b.conv(t, 16, 3, 1, 1, act="relu")
    t = b.conv(t, 32, 3, 1, 1, act="relu")
    t = b.conv(t, 64, 3, 1, 1, act="relu")
    t = b.pool(t, "max", 2, 2, 0)
    t = b.linear(t, 10, flatten="nchw")
    t = b.softmax(t)
    b.outputs = [t]
    return b.spec()


# ---------------------------------------------------------------------------
# C2 ResNet-50 v1.5, batch 1, 224x224 (BASELINE.json configs[1])
# ---------------------------------------------------------------------------
def resnet50(seed_weights=1, hw=224, batch=1, layers=(3, 4, 6, 3)):
    b = _Builder("resnet50", seed_weights)
    x = b.input((batch, 3, hw, hw), "f32")
    t = b.layout(x)
    t = b.conv(t, 64, 7, 2, 3, act="relu")
    t = b.pool(t, "max", 3, 2, 1)
    cin = 64
    for stage, (nblk, width) in enumerate(zip(layers, (64, 128, 256, 512))):
        for blk in range(nblk):
            stride = 2 if (blk == 0 and stage > 0) else 1
            cout = width * 4
            u = b.conv(t, width, 1, 1, 0, act="relu")
            u = b.conv(u, width, 3, stride, 1, act="relu")
            if blk == 0:
                idn = b.conv(t, cout, 1, stride, 0, act="none")
            else:
                idn = t
            t = b.conv(u, cout, 1, 1, 0, act="relu", res=idn, gain=0.3)
            cin = cout
    t = b.pool(t, "avg", "global")
    t = b.linear(t, 1000, flatten="nchw")
    t = b.softmax(t)
    b.outputs = [t]
    assert cin == 2048
    return b.spec()


# ---------------------------------------------------------------------------
# C3 MobileNetV2 width 1.0, batch 1, 224x224 (BASELINE.json configs[2])
# ---------------------------------------------------------------------------
def mobilenet_v2(seed_weights=1, hw=224, batch=1):
    b = _Builder("mobilenet_v2", seed_weights)
    x = b.input((batch, 3, hw, hw), "f32")
    t = b.layout(x)
    t = b.conv(t, 32, 3, 2, 1, act="relu6")
    cin = 32
    cfg = [(1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2),
           (6, 96, 3, 1), (6, 160, 3, 2), (6, 320, 1, 1)]
    for tr, c, n, s in cfg:
        for i in range(n):
            stride = s if i == 0 else 1
            hid = cin * tr
            u = t
            if tr != 1:
                u = b.conv(u, hid, 1, 1, 0, act="relu6")
            u = b.conv(u, hid, 3, stride, 1, groups=hid, act="relu6")
            use_res = stride == 1 and cin == c
            u = b.conv(u, c, 1, 1, 0, act="none", res=t if use_res else None,
                       gain=0.5 if use_res else 1.0)
            t = u
            cin = c
    t = b.conv(t, 1280, 1, 1, 0, act="relu6")
    t = b.pool(t, "avg", "global")
    t = b.linear(t, 1000, flatten="nchw")
    t = b.softmax(t)
    b.outputs = [t]
    return b.spec()


# ---------------------------------------------------------------------------
# C4 BERT-base encoder, seq 128, batch 1 (BASELINE.json configs[3])
# ---------------------------------------------------------------------------
def bert_base(seed_weights=1, seq=128, hidden=768, heads=12, ffn=3072, nlayers=12,
              eps=1e-12, fused_attention=False):
    b = _Builder("bert_base_fa" if fused_attention else "bert_base", seed_weights)
    dh = hidden // heads
    x = b.input((seq, hidden), "bf16")          # embedding sum (no gather)
    h = b.layernorm(x, eps)
    for _ in range(nlayers):
        qkv = b.linear(h, 3 * hidden, w_std=0.02, b_std=0.02)
        if fused_attention:
            ctx = b.attention(qkv, heads, dh, 1.0 / math.sqrt(dh))
        else:
            sc = b.qk(qkv, heads, dh)
            pr = b.softmax(sc, scale=1.0 / math.sqrt(dh))
            ctx = b.pv(pr, qkv, heads, dh)
        ao = b.linear(ctx, hidden, res=h, w_std=0.02, b_std=0.02)
        h1 = b.layernorm(ao, eps)
        f1 = b.linear(h1, ffn, act="gelu", w_std=0.02, b_std=0.02)
        f2 = b.linear(f1, hidden, res=h1, w_std=0.02, b_std=0.02)
        h = b.layernorm(f2, eps)
    pooled = b.linear(h, hidden, act="tanh", rows=1, w_std=0.02, b_std=0.02)
    b.outputs = [h, pooled]
    return b.spec()


MODELS = {
    "tiny_cnn": tiny_cnn,
    "resnet50": resnet50,
    "mobilenet_v2": mobilenet_v2,
    "bert_base": bert_base,
    # C4 with the qk -> softmax -> pv chain fused into one attention layer (NEXT #4)
    "bert_base_fa": lambda **kw: bert_base(fused_attention=True, **kw),
}


def make_input(spec, seed_input=0):
    """Seeded N(0,1) input for the spec's single input (bf16-exact when dtype is bf16)."""
    (name, shape, dtype), = spec["inputs"]
    g = _Gen(seed_input)
    x = g.normal(shape, 1.0)
    if dtype == "bf16":
        x = bf16_round(x)
    return x.astype(np.float32)


def build_model(name, seed_weights=1, seed_input=0, **kw):
    spec = MODELS[name](seed_weights=seed_weights, **kw)
    return spec, make_input(spec, seed_input)
