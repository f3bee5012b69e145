"""Plan oracle: PASK Algorithm 1 over the categorical solution cache.

TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``).

Follows PAPER.md:105-132 (Algorithm 1, EXECUTIONPLAN / GETSUBSOLUTION) and
PAPER.md:135-141 (§III-C categorical solution cache) step by step, with the
readings of SURVEY.md §8(c) R1-R9 (listed in DESIGN.md "Readings"):

* R1  milestone m is a config knob (default 0); layers i <= m load s*_i unconditionally.
* R2  a direct use of s*_i moves it to the head of its category list (:139 "loaded/invoked").
* R3  no eviction.
* R5  GETSUBSOLUTION scans the category list MRU -> LRU; first applicable wins.
* R6  on a miss s*_i itself is loaded and inserted at the head of its category.
* R7  a query is one GETSUBSOLUTION call; lookups count IsApplicable calls.
* R8  naive search (PaSK-R) scans every loaded solution in load order.
* R9  category key = (op class, dtype, layout); depthwise is its own op class.

The kernel catalog (ids, names, categories, IsApplicable predicates, the static
choice s*) is restated here from DESIGN.md's catalog table; the C++ planner
implements the same table independently.
"""
from __future__ import annotations

import math

# op classes
LAYOUT, CONV, DWCONV, POOL, GEMM, SOFTMAX, LAYERNORM, ATTENTION = range(8)

# kernel catalog ids
K_LAYOUT, K_IGEMM, K_CONV1X1, K_DW, K_POOL, K_GAVG, K_GEMM, K_SOFTMAX, K_LN, K_ATTN, K_IGEMM_PT, K_GEMV = \
    range(12)
KERNEL_NAMES = ["pask_layout", "pask_conv_igemm", "pask_conv_1x1", "pask_conv_dw",
                "pask_pool", "pask_pool_gavg", "pask_gemm", "pask_softmax", "pask_layernorm",
                "pask_attention", "pask_conv_igemm_pt", "pask_gemv"]
# s* of a GEMM with at most this many rows (an FC layer at batch <= 8, BERT's
# pooler) is the weight-streaming GEMV solution (reading D12)
GEMV_MAX_ROWS = 8
# s* of a dense conv with more output rows N*P*Q than 148 SMs x 128-row tiles is the
# persistent-tile implicit-GEMM solution
PERSISTENT_ROWS = 148 * 128

# Tuned catalog: one specialised conv solution per distinct dense
# conv problem (R, S, stride, pad, dilation, C) of configs C1-C3, ids 9 + i in
# sorted order; applicable to exactly that shape (any K, N, H, W).
SPECS = sorted([
    (1, 1, 1, 0, 1, c) for c in (16, 24, 32, 64, 96, 128, 144, 160, 192, 256, 320, 384, 512, 576,
                                 960, 1024, 2048)
] + [(1, 1, 2, 0, 1, c) for c in (256, 512, 1024)]
  + [(3, 3, 1, 1, 1, c) for c in (8, 16, 32, 64, 128, 256, 512)]
  + [(3, 3, 2, 1, 1, c) for c in (8, 128, 256, 512)] + [(7, 7, 2, 3, 1, 8)])
N_GENERIC = 12
KERNEL_NAMES = KERNEL_NAMES + ["pask_conv_spec_r%ds%du%dp%dd%dc%d" % sp for sp in SPECS]

# category key (op class, dtype, layout): dtype 0 = bf16 compute path, layouts
# 0 NCHW, 1 NHWC, 2 row-major
CATEGORY = {
    K_LAYOUT: (LAYOUT, 1, 0),
    K_IGEMM: (CONV, 0, 1),
    K_CONV1X1: (CONV, 0, 1),
    K_DW: (DWCONV, 0, 1),
    K_POOL: (POOL, 0, 1),
    K_GAVG: (POOL, 0, 1),
    K_GEMM: (GEMM, 0, 2),
    K_SOFTMAX: (SOFTMAX, 0, 2),
    K_LN: (LAYERNORM, 0, 2),
    K_ATTN: (ATTENTION, 0, 2),
    K_IGEMM_PT: (CONV, 0, 1),
    K_GEMV: (GEMM, 0, 2),
}
CATEGORY.update({N_GENERIC + i: (CONV, 0, 1) for i in range(len(SPECS))})


def _conv_class(p):
    return DWCONV if (p["groups"] > 1 and p["groups"] == p["c"] and p["k"] == p["c"]) else CONV


def is_applicable(kid, p):
    """IsApplicable(kernel, problem) -- PAPER.md:83, Alg. 1 l.15."""
    op = p["op"]
    if kid >= N_GENERIC:
        r, s, st, pd, dl, c = SPECS[kid - N_GENERIC]
        return (op == CONV and p["r"] == r and p["s"] == s and p["stride_h"] == st
                and p["stride_w"] == st and p["pad_h"] == pd and p["pad_w"] == pd
                and p["dil_h"] == dl and p["dil_w"] == dl and p["c"] == c and p["k"] % 8 == 0
                and p["p"] >= 1 and p["q"] >= 1)
    if kid == K_LAYOUT:
        return (op == LAYOUT and p["k"] % 8 == 0 and p["c"] <= p["k"]
                and p["n"] * p["h"] * p["w"] * max(p["c"], p["k"]) < 2 ** 31)
    if kid in (K_IGEMM, K_IGEMM_PT):
        return (op == CONV and p["groups"] == 1 and p["c"] % 8 == 0 and p["k"] % 8 == 0
                and 1 <= p["r"] <= 16 and 1 <= p["s"] <= 16
                and 1 <= p["stride_h"] <= 8 and 1 <= p["stride_w"] <= 8
                and 0 <= p["pad_h"] <= 64 and 0 <= p["pad_w"] <= 64
                and 1 <= p["dil_h"] <= 8 and 1 <= p["dil_w"] <= 8
                and p["p"] >= 1 and p["q"] >= 1)
    if kid == K_CONV1X1:
        return (op == CONV and p["groups"] == 1 and p["r"] == 1 and p["s"] == 1
                and p["stride_h"] == 1 and p["stride_w"] == 1
                and p["pad_h"] == 0 and p["pad_w"] == 0
                and p["c"] % 8 == 0 and p["k"] % 8 == 0)
    if kid == K_DW:
        return (op == DWCONV and p["c"] % 8 == 0 and p["n"] * p["h"] * p["w"] * p["c"] < 2 ** 31
                and 1 <= p["r"] <= 15 and 1 <= p["s"] <= 15
                and 1 <= p["stride_h"] <= 8 and 1 <= p["stride_w"] <= 8
                and 1 <= p["dil_h"] <= 8 and 1 <= p["dil_w"] <= 8
                and p["p"] >= 1 and p["q"] >= 1)
    if kid == K_POOL:
        return (op == POOL and p["c"] % 8 == 0 and p["n"] * p["h"] * p["w"] * p["c"] < 2 ** 31
                and p["r"] * p["s"] <= 1024
                and p["stride_h"] >= 1 and p["stride_w"] >= 1
                and p["pad_h"] < p["r"] and p["pad_w"] < p["s"])
    if kid == K_GAVG:
        return op == POOL and p["global"] == 1 and p["pool_mode"] == 1 and p["c"] % 8 == 0
    if kid == K_GEMM:
        return (op == GEMM and p["gk"] % 8 == 0 and p["lda"] % 8 == 0 and p["ldb"] % 8 == 0
                and p["off_a"] % 8 == 0 and p["off_b"] % 8 == 0
                and p["gm"] >= 1 and p["gn"] >= 1 and p["batch"] >= 1)
    if kid == K_GEMV:   # DESIGN.md D12: weight operand [N][K], one GEMM, few rows
        return (op == GEMM and p["b_weights"] == 1 and p["trans_b"] == 1 and p["batch"] == 1
                and 1 <= p["gm"] <= GEMV_MAX_ROWS and p["gn"] >= 1 and p["gk"] % 8 == 0
                and p["lda"] % 8 == 0 and p["ldb"] % 8 == 0
                and p["off_a"] % 8 == 0 and p["off_b"] % 8 == 0)
    if kid == K_SOFTMAX:
        return op == SOFTMAX and 1 <= p["cols"] <= 16384
    if kid == K_LN:
        return op == LAYERNORM and p["cols"] % 8 == 0 and 8 <= p["cols"] <= 8192
    if kid == K_ATTN:
        return (op == ATTENTION and p["gk"] == 64 and 1 <= p["gm"] <= 256
                and p["gn"] >= 1 and p["batch"] >= 1)
    raise ValueError(kid)


def static_choice(p, catalog="generic"):
    """s*_i: the library's statically 'best' (most specialised) solution.
    With the tuned catalog a dense conv's s* is its own specialised solution."""
    op = p["op"]
    if catalog == "tuned" and op == CONV:
        for i in range(len(SPECS)):
            if is_applicable(N_GENERIC + i, p):
                return N_GENERIC + i
    if op == LAYOUT:
        return K_LAYOUT
    if op == DWCONV:
        return K_DW
    if op == CONV:
        if p["n"] * p["p"] * p["q"] > PERSISTENT_ROWS:
            return K_IGEMM_PT
        if (p["r"] == 1 and p["s"] == 1 and p["stride_h"] == 1 and p["stride_w"] == 1
                and p["pad_h"] == 0 and p["pad_w"] == 0):
            return K_CONV1X1
        return K_IGEMM
    if op == POOL:
        return K_GAVG if (p["global"] == 1 and p["pool_mode"] == 1) else K_POOL
    if op == GEMM:
        return K_GEMV if is_applicable(K_GEMV, p) else K_GEMM
    if op == SOFTMAX:
        return K_SOFTMAX
    if op == LAYERNORM:
        return K_LN
    if op == ATTENTION:
        return K_ATTN
    raise ValueError(op)


_ZERO = dict(op=0, n=0, h=0, w=0, c=0, k=0, r=0, s=0, stride_h=0, stride_w=0, pad_h=0,
             pad_w=0, dil_h=0, dil_w=0, groups=0, p=0, q=0, pool_mode=0, **{"global": 0},
             gm=0, gn=0, gk=0, batch=0, lda=0, ldb=0, off_a=0, off_b=0, trans_b=0, b_weights=0,
             rows=0, cols=0)


def problems_from_spec(spec):
    """Extract the problem p_i of every spec layer (parse step P_i).
    Problems are stated on the device tensors (reading D1): the layout
    output carries C padded to c_pad; a pool keeps its input's (padded) channel
    count; a conv output has K channels; a flattened FC reduces over H*W*C_dev."""
    shapes = spec["tensors"]
    devc = {}
    out = []
    for layer in spec["layers"]:
        p = dict(_ZERO)
        op = layer["op"]
        if op == "layout":
            n, c, h, w = shapes[layer["inputs"][0]]
            p.update(op=LAYOUT, n=n, h=h, w=w, c=c, k=layer["c_pad"])
            devc[layer["out"]] = layer["c_pad"]
        elif op == "conv":
            n, c, h, w = shapes[layer["inputs"][0]]
            c = devc.get(layer["inputs"][0], c)
            k, cg, r, s = layer["w"].shape
            _, _, pp, qq = shapes[layer["out"]]
            p.update(n=n, h=h, w=w, c=c, k=k, r=r, s=s,
                     stride_h=layer["stride"][0], stride_w=layer["stride"][1],
                     pad_h=layer["pad"][0], pad_w=layer["pad"][1],
                     dil_h=layer["dil"][0], dil_w=layer["dil"][1],
                     groups=layer["groups"], p=pp, q=qq)
            p["op"] = _conv_class(p)
        elif op == "pool":
            n, c, h, w = shapes[layer["inputs"][0]]
            c = devc.get(layer["inputs"][0], c)
            devc[layer["out"]] = c
            _, _, pp, qq = shapes[layer["out"]]
            p.update(op=POOL, n=n, h=h, w=w, c=c, k=c, r=layer["kernel"][0],
                     s=layer["kernel"][1], stride_h=layer["stride"][0],
                     stride_w=layer["stride"][1], pad_h=layer["pad"][0], pad_w=layer["pad"][1],
                     p=pp, q=qq, pool_mode=0 if layer["mode"] == "max" else 1,
                     **{"global": 1 if layer["global_"] else 0})
        elif op == "linear":
            m, nout = shapes[layer["out"]]
            kin = layer["w"].shape[1]
            src = layer["inputs"][0]
            if len(shapes[src]) == 4:        # flattened image: K over the device channels
                _, c, h, w = shapes[src]
                kin = h * w * devc.get(src, c)
            p.update(op=GEMM, gm=m, gn=nout, gk=kin, batch=1, lda=kin, ldb=kin, trans_b=1, b_weights=1)
        elif op == "qk":
            s_, three_h = shapes[layer["inputs"][0]]
            hd = layer["head_dim"]
            p.update(op=GEMM, gm=s_, gn=s_, gk=hd, batch=layer["heads"], lda=three_h,
                     ldb=three_h, off_a=0, off_b=three_h // 3, trans_b=1, b_weights=0)
        elif op == "pv":
            heads, s_, _ = shapes[layer["inputs"][0]]
            three_h = shapes[layer["inputs"][1]][1]
            hd = layer["head_dim"]
            p.update(op=GEMM, gm=s_, gn=hd, gk=s_, batch=heads, lda=s_, ldb=three_h,
                     off_a=0, off_b=2 * (three_h // 3), trans_b=0, b_weights=0)
        elif op == "attention":
            s_, three_h = shapes[layer["inputs"][0]]
            p.update(op=ATTENTION, gm=s_, gn=layer["heads"], gk=layer["head_dim"], batch=1,
                     lda=three_h)
        elif op in ("softmax", "layernorm"):
            shp = shapes[layer["inputs"][0]]
            cols = shp[-1]
            rows = int(math.prod(shp[:-1]))
            p.update(op=SOFTMAX if op == "softmax" else LAYERNORM, rows=rows, cols=cols)
        else:
            raise ValueError(op)
        out.append(p)
    return out


DIRECT, REUSED, LOADED = 0, 1, 2


def execution_plan(problems, reuse=True, search="categorical", milestone=0, catalog="generic"):
    """Algorithm 1 EXECUTIONPLAN for layers 1..n.

    Returns dict(bindings=[(node, desired, bound, how, lookups)], loaded=[ids in load
    order], queries, hits, lookups)."""
    loaded = []               # S_m as a list in load order
    mru = {}                  # category key -> list of kernel ids, head = most recent
    bindings = []
    queries = hits = lookups = 0

    def touch(kid):           # insert / move to the head of its category list (:139)
        lst = mru.setdefault(CATEGORY[kid], [])
        if kid in lst:
            lst.remove(kid)
        lst.insert(0, kid)

    def load(kid):            # "wait for s*_i loading; add s*_i to S_m" (Alg. 1 l.10-11)
        loaded.append(kid)
        touch(kid)

    for i, p in enumerate(problems):
        s_star = static_choice(p, catalog)
        if not is_applicable(s_star, p):
            raise ValueError(f"node {i}: s* {KERNEL_NAMES[s_star]} not applicable")
        layer_no = i + 1
        if layer_no <= milestone or not reuse:
            if s_star in loaded:
                touch(s_star)
                bindings.append((i, s_star, s_star, DIRECT, 0))
            else:
                load(s_star)
                bindings.append((i, s_star, s_star, LOADED, 0))
            continue
        if s_star in loaded:                         # Alg. 1 l.3-4
            touch(s_star)
            bindings.append((i, s_star, s_star, DIRECT, 0))
            continue
        # Alg. 1 l.6: GETSUBSOLUTION(S, s*, p)
        queries += 1
        if search == "categorical":
            cand = list(mru.get(CATEGORY[s_star], []))   # l.13-14: MRU order
        else:
            cand = list(loaded)                           # R8: load order, all categories
        found = None
        nl = 0
        for s in cand:
            nl += 1
            if is_applicable(s, p):                       # l.15
                found = s
                break
        lookups += nl
        if found is not None:                             # l.7-8, l.16 lru.update
            hits += 1
            touch(found)
            bindings.append((i, s_star, found, REUSED, nl))
        else:                                             # l.9-11
            load(s_star)
            bindings.append((i, s_star, s_star, LOADED, nl))
    return dict(bindings=bindings, loaded=loaded, queries=queries, hits=hits, lookups=lookups)
