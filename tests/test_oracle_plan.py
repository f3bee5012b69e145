"""T1 (oracle side): pin the Algorithm 1 plan oracle.

Pins: the hand trace of PAPER.md Algorithm 1 on a MobileNetV2 prefix
(tests/golden/plan_mbv2_prefix.json), the survey's independent full-model
counts, brute-force re-derivation on tiny catalogs via an
exhaustive "which loaded kernels are applicable" enumeration, and invariants
(every binding applicable, reuse-off loads exactly the distinct s*, categorical
lookups <= naive lookups, milestone = n reproduces PaSK-I).
"""
import itertools
import random

import pytest

from oracle import plan as P
from workloads import build_model


def conv(c, k, r, stride=1, pad=0, groups=1, hw=56):
    p = dict(P._ZERO)
    q = (hw + 2 * pad - (r - 1) - 1) // stride + 1
    p.update(n=1, h=hw, w=hw, c=c, k=k, r=r, s=r, stride_h=stride, stride_w=stride, pad_h=pad,
             pad_w=pad, dil_h=1, dil_w=1, groups=groups, p=q, q=q)
    p["op"] = P._conv_class(p)
    return p


HOW = {0: "direct", 1: "reused", 2: "loaded"}


def test_mbv2_prefix_hand_trace(golden):
    g = golden("plan_mbv2_prefix.json")["categorical"]
    probs = [conv(8, 32, 3, 2, 1, hw=224), conv(32, 32, 3, 1, 1, groups=32, hw=112),
             conv(32, 16, 1, hw=112), conv(16, 96, 1, hw=112),
             conv(96, 96, 3, 2, 1, groups=96, hw=112), conv(96, 24, 1, hw=56)]
    pl = P.execution_plan(probs)
    assert [P.KERNEL_NAMES[k] for k in pl["loaded"]] == g["loaded"]
    assert (pl["queries"], pl["hits"], pl["lookups"]) == (g["queries"], g["hits"], g["lookups"])
    assert [HOW[b[3]] for b in pl["bindings"]] == g["how"]
    assert [b[4] for b in pl["bindings"]] == g["lookups_per_node"]


def test_full_model_counts_match_survey():
    """SURVEY.md §8(a) a3 (computed independently by the survey from the candidate
    catalog), with DESIGN.md D12's GEMV solution added to the catalog: the FC
    layers of C1-C3 (M = 1) have s* = pask_gemv instead of pask_gemm -- the GEMM
    category is still empty at their query, so the query / hit / lookup counts
    are the survey's -- and BERT's pooler (M = 1) now queries the GEMM category
    and reuses the loaded pask_gemm (one more query, one hit, one lookup)."""
    expect = {
        "tiny_cnn": (["pask_layout", "pask_conv_igemm", "pask_pool", "pask_gemv",
                      "pask_softmax"], 5, 0, 0),
        "resnet50": (["pask_layout", "pask_conv_igemm", "pask_pool", "pask_gemv",
                      "pask_softmax"], 39, 34, 34),
        "mobilenet_v2": (["pask_layout", "pask_conv_igemm", "pask_conv_dw", "pask_pool_gavg",
                          "pask_gemv", "pask_softmax"], 40, 34, 34),
        "bert_base": (["pask_layernorm", "pask_gemm", "pask_softmax"], 4, 1, 1),
        # NEXT #4: qk -> softmax -> pv fused; the attention solution replaces softmax
        "bert_base_fa": (["pask_layernorm", "pask_gemm", "pask_attention"], 4, 1, 1),
    }
    for name, (loaded, q, h, lk) in expect.items():
        spec, _ = build_model(name)
        pl = P.execution_plan(P.problems_from_spec(spec))
        assert [P.KERNEL_NAMES[k] for k in pl["loaded"]] == loaded, name
        assert (pl["queries"], pl["hits"], pl["lookups"]) == (q, h, lk), name
    # naive search lookups per hit: 2.32 (C2), 2.44 (C3)
    for name, per_hit in (("resnet50", 2.32), ("mobilenet_v2", 2.44)):
        spec, _ = build_model(name)
        pl = P.execution_plan(P.problems_from_spec(spec), search="naive")
        assert pl["lookups"] / pl["hits"] == pytest.approx(per_hit, abs=0.005)
    # batch 128: dense convs with N*P*Q > 148*128 rows take the persistent-tile
    # solution as s*; the smaller stage-3/4 convs reuse it (no conv_1x1 / igemm load)
    spec, _ = build_model("resnet50", batch=128)
    pl = P.execution_plan(P.problems_from_spec(spec))
    assert [P.KERNEL_NAMES[k] for k in pl["loaded"]] == [
        "pask_layout", "pask_conv_igemm_pt", "pask_pool", "pask_gemm", "pask_softmax"]   # FC M = 128: gemm
    # no reuse: ResNet-50 loads 7 distinct s* (adds conv_1x1 and gavg), MobileNetV2 7
    for name, n in (("resnet50", 7), ("mobilenet_v2", 7)):
        spec, _ = build_model(name)
        assert len(P.execution_plan(P.problems_from_spec(spec), reuse=False)["loaded"]) == n


def _invariants(probs, pl, reuse, search):
    loaded = set()
    for (i, want, bound, how, lk) in pl["bindings"]:
        assert P.is_applicable(bound, probs[i])
        assert want == P.static_choice(probs[i])
        if how == P.LOADED:
            assert bound == want and bound not in loaded
            loaded.add(bound)
        else:
            assert bound in loaded
        if how == P.REUSED:
            assert bound != want and lk >= 1
            if search == "categorical":
                assert P.CATEGORY[bound] == P.CATEGORY[want]
    assert set(pl["loaded"]) == loaded
    distinct = {P.static_choice(p) for p in probs}
    assert len(loaded) <= len(distinct)
    if not reuse:
        assert loaded == distinct


def _random_problem(rng):
    kind = rng.choice(["conv", "conv", "conv", "dw", "pool", "gemm"])
    if kind == "conv":
        r = rng.choice([1, 3, 5, 7])
        return conv(rng.choice([8, 16, 3]), rng.choice([8, 16, 24]), r, rng.choice([1, 2]),
                    rng.choice([0, r // 2]), hw=rng.choice([7, 14]))
    if kind == "dw":
        c = rng.choice([8, 16, 12])
        return conv(c, c, 3, rng.choice([1, 2]), 1, groups=c, hw=14)
    if kind == "pool":
        p = dict(P._ZERO)
        glob = rng.random() < 0.5
        p.update(op=P.POOL, n=1, h=7, w=7, c=rng.choice([8, 16, 4]), r=7 if glob else 3,
                 s=7 if glob else 3, stride_h=1 if glob else 2, stride_w=1 if glob else 2,
                 pad_h=0 if glob else 1, pad_w=0 if glob else 1, pool_mode=rng.choice([0, 1]),
                 **{"global": 1 if glob else 0})
        return p
    p = dict(P._ZERO)
    k = rng.choice([64, 60])
    p.update(op=P.GEMM, gm=rng.choice([4, 16]), gn=8, gk=k, batch=1, lda=k, ldb=k, trans_b=1,
             b_weights=rng.choice([0, 1]))
    return p


def test_random_sequences_invariants_and_determinism():
    rng = random.Random(7)
    for _ in range(300):
        probs = [_random_problem(rng) for _ in range(rng.randint(1, 12))]
        probs = [p for p in probs if P.is_applicable(P.static_choice(p), p)]
        if not probs:
            continue
        for reuse in (True, False):
            for search in ("categorical", "naive"):
                pl = P.execution_plan(probs, reuse, search)
                _invariants(probs, pl, reuse, search)
                assert pl == P.execution_plan(probs, reuse, search)      # deterministic
        # both searches issue the same queries (a query happens iff s* is absent)
        assert (P.execution_plan(probs)["queries"]
                == P.execution_plan(probs, search="naive")["queries"])
        # PaSK-I: milestone = n disables reuse entirely
        pi = P.execution_plan(probs, milestone=len(probs))
        assert pi["loaded"] == P.execution_plan(probs, reuse=False)["loaded"]
        assert pi["queries"] == 0


def test_bruteforce_small_catalog_trace():
    """Brute force: for every order of a 4-problem set, re-derive the plan by a
    direct simulation of 'bound = s* if loaded, else the first applicable
    loaded kernel of the same category in MRU order, else load s*' written as a
    recency-timestamp search (independent of the list-manipulation code)."""
    base = [conv(8, 16, 3, 1, 1, hw=14), conv(16, 16, 1, hw=14), conv(16, 16, 1, hw=14),
            conv(16, 16, 3, 1, 1, groups=16, hw=14), conv(16, 8, 1, hw=14)]
    pool_g = dict(P._ZERO)
    pool_g.update(op=P.POOL, n=1, h=7, w=7, c=8, r=7, s=7, stride_h=1, stride_w=1, pool_mode=1,
                  **{"global": 1})
    pool_m = dict(P._ZERO)
    pool_m.update(op=P.POOL, n=1, h=7, w=7, c=8, r=3, s=3, stride_h=2, stride_w=2, pad_h=1,
                  pad_w=1, pool_mode=0)
    base += [pool_g, pool_m]
    for combo in itertools.permutations(range(len(base)), 4):
        probs = [base[i] for i in combo]
        pl = P.execution_plan(probs)
        stamp = {}          # kernel -> last access time (load or use)
        t = 0
        q = h = lk = 0
        for i, p in enumerate(probs):
            t += 1
            want = P.static_choice(p)
            if want in stamp:
                stamp[want] = t
                assert pl["bindings"][i][2] == want
                continue
            q += 1
            same = sorted((k for k in stamp if P.CATEGORY[k] == P.CATEGORY[want]),
                          key=lambda k: -stamp[k])
            got = None
            for n_checked, k in enumerate(same, 1):
                if P.is_applicable(k, p):
                    got = k
                    lk += n_checked
                    break
            else:
                lk += len(same)
            if got is None:
                got = want
            else:
                h += 1
            stamp[got] = t
            assert pl["bindings"][i][2] == got
        assert (pl["queries"], pl["hits"], pl["lookups"]) == (q, h, lk)


def test_tuned_catalog_covers_every_config_conv_and_plans():
    """The tuned catalog holds exactly one specialisation per distinct dense-conv
    (R, S, stride, pad, dilation, C) of configs C1-C3; with it the reactive
    Baseline loads one conv kernel per such problem (ResNet-50: 17 + layout,
    pool, gavg, FC, softmax = 22), while reuse cannot help (specialisations are
    applicable only to their own shape)."""
    combos = set()
    for name in ("tiny_cnn", "resnet50", "mobilenet_v2"):
        spec, _ = build_model(name)
        for p in P.problems_from_spec(spec):
            if p["op"] == P.CONV:
                combos.add((p["r"], p["s"], p["stride_h"], p["pad_h"], p["dil_h"], p["c"]))
    assert combos == set(P.SPECS) and len(P.SPECS) == 32
    spec, _ = build_model("resnet50")
    probs = P.problems_from_spec(spec)
    base = P.execution_plan(probs, reuse=False, catalog="tuned")
    assert len(base["loaded"]) == 22
    pask = P.execution_plan(probs, catalog="tuned")
    assert len(pask["loaded"]) == 21 and pask["hits"] == 1      # only gavg -> pool
    for (i, want, bound, how, lk) in pask["bindings"]:
        assert P.is_applicable(bound, probs[i])


def test_gemv_predicate_and_choice():
    """DESIGN.md D12: the GEMV solution is s* (and applicable) exactly for a
    single GEMM with a weight operand stored [N][K] and 1..8 rows, K, lda, ldb and
    the offsets multiples of 8 (16-byte vectors); otherwise s* stays pask_gemm,
    which is applicable to every such GEMM too (so the pooler can reuse it)."""
    base = dict(P._ZERO)
    base.update(op=P.GEMM, gm=1, gn=1000, gk=2048, batch=1, lda=2048, ldb=2048, trans_b=1, b_weights=1)
    assert P.static_choice(base) == P.K_GEMV
    assert P.is_applicable(P.K_GEMM, base)
    for m in (1, 2, 8):
        assert P.static_choice({**base, "gm": m}) == P.K_GEMV
    for bad in (dict(gm=9), dict(gm=0), dict(batch=2), dict(trans_b=0), dict(b_weights=0), dict(gk=2044),
                dict(lda=2050), dict(ldb=2052), dict(off_a=4), dict(off_b=12), dict(gn=0)):
        q = {**base, **bad}
        assert not P.is_applicable(P.K_GEMV, q), bad
        if q["gm"] >= 1 and q["gn"] >= 1 and q["gk"] % 8 == 0:
            assert P.static_choice(q) == P.K_GEMM, bad
    assert P.CATEGORY[P.K_GEMV] == P.CATEGORY[P.K_GEMM]
