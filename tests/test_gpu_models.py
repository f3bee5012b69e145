"""T3/T5 on the GPU: every layer of every config, teacher-forced vs the oracle,
through the C ABI (pask_load_model -> pask_infer), plus plan / loaded-kernel
bit-exactness against the plan oracle and cuFuncIsLoaded."""
import os
import subprocess
import sys

import numpy as np
import pytest

from oracle import plan as OP
from paper_conf_dac_huangdxz25_b200 import pask as P
from workloads import build_model

from .gpu_harness import TOL, run_model, teacher_forced_errors

pytestmark = pytest.mark.gpu

MODELS = ["tiny_cnn", "resnet50", "mobilenet_v2", "bert_base", "bert_base_fa"]


@pytest.mark.parametrize("name", MODELS)
def test_model_layers_teacher_forced(name):
    spec, x = build_model(name)
    dm, ctx, plan = run_model(spec, x)
    errs = teacher_forced_errors(dm, spec, x)
    bad = [(i, op, e) for i, op, e in errs if not e <= TOL]
    assert not bad, f"layers over tolerance: {bad[:10]}"
    # integer bookkeeping: plan == plan oracle, loaded set == cuFuncIsLoaded
    o = OP.execution_plan(OP.problems_from_spec(spec))
    assert [tuple(b) for b in plan] == [tuple(b) for b in o["bindings"]]
    st = ctx.stats()
    assert st["kernels_loaded"] == len(o["loaded"])
    assert st["code_objects_loaded"] == len(o["loaded"])   # packaging 0: one object per kernel
    loaded = {k for k in range(P.num_kernels()) if ctx.kernel_is_loaded(k)}
    assert loaded == set(o["loaded"])
    assert len(loaded) <= 8
    ctx.close()


@pytest.mark.parametrize("name,batch", [("resnet50", 3), ("mobilenet_v2", 2), ("tiny_cnn", 5)])
def test_batched_models_teacher_forced(name, batch):
    """Batch > 1 (Table II sweep): pixels of several
    images share GEMM tiles (gather / TMA im2col wrap across images)."""
    spec, x = build_model(name, batch=batch)
    dm, ctx, plan = run_model(spec, x)
    errs = teacher_forced_errors(dm, spec, x)
    bad = [(i, op, e) for i, op, e in errs if not e <= TOL]
    assert not bad, f"layers over tolerance: {bad[:10]}"
    ctx.close()


@pytest.mark.parametrize("name", ["resnet50", "bert_base"])
def test_graph_replay_bitwise(name):
    """Hot inferences replayed from a captured CUDA graph equal direct issue, bitwise."""
    import torch
    spec, x = build_model(name)
    dm, ctx, _ = run_model(spec, x, cfg=P.config(graph=1))
    ref = [dm.read_raw(n) for n in spec["outputs"]]
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(3):
        ctx.infer(s)
    ctx.sync()
    for a, n in zip(ref, spec["outputs"]):
        np.testing.assert_array_equal(a, dm.read_raw(n))
    ctx.close()


@pytest.mark.parametrize("name", ["tiny_cnn", "resnet50", "mobilenet_v2"])
def test_tuned_catalog_specialised_kernels(name):
    """The per-problem specialised solutions (tuned catalog, Baseline scheme):
    every layer within tolerance, the loaded set = the plan oracle's, and every
    layer's output bitwise equal to the generic kernels' (same tiling and
    reduction order: a substitution never changes results)."""
    spec, x = build_model(name)
    dm, ctx, plan = run_model(spec, x, cfg=P.config(catalog=1, reuse=0, proactive=0))
    errs = teacher_forced_errors(dm, spec, x)
    assert max(e for _, _, e in errs) <= TOL
    o = OP.execution_plan(OP.problems_from_spec(spec), reuse=False, catalog="tuned")
    assert [tuple(b) for b in plan] == [tuple(b) for b in o["bindings"]]
    assert {k for k in range(P.num_kernels()) if ctx.kernel_is_loaded(k)} == set(o["loaded"])
    tuned = {L["out"]: dm.read_raw(L["out"]) for L in spec["layers"]}
    ctx.close()
    if dm.ws_bytes and os.environ.get("PASK_STEM_FOLD") != "0":
        # the generic solutions fold ResNet-50's stem (D16: another k
        # order), the specialised one cannot: compare with the fold off, in a
        # child (the runtime reads its switches once per process)
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                            f"{os.path.abspath(__file__)}::test_tuned_catalog_specialised_kernels[{name}]"],
                           cwd=root, env={**os.environ, "PASK_STEM_FOLD": "0"}, capture_output=True, text=True,
                           timeout=900)
        assert r.returncode == 0, r.stdout[-3000:]
        return
    dm2, ctx2, _ = run_model(spec, x)
    for L in spec["layers"]:
        np.testing.assert_array_equal(tuned[L["out"]], dm2.read_raw(L["out"]))
    ctx2.close()


@pytest.mark.parametrize("packaging", [0, 1, 2, 3])
@pytest.mark.parametrize("cfg", ["reactive", "pask_i", "pask_r", "no_pdl"])
def test_schemes_same_outputs(cfg, packaging):
    """Every scheme of PAPER.md:174-186 (reactive loading, PaSK-I = no reuse,
    PaSK-R = naive search) and both code-object packagings produce outputs
    within tolerance; plans match the plan oracle for the same config."""
    spec, x = build_model("resnet50")
    kw = dict(packaging=packaging)
    if cfg == "reactive":
        kw.update(proactive=0)
    elif cfg == "pask_i":
        kw.update(reuse=0)
    elif cfg == "pask_r":
        kw.update(search=1)
    else:
        kw.update(pdl=0)
    dm, ctx, plan = run_model(spec, x, cfg=P.config(**kw))
    errs = teacher_forced_errors(dm, spec, x)
    assert max(e for _, _, e in errs) <= TOL
    o = OP.execution_plan(OP.problems_from_spec(spec), reuse=bool(kw.get("reuse", 1)),
                          search="naive" if kw.get("search") else "categorical")
    assert [tuple(b) for b in plan] == [tuple(b) for b in o["bindings"]]
    st = ctx.stats()
    if packaging == 2:   # ResNet-50's solutions fall in two families, one code object
        assert st["kernels_loaded"] == 2 and st["code_objects_loaded"] == 1
    elif packaging == 3:  # ... and in one function under packaging 3
        assert st["kernels_loaded"] == 1 and st["code_objects_loaded"] == 1
    else:
        assert st["kernels_loaded"] == len(o["loaded"])
        assert st["code_objects_loaded"] == (1 if packaging == 1 else len(o["loaded"]))
    ctx.close()


@pytest.mark.parametrize("name", MODELS)
def test_family_packaging_bitwise(name):
    """Packaging 2 (D8): the same plan as packaging 0, every solution
    resident (cuFuncIsLoaded) after at most one upload per operator family, and
    every layer's output bitwise equal to the per-kernel code objects' (the family
    entries run the same bodies on the same parameters)."""
    spec, x = build_model(name)
    dm, ctx, plan = run_model(spec, x, cfg=P.config(packaging=2))
    o = OP.execution_plan(OP.problems_from_spec(spec))
    assert [tuple(b) for b in plan] == [tuple(b) for b in o["bindings"]]
    st = ctx.stats()
    fams = {("mem" if k in (P.K_LAYOUT, P.K_CONV_DW, P.K_POOL, P.K_POOL_GAVG, P.K_SOFTMAX, P.K_LAYERNORM,
                            P.K_GEMV)
             else "contract" if k in (P.K_CONV_IGEMM, P.K_CONV_1X1, P.K_GEMM) else k) for k in o["loaded"]}
    assert st["kernels_loaded"] == len(fams)
    # both families share one code object; other kernels keep their own
    assert st["code_objects_loaded"] == len(fams - {"mem", "contract"}) + 1
    assert {k for k in range(P.num_kernels()) if ctx.kernel_is_loaded(k)} >= set(o["loaded"])
    fam_out = {L["out"]: dm.read_raw(L["out"]) for L in spec["layers"]}
    ctx.close()
    dm2, ctx2, _ = run_model(spec, x)
    for L in spec["layers"]:
        np.testing.assert_array_equal(fam_out[L["out"]], dm2.read_raw(L["out"]))
    ctx2.close()


@pytest.mark.parametrize("name", MODELS)
def test_single_function_packaging_bitwise(name):
    """Packaging 3 (D10): the same plan as packaging 0, every
    contraction and memory-bound solution served by the one `pask_all` upload
    (attention keeps its own object), and every layer's output bitwise equal to
    the per-kernel code objects' (same bodies, same parameters)."""
    spec, x = build_model(name)
    dm, ctx, plan = run_model(spec, x, cfg=P.config(packaging=3))
    o = OP.execution_plan(OP.problems_from_spec(spec))
    assert [tuple(b) for b in plan] == [tuple(b) for b in o["bindings"]]
    st = ctx.stats()
    fam = {P.K_LAYOUT, P.K_CONV_DW, P.K_POOL, P.K_POOL_GAVG, P.K_SOFTMAX, P.K_LAYERNORM, P.K_GEMV,
           P.K_CONV_IGEMM, P.K_CONV_1X1, P.K_GEMM}
    own = set(o["loaded"]) - fam
    assert st["kernels_loaded"] == len(own) + 1
    assert st["code_objects_loaded"] == len(own) + 1
    assert {k for k in range(P.num_kernels()) if ctx.kernel_is_loaded(k)} >= set(o["loaded"])
    one_out = {L["out"]: dm.read_raw(L["out"]) for L in spec["layers"]}
    ctx.close()
    dm2, ctx2, _ = run_model(spec, x)
    for L in spec["layers"]:
        np.testing.assert_array_equal(one_out[L["out"]], dm2.read_raw(L["out"]))
    ctx2.close()


@pytest.mark.parametrize("name", MODELS)
def test_single_function_repack_bitwise(name):
    """Packaging 3 then pask_promote (D15): the cold inference runs on
    the single entry (one upload); the idle-interval repack uploads the two
    family entries of the variant with the same masks and re-lowers the nodes.
    Every later inference -- direct issue and CUDA-graph replay -- is bitwise
    equal to the cold one, and every solution stays resident."""
    import torch
    spec, x = build_model(name)
    dm, ctx, plan = run_model(spec, x, cfg=P.config(packaging=3, graph=1, branches=1))
    cold = {L["out"]: dm.read_raw(L["out"]) for L in spec["layers"]}
    k0 = ctx.stats()["kernels_loaded"]
    n = ctx.promote()
    fam = {P.K_LAYOUT, P.K_CONV_DW, P.K_POOL, P.K_POOL_GAVG, P.K_SOFTMAX, P.K_LAYERNORM, P.K_GEMV,
           P.K_CONV_IGEMM, P.K_CONV_1X1, P.K_GEMM}
    assert n == sum(1 for b in plan if b[2] in fam)
    bound_fams = {"mem" if b[2] in (P.K_LAYOUT, P.K_CONV_DW, P.K_POOL, P.K_POOL_GAVG, P.K_SOFTMAX,
                                    P.K_LAYERNORM, P.K_GEMV) else "contract" for b in plan if b[2] in fam}
    assert ctx.stats()["kernels_loaded"] == k0 + len(bound_fams)
    assert all(ctx.kernel_is_loaded(b[2]) for b in plan)
    assert [tuple(b) for b in ctx.bindings()] == [tuple(b) for b in plan]
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(3):                                   # direct, then capture + replays
        for L in spec["layers"]:
            dm.t[L["out"]].zero_()
        ctx.infer(s)
        ctx.sync()
        for L in spec["layers"]:
            np.testing.assert_array_equal(cold[L["out"]], dm.read_raw(L["out"]))
    ctx.close()


@pytest.mark.parametrize("name", MODELS)
def test_model_hot_repeat_bitwise(name):
    """A second (hot) inference reproduces the first bit for bit (deterministic
    split-K; no atomics in any reduction order)."""
    spec, x = build_model(name)
    dm, ctx, _ = run_model(spec, x)
    outs1 = [dm.read_raw(n) for n in spec["outputs"]]
    import torch
    ctx.infer(torch.cuda.current_stream().cuda_stream)
    ctx.sync()
    outs2 = [dm.read_raw(n) for n in spec["outputs"]]
    for a, b in zip(outs1, outs2):
        np.testing.assert_array_equal(a, b)
    ctx.close()


@pytest.mark.parametrize("name", ["resnet50", "mobilenet_v2"])
def test_promote_idle_interval(name):
    """Idle-interval loading: after the cold inference the skipped
    s* solutions are loaded and the reused nodes rebound; the next (hot, graph
    re-captured) inference stays within tolerance and every contraction layer is
    bitwise unchanged (a reused solution computes the same tiles in the same
    order, R6).  Promoting further to the tuned catalog loads the
    per-problem specialisations, again bitwise equal."""
    import torch
    spec, x = build_model(name)
    dm, ctx, plan = run_model(spec, x)
    before = {L["out"]: dm.read_raw(L["out"]) for L in spec["layers"]}
    reused = sum(1 for b in plan if b[3] == 1)
    assert ctx.promote() == reused > 0
    assert all(ctx.kernel_is_loaded(b[1]) for b in plan)
    stream = torch.cuda.current_stream().cuda_stream
    ctx.infer(stream)
    ctx.sync()
    errs = teacher_forced_errors(dm, spec, x)
    assert max(e for _, _, e in errs) <= TOL
    after = {L["out"]: dm.read_raw(L["out"]) for L in spec["layers"]}
    for L in spec["layers"]:
        if L["op"] in ("conv", "linear"):
            np.testing.assert_array_equal(before[L["out"]], after[L["out"]])
    n = ctx.promote(target_catalog=1)
    o = OP.execution_plan(OP.problems_from_spec(spec), reuse=False, catalog="tuned")
    assert n > 0 and all(ctx.kernel_is_loaded(k) for k in o["loaded"])
    ctx.infer(stream)
    ctx.sync()
    if dm.ws_bytes:
        # ResNet-50's stem was folded (D16: another k order); its
        # specialised solution runs it unfolded, so from the stem on the outputs
        # are compared with the oracle (the unfolded bitwise check is
        # test_tuned_catalog_specialised_kernels under PASK_STEM_FOLD=0)
        errs = teacher_forced_errors(dm, spec, x)
        assert max(e for _, _, e in errs) <= TOL
    else:
        for L in spec["layers"]:
            np.testing.assert_array_equal(after[L["out"]], dm.read_raw(L["out"]))
    ctx.close()


@pytest.mark.parametrize("graph", [0, 1])
def test_branches_bitwise(graph):
    """cfg.branches (D9): ResNet-50's downsample convs on a second
    stream give bitwise the same outputs as the one-stream issue, for the cold
    direct issue and for captured-graph replays."""
    import torch
    spec, x = build_model("resnet50")
    dm, ctx, _ = run_model(spec, x, cfg=P.config(branches=1, graph=graph, packaging=2))
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(3):          # hot: graph capture on the 2nd call when graph=1
        ctx.infer(s)
    ctx.sync()
    got = {L["out"]: dm.read_raw(L["out"]) for L in spec["layers"]}
    ctx.close()
    dm2, ctx2, _ = run_model(spec, x)
    for L in spec["layers"]:
        np.testing.assert_array_equal(got[L["out"]], dm2.read_raw(L["out"]))
    ctx2.close()


_STORE_MODE_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
from tests.gpu_harness import run_model
from workloads import build_model
spec, x = build_model(sys.argv[2])
dm, ctx, _ = run_model(spec, x)
np.savez(sys.argv[3], **{L["out"]: dm.read_raw(L["out"]) for L in spec["layers"]})  # bf16 -> f64 is exact
ctx.close()
"""


@pytest.mark.parametrize("name", ["resnet50", "bert_base"])
def test_direct_and_staged_epilogue_bitwise(name, tmp_path):
    """The direct epilogue (c_tma = 2: 256-bit stores from registers, the default)
    and the staged one (smem tile + TMA tensor store, PASK_STAGED_STORE=1) write
    bitwise identical outputs for every layer: same arithmetic, only the store
    path differs (DESIGN.md §6 K6 epilogue step 5).  Each mode runs in its own
    process (the switch is read once per process)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    outs = {}
    for mode in ("direct", "staged"):
        env = dict(os.environ)
        env.pop("PASK_STAGED_STORE", None)
        if mode == "staged":
            env["PASK_STAGED_STORE"] = "1"
        path = str(tmp_path / f"{mode}.npz")
        r = subprocess.run([sys.executable, "-c", _STORE_MODE_CHILD, root, name, path], env=env,
                           capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-2000:]
        outs[mode] = np.load(path)
    for k in outs["direct"].files:
        np.testing.assert_array_equal(outs["direct"][k], outs["staged"][k], err_msg=k)
