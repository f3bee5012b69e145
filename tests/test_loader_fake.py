"""T2: loader / issuer host logic on CPU through the fake driver
(include/pask_testing.h).  No GPU: every driver call goes to an in-library
fake that sleeps on loads and records loads and launches.

Checks, for every proactive / interleave / packaging / reuse mode:
* uploads happen once per planned kernel, in first-use order;
* no launch precedes the completed load of its kernel;
* the launch sequence is the plan's bound kernel of each node, in node order;
* a failed load propagates as PASK_ECUDA naming the kernel (no fallback);
* nothing deadlocks (pytest-timeout), including destroy with pending loads.
"""
import os
import pytest

from oracle import plan as OP
from paper_conf_dac_huangdxz25_b200 import build as pbuild
from paper_conf_dac_huangdxz25_b200 import pask as P
from paper_conf_dac_huangdxz25_b200.model import DeviceModel
from workloads import build_model

pytestmark = pytest.mark.timeout(120)


@pytest.fixture(scope="module", autouse=True)
def built():
    pbuild.build()
    P.use_testing_library(True)     # libpask_testing.so: the product library has no fake driver
    yield
    P.test_fake_driver(False)
    P.use_testing_library(False)


MODES = [
    dict(proactive=2), dict(proactive=1), dict(proactive=1, interleave=1), dict(proactive=0),
    dict(proactive=2, packaging=1), dict(proactive=2, reuse=0), dict(proactive=1, search=1),
    dict(proactive=0, reuse=0, catalog=1), dict(proactive=2, catalog=1),
    dict(proactive=2, packaging=2), dict(proactive=1, packaging=2), dict(proactive=0, packaging=2),
    dict(proactive=2, packaging=3), dict(proactive=1, packaging=3), dict(proactive=0, packaging=3),
]

# packaging 2 (D8): the CUfunction that serves a catalog solution, as
# the fake driver logs it (the memory family entry `pask_mem` is id 63)
FAM_MEM = 63
FAM_ALL = 62   # packaging 3 (D10): `pask_all`
MEM_SOLUTIONS = {P.K_LAYOUT, P.K_CONV_DW, P.K_POOL, P.K_POOL_GAVG, P.K_SOFTMAX, P.K_LAYERNORM, P.K_GEMV}
CONTRACT_SOLUTIONS = {P.K_CONV_IGEMM, P.K_CONV_1X1, P.K_GEMM}


def function_of(k, packaging):
    if packaging == 3:
        return FAM_ALL if k in MEM_SOLUTIONS | CONTRACT_SOLUTIONS else k
    if packaging != 2:
        return k
    if k in MEM_SOLUTIONS:
        return FAM_MEM
    if k in CONTRACT_SOLUTIONS:
        return P.K_CONV_IGEMM
    return k


def dedup(seq):
    out = []
    for x in seq:
        if x not in out:
            out.append(x)
    return out


@pytest.mark.parametrize("name", ["tiny_cnn", "resnet50", "bert_base", "bert_base_fa"])
@pytest.mark.parametrize("mode", MODES, ids=[str(m) for m in MODES])
def test_load_order_and_launch_safety(name, mode):
    spec, _ = build_model(name)
    dm = DeviceModel(spec, alloc=False)
    P.test_fake_driver(True, load_us=300)
    ctx = P.Context(0, P.config(**mode))
    plan = ctx.load_model(dm.graph)
    for _ in range(2):                      # cold, then hot
        ctx.infer(0)
        ctx.sync()
    st = ctx.stats()
    ctx.close()
    log = P.test_fake_log()
    loads = [k for k, kind in log if kind == 0]
    launches = [(k, kind) for k, kind in log if kind != 0]
    exp = OP.execution_plan(OP.problems_from_spec(spec), reuse=bool(mode.get("reuse", 1)),
                            search="naive" if mode.get("search") else "categorical",
                            catalog="tuned" if mode.get("catalog") else "generic")
    pk = mode.get("packaging", 0)
    want = dedup(function_of(k, pk) for k in exp["loaded"])
    assert loads == want                                            # once each, first-use order
    assert all(kind == 1 for _, kind in launches)                   # never before its load
    bound = [function_of(b[2], pk) for b in plan]
    assert [k for k, _ in launches] == bound + bound                # node order, 2 inferences
    assert st["kernels_loaded"] == len(want)
    assert st["launches"] == 2 * len(bound)
    if mode.get("proactive", 2) == 2:
        assert st["load_exposed_ns"] == 0                           # all uploads inside load_model


@pytest.mark.parametrize("mode", [dict(proactive=2), dict(proactive=1), dict(proactive=0),
                                  dict(proactive=1, interleave=1)])
def test_failed_load_propagates(mode):
    spec, _ = build_model("resnet50")
    dm = DeviceModel(spec, alloc=False)
    P.test_fake_driver(True, load_us=100, fail_kernel=P.K_CONV_IGEMM)
    ctx = P.Context(0, P.config(**mode))
    with pytest.raises(P.PaskError) as ei:
        ctx.load_model(dm.graph)
        ctx.infer(0)
    assert ei.value.code == P.ECUDA
    assert "pask_conv_igemm" in str(ei.value) and "CUDA_ERROR_INVALID_IMAGE" in str(ei.value)
    ctx.close()
    launched = [k for k, kind in P.test_fake_log() if kind != 0]
    assert P.K_CONV_IGEMM not in launched
    # only the layout node (before the first conv) may have been issued
    assert set(launched) <= {P.K_LAYOUT}


def test_destroy_with_pending_loads_and_reuse_across_models():
    P.test_fake_driver(True, load_us=2000)
    spec, _ = build_model("resnet50")
    dm = DeviceModel(spec, alloc=False)
    ctx = P.Context(0, P.config(proactive=1))
    ctx.load_model(dm.graph)
    ctx.close()                              # joins the loader with loads still queued
    # a second model in a fresh context after a first one: no stale state
    P.test_fake_driver(True, load_us=0)
    ctx = P.Context(0, P.config())
    spec2, _ = build_model("mobilenet_v2")
    ctx.load_model(DeviceModel(spec2, alloc=False).graph)
    ctx.infer(0)
    ctx.sync()
    assert ctx.stats()["kernels_loaded"] == 6
    ctx.close()


def test_rebinding_inputs_relowers_without_reloading():
    P.test_fake_driver(True, load_us=0)
    spec, _ = build_model("tiny_cnn")
    dm = DeviceModel(spec, alloc=False)
    ctx = P.Context(0, P.config())
    ctx.load_model(dm.graph)
    ctx.infer(0)
    ctx.infer(0, inputs=[1 << 22], outputs=[1 << 23])   # new buffers: parameters re-encoded
    ctx.sync()
    st = ctx.stats()
    ctx.close()
    assert st["kernels_loaded"] == 5 and st["launches"] == 14
    assert sum(1 for _, kind in P.test_fake_log() if kind == 0) == 5


def test_state_errors():
    P.test_fake_driver(True)
    ctx = P.Context(0, P.config())
    with pytest.raises(P.PaskError) as ei:
        ctx.infer(0)
    assert ei.value.code == P.ESTATE
    spec, _ = build_model("tiny_cnn")
    dm = DeviceModel(spec, alloc=False)
    ctx.load_model(dm.graph)
    with pytest.raises(P.PaskError) as ei:
        ctx.load_model(dm.graph)             # one model per context
    assert ei.value.code == P.ESTATE
    ctx.close()


def test_promote_loads_skipped_solutions_in_order():
    """Idle-interval loading: the solutions Algorithm 1 skipped are
    uploaded after the cold inference and the reused nodes rebound to them."""
    P.test_fake_driver(True, load_us=0)
    spec, _ = build_model("resnet50")
    dm = DeviceModel(spec, alloc=False)
    ctx = P.Context(0, P.config())
    plan = ctx.load_model(dm.graph)
    ctx.infer(0)
    n = ctx.promote()
    assert n == sum(1 for b in plan if b[3] == 1) == 34            # every reused node
    ctx.infer(0)
    ctx.sync()
    log = P.test_fake_log()
    loads = [k for k, kind in log if kind == 0]
    assert loads[5:] == [P.K_CONV_1X1, P.K_POOL_GAVG]             # skipped s*, first-use order
    hot = [k for k, kind in log if kind == 1][len(plan):]
    assert hot == [b[1] for b in plan]                             # every node on its s*
    assert ctx.promote() == 0                                      # idempotent
    n_tuned = ctx.promote(target_catalog=1)
    assert n_tuned == 53                                           # every conv -> its specialisation
    ctx.close()


def expected_side_nodes(spec):
    """Restatement of the branches rule (D9): node i goes to the side
    stream when it reads an earlier node's output but not node i-1's (its last
    producer is before i-1), and none of its producers is itself a side node."""
    producer, side = {}, []
    for i, L in enumerate(spec["layers"]):
        srcs = [t for t in list(L["inputs"]) + ([L["res"]] if L.get("res") else []) if t in producer]
        if srcs:
            prod = max(producer[t] for t in srcs)
            if prod < i - 1 and not any(producer[t] in side for t in srcs):
                side.append(i)
        producer[L["out"]] = i
    return side


@pytest.mark.parametrize("name", ["resnet50", "mobilenet_v2", "bert_base", "tiny_cnn"])
def test_branches_issue_side_nodes_after_their_producer(name):
    """cfg.branches: in the captured hot graph the side nodes (ResNet-50's four
    downsample convs; none in the other configs) launch on the second stream
    right after their last producer, everything else on the main stream in node
    order; the cold direct issue does the same on the context's side stream."""
    spec, _ = build_model(name)
    dm = DeviceModel(spec, alloc=False)
    P.test_fake_driver(True, load_us=0)
    ctx = P.Context(0, P.config(branches=1, graph=1))
    plan = ctx.load_model(dm.graph)
    for _ in range(3):   # cold direct issue, then capture (2nd call), then a replay
        ctx.infer(0)
    ctx.sync()
    ctx.close()
    log = [(k, kind) for k, kind in P.test_fake_log() if kind != 0]
    n = len(spec["layers"])
    assert len(log) == 2 * n                      # the replay launches nothing in the fake
    side = expected_side_nodes(spec)
    assert len(side) == (4 if name == "resnet50" else 0)
    # expected issue order: main nodes in order, each side node right after its producer
    producer = {L["out"]: i for i, L in enumerate(spec["layers"])}
    order = []
    for i, L in enumerate(spec["layers"]):
        if i in side:
            continue
        order.append((i, 1))
        for j in side:
            srcs = [t for t in list(spec["layers"][j]["inputs"]) +
                    ([spec["layers"][j]["res"]] if spec["layers"][j].get("res") else []) if t in producer]
            if max(producer[t] for t in srcs) == i:
                order.append((j, 3))
    bound = [b[2] for b in plan]
    for launches in (log[:n], log[n:]):           # cold direct issue, then the captured sequence
        assert [(k, kind) for k, kind in launches] == [(bound[i], kind) for i, kind in order]
        assert sum(1 for _, kind in launches if kind == 3) == len(side)


@pytest.mark.parametrize("packaging", [2, 3])
@pytest.mark.parametrize("name,variant", [("tiny_cnn", "cnng"), ("resnet50", "cnnf"), ("mobilenet_v2", "dwg"),
                                          ("bert_base", "tf"), ("bert_base_fa", "tf")])
def test_family_variant_covers_the_plan(name, variant, packaging):
    """Packaging 2 (D8): the families object is loaded in the smallest
    variant whose memory-bound cases cover every solution the plan binds (CNN:
    layout / pool / softmax / GEMV; layout / depthwise / global-average pool /
    softmax / GEMV for MobileNetV2; softmax / LayerNorm for BERT) and whose contraction entry compiles the paths the
    plan's contraction nodes take (D13: split-K / gather / im2col for
    the CNNs -- ResNet-50, its stem folded (D16), no gather --, staged epilogues for MobileNetV2's N = 24 layers, MN-major B and
    GELU for BERT); one code object, whose bytes are that variant's image
    (attention keeps its own object).  Packaging 3 (D10) picks the single-entry
    variant pask_single_<v> with the same masks: one CUfunction."""
    from paper_conf_dac_huangdxz25_b200 import build as B
    spec, _ = build_model(name)
    dm = DeviceModel(spec, alloc=False)
    P.test_fake_driver(True, load_us=0)
    ctx = P.Context(0, P.config(packaging=packaging))
    plan = ctx.load_model(dm.graph)
    ctx.infer(0)
    ctx.sync()
    st = ctx.stats()
    ctx.close()
    mask = B.FAMILY_VARIANTS[f"pask_families_{variant}"][0]
    kinds = {P.K_LAYOUT: 0, P.K_CONV_DW: 1, P.K_POOL: 2, P.K_POOL_GAVG: 3, P.K_SOFTMAX: 4, P.K_LAYERNORM: 5,
             P.K_GEMV: 6}
    need = {kinds[b[2]] for b in plan if b[2] in kinds}     # the bound solutions (D13)
    assert all((mask >> kd) & 1 for kd in need)
    # variants are tried smallest first; the ones before the chosen one lack a
    # memory case or a contraction path (D13) the plan needs
    names = list(B.FAMILY_VARIANTS)
    assert names.index(f"pask_families_{variant}") <= names.index("pask_families_dw")
    own = [b[2] for b in plan if b[2] == P.K_ATTENTION][:1]
    stem = "pask_families" if packaging == 2 else "pask_single"
    assert B.SINGLE_VARIANTS[f"pask_single_{variant}"] == B.FAMILY_VARIANTS[f"pask_families_{variant}"]
    expect = os.path.getsize(os.path.join(B.BUILD, f"{stem}_{variant}.fatbin"))
    expect += sum(os.path.getsize(os.path.join(B.BUILD, P.kernel_name(k) + ".fatbin")) for k in own)
    assert st["code_bytes_loaded"] == expect
    assert st["kernels_loaded"] == (2 if packaging == 2 else 1) + len(own)


@pytest.mark.parametrize("name,variant", [("resnet50", "cnnf"), ("mobilenet_v2", "dwg"), ("bert_base", "tf")])
def test_single_entry_repack(name, variant):
    """DESIGN.md D15: packaging 3 cold-starts on pask_single_<v> (one upload);
    pask_promote then repacks -- uploads pask_families_<v> (the same masks; one
    more parse, two more functions), moves every family-served node and leaves
    the plan alone; the next inferences issue from the family entries."""
    from paper_conf_dac_huangdxz25_b200 import build as B
    spec, _ = build_model(name)
    dm = DeviceModel(spec, alloc=False)
    P.test_fake_driver(True, load_us=0)
    ctx = P.Context(0, P.config(packaging=3, graph=1))
    plan = ctx.load_model(dm.graph)
    ctx.infer(0)
    ctx.sync()
    st0 = ctx.stats()
    fam = {P.K_LAYOUT, P.K_CONV_DW, P.K_POOL, P.K_POOL_GAVG, P.K_SOFTMAX, P.K_LAYERNORM, P.K_GEMV,
           P.K_CONV_IGEMM, P.K_CONV_1X1, P.K_GEMM}
    n = ctx.promote()
    assert n == sum(1 for b in plan if b[2] in fam)
    st1 = ctx.stats()
    assert st1["kernels_loaded"] == st0["kernels_loaded"] + 2
    single = os.path.getsize(os.path.join(B.BUILD, f"pask_single_{variant}.fatbin"))
    families = os.path.getsize(os.path.join(B.BUILD, f"pask_families_{variant}.fatbin"))
    assert st1["code_bytes_loaded"] - st0["code_bytes_loaded"] == families
    assert st0["code_bytes_loaded"] >= single
    assert all(ctx.kernel_is_loaded(b[2]) for b in plan)
    for _ in range(3):                       # direct issue, capture, replay
        ctx.infer(0)
        ctx.sync()
    ctx.close()


def test_create_refuses_a_context_of_another_device():
    """pask_create binds `device`'s primary context; a calling thread
    whose current context belongs to another device is refused (the ctx could not
    use the caller's device pointers) instead of silently issuing there."""
    P.test_fake_driver(True)
    P.test_fake_knob(P.FAKE_CURRENT_DEVICE, 0)
    with pytest.raises(P.PaskError) as ei:
        P.Context(1, P.config())
    assert ei.value.code == P.EINVAL and "device 0" in str(ei.value)
    ctx = P.Context(0, P.config())            # the current device's ctx is fine
    ctx.close()
    P.test_fake_knob(P.FAKE_CURRENT_DEVICE, 1)
    ctx = P.Context(1, P.config())            # ... and so is device 1 once it is current
    ctx.close()


def test_overlapping_tensors_run_on_one_stream():
    """branch dependencies are tracked by tensor index, so a graph whose
    tensors overlap in memory (or that is rebound onto an overlapping buffer)
    issues everything on one stream."""
    spec, _ = build_model("resnet50")
    dm = DeviceModel(spec, alloc=False)
    P.test_fake_driver(True)
    ctx = P.Context(0, P.config(branches=1))
    ctx.load_model(dm.graph)
    ctx.infer(0)
    ctx.sync()
    assert sum(1 for _, kind in P.test_fake_log() if kind == 3) == 4       # ResNet-50 downsample convs
    # rebind the output (softmax) onto the first activation: the tensors now overlap
    first_act = dm._tensors[dm.index[spec["layers"][0]["out"]]].dptr
    P.test_fake_driver(True)
    ctx.infer(0, outputs=[first_act])
    ctx.sync()
    ctx.close()
    assert sum(1 for _, kind in P.test_fake_log() if kind == 3) == 0
    # a graph that aliases from the start
    dm2 = DeviceModel(spec, alloc=False)
    dm2._tensors[dm2.index[spec["layers"][5]["out"]]].dptr = dm2._tensors[dm2.index[spec["layers"][1]["out"]]].dptr
    dm2._make_graph(dm2.graph.workspace, dm2.ws_bytes)
    P.test_fake_driver(True)
    ctx = P.Context(0, P.config(branches=1))
    ctx.load_model(dm2.graph)
    ctx.infer(0)
    ctx.sync()
    ctx.close()
    assert sum(1 for _, kind in P.test_fake_log() if kind == 3) == 0


def test_cluster_size_capped_by_device_occupancy():
    """the tiny CNN's FC (M = 1, K = 16384) on the tcgen05 GEMM plans a
    16-CTA split-K cluster; where the device cannot co-schedule one the node is lowered again
    with at most 8, before it is launched."""
    spec, _ = build_model("tiny_cnn")
    fc = [i for i, L in enumerate(spec["layers"]) if L["op"] == "linear"][0]
    sol = {fc: P.K_GEMM}       # the FC's s* is the GEMV solution; force the tcgen05 GEMM
    for occ, want in ((1, 16), (0, 8)):
        P.test_fake_driver(True)
        P.test_fake_knob(P.FAKE_OCCUPANCY, occ)
        for mode in (dict(), dict(proactive=1), dict(proactive=0)):
            P.test_fake_driver(True)
            P.test_fake_knob(P.FAKE_OCCUPANCY, occ)
            ctx = P.Context(0, P.config(**mode))
            ctx.load_model(DeviceModel(spec, alloc=False, solutions=sol).graph)
            ctx.infer(0)
            ctx.sync()
            st = ctx.stats()
            ctx.close()
            assert st["max_cluster"] == want, mode
            assert P.test_fake_knob(P.FAKE_MAX_CLUSTER_LAUNCHED) == want, mode


def test_timeline_api_states():
    """cfg.timeline: pask_node_intervals returns one (start, end) per node after a
    sync (the fake runs no kernel: all zero, busy 0); without timeline it is
    PASK_ESTATE."""
    spec, _ = build_model("tiny_cnn")
    P.test_fake_driver(True)
    ctx = P.Context(0, P.config(timeline=1))
    ctx.load_model(DeviceModel(spec, alloc=False).graph)
    ctx.infer(0)
    ctx.sync()
    assert ctx.node_intervals() == [(0, 0)] * len(spec["layers"])
    assert ctx.stats()["gpu_busy_ns"] == 0
    ctx.close()
    ctx = P.Context(0, P.config())
    ctx.load_model(DeviceModel(spec, alloc=False).graph)
    ctx.infer(0)
    ctx.sync()
    with pytest.raises(P.PaskError) as ei:
        ctx.node_intervals()
    assert ei.value.code == P.ESTATE
    ctx.close()


def test_primer_outside_the_plan():
    """pask_create's driver primer (D11) uploads its own trivial kernel
    once per context, never a catalog solution, and not with no_prime = 1; the
    model's loads and launches are unchanged by it."""
    spec, _ = build_model("tiny_cnn")
    for no_prime, want in ((0, 1), (1, 0)):
        P.test_fake_driver(True)
        ctx = P.Context(0, P.config(no_prime=no_prime))
        assert P.test_fake_knob(P.FAKE_PRIMER_LOADS) == want
        plan = ctx.load_model(DeviceModel(spec, alloc=False).graph)
        ctx.infer(0)
        ctx.sync()
        ctx.close()
        log = P.test_fake_log()
        assert [k for k, kind in log if kind == 1] == [b[2] for b in plan]
