"""C-ABI boundary tests that need no GPU (-m "not gpu").

* libpask.so loads and exports every function declared in include/pask.h;
* the ctypes mirror of every struct has the C layout (offsets / sizes checked
  against a compiled C probe of the header);
* the host planner (pask_plan) reproduces the plan oracle bit for bit on all
  four configs and on random graphs, for categorical / naive / no-reuse /
  milestone configurations;
* errors fail loudly: EUNSUPPORTED for an inapplicable solution, EINVAL for a
  malformed graph, ECUDA (driver unavailable) from pask_create without a GPU.
"""
import ctypes as C
import os
import random
import re
import subprocess

import pytest

from oracle import plan as OP
from paper_conf_dac_huangdxz25_b200 import build as pbuild
from paper_conf_dac_huangdxz25_b200 import pask as P
from paper_conf_dac_huangdxz25_b200.model import DeviceModel
from workloads import build_model
from workloads.models import _Builder

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "pask.h")
TEST_HEADER = os.path.join(ROOT, "include", "pask_testing.h")


@pytest.fixture(scope="module", autouse=True)
def built():
    pbuild.build()


def header_functions(path=HEADER):
    src = open(path).read()
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(pask_\w+)\s*\(", src, re.M)))


def _exported(path):
    out = subprocess.run(["nm", "-D", "--defined-only", path], capture_output=True, text=True).stdout
    return set(re.findall(r" T (pask_\w+)", out))


def test_exports_every_declared_symbol():
    """The product library exports exactly include/pask.h; the test-only build
    exports pask.h plus include/pask_testing.h (the fake driver is not in the
    product library)."""
    names = header_functions()
    test_names = header_functions(TEST_HEADER)
    assert len(names) >= 18
    assert set(names) == _exported(P.LIB_PATH), (set(names) ^ _exported(P.LIB_PATH))
    assert set(names) | set(test_names) == _exported(P.TESTING_LIB_PATH)
    lib = P.lib()
    for n in names:
        assert hasattr(lib, n)
    assert set(P.EXPORTS) == set(names)
    assert set(P.TEST_EXPORTS) == set(test_names)
    assert lib.pask_version() >= 100


def test_struct_layouts_match_header(tmp_path):
    probe = tmp_path / "probe.c"
    structs = {"pask_tensor": P.Tensor, "pask_node": P.Node, "pask_graph": P.Graph,
               "pask_config": P.Config, "pask_binding": P.Binding, "pask_stats_t": P.Stats}
    lines = ['#include <stdio.h>', '#include <stddef.h>', f'#include "{HEADER}"', "int main(){"]
    for cname, py in structs.items():
        lines.append(f'printf("{cname} size %zu\\n", sizeof({cname}));')
        for f, _ in py._fields_:
            lines.append(f'printf("{cname}.{f} %zu\\n", offsetof({cname}, {f}));')
    lines.append("return 0;}")
    probe.write_text("\n".join(lines))
    exe = tmp_path / "probe"
    subprocess.run(["gcc", "-o", str(exe), str(probe)], check=True)
    got = dict(l.rsplit(" ", 1) for l in subprocess.run([str(exe)], capture_output=True,
                                                        text=True).stdout.splitlines())
    for cname, py in structs.items():
        assert int(got[f"{cname} size"]) == C.sizeof(py), cname
        for f, _ in py._fields_:
            assert int(got[f"{cname}.{f}"]) == getattr(py, f).offset, (cname, f)


CFGS = [dict(), dict(search=1), dict(reuse=0), dict(milestone=5), dict(milestone=1000),
        dict(catalog=1), dict(catalog=1, reuse=0), dict(catalog=1, search=1)]


@pytest.mark.parametrize("name", ["tiny_cnn", "resnet50", "mobilenet_v2", "bert_base", "bert_base_fa"])
def test_planner_matches_oracle_on_models(name):
    spec, _ = build_model(name)
    dm = DeviceModel(spec, alloc=False)
    probs = OP.problems_from_spec(spec)
    for kw in CFGS:
        cfg = P.config(**kw)
        got, st = P.plan(dm.graph, cfg)
        exp = OP.execution_plan(probs, reuse=bool(cfg.reuse),
                                search="naive" if cfg.search else "categorical",
                                milestone=cfg.milestone,
                                catalog="tuned" if cfg.catalog else "generic")
        assert [tuple(b) for b in got] == [tuple(b) for b in exp["bindings"]], kw
        assert (st["queries"], st["hits"], st["lookups"]) == \
            (exp["queries"], exp["hits"], exp["lookups"])
        assert st["kernels_loaded"] == len(exp["loaded"])


def _random_spec(rng, idx):
    b = _Builder(f"r{idx}", idx)
    c = rng.choice([3, 8, 16])
    hw = rng.choice([9, 14, 16])
    t = b.layout(b.input((1, c, hw, hw), "f32"))
    for _ in range(rng.randint(1, 9)):
        _, ch, h, _ = b.shape(t)
        kind = rng.choice(["conv", "conv", "conv1", "dw", "pool", "gpool"])
        if kind == "conv" and h >= 3:
            r = rng.choice([1, 3, 5]) if h >= 5 else 1
            t = b.conv(t, rng.choice([8, 16, 24]), r, rng.choice([1, 2]), r // 2, act="relu")
        elif kind == "conv1":
            t = b.conv(t, rng.choice([8, 16, 32]), 1, act="relu")
        elif kind == "dw" and h >= 3:
            t = b.conv(t, ch, 3, 1, 1, groups=ch, act="relu6")
        elif kind == "pool" and h >= 3:
            t = b.pool(t, rng.choice(["max", "avg"]), 3, 2, 1)
        elif kind == "gpool":
            t = b.pool(t, rng.choice(["max", "avg"]), "global")
            break
    t = b.linear(t, 10)
    t = b.softmax(t)
    b.outputs = [t]
    return b.spec()


def test_planner_matches_oracle_on_random_graphs():
    rng = random.Random(11)
    n_ok = 0
    for i in range(120):
        spec = _random_spec(rng, i)
        probs = OP.problems_from_spec(spec)
        for kw in CFGS[:3]:
            cfg = P.config(**kw)
            try:
                exp = OP.execution_plan(probs, reuse=bool(cfg.reuse),
                                        search="naive" if cfg.search else "categorical")
            except ValueError:
                with pytest.raises(P.PaskError) as ei:     # both sides reject the graph
                    P.plan(DeviceModel(spec, alloc=False).graph, cfg)
                assert ei.value.code in (P.EUNSUPPORTED, P.EINVAL)
                continue
            got, _ = P.plan(DeviceModel(spec, alloc=False).graph, cfg)
            assert [tuple(b) for b in got] == [tuple(b) for b in exp["bindings"]]
            n_ok += 1
    assert n_ok > 200


def test_unsupported_and_invalid_fail_loudly():
    spec, _ = build_model("tiny_cnn")
    dm = DeviceModel(spec, alloc=False, solutions={1: P.K_CONV_1X1})   # 3x3 conv on the 1x1 kernel
    with pytest.raises(P.PaskError) as ei:
        P.plan(dm.graph)
    assert ei.value.code == P.EUNSUPPORTED and "node 1" in str(ei.value)
    dm = DeviceModel(spec, alloc=False)
    dm._nodes[2].in0 = 999          # tensor index out of range
    dm._make_graph(None, 0)
    with pytest.raises(P.PaskError) as ei:
        P.plan(dm.graph)
    assert ei.value.code == P.EINVAL and "node 2" in str(ei.value)
    dm = DeviceModel(spec, alloc=False)
    dm._nodes[1].k = 17             # conv output channels mismatch the out tensor
    dm._make_graph(None, 0)
    with pytest.raises(P.PaskError) as ei:
        P.plan(dm.graph)
    assert ei.value.code == P.EINVAL


def test_catalog_introspection_and_workspace():
    lib = P.lib()
    assert lib.pask_num_kernels() == len(OP.KERNEL_NAMES) == P.NUM_KERNELS + len(OP.SPECS)
    assert [P.kernel_name(k) for k in range(P.num_kernels())] == OP.KERNEL_NAMES
    assert P.kernel_name(99) == ""
    # the only workspace is the stem fold (D16): ResNet-50's 7x7 s2
    # C = 3 stem reads Y [n][P + R2 - 1][Q][64] and weights [K][R2][64], R2 = 4;
    # MobileNetV2's 3x3 s2 stem and the tiny CNN's 3x3 s1 conv would not take
    # fewer k-blocks folded (2 vs 2, 3 vs 2), BERT has no conv
    al = lambda b: (b + 255) // 256 * 256
    for batch in (1, 3):
        spec, _ = build_model("resnet50", batch=batch)
        assert P.workspace_bytes(DeviceModel(spec, alloc=False).graph) == \
            al(batch * (112 + 3) * 112 * 64 * 2) + al(64 * 4 * 64 * 2)
    for name in ("mobilenet_v2", "tiny_cnn", "bert_base"):
        spec, _ = build_model(name)
        assert P.workspace_bytes(DeviceModel(spec, alloc=False).graph) == 0, name


@pytest.mark.skipif(os.path.exists("/dev/nvidia0"), reason="GPU present")
def test_create_without_driver_fails_loudly():
    with pytest.raises(P.PaskError) as ei:
        P.Context(0)
    assert ei.value.code == P.ECUDA
    assert "driver unavailable" in str(ei.value)


def test_kernel_function_families():
    """pask_kernel_function: the CUfunction serving each solution per packaging
    (D8).  Packaging 0/1: the solution's own entry; packaging 2: the
    memory-bound family entry or the generic implicit-GEMM entry."""
    mem = {P.K_LAYOUT, P.K_CONV_DW, P.K_POOL, P.K_POOL_GAVG, P.K_SOFTMAX, P.K_LAYERNORM, P.K_GEMV}
    contract = {P.K_CONV_IGEMM, P.K_CONV_1X1, P.K_GEMM}
    for k in range(P.num_kernels()):
        assert P.function_name(k, 0) == P.function_name(k, 1) == P.kernel_name(k)
        want = "pask_mem" if k in mem else "pask_conv_igemm" if k in contract else P.kernel_name(k)
        assert P.function_name(k, 2) == want
        assert P.function_name(k, 3) == ("pask_all" if k in mem | contract else P.kernel_name(k))
    assert P.function_name(-1, 2) == "" and P.function_name(P.num_kernels(), 0) == ""
