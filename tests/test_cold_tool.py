"""The native cold-start sampler (csrc/tools/pask_cold.cpp) and its model image
(DeviceModel.save_image), without a GPU: the image round-trips the lowered
graph -- pask_cold --plan-only parses it and runs the host planner, whose
bindings must equal the plan oracle's (Algorithm 1) -- and
every weight / bias / gamma / beta plus the input is stored as a blob."""
import json
import os
import subprocess

import numpy as np
import pytest

from oracle import plan as OP
from paper_conf_dac_huangdxz25_b200 import build as pbuild
from paper_conf_dac_huangdxz25_b200.model import DeviceModel
from workloads import build_model

EXE = os.path.join(os.path.dirname(pbuild.__file__), "pask_cold")


@pytest.fixture(scope="module", autouse=True)
def built():
    pbuild.build()


@pytest.mark.parametrize("name", ["tiny_cnn", "resnet50", "mobilenet_v2", "bert_base", "bert_base_fa"])
@pytest.mark.parametrize("cfg", ["reuse=1", "reuse=0", "search=1", "catalog=1"])
def test_image_round_trip_plan(name, cfg, tmp_path):
    spec, x = build_model(name)
    path = str(tmp_path / f"{name}.pmodel")
    DeviceModel(spec, alloc=False).save_image(path, x)
    r = subprocess.run([EXE, path, "--plan-only", "--cfg", cfg], capture_output=True, text=True, timeout=60)
    assert r.returncode == 0, r.stderr
    got = json.loads(r.stdout)
    kw = dict(reuse=cfg != "reuse=0", search="naive" if cfg == "search=1" else "categorical",
              catalog="tuned" if cfg == "catalog=1" else "generic")
    exp = OP.execution_plan(OP.problems_from_spec(spec), **kw)
    assert [tuple(b) for b in got["bindings"]] == [tuple(b) for b in exp["bindings"]]
    assert got["n_nodes"] == len(spec["layers"])
    # blobs: every weight / vector array of the spec once, plus the input
    arrays = [L[k] for L in spec["layers"] for k in ("w", "b", "gamma", "beta") if L.get(k) is not None]
    assert got["n_blobs"] == len(arrays) + 1
    in_bytes = x.size * (4 if spec["inputs"][0][2] == "f32" else 2)
    wbytes = 0
    for L in spec["layers"]:
        for k in ("b", "gamma", "beta"):
            if L.get(k) is not None:
                wbytes += L[k].size * 4
    assert got["blob_bytes"] > wbytes + in_bytes


def test_image_input_blob_is_the_input(tmp_path):
    """The last blob is the graph input in its device dtype (fp32 NCHW image)."""
    spec, x = build_model("tiny_cnn")
    path = str(tmp_path / "t.pmodel")
    DeviceModel(spec, alloc=False).save_image(path, x)
    raw = open(path, "rb").read()
    tail = raw[-((x.nbytes + 255) // 256 * 256):][:x.nbytes]
    assert np.array_equal(np.frombuffer(tail, np.float32).reshape(x.shape), x.astype(np.float32))


def test_bad_image_fails_loudly(tmp_path):
    p = tmp_path / "bad.pmodel"
    p.write_bytes(b"NOTAMODEL" * 8)
    r = subprocess.run([EXE, str(p), "--plan-only"], capture_output=True, text=True, timeout=60)
    assert r.returncode != 0 and "not a pask model image" in r.stderr
