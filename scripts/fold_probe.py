"""Run a few inferences of a model (packaging 2, as the bench's hot path) for an
ncu capture of one kernel, e.g. the layout (first pask_mem launch):
    ncu --kernel-name pask_mem --launch-count 1 --set full python scripts/fold_probe.py resnet50 --batch 128
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_dac_huangdxz25_b200 import pask as P  # noqa: E402
from paper_conf_dac_huangdxz25_b200.model import DeviceModel  # noqa: E402
from workloads import build_model  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("model", nargs="?", default="resnet50")
ap.add_argument("--batch", type=int, default=1)
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
spec, x = build_model(a.model, **({"batch": a.batch} if a.batch != 1 else {}))
dm = DeviceModel(spec)
dm.set_input(x)
ctx = P.Context(0, P.config(packaging=2))
ctx.load_model(dm.graph)
s = torch.cuda.current_stream().cuda_stream
for _ in range(a.reps):
    ctx.infer(s)
    ctx.sync()
ctx.close()
print("ok")
