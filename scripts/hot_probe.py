"""Hot-path A/B probe: the bench's hot loop (packaging 3 cold start, repacked into
the families by pask_promote, graph replay, branches, L2 flushed before every
inference, CUDA events around each inference) on one model, printing mean and
median ms.  Run it in separate processes per experiment switch (the runtime
reads its switches once per process):
    PASK_NO_SPAN_EVENTS=1 python scripts/hot_probe.py resnet50 --steps 400
"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_dac_huangdxz25_b200 import pask as P  # noqa: E402
from paper_conf_dac_huangdxz25_b200.model import DeviceModel  # noqa: E402
from workloads import build_model  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("model", nargs="?", default="resnet50")
ap.add_argument("--batch", type=int, default=1)
ap.add_argument("--steps", type=int, default=400)
a = ap.parse_args()
spec, x = build_model(a.model, **({"batch": a.batch} if a.batch != 1 else {}))
dm = DeviceModel(spec)
dm.set_input(x)
flush_buf = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
stream = torch.cuda.current_stream()
sp = stream.cuda_stream
ctx = P.Context(0, P.config(packaging=3, graph=1, branches=1))
ctx.load_model(dm.graph, plan=False)
ctx.infer(sp)
ctx.sync()
ctx.promote()
for _ in range(10):
    flush_buf.zero_()
    ctx.infer(sp)
torch.cuda.synchronize()
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
for i in range(a.steps):
    flush_buf.zero_()
    ev[i][0].record(stream)
    ctx.infer(sp)
    ev[i][1].record(stream)
torch.cuda.synchronize()
ms = [s.elapsed_time(e) for s, e in ev]
env = ",".join(f"{k}={v}" for k, v in os.environ.items() if k.startswith("PASK_")) or "default"
print(f"{a.model} b{a.batch} [{env}] hot mean {statistics.mean(ms):.4f} median {statistics.median(ms):.4f} ms")
ctx.close()
