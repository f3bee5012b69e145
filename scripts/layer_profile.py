"""Per-layer GPU time (instrumented, events around each node, no PDL) of one
model at a given batch: achieved TFLOP/s and GB/s per layer, to see which layers
bound throughput.  usage: python scripts/layer_profile.py resnet50 128"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_dac_huangdxz25_b200 import pask as P  # noqa: E402
from paper_conf_dac_huangdxz25_b200.model import DeviceModel  # noqa: E402
from workloads import build_model  # noqa: E402
import bench  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "resnet50"
batch = int(sys.argv[2]) if len(sys.argv) > 2 else 1
spec, x = build_model(name, **({"batch": batch} if batch != 1 else {}))
dm = DeviceModel(spec)
dm.set_input(x)
ctx = P.Context(0, P.config(instrument=1))
plan = ctx.load_model(dm.graph)
s = torch.cuda.current_stream().cuda_stream
acc = None
for it in range(6):
    ctx.infer(s)
    ctx.sync()
    if it >= 1:
        t = ctx.node_times()
        acc = t if acc is None else [a + b for a, b in zip(acc, t)]
n = 5
tot = sum(acc) / n / 1e3
rows = []
for i, L in enumerate(spec["layers"]):
    us = acc[i] / n / 1e3
    by, fl = bench.node_work(spec, i)
    rows.append((us, i, L["op"], P.kernel_name(plan[i][2]), fl / us / 1e6 if us else 0, by / us / 1e3 if us else 0,
                 L.get("w").shape if L.get("w") is not None else ""))
print(f"{name} batch {batch}: sum of node times {tot:.1f} us")
print(f"{'us':>8} {'%':>5} {'node':>4} {'op':8} {'kernel':18} {'TFLOP/s':>8} {'GB/s':>8} shape")
for us, i, op, k, tf, gb, shp in sorted(rows, reverse=True)[:25]:
    print(f"{us:8.1f} {100*us/tot:5.1f} {i:4d} {op:8} {k:18} {tf:8.1f} {gb:8.0f} {shp}")
