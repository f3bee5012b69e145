"""Debug: GPU timeline of one hot inference (PDL on, graph replay as bench.py): per
contraction node, first CTA start / last CTA end and median phase times."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_dac_huangdxz25_b200 import pask as P  # noqa: E402
from paper_conf_dac_huangdxz25_b200.model import DeviceModel  # noqa: E402
from workloads import build_model  # noqa: E402

args = [a for a in sys.argv[1:] if not a.startswith("--")]
CLOCK = "--clock" in sys.argv  # per-CTA phase durations in SM cycles (clock64) instead of %globaltimer
name = args[0] if args else "resnet50"
if CLOCK:
    os.environ["PASK_TRACE_CLOCK"] = "1"
spec, x = build_model(name)
dm = DeviceModel(spec)
dm.set_input(x)
n = len(spec["layers"])
buf = torch.zeros(n * 8 * 4096, dtype=torch.int64, device="cuda")
os.environ["PASK_TRACE_NODE"] = "-1"
os.environ["PASK_TRACE_PTR"] = str(buf.data_ptr())
# the bench configuration: families packaging, hot graph with branches
ctx = P.Context(0, P.config(packaging=2, graph=1, branches=1))
ctx.load_model(dm.graph)
s = torch.cuda.current_stream().cuda_stream
for _ in range(5):
    ctx.infer(s)
ctx.sync()
buf.zero_()
torch.cuda.synchronize()
ctx.infer(s)
ctx.sync()
torch.cuda.synchronize()
tr = buf.view(n, 4096, 8).cpu().numpy().astype(np.float64)
plan = ctx.bindings()
t0 = None
rows = []
for i in range(n):
    t = tr[i]
    t = t[t[:, 0] > 0]
    if not len(t):
        continue
    if t0 is None:
        t0 = t[:, 0].min()
    rel = (t - t0) / 1e3
    rows.append((i, len(t), rel[:, 0].min(), rel[:, 7].max(), np.median(rel[:, 2] - rel[:, 0]),
                 np.median(rel[:, 3] - rel[:, 2]), np.median(rel[:, 5] - rel[:, 3]),
                 np.median(rel[:, 6] - rel[:, 5]), np.median(rel[:, 7] - rel[:, 6]),
                 rel[:, 2].min(), rel[:, 7].max()))
if CLOCK:
    print(f"{'node':>4} {'ctas':>4} | median SM cycles: prologue pre-wait first-load mainloop epi-1st-chunk epi-rest store")
    for i in range(n):
        t = tr[i]
        t = t[t[:, 0] > 0]
        if not len(t):
            continue
        d = lambda a, b: int(np.median(t[:, b] - t[:, a]))
        L = spec["layers"][i]
        desc = L["op"] + (str(tuple(L["w"].shape)) + f" s{L['stride'][0]}" if L["op"] == "conv" else "")
        print(f"{i:4d} {len(t):4d} | {d(0,1):6d} {d(0,2):6d} {d(2,3):6d} {d(3,5):6d} {d(5,4):6d} {d(4,6):6d} {d(6,7):6d}  {desc}")
    sys.exit(0)
prev_end = None
print(f"{'node':>4} {'ctas':>4} {'start':>8} {'end':>8} {'dur':>6} {'gap':>6} {'dep':>6} | pre-wait first-load mainloop epilogue store (median us)")
deps = []
prev_i = None
for r in rows:
    i, nc, st, en = r[:4]
    gap = st - prev_end if prev_end is not None else 0.0
    # dependency latency: previous traced node's last CTA end -> this node's first
    # CTA past griddepcontrol.wait (only meaningful when that node is the predecessor)
    dep = r[9] - prev_end if prev_end is not None else 0.0
    if prev_i is not None and i == prev_i + 1:
        deps.append(dep)
    prev_i = i
    L = spec["layers"][i]
    desc = L["op"] + (str(tuple(L["w"].shape)) + f" s{L['stride'][0]}" if L["op"] == "conv" else "")
    print(f"{i:4d} {nc:4d} {st:8.2f} {en:8.2f} {en-st:6.2f} {gap:6.2f} {dep:6.2f} | {r[4]:5.2f} {r[5]:5.2f} {r[6]:5.2f} {r[7]:5.2f} {r[8]:5.2f}  {desc}")
    prev_end = en
print("total span of traced nodes (us):", rows[-1][3] - rows[0][2])
if deps:
    print(f"dependency latency (prev end -> first wait return), adjacent nodes: median {np.median(deps):.2f} us,"
          f" min {np.min(deps):.2f}, max {np.max(deps):.2f}")
