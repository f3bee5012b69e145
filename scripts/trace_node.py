"""Debug: per-CTA phase trace of one contraction node of a model (globaltimer)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_dac_huangdxz25_b200 import pask as P  # noqa: E402
from paper_conf_dac_huangdxz25_b200.model import DeviceModel  # noqa: E402
from workloads import build_model  # noqa: E402

name = sys.argv[1]
nodes = [int(a) for a in sys.argv[2:]]
spec, x = build_model(name)
dm = DeviceModel(spec)
dm.set_input(x)
buf = torch.zeros(8 * 4096, dtype=torch.int64, device="cuda")
names = ["start", "prologue", "pdl_wait", "first_full", "mma_done", "accum_seen", "epi_done", "end"]
for node in nodes:
    buf.zero_()
    os.environ["PASK_TRACE_NODE"] = str(node)
    os.environ["PASK_TRACE_PTR"] = str(buf.data_ptr())
    ctx = P.Context(0, P.config(pdl=0))
    ctx.load_model(dm.graph)
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(3):
        ctx.infer(s)
    ctx.sync()
    torch.cuda.synchronize()
    tr = buf.view(-1, 8).cpu().numpy().astype(np.float64)
    tr = tr[tr[:, 0] > 0]
    t0 = tr[:, 0].min()
    rel = (tr - t0) / 1e3
    L = spec["layers"][node]
    print(f"node {node} {L['op']} w{getattr(L.get('w'), 'shape', None)} ctas {len(tr)}")
    for j, nm in enumerate(names):
        col = rel[:, j]
        col = col[tr[:, j] > 0]
        if len(col):
            print(f"   {nm:11s} min {col.min():7.2f}  med {np.median(col):7.2f}  max {col.max():7.2f} us")
    ctx.close()
