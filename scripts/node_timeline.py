"""Per-layer GPU timeline of one hot inference from the kernels' own timeline
stamps (pask_config.timeline: first-CTA start / last-CTA end, %globaltimer),
under the bench's issue mode (CUDA-graph replay, PDL, branches), L2 flushed
before each inference.  Prints per node: start, end, the interval, and its
charge on the critical path (end minus the latest earlier end: the time by
which the node extended the inference), then per solution totals.

    python scripts/node_timeline.py [model] [--batch B] [--reps N] [--direct]
"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_dac_huangdxz25_b200 import build as pbuild  # noqa: E402
from paper_conf_dac_huangdxz25_b200 import pask as P  # noqa: E402
from paper_conf_dac_huangdxz25_b200.model import DeviceModel  # noqa: E402
from workloads import build_model  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("model", nargs="?", default="resnet50")
    ap.add_argument("--batch", type=int, default=1)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--direct", action="store_true", help="direct issue instead of graph replay")
    a = ap.parse_args()
    pbuild.build()
    spec, x = build_model(a.model, **({"batch": a.batch} if a.batch != 1 else {}))
    dm = DeviceModel(spec)
    dm.set_input(x)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    ctx = P.Context(0, P.config(packaging=2, branches=1, graph=0 if a.direct else 1, timeline=1))
    plan = ctx.load_model(dm.graph)
    s = torch.cuda.current_stream().cuda_stream
    n = len(spec["layers"])
    runs = []
    for r in range(a.reps + 3):
        flush.zero_()
        ctx.infer(s)
        ctx.sync()
        if r >= 3:
            runs.append((ctx.node_intervals(), ctx.stats()))
    ctx.close()
    med = lambda v: statistics.median(v)  # noqa: E731
    print(f"{a.model} batch {a.batch} ({'direct' if a.direct else 'graph'}), median of {a.reps}: "
          f"busy {med([st['gpu_busy_ns'] for _, st in runs]) / 1e3:.1f} us, kernel span "
          f"{med([st['kernel_span_ns'] for _, st in runs]) / 1e3:.1f} us")
    print(f"{'node':>4} {'solution':22s} {'start':>8} {'end':>8} {'dur':>7} {'charge':>7}  layer")
    per_sol = {}
    for i in range(n):
        st_ = med([iv[i][0] for iv, _ in runs]) / 1e3
        en_ = med([iv[i][1] for iv, _ in runs]) / 1e3
        ch = []
        for iv, _ in runs:
            prev = max([iv[j][1] for j in range(n) if iv[j][1] < iv[i][1]] or [iv[i][0]])
            ch.append(max(0, iv[i][1] - max(prev, iv[i][0])) / 1e3)
        ch_ = med(ch)
        L = spec["layers"][i]
        desc = L["op"] + (f" {tuple(L['w'].shape)} s{L['stride'][0]}" if L["op"] == "conv" else "")
        name = P.kernel_name(plan[i][2])
        d = per_sol.setdefault(name, [0, 0.0])
        d[0] += 1
        d[1] += ch_
        print(f"{i:4d} {name:22s} {st_:8.2f} {en_:8.2f} {en_ - st_:7.2f} {ch_:7.2f}  {desc}")
    print("per solution: launches, critical-path charge us, us per launch")
    for k, (cnt, tot) in sorted(per_sol.items(), key=lambda kv: -kv[1][1]):
        print(f"  {k:22s} {cnt:4d} {tot:8.1f} {tot / cnt:6.2f}")


if __name__ == "__main__":
    main()
