"""Debug helper: run configs through the C ABI and print per-layer teacher-forced errors."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_dac_huangdxz25_b200 import pask as P  # noqa: E402
from tests.gpu_harness import run_model, teacher_forced_errors  # noqa: E402
from workloads import build_model  # noqa: E402

for name in sys.argv[1:]:
    spec, x = build_model(name)
    t0 = time.time()
    dm, ctx, plan = run_model(spec, x)
    t1 = time.time()
    errs = teacher_forced_errors(dm, spec, x)
    st = ctx.stats()
    print(f"== {name}: infer+sync {1e3*(t1-t0):.1f} ms  stats {st}")
    for k in range(P.num_kernels()):
        ld, rd, lb = ctx.kernel_timeline(k)
        if ld:
            print(f"  load {P.kernel_name(k):16s} load {ld/1e3:8.1f} us  ready@ {rd/1e3:8.1f} us  lib {lb/1e3:8.1f} us")
    for (li, op, e), b in zip(errs, plan):
        L = spec["layers"][li]
        extra = ""
        if op == "conv":
            extra = f"w{tuple(L['w'].shape)} s{L['stride']} p{L['pad']} g{L['groups']}"
        print(f"  {li:3d} {op:9s} {P.kernel_name(b[2]):16s} err {e:.3e} {'BAD' if not e <= 1e-2 else ''} {extra}")
    worst = max(e for _, _, e in errs)
    print(f"== {name} worst {worst:.3e}")
    # hot timing
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(5):
        ctx.infer(s)
    ctx.sync()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    ev0.record()
    n = 20
    for _ in range(n):
        ctx.infer(s)
    ev1.record()
    torch.cuda.synchronize()
    print(f"== {name} hot {ev0.elapsed_time(ev1)/n:.3f} ms/inference")
    if os.environ.get("PASK_DEBUG_SKIP_CLOSE") != "1":
        ctx.close()
    sys.stdout.flush()
