"""Tiny shapes of every catalog kernel and code path, for compute-sanitizer
(SURVEY.md §4 T8 / §5): memcheck, racecheck, synccheck, initcheck.

    compute-sanitizer --tool memcheck --error-exitcode 99 python scripts/sanitize_cases.py

Each case is a small single-layer (or few-layer) graph run once through the C
ABI and checked teacher-forced against the oracle, so a sanitizer-clean run is
also a correct one.  Covered: layout; the contraction kernel's A paths (TMA
plain matrix, TMA im2col, cp.async gather), split-K clusters of 2..8 and 16,
the direct / staged / scalar epilogues with residual, GEMM batched with K- and
MN-major B (QK^T / PV); the persistent-tile solution; depthwise; windowed and
global pooling; softmax; LayerNorm; fused attention; and the packaging 2 / 3
family entries.
"""
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_dac_huangdxz25_b200 import build as pbuild  # noqa: E402
from paper_conf_dac_huangdxz25_b200 import pask as P  # noqa: E402
from tests.gpu_harness import TOL, run_model, teacher_forced_errors  # noqa: E402
from workloads.models import _Builder, make_input  # noqa: E402


def conv(c, k, hw, r, s=1, p=0, d=1, act="relu", res=False, groups=1):
    b = _Builder("conv", 3)
    x = b.input((1, c, hw, hw), "f32")
    t = b.layout(x, c_pad=max(8, (c + 7) // 8 * 8))
    rr = b.conv(t, k, r, s, p, d, act="none") if res else None
    b.outputs = [b.conv(t, k, r, s, p, d, groups=groups, act=act, res=rr)]
    return b.spec()


def linear(m, kin, nout, act="none", res=False):
    b = _Builder("lin", 4)
    x = b.input((m, kin), "bf16")
    rr = b.linear(x, nout) if res else None
    b.outputs = [b.linear(x, nout, act=act, res=rr)]
    return b.spec()


def pool(kind):
    b = _Builder("pool", 5)
    x = b.input((1, 16, 9, 9), "f32")
    t = b.layout(x)
    if kind == "max":
        y = b.pool(t, "max", 3, 2, 1)
    elif kind == "avg":
        y = b.pool(t, "avg", 3, 1, 1)
    else:
        y = b.pool(t, "avg", "global")
    b.outputs = [y]
    return b.spec()


def rows(op):
    b = _Builder("rows", 6)
    x = b.input((24, 72), "bf16")
    b.outputs = [b.softmax(x, 0.5) if op == "softmax" else b.layernorm(x, 1e-5)]
    return b.spec()


def attention(fused, s=40, heads=2):
    b = _Builder("attn", 7)
    dh = 64
    x = b.input((s, heads * dh), "bf16")
    qkv = b.linear(x, 3 * heads * dh, w_std=0.08, b_std=0.02)
    if fused:
        y = b.attention(qkv, heads, dh, 1 / math.sqrt(dh))
    else:
        sc = b.qk(qkv, heads, dh)
        pr = b.softmax(sc, 1 / math.sqrt(dh))
        y = b.pv(pr, qkv, heads, dh)
    b.outputs = [y]
    return b.spec()


CASES = [
    ("layout+conv 3x3 gather (C=8)", conv(3, 16, 12, 3, 1, 1), {}),
    ("conv 3x3 im2col C=64 split-K", conv(64, 64, 7, 3, 1, 1, res=True), {}),
    ("conv 1x1 TMA A + residual", conv(64, 128, 10, 1, res=True), {}),
    ("conv 1x1 stride 2 im2col", conv(128, 64, 9, 1, 2, 0), {}),
    ("conv 5x5 dil 2 narrow-C gather", conv(24, 32, 11, 5, 1, 4, 2, act="tanh"), {}),
    ("conv N tail 40", conv(16, 40, 9, 3, 1, 1, act="relu6"), {}),
    ("depthwise 3x3 s2", conv(32, 32, 9, 3, 2, 1, act="relu6", groups=32), {}),
    ("persistent tiles", conv(8, 64, 140, 3, 1, 1), {}),   # M = 19600 > 148 x 128 rows
    ("gemm scalar epilogue N=10", linear(3, 256, 10), {}),
    ("gemm split-16 cluster + residual", linear(8, 8192, 64, res=True), {}),
    ("gemm GELU, staged tail", linear(40, 128, 96, act="gelu"), {}),
    ("pool max 3x3 s2 p1", pool("max"), {}),
    ("pool avg 3x3", pool("avg"), {}),
    ("pool global avg", pool("global"), {}),
    ("softmax rows", rows("softmax"), {}),
    ("layernorm rows", rows("layernorm"), {}),
    ("attention unfused (QK^T, softmax, PV MN-major)", attention(False), {}),
    ("attention fused", attention(True), {}),
    ("families packaging (pask_mem + contraction)", conv(32, 32, 8, 3, 1, 1, groups=32), dict(packaging=2)),
    ("single-function packaging (pask_all)", pool("max"), dict(packaging=3)),
    ("timeline stamps", conv(16, 32, 8, 3, 1, 1), dict(timeline=1)),
    ("async loader + interleave", conv(16, 32, 8, 3, 1, 1), dict(proactive=1, interleave=1)),
]


def main():
    pbuild.build()
    only = sys.argv[1:]
    failed = []
    for name, spec, cfg in CASES:
        if only and not any(o in name for o in only):
            continue
        x = make_input(spec, 0)
        dm, ctx, _ = run_model(spec, x, cfg=P.config(**cfg) if cfg else None)
        errs = teacher_forced_errors(dm, spec, x)
        ctx.close()
        worst = max(e for _, _, e in errs)
        ok = worst <= TOL
        print(f"{'ok ' if ok else 'BAD'} {name}: worst rel err {worst:.2e}", flush=True)
        if not ok:
            failed.append(name)
    if failed:
        print("FAILED:", failed)
        sys.exit(1)
    print("all sanitizer cases ok")


if __name__ == "__main__":
    main()
