"""Shared GPU parity helpers (test infrastructure).

Teacher-forced per-layer parity: after one inference
through the C ABI, every layer's GPU inputs (caller-owned device tensors) are
read back and fed to the oracle layer; the oracle output is compared with the
GPU output, max|gpu - ref| <= 1e-2 * max|ref| (BASELINE.json north_star tolerance
for bf16-in / fp32-accumulate).  The layout layer is compared bit-exactly.
"""
from __future__ import annotations

import numpy as np
import torch

from oracle import models as om
from oracle import ops as oops
from paper_conf_dac_huangdxz25_b200 import pask as P
from paper_conf_dac_huangdxz25_b200.model import DeviceModel

TOL = 1e-2


def rel_err(gpu, ref):
    return float(np.abs(gpu - ref).max() / max(float(np.abs(ref).max()), 1e-30))


def run_model(spec, x, cfg=None, solutions=None):
    dm = DeviceModel(spec, solutions=solutions)
    dm.set_input(x)
    ctx = P.Context(0, cfg)
    plan = ctx.load_model(dm.graph)
    stream = torch.cuda.current_stream().cuda_stream
    ctx.infer(stream)
    ctx.sync()
    torch.cuda.synchronize()
    return dm, ctx, plan


def teacher_forced_errors(dm, spec, x):
    errs = []
    for li, L in enumerate(spec["layers"]):
        ins = [dm.read(t) for t in L["inputs"]]
        if L["op"] == "layout":
            ins = [np.asarray(x, np.float64)]
        res = dm.read(L["res"]) if L.get("res") else None
        ref = om.run_layer(L, ins, res)
        gpu = dm.read(L["out"])
        if L["op"] == "layout":
            raw = dm.read_raw(L["out"])
            exp = oops.layout_nchw_to_nhwc(x, L["c_pad"])
            e = 0.0 if np.array_equal(raw, exp) else float("inf")
        else:
            e = rel_err(gpu.reshape(ref.shape), ref)
        errs.append((li, L["op"], e))
    return errs
