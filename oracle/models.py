"""Oracle execution of a model spec (``workloads.models``), layer by layer.

TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``).

``run_layer`` evaluates one lowered layer on float64 inputs in logical layout
(NCHW images, row-major matrices).  ``run_model`` chains the layers
free-running in float64.  Teacher-forced parity calls
``run_layer`` on the GPU's own bf16 inputs of each layer.
"""
from __future__ import annotations

import numpy as np

from . import ops


def run_layer(layer, ins, res=None):
    """Evaluate one spec layer.  ``ins`` is the list of float64 input arrays in
    logical layout, ``res`` the residual operand (or None)."""
    op = layer["op"]
    if op == "layout":
        # logical result is the bf16-rounded NCHW image (channel padding is a
        # device-layout detail checked separately)
        return ops.bf16_rne(ins[0])
    if op == "conv":
        return ops.conv_layer(ins[0], layer["w"], layer["b"], layer["stride"], layer["pad"],
                              layer["dil"], layer["groups"], layer["act"], res)
    if op == "pool":
        x = ins[0]
        if layer["global_"]:
            if layer["mode"] == "avg":
                return ops.global_avg_pool(x)
            return ops.max_pool2d(x, layer["kernel"], (1, 1), (0, 0))
        if layer["mode"] == "max":
            return ops.max_pool2d(x, layer["kernel"], layer["stride"], layer["pad"])
        return ops.avg_pool2d(x, layer["kernel"], layer["stride"], layer["pad"],
                              layer["count_include_pad"])
    if op == "linear":
        x = ins[0]
        if layer["flatten"] == "nchw":
            x = x.reshape(x.shape[0], -1)
        if layer["rows"] is not None:
            x = x[:layer["rows"]]
        return ops.linear(x, layer["w"], layer["b"], layer["act"], res)
    if op == "softmax":
        return ops.softmax(ins[0], layer["scale"])
    if op == "layernorm":
        return ops.layernorm(ins[0], layer["gamma"], layer["beta"], layer["eps"])
    if op == "qk":
        return ops.attn_qk(ins[0], layer["heads"], layer["head_dim"])
    if op == "pv":
        return ops.attn_pv(ins[0], ins[1], layer["heads"], layer["head_dim"])
    if op == "attention":
        return ops.attention(ins[0], layer["heads"], layer["head_dim"], layer["scale"])
    raise ValueError(f"unknown op {op}")


def run_model(spec, x):
    """Free-running float64 forward.  Returns {tensor_name: float64 array}."""
    (in_name, _, _), = spec["inputs"]
    env = {in_name: np.asarray(x, dtype=np.float64)}
    for layer in spec["layers"]:
        ins = [env[t] for t in layer["inputs"]]
        res = env[layer["res"]] if layer.get("res") else None
        env[layer["out"]] = run_layer(layer, ins, res)
    return env


def model_flops(spec):
    """Algorithmic multiply-add FLOPs (2 per MAC) of the conv / linear / attention layers."""
    tot = 0
    shapes = spec["tensors"]
    for layer in spec["layers"]:
        op = layer["op"]
        if op == "conv":
            k, cg, r, s = layer["w"].shape
            n, _, p, q = shapes[layer["out"]]
            tot += 2 * n * k * p * q * cg * r * s
        elif op == "linear":
            m, nout = shapes[layer["out"]]
            tot += 2 * m * nout * layer["w"].shape[1]
        elif op in ("qk", "pv"):
            s = shapes[layer["inputs"][-1]][0]
            tot += 2 * layer["heads"] * s * s * layer["head_dim"]
        elif op == "attention":  # QK^T and PV
            s = shapes[layer["inputs"][0]][0]
            tot += 4 * layer["heads"] * s * s * layer["head_dim"]
    return tot
