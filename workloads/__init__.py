"""Seeded synthetic workloads shared by the oracle and the CUDA path.

This package holds ONLY input generation: model *specs* (the lowered layer
sequence PASK receives as input, Fig. 5 caption "PASK receives the
lowered model (a sequence of n solutions) as input"), seeded random weights and
seeded input tensors.  It contains none of the method's arithmetic (no
convolution, GEMM, pooling, softmax, LayerNorm or planning); both ``oracle/``
and ``paper_conf_dac_huangdxz25_b200/`` interpret the specs independently.
"""
from .models import (  # noqa: F401
    MODELS,
    build_model,
    bf16_round,
    tiny_cnn,
    resnet50,
    mobilenet_v2,
    bert_base,
)
