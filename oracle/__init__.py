"""PASK oracle -- TEST INFRASTRUCTURE, not the product.

A plain, slow, obviously-correct CPU implementation of what the PASK hot path
computes (§III):

* ``oracle.ops``    float64 definitions of the canonical operators (conv, depthwise
                    conv, GEMM, pooling, activations, softmax, LayerNorm, layout);
* ``oracle.models`` spec execution, layer by layer (teacher-forced) or free-running;
* ``oracle.plan``   Algorithm 1 (EXECUTIONPLAN / GETSUBSOLUTION) over the categorical
                    MRU cache, producing the exact integer plan.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import, call or execute anything under ``oracle/``.
It shares no code with ``paper_conf_dac_huangdxz25_b200`` (the CUDA path), and the
CUDA path never imports it.  Seeded inputs come from ``workloads`` (no arithmetic
of the method lives there).

Parity pins: every function is pinned in ``tests/test_oracle_*.py`` against worked
examples (``tests/golden/``), closed forms, invariants, brute force and independent
library routines (torch float64).  No function is "parity unpinned".
"""
