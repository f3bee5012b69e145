"""PASK on B200: proactive and selective kernel loading for cold-start DNN inference.

The product is libpask.so (C ABI in include/pask.h): planner (Algorithm 1 over a
categorical kernel cache), proactive loader thread, issue loop and a handful of
shape-generic sm_100a kernels in one code object.  This package holds the
in-tree build (``build.py``), the ctypes binding (``pask.py``) and the lowering of
model specs to pask_graph (``model.py``).
"""
from . import pask  # noqa: F401
