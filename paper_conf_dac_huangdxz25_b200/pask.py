"""Thin ctypes binding of libpask.so (include/pask.h): argument marshalling only.

Every step of the hot path (planning, loading, issuing, all kernels) runs in
libpask.so; this module only mirrors the C structs and forwards calls.  It
fails loudly when the library is missing -- there is no Python or CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libpask.so")
# test-only build of the same library plus the fake CUDA driver of
# include/pask_testing.h (never loaded by the product path)
TESTING_LIB_PATH = os.environ.get("PASK_TESTING_LIB", os.path.join(_PKG, "libpask_testing.so"))

# ---------------------------------------------------------------- enums (pask.h)
OK, EINVAL, EUNSUPPORTED, ECUDA, ENOMEM, ESTATE = 0, -1, -2, -3, -4, -5
BF16, F32 = 0, 1
NCHW, NHWC, ROWMAJOR = 0, 1, 2
OP_LAYOUT, OP_CONV2D, OP_GEMM, OP_POOL, OP_SOFTMAX, OP_LAYERNORM, OP_ATTENTION = range(7)
ACT = {"none": 0, "relu": 1, "relu6": 2, "gelu": 3, "tanh": 4}
K_LAYOUT, K_CONV_IGEMM, K_CONV_1X1, K_CONV_DW, K_POOL, K_POOL_GAVG, K_GEMM, K_SOFTMAX, \
    K_LAYERNORM, K_ATTENTION, K_CONV_IGEMM_PT, K_GEMV = range(12)
NUM_KERNELS = 12         # generic catalog (PASK_NUM_KERNELS); num_kernels() adds the specialisations
HOW = {0: "direct", 1: "reused", 2: "loaded"}


class Tensor(C.Structure):
    _fields_ = [("dtype", C.c_int32), ("layout", C.c_int32), ("n", C.c_int32),
                ("h", C.c_int32), ("w", C.c_int32), ("c", C.c_int32), ("dptr", C.c_void_p)]


class Node(C.Structure):
    _fields_ = [("op", C.c_int32), ("in0", C.c_int32), ("in1", C.c_int32), ("res", C.c_int32),
                ("out", C.c_int32), ("w", C.c_void_p), ("bias", C.c_void_p),
                ("gamma", C.c_void_p), ("beta", C.c_void_p), ("k", C.c_int32),
                ("r", C.c_int32), ("s", C.c_int32), ("stride", C.c_int32 * 2),
                ("pad", C.c_int32 * 2), ("dil", C.c_int32 * 2), ("groups", C.c_int32),
                ("m", C.c_int32), ("n", C.c_int32), ("kk", C.c_int32), ("batch", C.c_int32),
                ("trans_b", C.c_int32), ("lda", C.c_int64), ("ldb", C.c_int64),
                ("ldc", C.c_int64), ("off_a", C.c_int64), ("off_b", C.c_int64),
                ("off_c", C.c_int64), ("stride_a", C.c_int64), ("stride_b", C.c_int64),
                ("stride_c", C.c_int64), ("pool_mode", C.c_int32),
                ("count_include_pad", C.c_int32), ("global_pool", C.c_int32),
                ("eps", C.c_float), ("scale", C.c_float), ("act", C.c_int32),
                ("solution", C.c_int32)]


class Graph(C.Structure):
    _fields_ = [("n_tensors", C.c_int32), ("tensors", C.POINTER(Tensor)),
                ("n_nodes", C.c_int32), ("nodes", C.POINTER(Node)),
                ("n_inputs", C.c_int32), ("inputs", C.POINTER(C.c_int32)),
                ("n_outputs", C.c_int32), ("outputs", C.POINTER(C.c_int32)),
                ("workspace", C.c_void_p), ("workspace_bytes", C.c_uint64)]


class Config(C.Structure):
    _fields_ = [("reuse", C.c_int32), ("search", C.c_int32), ("milestone", C.c_int32),
                ("proactive", C.c_int32), ("pdl", C.c_int32), ("instrument", C.c_int32),
                ("packaging", C.c_int32), ("interleave", C.c_int32), ("graph", C.c_int32),
                ("catalog", C.c_int32), ("branches", C.c_int32), ("timeline", C.c_int32),
                ("no_prefault", C.c_int32), ("no_prime", C.c_int32)]


class Binding(C.Structure):
    _fields_ = [("node", C.c_int32), ("desired_kernel", C.c_int32), ("bound_kernel", C.c_int32),
                ("how", C.c_int32), ("lookups", C.c_int32)]


class Stats(C.Structure):
    _fields_ = [("n_nodes", C.c_int32), ("kernels_loaded", C.c_int32),
                ("code_objects_loaded", C.c_int32), ("queries", C.c_int32), ("hits", C.c_int32),
                ("lookups", C.c_int32), ("code_bytes_loaded", C.c_uint64), ("plan_ns", C.c_uint64),
                ("load_ns", C.c_uint64), ("load_exposed_ns", C.c_uint64), ("issue_ns", C.c_uint64),
                ("encode_ns", C.c_uint64), ("gpu_span_ns", C.c_uint64), ("gpu_busy_ns", C.c_uint64),
                ("cold_wall_ns", C.c_uint64), ("infer_count", C.c_uint64), ("launches", C.c_uint64),
                ("load_done_ns", C.c_uint64), ("infer_entry_ns", C.c_uint64),
                ("first_launch_ns", C.c_uint64), ("last_launch_ns", C.c_uint64),
                ("encode_begin_ns", C.c_uint64), ("encode_end_ns", C.c_uint64),
                ("kernel_span_ns", C.c_uint64), ("prefault_ns", C.c_uint64),
                ("prefault_bytes", C.c_uint64), ("max_cluster", C.c_int32), ("reserved0", C.c_int32),
                ("prime_ns", C.c_uint64)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


EXPORTS = ["pask_version", "pask_create", "pask_plan", "pask_workspace_bytes", "pask_load_model",
           "pask_infer", "pask_infer_host", "pask_sync", "pask_stats", "pask_kernel_is_loaded",
           "pask_destroy", "pask_last_error", "pask_num_kernels", "pask_kernel_name",
           "pask_kernel_function",
           "pask_kernel_timeline", "pask_node_times", "pask_node_intervals", "pask_promote"]
TEST_EXPORTS = ["pask_test_fake_driver", "pask_test_fake_log", "pask_test_fake_knob"]   # pask_testing.h
FAKE_OCCUPANCY, FAKE_CURRENT_DEVICE, FAKE_MAX_CLUSTER_LAUNCHED, FAKE_PRIMER_LOADS = 1, 2, 3, 4

_libs = {}
_use_testing = False


def use_testing_library(enable=True):
    """Test-only: route lib() (and so every Context created afterwards) to
    libpask_testing.so, which adds the fake driver hooks of pask_testing.h."""
    global _use_testing
    _use_testing = bool(enable)


def lib():
    """Load libpask.so (build it first with paper_conf_dac_huangdxz25_b200.build)."""
    path = TESTING_LIB_PATH if _use_testing else LIB_PATH
    if path in _libs:
        return _libs[path]
    if not os.path.exists(path):
        raise RuntimeError(f"{path} is missing: run `python -m paper_conf_dac_huangdxz25_b200."
                           "build` (there is no fallback path)")
    L = C.CDLL(path)
    P = C.c_void_p
    sig = {
        "pask_version": (C.c_int, []),
        "pask_create": (C.c_int, [C.POINTER(P), C.c_int, C.POINTER(Config)]),
        "pask_plan": (C.c_int, [C.POINTER(Graph), C.POINTER(Config), C.POINTER(Binding),
                                C.POINTER(Stats)]),
        "pask_workspace_bytes": (C.c_int, [C.POINTER(Graph), C.POINTER(C.c_uint64)]),
        "pask_load_model": (C.c_int, [P, C.POINTER(Graph), C.POINTER(Binding)]),
        "pask_infer": (C.c_int, [P, C.POINTER(P), C.POINTER(P), P]),
        "pask_infer_host": (C.c_int, [P, C.POINTER(P), C.POINTER(P), P]),
        "pask_sync": (C.c_int, [P]),
        "pask_stats": (C.c_int, [P, C.POINTER(Stats)]),
        "pask_kernel_is_loaded": (C.c_int, [P, C.c_int32, C.POINTER(C.c_int32)]),
        "pask_destroy": (C.c_int, [P]),
        "pask_kernel_timeline": (C.c_int, [P, C.c_int32, C.POINTER(C.c_uint64),
                                           C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]),
        "pask_node_times": (C.c_int, [P, C.POINTER(C.c_uint64), C.c_int32]),
        "pask_node_intervals": (C.c_int, [P, C.POINTER(C.c_uint64), C.POINTER(C.c_uint64), C.c_int32]),
        "pask_promote": (C.c_int, [P, C.c_int32, C.POINTER(C.c_int32)]),
        "pask_last_error": (C.c_char_p, []),
        "pask_num_kernels": (C.c_int32, []),
        "pask_kernel_name": (C.c_char_p, [C.c_int32]),
        "pask_kernel_function": (C.c_char_p, [C.c_int32, C.c_int32]),
    }
    if path == TESTING_LIB_PATH:
        sig["pask_test_fake_driver"] = (C.c_int, [C.c_int32, C.c_int32, C.c_int32])
        sig["pask_test_fake_log"] = (C.c_int32, [C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.c_int32])
        sig["pask_test_fake_knob"] = (C.c_int32, [C.c_int32, C.c_int32])
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _libs[path] = L
    return L


class PaskError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"pask error {code}: {msg}")
        self.code = code


def _check(rc, L=None):
    if rc != OK:
        raise PaskError(rc, (L or lib()).pask_last_error().decode())
    return rc


def kernel_name(k):
    return lib().pask_kernel_name(k).decode()


def function_name(k, packaging):
    """CUfunction entry serving catalog solution k under a packaging (pask_kernel_function)."""
    return lib().pask_kernel_function(k, packaging).decode()


def config(reuse=1, search=0, milestone=0, proactive=2, pdl=1, instrument=0, packaging=0,
           interleave=0, graph=0, catalog=0, branches=0, timeline=0, no_prefault=0, no_prime=0):
    return Config(reuse, search, milestone, proactive, pdl, instrument, packaging, interleave, graph,
                  catalog, branches, timeline, no_prefault, no_prime)


def test_fake_driver(enable=True, load_us=0, fail_kernel=-1):
    """Test-only (include/pask_testing.h, libpask_testing.so): route new contexts
    to the fake driver.  Call use_testing_library() first."""
    _check(lib().pask_test_fake_driver(1 if enable else 0, load_us, fail_kernel))


def test_fake_knob(knob, value=0):
    """Test-only: set / read a fake-driver knob (pask_test_fake_knob)."""
    return lib().pask_test_fake_knob(knob, value)


def test_fake_log(cap=4096):
    """[(kernel_id, kind)], kind 0 = load completed, 1 = launch, 2 = launch before load."""
    ids = (C.c_int32 * cap)()
    kinds = (C.c_int32 * cap)()
    n = lib().pask_test_fake_log(ids, kinds, cap)
    return [(ids[i], kinds[i]) for i in range(min(n, cap))]


def num_kernels():
    """Generic + specialised catalog size (pask_num_kernels)."""
    return lib().pask_num_kernels()


def plan(graph: Graph, cfg: Config | None = None):
    """Host-only Algorithm 1 plan: (bindings list of tuples, stats dict)."""
    n = graph.n_nodes
    out = (Binding * max(n, 1))()
    st = Stats()
    _check(lib().pask_plan(C.byref(graph), C.byref(cfg) if cfg else None, out, C.byref(st)))
    return [(b.node, b.desired_kernel, b.bound_kernel, b.how, b.lookups) for b in out[:n]], \
        st.as_dict()


def workspace_bytes(graph: Graph) -> int:
    v = C.c_uint64()
    _check(lib().pask_workspace_bytes(C.byref(graph), C.byref(v)))
    return v.value


class Context:
    """One pask_ctx (not thread-safe; one per thread)."""

    def __init__(self, device=0, cfg: Config | None = None):
        self.h = C.c_void_p()
        self.L = lib()   # the library this ctx lives in (product, or the testing build)
        self._ck(self.L.pask_create(C.byref(self.h), device, C.byref(cfg) if cfg else None))
        self.n_nodes = 0

    def load_model(self, graph: Graph, plan=True):
        """pask_load_model.  plan=False skips converting the bindings to Python
        (keeps ctypes field access out of a timed cold window); call
        ``bindings()`` afterwards."""
        self.n_nodes = graph.n_nodes
        self._plan_arr = (Binding * max(graph.n_nodes, 1))()
        self._ck(self.L.pask_load_model(self.h, C.byref(graph), self._plan_arr))
        return self.bindings() if plan else None

    def bindings(self):
        return [(b.node, b.desired_kernel, b.bound_kernel, b.how, b.lookups)
                for b in self._plan_arr[:self.n_nodes]]

    def infer(self, stream=0, inputs=None, outputs=None):
        ip = (C.c_void_p * len(inputs))(*inputs) if inputs else None
        op = (C.c_void_p * len(outputs))(*outputs) if outputs else None
        self._ck(self.L.pask_infer(self.h, ip, op, C.c_void_p(stream)))

    def infer_host(self, host_inputs, host_outputs, stream=0):
        ip = (C.c_void_p * len(host_inputs))(*host_inputs)
        op = (C.c_void_p * len(host_outputs))(*host_outputs)
        self._ck(self.L.pask_infer_host(self.h, ip, op, C.c_void_p(stream)))

    def sync(self):
        self._ck(self.L.pask_sync(self.h))

    def stats(self):
        st = Stats()
        self._ck(self.L.pask_stats(self.h, C.byref(st)))
        return st.as_dict()

    def kernel_is_loaded(self, k):
        v = C.c_int32()
        self._ck(self.L.pask_kernel_is_loaded(self.h, k, C.byref(v)))
        return bool(v.value)

    def kernel_timeline(self, k):
        """(load_ns, ready_ns since load_model entry, lib_ns) of catalog kernel k."""
        a, b, c = C.c_uint64(), C.c_uint64(), C.c_uint64()
        self._ck(self.L.pask_kernel_timeline(self.h, k, C.byref(a), C.byref(b), C.byref(c)))
        return a.value, b.value, c.value

    def promote(self, target_catalog=-1):
        """Idle-interval loading of skipped / specialised solutions."""
        n = C.c_int32()
        self._ck(self.L.pask_promote(self.h, target_catalog, C.byref(n)))
        return n.value

    def node_times(self):
        """Per-node GPU ns of the last instrumented inference (cfg.instrument = 1)."""
        arr = (C.c_uint64 * max(self.n_nodes, 1))()
        self._ck(self.L.pask_node_times(self.h, arr, self.n_nodes))
        return list(arr[:self.n_nodes])

    def node_intervals(self):
        """[(start_ns, end_ns)] per node of the last synced inference of a
        timeline = 1 context (first CTA start / last CTA end, ns after the
        inference's first kernel start)."""
        a = (C.c_uint64 * max(self.n_nodes, 1))()
        b = (C.c_uint64 * max(self.n_nodes, 1))()
        self._ck(self.L.pask_node_intervals(self.h, a, b, self.n_nodes))
        return list(zip(a[:self.n_nodes], b[:self.n_nodes]))

    def _ck(self, rc):
        return _check(rc, self.L)

    def close(self):
        if self.h:
            self._ck(self.L.pask_destroy(self.h))
            self.h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
