"""Loader microbenchmark (driver API via ctypes): what does code loading cost on B200?"""
import ctypes as C
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LB = os.path.join(ROOT, "_loadbench")
KERNELS = ["pask_layout", "pask_conv_igemm", "pask_pool", "pask_gemm", "pask_softmax"]


def child(scn):
    import torch
    torch.zeros(1, device="cuda")
    torch.cuda.synchronize()
    cu = C.CDLL("libcuda.so.1")
    def ns():
        return time.perf_counter_ns()
    res = {"scenario": scn}
    def lib_load(path, preserved=False):
        data = open(path, "rb").read()
        buf = C.create_string_buffer(data, len(data))
        lib = C.c_void_p()
        if preserved:
            opts = (C.c_int * 1)(1)   # CU_LIBRARY_BINARY_IS_PRESERVED
            vals = (C.c_void_p * 1)(1)
            t = ns(); r = cu.cuLibraryLoadData(C.byref(lib), buf, None, None, 0, opts, vals, 1); dt = ns() - t
        else:
            t = ns(); r = cu.cuLibraryLoadData(C.byref(lib), buf, None, None, 0, None, None, 0); dt = ns() - t
        assert r == 0, r
        return lib, dt, buf
    def func_load(lib, name):
        k = C.c_void_p(); f = C.c_void_p()
        t0 = ns(); r = cu.cuLibraryGetKernel(C.byref(k), lib, name.encode()); t1 = ns()
        r2 = cu.cuKernelGetFunction(C.byref(f), k); t2 = ns()
        r3 = cu.cuFuncLoad(f); t3 = ns()
        assert r == 0 and r2 == 0 and r3 == 0, (r, r2, r3)
        return {"get_kernel": (t1 - t0) / 1e3, "get_function": (t2 - t1) / 1e3, "func_load": (t3 - t2) / 1e3}
    if scn in ("fatbin", "fatbin_preserved", "cubin"):
        path = os.path.join(LB, "all.cubin" if scn == "cubin" else "all.fatbin")
        lib, dt, keep = lib_load(path, preserved=(scn == "fatbin_preserved"))
        res["lib_us"] = dt / 1e3
        res["funcs"] = {k: func_load(lib, k) for k in KERNELS}
        lib2, dt2, keep2 = lib_load(path)
        res["second_lib_us"] = dt2 / 1e3
        res["second_funcs"] = {k: func_load(lib2, k) for k in KERNELS[:2]}
    elif scn == "per_kernel":
        out = {}
        keep = []
        for k in KERNELS:
            lib, dt, b = lib_load(os.path.join(LB, k + ".fatbin"))
            keep.append(b)
            out[k] = {"lib_us": dt / 1e3, **func_load(lib, k)}
        res["kernels"] = out
    elif scn == "module":
        data = open(os.path.join(LB, "all.fatbin"), "rb").read()
        buf = C.create_string_buffer(data, len(data))
        mod = C.c_void_p()
        t = ns(); r = cu.cuModuleLoadData(C.byref(mod), buf); dt = ns() - t
        assert r == 0, r
        res["module_load_us"] = dt / 1e3
        fl = {}
        for k in KERNELS:
            f = C.c_void_p()
            t0 = ns(); r = cu.cuModuleGetFunction(C.byref(f), mod, k.encode()); t1 = ns()
            r2 = cu.cuFuncLoad(f); t2 = ns()
            fl[k] = {"get_function": (t1 - t0) / 1e3, "func_load": (t2 - t1) / 1e3}
        res["funcs"] = fl
    elif scn == "eager":
        lib, dt, keep = lib_load(os.path.join(LB, "all.fatbin"))
        res["lib_us_eager"] = dt / 1e3
        res["funcs"] = {k: func_load(lib, k) for k in KERNELS}
    print(json.dumps(res))


if __name__ == "__main__":
    if len(sys.argv) > 1:
        child(sys.argv[1])
        sys.exit(0)
    for scn in ["fatbin", "fatbin", "fatbin_preserved", "cubin", "per_kernel", "module", "eager"]:
        env = dict(os.environ)
        if scn == "eager":
            env["CUDA_MODULE_LOADING"] = "EAGER"
        out = subprocess.run([sys.executable, __file__, scn], capture_output=True, text=True, env=env)
        print(out.stdout.strip() or out.stderr[-2000:])
