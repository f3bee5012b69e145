"""Code-upload cost vs code-object layout (D10 experiment).

Each sample is a fresh process: torch initialises the context and runs one
kernel (so the context's own code memory is set up, as in a real cold start),
then the code object is parsed (cuLibraryLoadData, BINARY_IS_PRESERVED, as in
libpask) and each listed function is fetched and uploaded (cuLibraryGetKernel ->
cuKernelGetFunction -> cuFuncLoad), timed on the host.

    python scripts/upload_microbench.py [--n 9] [--dir _loadbench]
Variants (fatbins built by the caller into --dir): name:fn1,fn2,...
"""
import argparse
import ctypes as C
import json
import os
import statistics
import subprocess
import sys
import time

DEFAULT = ["fam:pask_mem,pask_conv_igemm", "all:pask_all", "all_cnn:pask_all", "fam_cnn:pask_mem,pask_conv_igemm",
           "all_bert:pask_all"]


def child(path, fns):
    import torch
    torch.ones(1, device="cuda").add_(1)
    torch.cuda.synchronize()
    cu = C.CDLL("libcuda.so.1")
    data = open(path, "rb").read()
    buf = C.create_string_buffer(data, len(data))
    ns = time.perf_counter_ns
    time.sleep(0.02)
    lib = C.c_void_p()
    opts = (C.c_int * 1)(1)  # CU_LIBRARY_BINARY_IS_PRESERVED
    vals = (C.c_void_p * 1)(1)
    t0 = ns()
    assert cu.cuLibraryLoadData(C.byref(lib), buf, None, None, 0, opts, vals, 1) == 0
    t1 = ns()
    out = {"lib_us": (t1 - t0) / 1e3, "funcs": {}}
    for name in fns:
        k, f = C.c_void_p(), C.c_void_p()
        a = ns()
        assert cu.cuLibraryGetKernel(C.byref(k), lib, name.encode()) == 0
        assert cu.cuKernelGetFunction(C.byref(f), k) == 0
        b = ns()
        assert cu.cuFuncLoad(f) == 0
        c = ns()
        out["funcs"][name] = {"get_us": (b - a) / 1e3, "upload_us": (c - b) / 1e3}
    out["total_us"] = (ns() - t0) / 1e3
    print(json.dumps(out))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=9)
    ap.add_argument("--dir", default=os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                   "_loadbench"))
    ap.add_argument("--child", nargs=2)
    ap.add_argument("variants", nargs="*")
    a = ap.parse_args()
    if a.child:
        child(a.child[0], a.child[1].split(","))
        return
    variants = [v.split(":") for v in (a.variants or DEFAULT)]
    res = {v[0]: [] for v in variants}
    for _ in range(a.n):  # interleaved so drift hits every variant alike
        for name, fns in variants:
            p = os.path.join(a.dir, name + ".fatbin")
            r = subprocess.run([sys.executable, __file__, "--child", p, fns], capture_output=True, text=True)
            js = [l for l in r.stdout.splitlines() if l.startswith("{")]
            if not js:
                print(name, "FAILED", r.stderr[-500:])
                continue
            res[name].append(json.loads(js[-1]))
    for name, fns in variants:
        s = res[name]
        if not s:
            continue
        med = lambda f: round(statistics.median(f(x) for x in s), 1)
        per = {fn: med(lambda x, fn=fn: x["funcs"][fn]["upload_us"]) for fn in fns.split(",")}
        print(f"{name:10s} size {os.path.getsize(os.path.join(a.dir, name + '.fatbin')):7d} B  "
              f"lib {med(lambda x: x['lib_us']):6.1f}  uploads {per}  total {med(lambda x: x['total_us']):6.1f} us "
              f"(median of {len(s)})")


if __name__ == "__main__":
    main()
