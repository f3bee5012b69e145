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


def child(path, fns, pre=None):
    import torch
    torch.ones(1, device="cuda").add_(1)
    torch.cuda.synchronize()
    cu = C.CDLL("libcuda.so.1")
    ns = time.perf_counter_ns
    opts = (C.c_int * 1)(1)  # CU_LIBRARY_BINARY_IS_PRESERVED
    vals = (C.c_void_p * 1)(1)
    keep = []

    def load(p):
        data = open(p, "rb").read()
        buf = C.create_string_buffer(data, len(data))
        keep.append(buf)
        lib = C.c_void_p()
        assert cu.cuLibraryLoadData(C.byref(lib), buf, None, None, 0, opts, vals, 1) == 0
        return lib

    out = {"funcs": {}}
    spin_until = ns() + 20_000_000   # keep the core hot (as libpask's loader does), no sleep
    while ns() < spin_until:
        pass
    if pre:  # warm-up upload of an unrelated small function (another code object)
        ppath, pfn = pre.split(":")
        a = ns()
        plib = load(ppath)
        k, f = C.c_void_p(), C.c_void_p()
        assert cu.cuLibraryGetKernel(C.byref(k), plib, pfn.encode()) == 0
        assert cu.cuKernelGetFunction(C.byref(f), k) == 0
        assert cu.cuFuncLoad(f) == 0
        out["pre_us"] = (ns() - a) / 1e3
    t0 = ns()
    lib = load(path)
    t1 = ns()
    out["lib_us"] = (t1 - t0) / 1e3
    for name in fns:
        k, f = C.c_void_p(), C.c_void_p()
        a = ns()
        assert cu.cuLibraryGetKernel(C.byref(k), lib, name.encode()) == 0
        assert cu.cuKernelGetFunction(C.byref(f), k) == 0
        b = ns()
        assert cu.cuFuncLoad(f) == 0
        c = ns()
        out["funcs"][name] = {"get_us": (b - a) / 1e3, "upload_us": (c - b) / 1e3, "total_us": (c - a) / 1e3}
    out["total_us"] = (ns() - t0) / 1e3
    print(json.dumps(out))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=9)
    ap.add_argument("--dir", default=os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                   "_loadbench"))
    ap.add_argument("--child", nargs=2)
    ap.add_argument("--pre", default=None, help="path:function uploaded before the timed library")
    ap.add_argument("variants", nargs="*")
    a = ap.parse_args()
    if a.child:
        child(a.child[0], a.child[1].split(","), a.pre)
        return
    variants = [v.split(":") for v in (a.variants or DEFAULT)]
    # name:fns[:pre-object:pre-function] -> optional warm-up upload before the timed one
    variants = [(v[0], v[1], (os.path.join(a.dir, v[2] + ".fatbin") + ":" + v[3]) if len(v) > 3 else None)
                for v in variants]
    res = {v[0] + (" +pre" if v[2] else ""): [] for v in variants}
    for _ in range(a.n):  # interleaved so drift hits every variant alike
        for name, fns, pre in variants:
            p = os.path.join(a.dir, name + ".fatbin")
            r = subprocess.run([sys.executable, __file__, "--child", p, fns] + (["--pre", pre] if pre else []),
                               capture_output=True, text=True)
            js = [l for l in r.stdout.splitlines() if l.startswith("{")]
            if not js:
                print(name, "FAILED", r.stderr[-500:])
                continue
            res[name + (" +pre" if pre else "")].append(json.loads(js[-1]))
    for name, fns, pre in variants:
        name = name + (" +pre" if pre else "")
        s = res[name]
        if not s:
            continue
        med = lambda f: round(statistics.median(f(x) for x in s), 1)
        per = {fn: med(lambda x, fn=fn: x["funcs"][fn]["total_us"]) for fn in fns.split(",")}
        pre_us = f" pre {med(lambda x: x['pre_us']):6.1f}" if pre else ""
        print(f"{name:14s} size {os.path.getsize(os.path.join(a.dir, name.split()[0] + '.fatbin')):7d} B {pre_us} "
              f"lib {med(lambda x: x['lib_us']):6.1f}  uploads {per}  total {med(lambda x: x['total_us']):6.1f} us "
              f"(median of {len(s)})")


if __name__ == "__main__":
    main()
