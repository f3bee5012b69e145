"""Build libpask.so in-tree: one SASS-only sm_100a fatbin (the whole kernel
catalog in one code object) embedded into a C++17 shared library that talks to
the CUDA driver through dlopen (no link-time libcuda dependency).

    python -m paper_conf_dac_huangdxz25_b200.build [--force]
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libpask.so")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]

KERNEL_SRC = [os.path.join(CSRC, "kernels", f) for f in
              ("pask_kernels.cu", "conv_gemm.cuh", "elementwise.cuh", "ptx.cuh", "pask_params.h")]
HOST_SRC = [os.path.join(CSRC, "runtime", f) for f in ("pask.cpp", "plan.cpp", "driver.cpp")]
HOST_DEPS = HOST_SRC + [os.path.join(CSRC, "runtime", f) for f in
                         ("plan.h", "driver.h", "exports.map")] + [
    os.path.join(CSRC, "kernels", "pask_params.h"),
    os.path.join(os.path.dirname(PKG), "include", "pask.h")]


def _run(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
        raise RuntimeError(f"build step failed: {cmd[0]}")
    return r.stdout + r.stderr


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


# catalog order (include/pask.h PASK_K_*)
KERNELS = ["pask_layout", "pask_conv_igemm", "pask_conv_1x1", "pask_conv_dw", "pask_pool",
           "pask_pool_gavg", "pask_gemm", "pask_softmax", "pask_layernorm"]


def _nvcc_fatbin(out, defines=()):
    # -lineinfo (ncu source page) embeds the PTX text in the code object and
    # makes every cold load parse ~1 MB more, so it is opt-in (PASK_LINEINFO=1)
    extra = ["-lineinfo"] if os.environ.get("PASK_LINEINFO") == "1" else []
    return subprocess.Popen([NVCC, *ARCH, "-fatbin", "-O3", *extra, "-std=c++17", "-Xptxas", "-v",
                             *defines, "-o", out, KERNEL_SRC[0]],
                            stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    fatbin = os.path.join(BUILD, "pask.fatbin")
    per_kernel = [os.path.join(BUILD, k + ".fatbin") for k in KERNELS]
    if force or any(_stale(f, KERNEL_SRC) for f in [fatbin] + per_kernel):
        # the whole catalog as one code object, and one code object per kernel
        jobs = [(fatbin, _nvcc_fatbin(fatbin))]
        for k, f in zip(KERNELS, per_kernel):
            jobs.append((f, _nvcc_fatbin(f, ["-DPASK_ONLY_KERNEL", f"-DPASK_ONLY_KERNEL_{k}=1"])))
        logs = []
        for f, proc in jobs:
            out, _ = proc.communicate()
            logs.append(out)
            if proc.returncode != 0:
                sys.stderr.write(out)
                raise RuntimeError(f"nvcc failed for {f}")
        with open(os.path.join(BUILD, "ptxas.log"), "w") as fh:
            fh.write(logs[0])
        if verbose:
            print(logs[0])
    asm = os.path.join(BUILD, "fatbins.S")
    with open(asm, "w") as fh:
        fh.write('        .section .rodata.pask_fatbin,"a",@progbits\n')
        for sym, path in [("pask_fatbin", fatbin)] + [(f"pask_fb_{k}", f) for k, f in
                                                       zip(KERNELS, per_kernel)]:
            fh.write(f"        .balign 64\n        .globl {sym}_start\n        .hidden {sym}_start\n"
                     f"{sym}_start:\n        .incbin \"{path}\"\n        .globl {sym}_end\n"
                     f"        .hidden {sym}_end\n{sym}_end:\n        .byte 0\n")
        fh.write('        .section .note.GNU-stack,"",@progbits\n')
    if force or _stale(LIB, HOST_DEPS + [fatbin] + per_kernel):
        cxx = os.environ.get("CXX", "g++")
        flags = ["-O2", "-std=c++17", "-fPIC", "-fvisibility=hidden", "-Wall", "-Wno-unused-function",
                 f"-I{CUDA}/include"]
        objs = []
        for src in HOST_SRC:
            obj = os.path.join(BUILD, os.path.basename(src) + ".o")
            _run([cxx, *flags, "-c", src, "-o", obj])
            objs.append(obj)
        fobj = os.path.join(BUILD, "fatbin.o")
        _run([cxx, "-c", asm, "-o", fobj])
        tmp = LIB + ".tmp"
        _run([cxx, "-shared", "-o", tmp, *objs, fobj, "-ldl", "-lpthread", "-Wl,--no-undefined",
              "-Wl,--version-script=" + os.path.join(CSRC, "runtime", "exports.map")])
        shutil.move(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
