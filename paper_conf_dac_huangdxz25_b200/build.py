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
              ("pask_kernels.cu", "conv_gemm.cuh", "attention.cuh", "elementwise.cuh", "ptx.cuh",
               "pask_params.h", "primer.cuh")]
HOST_SRC = [os.path.join(CSRC, "runtime", f) for f in ("pask.cpp", "plan.cpp", "driver.cpp")]
# the fake CUDA driver (include/pask_testing.h) is compiled only into the
# test-only library libpask_testing.so, never into the product libpask.so
TEST_SRC = [os.path.join(CSRC, "runtime", "fake_driver.cpp")]
TEST_LIB = os.path.join(PKG, "libpask_testing.so")
COLD_SRC = os.path.join(CSRC, "tools", "pask_cold.cpp")
COLD_EXE = os.path.join(PKG, "pask_cold")   # native cold-start sampler (scripts/cold_samples.py)
HOST_DEPS = HOST_SRC + TEST_SRC + [os.path.join(CSRC, "runtime", f) for f in
                                   ("plan.h", "driver.h", "tuning.h", "exports.map")] + [
    os.path.join(CSRC, "kernels", "pask_params.h"),
    os.path.join(os.path.dirname(PKG), "include", "pask.h"),
    os.path.join(os.path.dirname(PKG), "include", "pask_testing.h")]


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
           "pask_pool_gavg", "pask_gemm", "pask_softmax", "pask_layernorm", "pask_attention",
           "pask_conv_igemm_pt", "pask_gemv"]
# Extra code objects that are not catalog ids: packaging 2's operator families
# (D8) -- the generic implicit-GEMM entry and the memory-bound family
# entry `pask_mem` in ONE code object.  name -> entries compiled into it.
# The families object comes in variants by the memory cases compiled in
# (PASK_MEM_MASK, bit per MemKind: layout 0, dw 1, pool 2, gavg 3, softmax 4,
# LayerNorm 5, GEMV 6; bit 7 the layout's stem-fold path); the runtime loads the smallest covering the model's solutions
# (dwg = depthwise + global pool without the windowed pool: MobileNetV2).
# Packaging 3 (D10): both families behind the single entry `pask_all`.
# Each variant also compiles only some contraction paths (PASK_GEMM_FEAT, bit per
# GemmFeat of conv_gemm.cuh: split-K 1, MN-major B 2, staged epilogue 4, scalar
# epilogue 8, GELU / tanh 16, cp.async gather 32, TMA im2col 64; D13).
# Smallest first: the runtime takes the first variant covering the plan (the
# table is generated into _build/spec_catalog.h as PASK_FAMILY_VARIANTS).
# The CNN variants also drop softmax's register-resident row path (their one
# softmax row of 10 / 1000 classes takes the two-pass loop: same arithmetic,
# bitwise equal) -- PASK_SOFTMAX_REG.
FAMILY_VARIANTS = {"pask_families_tf": (0x30, 0x17), "pask_families_cnng": (0x55, 0x21),
                   "pask_families_cnnf": (0xd5, 0x41),
                   "pask_families_dwg": (0x5b, 0x25),
                   "pask_families_cnn": (0x55, 0x61), "pask_families_dw": (0x5f, 0x7f),
                   "pask_families": (0xff, 0x7f)}
# (cnng: a small CNN whose contractions all take the gather (and split-K), no
# TMA im2col -- the tiny CNN;
#  cnnf: a CNN whose narrow stem is folded (D16): the layout's fold path, memory
# bit 7, and no cp.async gather -- ResNet-50; only cnnf and the full variant
# carry the fold path)
FAMILY_SOFTMAX_REG = {"pask_families_tf": 1, "pask_families_cnng": 0, "pask_families_cnnf": 0,
                      "pask_families_dwg": 0,
                      "pask_families_cnn": 0, "pask_families_dw": 1, "pask_families": 1}
# Packaging 3 comes in the same variants: pask_single_<v> has the cases and paths
# of pask_families_<v> behind the one entry pask_all (pask_single: everything).
SINGLE_VARIANTS = {k.replace("pask_families", "pask_single"): v for k, v in FAMILY_VARIANTS.items()}
SINGLE_SOFTMAX_REG = {k.replace("pask_families", "pask_single"): v for k, v in FAMILY_SOFTMAX_REG.items()}
EXTRA_OBJECTS = {**{k: ["pask_conv_igemm", "pask_mem"] for k in FAMILY_VARIANTS},
                 **{k: ["pask_all"] for k in SINGLE_VARIANTS},
                 "pask_primer": ["pask_primer"]}   # pask_create's driver primer (not a solution)
EXTRA_DEFINES = {k: [f"-DPASK_MEM_MASK={m:#x}", f"-DPASK_GEMM_FEAT={g:#x}",
                     f"-DPASK_SOFTMAX_REG={({**FAMILY_SOFTMAX_REG, **SINGLE_SOFTMAX_REG})[k]}"]
                 for k, (m, g) in {**FAMILY_VARIANTS, **SINGLE_VARIANTS}.items()}

# The "tuned library": one specialised conv solution per distinct
# dense-conv problem (R, S, stride, pad, dilation, input channels C) of configs
# C1-C3, i.e. the per-problem solutions a library's find step would pick
# (PAPER.md:69, :83).  Catalog ids PASK_NUM_KERNELS + i, in this sorted order.
SPECS = sorted([
    (1, 1, 1, 0, 1, 16), (1, 1, 1, 0, 1, 24), (1, 1, 1, 0, 1, 32), (1, 1, 1, 0, 1, 64),
    (1, 1, 1, 0, 1, 96), (1, 1, 1, 0, 1, 128), (1, 1, 1, 0, 1, 144), (1, 1, 1, 0, 1, 160),
    (1, 1, 1, 0, 1, 192), (1, 1, 1, 0, 1, 256), (1, 1, 1, 0, 1, 320), (1, 1, 1, 0, 1, 384),
    (1, 1, 1, 0, 1, 512), (1, 1, 1, 0, 1, 576), (1, 1, 1, 0, 1, 960), (1, 1, 1, 0, 1, 1024),
    (1, 1, 1, 0, 1, 2048), (1, 1, 2, 0, 1, 256), (1, 1, 2, 0, 1, 512), (1, 1, 2, 0, 1, 1024),
    (3, 3, 1, 1, 1, 8), (3, 3, 1, 1, 1, 16), (3, 3, 1, 1, 1, 32), (3, 3, 1, 1, 1, 64),
    (3, 3, 1, 1, 1, 128), (3, 3, 1, 1, 1, 256), (3, 3, 1, 1, 1, 512), (3, 3, 2, 1, 1, 8),
    (3, 3, 2, 1, 1, 128), (3, 3, 2, 1, 1, 256), (3, 3, 2, 1, 1, 512), (7, 7, 2, 3, 1, 8),
])


def spec_name(spec):
    r, s, st, pd, dl, c = spec
    return f"pask_conv_spec_r{r}s{s}u{st}p{pd}d{dl}c{c}"


def _gen_spec_sources():
    """_build/spec_kernels.inc (device entries) and _build/spec_catalog.h (host table)."""
    ker = []
    for sp in SPECS:
        n = spec_name(sp)
        ker.append(f"#if !defined(PASK_NO_SPECS) && (!defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_{n})\n"
                   f"__global__ void __launch_bounds__(kGemmThreads, 1) {n}(const __grid_constant__ GemmParams p) "
                   f"{{ TimelineScope ts(p.tl); conv_gemm_body<true, FixGeo<{', '.join(map(str, sp))}>>(p); }}\n#endif\n")
    host = ["// generated by build.py: the specialised conv solutions (catalog ids PASK_NUM_KERNELS + i)",
            "#pragma once", "namespace pask {",
            "struct SpecEntry { int r, s, st, pd, dl, c; const char* name; };",
            "constexpr int kNumSpecs = %d;" % len(SPECS),
            "constexpr SpecEntry kSpecs[kNumSpecs] = {"]
    host += ["    {%d, %d, %d, %d, %d, %d, \"%s\"}," % (*sp, spec_name(sp)) for sp in SPECS]
    host += ["};", "}  // namespace pask", ""]
    host += ["#define PASK_SPEC_IMAGES(X) \\"] + [f"  X({spec_name(sp)}) \\" for sp in SPECS] + [""]
    host += ["// packaging 2 families variants (name, memory-case mask, contraction-path mask),",
             "// smallest first",
             "#define PASK_FAMILY_VARIANTS(X) \\"] + \
        [f"  X({k}, {m:#x}, {g:#x}) \\" for k, (m, g) in FAMILY_VARIANTS.items()] + ["", ""]
    host += ["// packaging 3 single-entry variants, the same masks, smallest first",
             "#define PASK_SINGLE_VARIANTS(X) \\"] + \
        [f"  X({k}, {m:#x}, {g:#x}) \\" for k, (m, g) in SINGLE_VARIANTS.items()] + ["", ""]
    for path, text in ((os.path.join(BUILD, "spec_kernels.inc"), "".join(ker)),
                       (os.path.join(BUILD, "spec_catalog.h"), "\n".join(host))):
        old = open(path).read() if os.path.exists(path) else None
        if old != text:
            with open(path, "w") as f:
                f.write(text)


def _defines_stamp():
    """_build/defines.stamp: rewritten only when the build-affecting environment
    changes, so an experiment build (PASK_NVCC_DEFINES / PASK_LINEINFO) never
    leaves stale fatbins behind."""
    text = f"PASK_NVCC_DEFINES={os.environ.get('PASK_NVCC_DEFINES', '')}\n" \
           f"PASK_LINEINFO={os.environ.get('PASK_LINEINFO', '')}\n"
    path = os.path.join(BUILD, "defines.stamp")
    old = open(path).read() if os.path.exists(path) else None
    if old != text:
        with open(path, "w") as f:
            f.write(text)
    return path


def _nvcc_fatbin_cmd(out, defines=()):
    # -lineinfo (ncu source page) embeds the PTX text in the code object and
    # makes every cold load parse ~1 MB more, so it is opt-in (PASK_LINEINFO=1)
    extra = ["-lineinfo"] if os.environ.get("PASK_LINEINFO") == "1" else []
    extra += os.environ.get("PASK_NVCC_DEFINES", "").split()  # experiment builds only
    return [NVCC, *ARCH, "-fatbin", "-O3", *extra, "-std=c++17", "-Xptxas", "-v", f"-I{BUILD}",
            *defines, "-o", out, KERNEL_SRC[0]]


def _run_parallel(cmds, jobs=None):
    jobs = jobs or max(2, min(8, os.cpu_count() or 2))
    pending = list(cmds)
    running = []
    logs = {}
    while pending or running:
        while pending and len(running) < jobs:
            out, cmd = pending.pop(0)
            running.append((out, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT,
                                                  text=True)))
        out, proc = running.pop(0)
        text, _ = proc.communicate()
        if proc.returncode != 0:
            sys.stderr.write(text)
            raise RuntimeError(f"nvcc failed for {out}")
        logs[out] = text
    return logs


def build(force: bool = False, verbose: bool = False) -> str:
    """Build (if stale) and return the path of libpask.so.  Serialised across
    processes by an flock on _build/.lock (torchrun ranks, pytest workers)."""
    import fcntl
    os.makedirs(BUILD, exist_ok=True)
    with open(os.path.join(BUILD, ".lock"), "w") as lock:
        fcntl.flock(lock, fcntl.LOCK_EX)
        try:
            return _build_locked(force, verbose)
        finally:
            fcntl.flock(lock, fcntl.LOCK_UN)


def _build_locked(force: bool, verbose: bool) -> str:
    _gen_spec_sources()
    fatbin = os.path.join(BUILD, "pask.fatbin")
    names = KERNELS + list(EXTRA_OBJECTS) + [spec_name(sp) for sp in SPECS]
    per_kernel = [os.path.join(BUILD, k + ".fatbin") for k in names]
    deps = KERNEL_SRC + [os.path.join(BUILD, "spec_kernels.inc"), os.path.abspath(__file__), _defines_stamp()]
    if force or any(_stale(f, deps) for f in [fatbin] + per_kernel):
        # the generic catalog as one code object, and one code object per kernel
        cmds = [(fatbin, _nvcc_fatbin_cmd(fatbin, ["-DPASK_NO_SPECS"]))]
        for k, f in zip(names, per_kernel):
            if force or _stale(f, deps):
                entries = EXTRA_OBJECTS.get(k, [k])
                cmds.append((f, _nvcc_fatbin_cmd(f, ["-DPASK_ONLY_KERNEL"] + EXTRA_DEFINES.get(k, []) +
                                                 [f"-DPASK_ONLY_KERNEL_{e}=1" for e in entries])))
        logs = _run_parallel(cmds)
        if fatbin in logs:
            with open(os.path.join(BUILD, "ptxas.log"), "w") as fh:
                fh.write(logs[fatbin])
            if verbose:
                print(logs[fatbin])
    asm = os.path.join(BUILD, "fatbins.S")
    with open(asm, "w") as fh:
        fh.write('        .section .rodata.pask_fatbin,"a",@progbits\n')
        for sym, path in [("pask_fatbin", fatbin)] + [(f"pask_fb_{k}", f) for k, f in
                                                       zip(names, per_kernel)]:
            fh.write(f"        .balign 64\n        .globl {sym}_start\n        .hidden {sym}_start\n"
                     f"{sym}_start:\n        .incbin \"{path}\"\n        .globl {sym}_end\n"
                     f"        .hidden {sym}_end\n{sym}_end:\n        .byte 0\n")
        fh.write('        .section .note.GNU-stack,"",@progbits\n')
    host_deps = HOST_DEPS + [fatbin] + per_kernel + [os.path.join(BUILD, "spec_catalog.h"), _defines_stamp(),
                                                      os.path.abspath(__file__)]
    if force or _stale(LIB, host_deps) or _stale(TEST_LIB, host_deps):
        cxx = os.environ.get("CXX", "g++")
        flags = ["-O2", "-std=c++17", "-fPIC", "-fvisibility=hidden", "-Wall", "-Wno-unused-function",
                 f"-I{CUDA}/include", f"-I{BUILD}"]
        flags += os.environ.get("PASK_NVCC_DEFINES", "").split()  # experiment builds: same -D for host
        objs = {}
        for src in HOST_SRC + TEST_SRC:
            obj = os.path.join(BUILD, os.path.basename(src) + ".o")
            _run([cxx, *flags, "-c", src, "-o", obj])
            objs[src] = obj
        fobj = os.path.join(BUILD, "fatbin.o")
        _run([cxx, "-c", asm, "-o", fobj])
        for lib, srcs in ((LIB, HOST_SRC), (TEST_LIB, HOST_SRC + TEST_SRC)):
            tmp = lib + ".tmp"
            _run([cxx, "-shared", "-o", tmp, *[objs[x] for x in srcs], fobj, "-ldl", "-lpthread",
                  "-Wl,--no-undefined", "-Wl,--version-script=" + os.path.join(CSRC, "runtime", "exports.map")])
            shutil.move(tmp, lib)
    if force or _stale(COLD_EXE, [LIB, COLD_SRC, os.path.join(os.path.dirname(PKG), "include", "pask.h")]):
        # the native fresh-process cold-start sampler (links libpask.so, dlopens libcuda)
        cxx = os.environ.get("CXX", "g++")
        tmp = COLD_EXE + ".tmp"
        _run([cxx, "-O2", "-std=c++17", "-Wall", f"-I{CUDA}/include", COLD_SRC, "-o", tmp, f"-L{PKG}", "-lpask",
              "-ldl", "-Wl,-rpath,$ORIGIN"])
        shutil.move(tmp, COLD_EXE)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
