// The whole PASK kernel catalog in ONE translation unit -> ONE SASS-only
// cubin -> ONE code object embedded in libpask.so ("a single fatbin layout
// that minimises distinct code objects"; BASELINE.json north_star).  Each
// extern "C" entry is one catalog solution (include/pask.h PASK_K_*); the
// loader fetches them individually with cuLibraryGetKernel + cuFuncLoad.
#include "conv_gemm.cuh"
#include "attention.cuh"
#include "elementwise.cuh"
#include "primer.cuh"

using namespace pask;

// resident CTAs per SM the one-tile contraction entries are compiled for
// (register budget); experiment builds may ask for 2
#ifndef PASK_GEMM_MIN_BLOCKS
#define PASK_GEMM_MIN_BLOCKS 1
#endif

static_assert(kTimelineStride == 4096, "TimelineScope (ptx.cuh) hard-codes the end-slot offset");

// PASK_MEM_MASK (bit per MemKind) selects the memory-family cases compiled into
// a code object: packaging 2 ships the families object in variants (all cases,
// CNN, CNN + depthwise, transformer) and loads the smallest one covering the
// model's bound solutions (D8).  A case compiled out traps: the host
// never binds it, and if it did the launch fails loudly instead of writing nothing.
// (bit 7, MEM_FOLD_BIT: the layout's stem-fold path, D16)
#ifndef PASK_MEM_MASK
#define PASK_MEM_MASK 0xff
#endif
#define PASK_MEM_CASE(k, body) \
  case k:                     \
    if ((PASK_MEM_MASK >> (k)) & 1) { body; } else { __trap(); } \
    break;

// The memory-bound family: the solution's own body selected by p.kind.
__device__ __forceinline__ void mem_dispatch(const MemParams& p) {
  switch (p.kind) {
    PASK_MEM_CASE(MEM_LAYOUT, TimelineScope ts(p.l.tl); layout_body(p.l))
    PASK_MEM_CASE(MEM_DW, TimelineScope ts(p.d.tl); dw_body(p.d))
    PASK_MEM_CASE(MEM_POOL, TimelineScope ts(p.p.tl); pool_body(p.p))
    PASK_MEM_CASE(MEM_GAVG, TimelineScope ts(p.p.tl); gavg_body(p.p))
    PASK_MEM_CASE(MEM_SOFTMAX, TimelineScope ts(p.r.tl); softmax_body(p.r))
    PASK_MEM_CASE(MEM_LAYERNORM, TimelineScope ts(p.r.tl); layernorm_body(p.r))
    PASK_MEM_CASE(MEM_GEMV, TimelineScope ts(p.v.tl); gemv_body(p.v))
    default: __trap();
  }
}

extern "C" {

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_layout
// PASK_K_LAYOUT
__global__ void __launch_bounds__(256) pask_layout(const __grid_constant__ LayoutParams p) {
  TimelineScope ts(p.tl);
  layout_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_conv_igemm
// PASK_K_CONV_IGEMM: generic implicit-GEMM conv (A by gather, or TMA for 1x1 s1 p0)
__global__ void __launch_bounds__(kGemmThreads, PASK_GEMM_MIN_BLOCKS) pask_conv_igemm(const __grid_constant__ GemmParams p) {
  TimelineScope ts(p.tl);
  conv_gemm_body<true>(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_conv_igemm_pt
// PASK_K_CONV_IGEMM_PT: the implicit-GEMM conv as persistent tiles (<= #SMs CTAs
// loop over the tiles, double-buffered TMEM accumulator / staging, store agent)
__global__ void __launch_bounds__(kGemmThreadsPT, 1) pask_conv_igemm_pt(const __grid_constant__ GemmParams p) {
  TimelineScope ts(p.tl);
  conv_gemm_body_pt<true>(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_conv_1x1
// PASK_K_CONV_1X1: specialised 1x1 / stride 1 / pad 0 conv (A by TMA only)
__global__ void __launch_bounds__(kGemmThreads, PASK_GEMM_MIN_BLOCKS) pask_conv_1x1(const __grid_constant__ GemmParams p) {
  TimelineScope ts(p.tl);
  conv_gemm_body<false>(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_conv_dw
// PASK_K_CONV_DW
__global__ void __launch_bounds__(256) pask_conv_dw(const __grid_constant__ DwParams p) {
  TimelineScope ts(p.tl);
  dw_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_pool
// PASK_K_POOL
__global__ void __launch_bounds__(256) pask_pool(const __grid_constant__ PoolParams p) {
  TimelineScope ts(p.tl);
  pool_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_pool_gavg
// PASK_K_POOL_GAVG
__global__ void __launch_bounds__(128) pask_pool_gavg(const __grid_constant__ PoolParams p) {
  TimelineScope ts(p.tl);
  gavg_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_gemm
// PASK_K_GEMM: batched GEMM (A K-major by TMA; B K- or MN-major by TMA)
__global__ void __launch_bounds__(kGemmThreads, PASK_GEMM_MIN_BLOCKS) pask_gemm(const __grid_constant__ GemmParams p) {
  TimelineScope ts(p.tl);
  conv_gemm_body<false>(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_attention
// PASK_K_ATTENTION: fused QK^T -> softmax -> PV (tcgen05, scores in TMEM)
__global__ void __launch_bounds__(320, 1) pask_attention(const __grid_constant__ AttnParams p) {
  TimelineScope ts(p.tl);
  attention_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_softmax
// PASK_K_SOFTMAX
__global__ void __launch_bounds__(256) pask_softmax(const __grid_constant__ RowParams p) {
  TimelineScope ts(p.tl);
  softmax_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_layernorm
// PASK_K_LAYERNORM
__global__ void __launch_bounds__(256) pask_layernorm(const __grid_constant__ RowParams p) {
  TimelineScope ts(p.tl);
  layernorm_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_gemv
// PASK_K_GEMV (D12)
__global__ void __launch_bounds__(kGemvThreads) pask_gemv(const __grid_constant__ GemvParams p) {
  TimelineScope ts(p.tl);
  gemv_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_mem
// Family entry of packaging 2 (D8): the memory-bound solutions in one
// CUfunction -- one code upload instead of up to six (a function upload costs a
// fixed ~20-40 us on top of its size, profiles/r01_loader_microbench.md).  Each
// case is the same body as the solution's own entry, so outputs are bitwise equal.
__global__ void __launch_bounds__(256) pask_mem(const __grid_constant__ MemParams p) { mem_dispatch(p); }
#endif

#if defined(PASK_ONLY_KERNEL) && PASK_ONLY_KERNEL_pask_all  // own code object only
// Single-function entry of packaging 3 (D10): the generic contraction
// body and the memory family behind one branch on a uniform parameter -- one code
// upload for a whole CNN / transformer catalog.  Same bodies as the solutions' own
// entries, so outputs are bitwise equal.
__global__ void __launch_bounds__(kGemmThreads, 1) pask_all(const __grid_constant__ AllParams p) {
  if (p.g.family == 0) {
    TimelineScope ts(p.g.tl);
    conv_gemm_body<true>(p.g);
  } else {
    mem_dispatch(p.m);
  }
}
#endif

#if defined(PASK_ONLY_KERNEL) && PASK_ONLY_KERNEL_pask_primer  // own code object only
// Not a solution: pask_create's driver primer (primer.cuh, D11).
__global__ void __launch_bounds__(128, 1) pask_primer(const __grid_constant__ PrimerParams p) { primer_body(p); }
#endif

// Per-problem specialised conv solutions (the tuned library of the Baseline
// scheme; generated by build.py from its SPECS table).
#include "spec_kernels.inc"

}  // extern "C"
