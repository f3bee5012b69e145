// The whole PASK kernel catalog in ONE translation unit -> ONE SASS-only
// cubin -> ONE code object embedded in libpask.so ("a single fatbin layout
// that minimises distinct code objects"; BASELINE.json north_star).  Each
// extern "C" entry is one catalog solution (include/pask.h PASK_K_*); the
// loader fetches them individually with cuLibraryGetKernel + cuFuncLoad.
#include "conv_gemm.cuh"
#include "elementwise.cuh"

using namespace pask;

extern "C" {

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_layout
// PASK_K_LAYOUT
__global__ void __launch_bounds__(256) pask_layout(const __grid_constant__ LayoutParams p) {
  layout_body(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_conv_igemm
// PASK_K_CONV_IGEMM: generic implicit-GEMM conv (A by gather, or TMA for 1x1 s1 p0)
__global__ void __launch_bounds__(kGemmThreads, 1) pask_conv_igemm(const __grid_constant__ GemmParams p) {
  conv_gemm_body<true>(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_conv_1x1
// PASK_K_CONV_1X1: specialised 1x1 / stride 1 / pad 0 conv (A by TMA only)
__global__ void __launch_bounds__(kGemmThreads, 1) pask_conv_1x1(const __grid_constant__ GemmParams p) {
  conv_gemm_body<false>(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_conv_dw
// PASK_K_CONV_DW
__global__ void __launch_bounds__(256) pask_conv_dw(const __grid_constant__ DwParams p) { dw_body(p); }
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_pool
// PASK_K_POOL
__global__ void __launch_bounds__(256) pask_pool(const __grid_constant__ PoolParams p) { pool_body(p); }
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_pool_gavg
// PASK_K_POOL_GAVG
__global__ void __launch_bounds__(128) pask_pool_gavg(const __grid_constant__ PoolParams p) { gavg_body(p); }
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_gemm
// PASK_K_GEMM: batched GEMM (A K-major by TMA; B K- or MN-major by TMA)
__global__ void __launch_bounds__(kGemmThreads, 1) pask_gemm(const __grid_constant__ GemmParams p) {
  conv_gemm_body<false>(p);
}
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_softmax
// PASK_K_SOFTMAX
__global__ void __launch_bounds__(256) pask_softmax(const __grid_constant__ RowParams p) { softmax_body(p); }
#endif

#if !defined(PASK_ONLY_KERNEL) || PASK_ONLY_KERNEL_pask_layernorm
// PASK_K_LAYERNORM
__global__ void __launch_bounds__(256) pask_layernorm(const __grid_constant__ RowParams p) { layernorm_body(p); }
#endif

}  // extern "C"
