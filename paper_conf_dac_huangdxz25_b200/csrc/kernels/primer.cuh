// pask_create's driver primer (D11) -- NOT a catalog solution and
// never bound to a layer.  One 128 x 64 x 64 bf16 tile through the same kind
// of instruction mix as the library's tensor-core solutions (TMA tile loads,
// mbarrier phases, tcgen05 alloc / mma / commit / ld, PDL), so that loading it
// once at pask_create takes the driver's one-time processing of such code out
// of the first model's cold window -- the state any framework process is in
// after loading its own kernels.  pask_create launches it with run = 0 (an
// immediate return); it shares no body with any solution.
#pragma once
#include "pask_params.h"
#include "ptx.cuh"

namespace pask {

template <int kN, int kK>
__device__ __forceinline__ void primer_tile(const PrimerParams& p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const uint32_t sa = smem_u32(smem), sb = sa + 16384;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + 16384 + 8192);
  uint32_t* slot = reinterpret_cast<uint32_t*>(bars + 2);
  const uint32_t full = smem_u32(bars), done = smem_u32(bars + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    mbar_init(full, 1);
    mbar_init(done, 1);
    fence_barrier_init();
    tma_prefetch_desc(&p.tmap_a);
  }
  if (warp == 0) tmem_alloc(smem_u32(slot), kN < 32 ? 32 : kN);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *slot;
  pdl_wait();
  if (threadIdx.x == 0) {
    mbar_arrive_expect_tx(full, 16384 + 8192);
    tma_load_3d(sa, &p.tmap_a, full, 0, 0, 0);
    tma_load_3d(sb, &p.tmap_b, full, 0, 0, 0);
    mbar_wait(full, 0);
    tc_fence_after();
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | (static_cast<uint32_t>(kN >> 3) << 17) |
                           (8u << 24);  // M128 N kN bf16 -> f32
#pragma unroll
    for (int k = 0; k < kK; ++k)
      umma_f16(tmem, umma_desc_sw128(sa + k * 32, 16, 1024), umma_desc_sw128(sb + k * 32, 16, 1024), idesc,
               k ? 1u : 0u);
    umma_commit(done);
  }
  __syncwarp();
  mbar_wait(done, 0);
  tc_fence_after();
  float v[16];
  for (int c = 0; c < kN; c += 16) {
    tmem_ld16(tmem + (static_cast<uint32_t>(warp * 32) << 16) + c, v);
#pragma unroll
    for (int i = 0; i < 16; ++i) p.out[(warp * 32 + lane) * 64 + c + i] = v[i];
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tmem, kN < 32 ? 32 : kN);
}

__device__ __forceinline__ void primer_body(const PrimerParams& p) {
  if (p.run == 0) return;
  primer_tile<64, 4>(p);
}

}  // namespace pask
