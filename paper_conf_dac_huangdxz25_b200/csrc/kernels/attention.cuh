// K12 -- fused multi-head attention ("QK^T -> softmax ->
// PV in one tcgen05 kernel, since seq 128 <= N-tile 256").  Replaces the qk,
// softmax and pv layers of a transformer block by one launch; the scores never
// leave the SM.
//
// Computation, for sequence b, head h, query i (no mask):
//   s_ij = sum_e Q[i][h*64+e] K[j][h*64+e]            (tcgen05.mma, fp32 in TMEM)
//   p_ij = exp(scale*s_ij - max_j scale*s_ij)         (fp32; stored bf16 as MMA operand)
//   O[i][h*64+d] = (sum_j p_ij V[j][h*64+d]) / sum_j p_ij   (tcgen05.mma, fp32 in TMEM)
// i.e. softmax(scale * Q K^T) V with the normalisation applied to the fp32
// accumulator (flash-attention order) instead of to the bf16 probabilities.
//
// Structure (320 threads, one CTA per 128 queries x head x sequence):
//   warp 8    : TMA producer: Q tile (128 x 64), K and V (s_pad x 64 each) from
//               the packed QKV rows; tails beyond S are zero-filled by TMA
//   warp 9    : TMEM allocator + MMA issuer: S = Q K^T into TMEM cols [0, s_pad),
//               then O = P V into TMEM cols [s_pad, s_pad + 64)
//   warps 0-7 : two warps per TMEM lane quarter; warp w owns query rows
//               32 (w % 4) .. + 31 (TMEM lanes) and key half w / 4 of them: a
//               max pass and an exp / sum pass over its half of the row's
//               scores, the two halves combined through smem in fixed order,
//               writing bf16 P into smem in the UMMA K-major SWIZZLE_128B
//               layout; then half of the O epilogue (x 1/sum).
#pragma once
#include "pask_params.h"
#include "ptx.cuh"

namespace pask {

__device__ __forceinline__ void named_bar_sync_attn(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

__device__ __forceinline__ void attention_body(const AttnParams& p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int t = threadIdx.x;
  const int nkb = p.s_pad >> 6;  // 64-key blocks
  const int m0 = blockIdx.x * 128;
  const int h = blockIdx.y;
  const int b = blockIdx.z;
  // smem: Q 16 KB | K nkb x 8 KB | V nkb x 8 KB | P nkb x 16 KB | barriers
  const uint32_t base = smem_u32(smem);
  const uint32_t sq = base;
  const uint32_t sk = sq + 16384;
  const uint32_t sv = sk + nkb * 8192;
  const uint32_t sp = sv + nkb * 8192;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + 16384 + nkb * (8192 * 2 + 16384));
  const uint32_t bar_qk = smem_u32(bars), bar_v = smem_u32(bars + 1), bar_s = smem_u32(bars + 2);
  const uint32_t bar_p = smem_u32(bars + 3), bar_o = smem_u32(bars + 4);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 5);
  float* red = reinterpret_cast<float*>(bars + 8);  // [2 halves][128 rows] partial max / sum

  if (t == 0) {
    mbar_init(bar_qk, 1);
    mbar_init(bar_v, 1);
    mbar_init(bar_s, 1);
    mbar_init(bar_p, 256);
    mbar_init(bar_o, 1);
    fence_barrier_init();
  }
  if (warp == 8 && lane == 0) tma_prefetch_desc(&p.tmap_qkv);
  if (warp == 9) tmem_alloc(smem_u32(tmem_slot), p.tmem_cols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_launch_dependents();
  pdl_wait();  // Q, K, V are the previous layer's output

  if (warp == 8) {
    if (lane == 0) {
      const int qc = h * 64, kc = p.H + h * 64, vc = 2 * p.H + h * 64;
      mbar_arrive_expect_tx(bar_qk, 16384u + nkb * 8192u);
      tma_load_3d(sq, &p.tmap_qkv, bar_qk, qc, m0, b);
      tma_load_3d(sq + 8192, &p.tmap_qkv, bar_qk, qc, m0 + 64, b);
      for (int j = 0; j < nkb; ++j) tma_load_3d(sk + j * 8192, &p.tmap_qkv, bar_qk, kc, 64 * j, b);
      mbar_arrive_expect_tx(bar_v, nkb * 8192u);
      for (int j = 0; j < nkb; ++j) tma_load_3d(sv + j * 8192, &p.tmap_qkv, bar_v, vc, 64 * j, b);
    }
    __syncwarp();
  } else if (warp == 9) {
    if (lane == 0) {
      mbar_wait(bar_qk, 0);
      tc_fence_after();
#pragma unroll
      for (int k = 0; k < 4; ++k)  // head dim 64 = 4 x K16
        umma_f16(tmem, umma_desc_sw128(sq + k * 32, 16, 1024), umma_desc_sw128(sk + k * 32, 16, 1024),
                 p.idesc_qk, k > 0 ? 1u : 0u);
      umma_commit(bar_s);
      mbar_wait(bar_p, 0);  // bf16 P written by the 256 softmax threads
      mbar_wait(bar_v, 0);
      tc_fence_after();
      for (int j = 0; j < nkb; ++j)
#pragma unroll
        for (int k = 0; k < 4; ++k)  // 64 keys = 4 x K16; V is MN-major (+16 key rows = 2048 B)
          umma_f16(tmem + p.s_pad, umma_desc_sw128(sp + j * 16384 + k * 32, 16, 1024),
                   umma_desc_sw128(sv + j * 8192 + k * 2048, 8192, 1024), p.idesc_pv, (j | k) != 0 ? 1u : 0u);
      umma_commit(bar_o);
    }
    __syncwarp();
  } else {
    // ---- softmax: row r = TMEM lane r of quarter warp % 4, key half warp / 4
    const int q4 = warp & 3, hf = warp >> 2;
    const int r = q4 * 32 + lane;
    const uint32_t taddr = tmem + (static_cast<uint32_t>(q4 * 32) << 16);
    mbar_wait(bar_s, 0);
    tc_fence_after();
    const int nc = p.s_pad >> 4;  // 16-column chunks (a multiple of 4)
    const int c0 = hf * (nc >> 1), c1 = c0 + (nc >> 1);
    float mx = -INFINITY;
    for (int c = c0; c < c1; ++c) {
      float v[16];
      tmem_ld16(taddr + c * 16, v);
#pragma unroll
      for (int i = 0; i < 16; ++i)
        if (c * 16 + i < p.S) mx = fmaxf(mx, v[i]);
    }
    red[hf * 128 + r] = mx;
    named_bar_sync_attn(1, 256);
    mx = fmaxf(red[r], red[128 + r]);
    const float msc = mx * p.scale_log2e;
    float sum = 0.f;
    for (int c = c0; c < c1; ++c) {
      float v[16];
      tmem_ld16(taddr + c * 16, v);
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        v[i] = (c * 16 + i < p.S) ? exp2f(fmaf(v[i], p.scale_log2e, -msc)) : 0.f;
        sum += v[i];
      }
      // key block j = c / 4, 16 B chunks cc, cc + 1 of row r (K-major SWIZZLE_128B)
      const int j = c >> 2, cc = (c & 3) * 2;
      const uint32_t row = sp + j * 16384 + r * 128;
      sts_u4(row + ((cc ^ (r & 7)) << 4), pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]),
             pack_bf16x2(v[4], v[5]), pack_bf16x2(v[6], v[7]));
      sts_u4(row + (((cc + 1) ^ (r & 7)) << 4), pack_bf16x2(v[8], v[9]), pack_bf16x2(v[10], v[11]),
             pack_bf16x2(v[12], v[13]), pack_bf16x2(v[14], v[15]));
    }
    fence_proxy_async_smem();  // generic-proxy P writes -> tcgen05.mma (async proxy)
    mbar_arrive(bar_p);
    named_bar_sync_attn(1, 256);  // every max read before the slots are reused for sums
    red[hf * 128 + r] = sum;
    named_bar_sync_attn(1, 256);
    const float inv = 1.f / (red[r] + red[128 + r]);  // halves in fixed order
    // ---- O epilogue: O / sum -> bf16 -> out[b][m0 + r][h*64 ...], 32 columns per half
    mbar_wait(bar_o, 0);
    tc_fence_after();
    const bool live = m0 + r < p.S;
    uint4* o = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.out) +
                                        (static_cast<int64_t>(b) * p.S + m0 + r) * p.H + h * 64);
#pragma unroll 1
    for (int c = 2 * hf; c < 2 * hf + 2; ++c) {
      float v[16];
      tmem_ld16(taddr + p.s_pad + c * 16, v);
      if (live) {
        o[2 * c] = make_uint4(pack_bf16x2(v[0] * inv, v[1] * inv), pack_bf16x2(v[2] * inv, v[3] * inv),
                              pack_bf16x2(v[4] * inv, v[5] * inv), pack_bf16x2(v[6] * inv, v[7] * inv));
        o[2 * c + 1] = make_uint4(pack_bf16x2(v[8] * inv, v[9] * inv), pack_bf16x2(v[10] * inv, v[11] * inv),
                                  pack_bf16x2(v[12] * inv, v[13] * inv), pack_bf16x2(v[14] * inv, v[15] * inv));
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 9) {
    tc_fence_after();
    tmem_dealloc(tmem, p.tmem_cols);
  }
}

}  // namespace pask
