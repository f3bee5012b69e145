// K6 -- the shape-generic contraction kernel: implicit-GEMM convolution and
// batched GEMM on the 5th-generation tensor cores (tcgen05, accumulator in
// TMEM), one code object reused across every conv / FC layer of a model.
//
// This is the "ImplicitGEMM pattern" solution of PAPER.md:83 (§II-B), built
// generic on purpose: padding, stride, dilation, filter size, channel counts
// and the N tile are runtime parameters, so the single loaded kernel is
// applicable to every dense conv problem of ResNet-50 / MobileNetV2 (the reuse
// opportunity of PAPER.md:101, §III-B, Fig. 2).  The GEMM mode is the
// hipBLAS extension of PAPER.md:238 (§VI).
//
// Computation (GEMM view, fp32 accumulate, bf16 RNE output):
//   C[b][m][n] = act( sum_k A[b][m][k] * B[b][n][k] + bias[n] + R[b][m][n] )
//   conv: m = output pixel (n, p, q), n = output channel, k = (r, s, c) in KRSC order,
//         A[m][k] = X[n, p*sh - ph + r*dh, q*sw - pw + s*dw, c] (0 outside)
//
// Structure (192 threads, one 128 x BN output tile per CTA):
//   warps 0-3 : A_GATHER -> implicit im2col producer (cp.async, 16 B per lane,
//               SWIZZLE_128B placement); then the epilogue (TMEM -> registers ->
//               bias / residual / activation -> bf16 NHWC stores, or split-K)
//   warp 4    : TMA producer (B always; A in A_TMA mode)
//   warp 5    : TMEM allocator + single-thread tcgen05.mma issuer
//   smem ring : `stages` x {A 128x64, B BNx64} bf16, full/empty mbarriers
//   split-K   : deterministic -- every split writes an fp32 partial tile; the
//               last-arriving CTA (atomic ticket) sums the partials in split
//               order 0..S-1 and runs the epilogue, so a given (kernel, problem)
//               is bitwise reproducible (SURVEY.md §7 hard part 8).
#pragma once
#include "pask_params.h"
#include "ptx.cuh"

namespace pask {

__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Epilogue for 16 consecutive output columns of one row.
__device__ __forceinline__ void store_row16(const GemmParams& p, int b, int m, int n0,
                                            float (&v)[16]) {
  const int64_t base = p.off_c + (int64_t)b * p.stride_c + (int64_t)m * p.ldc + n0;
  const bool full = (n0 + 16 <= p.N) && ((base & 7) == 0);
  if (p.bias) {
#pragma unroll
    for (int i = 0; i < 16; ++i)
      if (n0 + i < p.N) v[i] += __ldg(p.bias + n0 + i);
  }
  const __nv_bfloat16* res = reinterpret_cast<const __nv_bfloat16*>(p.res);
  __nv_bfloat16* out = reinterpret_cast<__nv_bfloat16*>(p.out);
  if (full) {
    if (res) {
      uint4 r0 = *reinterpret_cast<const uint4*>(res + base);
      uint4 r1 = *reinterpret_cast<const uint4*>(res + base + 8);
      float f0[8], f1[8];
      unpack_bf16x8(r0, f0);
      unpack_bf16x8(r1, f1);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        v[i] += f0[i];
        v[8 + i] += f1[i];
      }
    }
    float a0[8], a1[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      a0[i] = apply_act(v[i], p.act);
      a1[i] = apply_act(v[8 + i], p.act);
    }
    *reinterpret_cast<uint4*>(out + base) = pack_bf16x8(a0);
    *reinterpret_cast<uint4*>(out + base + 8) = pack_bf16x8(a1);
  } else {
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      if (n0 + i < p.N) {
        float t = v[i];
        if (res) t += __bfloat162float(res[base + i]);
        out[base + i] = __float2bfloat16_rn(apply_act(t, p.act));
      }
    }
  }
}

template <bool kAllowGather>
__device__ __forceinline__ void conv_gemm_body(const GemmParams& p) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ uint32_t s_last;
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int stages = p.stages;
  const int bn = p.bn;
  constexpr uint32_t kABytes = kBM * kBK * 2;  // 16 KB
  const uint32_t b_bytes = static_cast<uint32_t>(bn) * kBK * 2;
  const uint32_t stage_bytes = kABytes + b_bytes;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + stages * stage_bytes);
  const uint32_t full0 = smem_u32(bars);
  const uint32_t empty0 = smem_u32(bars + stages);
  const uint32_t accum_bar = smem_u32(bars + 2 * stages);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * stages + 1);
  const uint32_t smem_base = smem_u32(smem);

  const bool gather = kAllowGather && (p.a_mode == A_GATHER);
  const int mt = blockIdx.x, nt = blockIdx.y;
  const int b = blockIdx.z / p.splits;
  const int split = blockIdx.z - b * p.splits;
  const int kb_begin = split * p.kb_per_split;
  const int kb_end = min(p.num_kb, kb_begin + p.kb_per_split);
  const int nk = kb_end - kb_begin;  // >= 1 (host guarantees)

  // ---------------- prologue (overlaps the previous kernel under PDL)
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      mbar_init(full0 + 8 * s, gather ? 129u : 1u);
      mbar_init(empty0 + 8 * s, 1u);
    }
    mbar_init(accum_bar, 1u);
    fence_barrier_init();
  }
  if (warp == 4 && lane == 0) {
    if (!gather) tma_prefetch_desc(&p.tmap_a);
    tma_prefetch_desc(&p.tmap_b);
  }
  if (warp == 5) tmem_alloc(smem_u32(tmem_slot), p.tmem_cols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  pdl_wait();               // inputs of this layer are complete and visible
  pdl_launch_dependents();  // let the next layer's prologue start

  if (warp == 4) {
    // ================= TMA producer
    if (lane == 0) {
      for (int i = 0; i < nk; ++i) {
        const int s = i % stages;
        const uint32_t ph = (i / stages) & 1;
        mbar_wait(empty0 + 8 * s, ph ^ 1);
        const uint32_t sa = smem_base + s * stage_bytes;
        const uint32_t sb = sa + kABytes;
        const int kb = kb_begin + i;
        mbar_arrive_expect_tx(full0 + 8 * s, b_bytes + (gather ? 0u : kABytes));
        if (!gather) tma_load_3d(sa, &p.tmap_a, full0 + 8 * s, kb * kBK, mt * kBM, b);
        if (p.b_major == 0) {
          tma_load_3d(sb, &p.tmap_b, full0 + 8 * s, kb * kBK, nt * bn, b);
        } else {
          for (int j = 0; j < bn / 64; ++j)
            tma_load_3d(sb + j * 8192, &p.tmap_b, full0 + 8 * s, nt * bn + j * 64, kb * kBK, b);
        }
      }
    }
  } else if (warp == 5) {
    // ================= MMA issuer (one thread issues for the whole CTA)
    if (lane == 0) {
      for (int i = 0; i < nk; ++i) {
        const int s = i % stages;
        const uint32_t ph = (i / stages) & 1;
        mbar_wait(full0 + 8 * s, ph);
        tc_fence_after();
        const uint32_t sa = smem_base + s * stage_bytes;
        const uint32_t sb = sa + kABytes;
#pragma unroll
        for (int k = 0; k < kBK / 16; ++k) {
          // K-major SWIZZLE_128B: +32 B per 16-element K step inside the 128 B row
          const uint64_t adesc = umma_desc_sw128(sa + k * 32, 16, 1024);
          const uint64_t bdesc = (p.b_major == 0)
                                     ? umma_desc_sw128(sb + k * 32, 16, 1024)
                                     // MN-major: +16 K rows of 128 B; 64-wide N chunks 8 KB apart
                                     : umma_desc_sw128(sb + k * 2048, 8192, 1024);
          umma_f16(tmem_base, adesc, bdesc, p.idesc, (i | k) != 0 ? 1u : 0u);
        }
        umma_commit(empty0 + 8 * s);  // frees the smem slot when these MMAs complete
      }
      umma_commit(accum_bar);  // accumulator complete -> epilogue
    }
    __syncwarp();
  } else {
    // ================= warps 0-3
    const int t = threadIdx.x;  // 0..127
    if (kAllowGather && gather) {
      // implicit im2col: lane t owns 16 B chunk j = t % 8 of rows rg + 16 * ri
      const int j = t & 7;
      const int rg = t >> 3;
      const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(p.x);
      int ih0[8], iw0[8], nb[8];
      bool rv[8];
      const int pq = p.P * p.Q;
#pragma unroll
      for (int ri = 0; ri < 8; ++ri) {
        const int m = mt * kBM + rg + 16 * ri;
        rv[ri] = m < p.M;
        const int mm = rv[ri] ? m : 0;
        const int n = mm / pq;
        const int rem = mm - n * pq;
        const int pp = rem / p.Q;
        const int qq = rem - pp * p.Q;
        ih0[ri] = pp * p.sh - p.ph;
        iw0[ri] = qq * p.sw - p.pw;
        nb[ri] = n * p.H;
      }
      int kk = kb_begin * kBK + 8 * j;
      int tap = kk / p.C;
      int c = kk - tap * p.C;
      int r = tap / p.S;
      int s = tap - r * p.S;
      const int lag = min(2, stages - 1);
      for (int i = 0; i < nk; ++i) {
        const int st = i % stages;
        const uint32_t ph = (i / stages) & 1;
        mbar_wait(empty0 + 8 * st, ph ^ 1);
        const uint32_t sa = smem_base + st * stage_bytes;
        const bool kval = kk < p.K;
        const int dih = r * p.dh, diw = s * p.dw;
#pragma unroll
        for (int ri = 0; ri < 8; ++ri) {
          const int row = rg + 16 * ri;
          const uint32_t dst = sa + row * 128 + ((j ^ (row & 7)) << 4);
          const int ih = ih0[ri] + dih;
          const int iw = iw0[ri] + diw;
          const bool ok = kval && rv[ri] && ih >= 0 && ih < p.H && iw >= 0 && iw < p.W;
          const __nv_bfloat16* src =
              ok ? x + ((static_cast<int64_t>(nb[ri] + ih) * p.W + iw) * p.C + c) : x;
          cp_async_16(dst, src, ok ? 16u : 0u);
        }
        cp_async_commit();
        if (i >= lag) {
          cp_async_wait_dyn(lag);
          fence_proxy_async_smem();  // generic-proxy smem writes -> tcgen05 (async proxy)
          mbar_arrive(full0 + 8 * ((i - lag) % stages));
        }
        kk += kBK;
        c += kBK;
        while (c >= p.C) {
          c -= p.C;
          if (++s == p.S) {
            s = 0;
            ++r;
          }
        }
      }
      cp_async_wait<0>();
      fence_proxy_async_smem();
      for (int i = max(0, nk - lag); i < nk; ++i) mbar_arrive(full0 + 8 * (i % stages));
    }

    // ---------------- epilogue: TMEM lane == tile row
    mbar_wait(accum_bar, 0);
    tc_fence_after();
    const int row = warp * 32 + lane;
    const int m = mt * kBM + row;
    const uint32_t taddr = tmem_base + (static_cast<uint32_t>(warp * 32) << 16);
    if (p.splits == 1) {
      for (int cb = 0; cb < bn; cb += 16) {
        float v[16];
        tmem_ld16(taddr + cb, v);
        const int n0 = nt * bn + cb;
        if (m < p.M && n0 < p.N) store_row16(p, b, m, n0, v);
      }
    } else {
      const int tile = (b * p.m_tiles + mt) * p.n_tiles + nt;
      float* part = p.ws_partial + (static_cast<int64_t>(tile * p.splits + split) * kBM + row) * bn;
      for (int cb = 0; cb < bn; cb += 16) {
        float v[16];
        tmem_ld16(taddr + cb, v);
#pragma unroll
        for (int q4 = 0; q4 < 4; ++q4)
          __stcg(reinterpret_cast<float4*>(part + cb) + q4,
                 make_float4(v[4 * q4], v[4 * q4 + 1], v[4 * q4 + 2], v[4 * q4 + 3]));
      }
      __threadfence();
      named_bar_sync(1, 128);
      if (t == 0) {
        const uint32_t old = atomicAdd(p.ws_counter + tile, 1u);
        s_last = (old == static_cast<uint32_t>(p.splits - 1)) ? 1u : 0u;
      }
      named_bar_sync(1, 128);
      if (s_last) {
        __threadfence();
        const float* base = p.ws_partial + (static_cast<int64_t>(tile * p.splits) * kBM + row) * bn;
        if (m < p.M) {
          for (int cb = 0; cb < bn; cb += 16) {
            const int n0 = nt * bn + cb;
            if (n0 >= p.N) break;
            float v[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) v[i] = 0.f;
            for (int sp = 0; sp < p.splits; ++sp) {  // fixed order: deterministic
              const float4* src = reinterpret_cast<const float4*>(
                  base + static_cast<int64_t>(sp) * kBM * bn + cb);
#pragma unroll
              for (int q4 = 0; q4 < 4; ++q4) {
                const float4 f = __ldcg(src + q4);
                v[4 * q4] += f.x;
                v[4 * q4 + 1] += f.y;
                v[4 * q4 + 2] += f.z;
                v[4 * q4 + 3] += f.w;
              }
            }
            store_row16(p, b, m, n0, v);
          }
        }
        if (t == 0) p.ws_counter[tile] = 0u;  // self-reset for the next layer / inference
      }
    }
  }

  // ---------------- teardown
  tc_fence_before();
  __syncthreads();
  if (warp == 5) {
    tc_fence_after();
    tmem_dealloc(tmem_base, p.tmem_cols);
  }
}

}  // namespace pask
