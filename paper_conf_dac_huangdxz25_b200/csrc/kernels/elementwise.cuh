// HBM-bound kernels of the catalog: input layout (K10), depthwise conv (K5,
// the DirectConv pattern of PAPER.md:83), pooling (K7), softmax
// and LayerNorm (K11).  All use 128-bit vectors over the contiguous channel /
// column dimension and fp32 arithmetic; reductions use warp shuffles.
#pragma once
#include "pask_params.h"
#include "ptx.cuh"

namespace pask {

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// Activation over 8 values: ReLU / ReLU6 inline, GELU / tanh through one
// out-of-line scalar routine (rare on the memory-bound path; one copy of its
// body keeps the code object small -- uploads cost ~1.1 us per KB of SASS).
// Same arithmetic as apply_act either way.
__device__ __noinline__ float act1_slow(float v, int act) { return apply_act(v, act); }
__device__ __forceinline__ void act8(float (&v)[8], int act) {
  if (act == 1) {
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = fmaxf(v[i], 0.f);
  } else if (act == 2) {
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = fminf(fmaxf(v[i], 0.f), 6.f);
  } else if (act >= 3) {
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = act1_slow(v[i], act);
  }
}

// ---------------------------------------------------------------- K10 layout
// NCHW fp32 -> NHWC bf16 (RNE), channels c..c_out-1 zero.  One thread per
// (pixel, 8-channel chunk): coalesced fp32 reads across pixels, one 16 B store.
__device__ __noinline__ void layout_fold(const LayoutParams& p);
#ifndef PASK_MEM_MASK
#define PASK_MEM_MASK 0xff
#endif
__device__ __forceinline__ void layout_body(const LayoutParams& p) {
  if (p.yf) {  // stem fold (D16): compiled into the variants whose mask has MEM_FOLD_BIT
    if ((PASK_MEM_MASK >> MEM_FOLD_BIT) & 1)
      layout_fold(p);
    else
      __trap();
    return;
  }
  pdl_wait();
  pdl_launch_dependents();
  // 32-bit indices: the planner guarantees n*h*w*c_out < 2^31
  const int chunks = p.c_out >> 3;
  const int hw = p.h * p.w;
  const int total = p.n * hw * chunks;
  for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < total; idx += gridDim.x * blockDim.x) {
    const int pix = idx / chunks;
    const int ch = idx - pix * chunks;
    const int n = pix / hw;
    const int off = pix - n * hw;
    float f[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int c = ch * 8 + i;
      f[i] = (c < p.c) ? __ldg(p.x + (n * p.c + c) * hw + off) : 0.f;
    }
    reinterpret_cast<uint4*>(p.y)[idx] = pack_bf16x8(f);
  }
}

// Stem fold (D16, LayoutParams).  Persistent CTAs walk the folded
// rows (n, t) = blockIdx.x, +gridDim.x, ...  A row's fsh input rows
// fsh*t - fph + j (all c channels, bf16 RNE, zero outside the image; fpw zero
// columns in front) are staged in smem, double-buffered: the 16 B loads of the
// next row are in flight while the current one is written out as
//   - the NHWC output rows among them (every input row belongs to exactly one
//     folded row): the same bits as the unfolded layout;
//   - the folded row yf[n][t][0..fQ) (16 B per (q, 8-channel chunk)), each
//     value one smem read at a per-thread offset + fsw*q.
// The regrouped weights wf (constant) are written by extra CTAs, on the first
// inference only.
__device__ __forceinline__ uint16_t bf16_bits(float f) {
  return static_cast<uint16_t>(pack_bf16x2(f, 0.f) & 0xffffu);
}
__device__ __forceinline__ uint4 pack_u16x8(const uint16_t (&v)[8]) {
  return make_uint4(v[0] | (uint32_t(v[1]) << 16), v[2] | (uint32_t(v[3]) << 16), v[4] | (uint32_t(v[5]) << 16),
                    v[6] | (uint32_t(v[7]) << 16));
}
constexpr int kFoldItems = 4;  // 4-column input items per thread per row (host: rows * ceil(w / 4) <= 4 * 256)
__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts_u16(uint32_t a, uint16_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"(v) : "memory");
}
__device__ __noinline__ void layout_fold(const LayoutParams& pp) {
  extern __shared__ uint8_t smem_raw[];
  // every parameter the loops use in a register: read through the reference,
  // each would be reloaded after every global store (possible aliasing)
  const float* __restrict__ x = pp.x;
  uint4* const y = static_cast<uint4*>(pp.y);
  uint4* const yf = static_cast<uint4*>(pp.yf);
  const int C = pp.c, H = pp.h, W = pp.w;  // host: W % 4 == 0, c_out == 8 (one NHWC chunk)
  const int fT = pp.fT, fQ = pp.fQ, fsh = pp.fsh, fsw = pp.fsw, fph = pp.fph, fpw = pp.fpw;
  const int Wp = pp.fWp, hw = H * W;
  const int tid = threadIdx.x, bd = blockDim.x;
  const int stage = fsh * C * Wp;  // elements per staging buffer
  const uint32_t s0 = smem_u32(smem_raw);
  pdl_wait();
  pdl_launch_dependents();
  if (static_cast<int>(blockIdx.x) >= pp.frow_ctas) {
    // regrouped weights (k, r2, chunk), 16 B per thread; host tables give each
    // folded channel's source offset within a (k, sh*r2) filter block and its j
    const int wi = (blockIdx.x - pp.frow_ctas) * bd + tid;
    if (wi < pp.fK * pp.fR2 * 8) {
      const int r2 = (wi >> 3) % pp.fR2, k = (wi >> 3) / pp.fR2;
      const int blk = pp.fS * pp.fcw;
      const uint16_t* w = static_cast<const uint16_t*>(pp.wsrc) + (k * pp.fR + fsh * r2) * blk;
      uint64_t lo = 0, hi = 0;
#pragma unroll 1
      for (int e2 = 0; e2 < 8; ++e2) {
        const int cc = (wi & 7) * 8 + e2, j = pp.fwj[cc];
        const uint64_t v = (j != 0xff && fsh * r2 + j < pp.fR) ? w[pp.fwoff[cc]] : 0;
        if (e2 < 4) lo |= v << (16 * e2); else hi |= v << (16 * (e2 - 4));
      }
      reinterpret_cast<uint4*>(pp.wf)[wi] =
          make_uint4(static_cast<uint32_t>(lo), static_cast<uint32_t>(lo >> 32), static_cast<uint32_t>(hi),
                     static_cast<uint32_t>(hi >> 32));
    }
    return;
  }
#pragma unroll 1
  for (int i = tid; i < 2 * stage; i += bd) sts_u16(s0 + 2 * i, 0);  // padding columns stay zero
  // this thread's input items (4 columns of one (j, c) row), the same every row
  const int w4n = W >> 2, items = fsh * C * w4n;
  int it_j[kFoldItems], it_src[kFoldItems], it_dst[kFoldItems];
#pragma unroll
  for (int u = 0; u < kFoldItems; ++u) {
    const int it = tid + u * bd;
    const int row = it / w4n, w0 = (it - row * w4n) * 4;
    const int j = row / C, ci = row - j * C;
    it_j[u] = it < items ? j : -(1 << 20);  // out of every image row: never loaded or stored
    it_src[u] = ci * hw + w0;
    it_dst[u] = 2 * (row * Wp + fpw + w0);
  }
  // the Y chunk of this thread (blockDim % 8 == 0): smem byte offsets of its 8
  // folded channels and a mask zeroing the padding channels (branch-free reads:
  // a padding channel reads offset 0 and masks it)
  uint32_t off[8], msk = 0;
#pragma unroll
  for (int e2 = 0; e2 < 8; ++e2) {
    const uint32_t o = pp.foff[(tid & 7) * 8 + e2];  // host table (no divisions here)
    off[e2] = o == 0xffffu ? 0u : 2u * o;
    msk |= (o == 0xffffu ? 0u : 1u) << e2;
  }
  const int nrow = pp.n * fT, rstep = pp.frow_ctas;
  __syncthreads();  // zero fill done
  // skewed pipeline, one barrier per row: iteration i issues row r_i's loads,
  // writes row r_(i-1) out of buffer (i-1)&1 while they fly, then stages r_i in
  // buffer i&1.  A buffer is restaged two iterations after it was staged, behind
  // the barrier that ends the iteration which read it.
  for (int i = 0, r = blockIdx.x;; ++i, r += rstep) {
    float4 pf[kFoldItems];
    const int t = r % fT, n = r / fT;
#pragma unroll
    for (int u = 0; u < kFoldItems; ++u) {
      const int hh = fsh * t - fph + it_j[u];
      const float* src = x + n * C * hw + it_src[u] + hh * W;
      pf[u] = (r < nrow && hh >= 0 && hh < H) ? __ldg(reinterpret_cast<const float4*>(src))
                                               : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    if (i > 0) {  // write out the previous row
      const int rp = r - rstep, tp = rp % fT, np = rp / fT;
      const uint32_t sb = s0 + 2u * static_cast<uint32_t>(((i - 1) & 1) * stage);
      // NHWC rows of that folded row (branch-free channel reads: channel
      // min(c, C - 1), masked)
#pragma unroll 1
      for (int j = 0; j < fsh; ++j) {
        const int hh = fsh * tp - fph + j;
        if (hh < 0 || hh >= H) continue;
        const uint32_t a = sb + 2u * static_cast<uint32_t>(j * C * Wp + fpw);
        uint4* yo = y + static_cast<size_t>(np * H + hh) * W;
        for (int w = tid; w < W; w += bd) {
          uint32_t v[8];
#pragma unroll
          for (int e2 = 0; e2 < 8; ++e2)
            v[e2] = lds_u16(a + 2u * static_cast<uint32_t>(min(e2, C - 1) * Wp + w)) & (e2 < C ? 0xffffu : 0u);
          yo[w] = make_uint4(v[0] | (v[1] << 16), v[2] | (v[3] << 16), v[4] | (v[5] << 16), v[6] | (v[7] << 16));
        }
      }
      uint4* yrow = yf + static_cast<size_t>(rp) * fQ * 8 + (tid & 7);
      for (int q = tid >> 3; q < fQ; q += bd >> 3) {
        const uint32_t qo = sb + 2u * static_cast<uint32_t>(fsw * q);
        uint32_t v[8];
#pragma unroll
        for (int e2 = 0; e2 < 8; ++e2) v[e2] = lds_u16(qo + off[e2]) & ((msk >> e2) & 1u ? 0xffffu : 0u);
        yrow[q * 8] = make_uint4(v[0] | (v[1] << 16), v[2] | (v[3] << 16), v[4] | (v[5] << 16), v[6] | (v[7] << 16));
      }
    }
    if (r >= nrow) break;
    const uint32_t sb = s0 + 2u * static_cast<uint32_t>((i & 1) * stage);
#pragma unroll
    for (int u = 0; u < kFoldItems; ++u) {
      if (it_j[u] < 0) continue;
      const float* f = &pf[u].x;
#pragma unroll
      for (int e2 = 0; e2 < 4; ++e2) sts_u16(sb + it_dst[u] + 2 * e2, bf16_bits(f[e2]));
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- K7 pool
// Small windows: one thread per (output pixel, 8-channel chunk).  Large windows
// (per_warp, e.g. a 7x7 global pool): one warp per output chunk, lanes stride
// over the window taps and combine with a fixed shuffle tree (deterministic).
// Max pads with -inf; avg divides by the window or by the in-range count.
__device__ __forceinline__ void pool_body(const PoolParams& p) {
  pdl_wait();
  pdl_launch_dependents();
  // 32-bit indices: the planner guarantees n*H*W*C < 2^31
  const int chunks = p.C >> 3;
  const int total = p.n * p.P * p.Q * chunks;
  const uint4* x = reinterpret_cast<const uint4*>(p.x);
  const int lane = threadIdx.x & 31;
  const int gtid = blockIdx.x * blockDim.x + threadIdx.x;
  const int first = p.per_warp ? (gtid >> 5) : gtid;
  const int step = p.per_warp ? ((gridDim.x * blockDim.x) >> 5) : gridDim.x * blockDim.x;
  const int taps = p.R * p.S;
  for (int idx = first; idx < total; idx += step) {
    int t = idx;
    const int ch = t % chunks;
    t /= chunks;
    const int q = t % p.Q;
    t /= p.Q;
    const int pp = t % p.P;
    const int n = t / p.P;
    const int ih0 = pp * p.sh - p.ph, iw0 = q * p.sw - p.pw;
    const bool is_max = p.mode == 0;
    if (is_max && !p.per_warp && taps <= 9) {
      // small max windows (ResNet-50's 3x3 s2, the tiny CNN's 2x2): every tap load
      // issued before the first combine, combined as packed bf16x2.  The max of
      // bf16 values is one of them, so this is bit-identical to the fp32 max
      // followed by RNE (the loop below), in a fifth of the code (uploads cost
      // ~1.1 us per KB of SASS).  Out-of-window taps read as -inf.
      const uint32_t ninf2 = 0xff80ff80u;
      uint4 xv[9];
      int r = 0, s = 0;
#pragma unroll
      for (int tap = 0; tap < 9; ++tap) {
        const int ih = ih0 + r, iw = iw0 + s;
        const bool ok = tap < taps && ih >= 0 && ih < p.H && iw >= 0 && iw < p.W;
        xv[tap] = ok ? __ldg(x + ((n * p.H + ih) * p.W + iw) * chunks + ch) : make_uint4(ninf2, ninf2, ninf2, ninf2);
        if (++s == p.S) {
          s = 0;
          ++r;
        }
      }
      uint4 m = xv[0];
#pragma unroll
      for (int tap = 1; tap < 9; ++tap) m = bf16x8_max(m, xv[tap]);
      reinterpret_cast<uint4*>(p.y)[idx] = m;
      continue;
    }
    float acc[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] = is_max ? -INFINITY : 0.f;
    float cnt = 0.f;
    {
#pragma unroll 1
      for (int tap = p.per_warp ? lane : 0; tap < taps; tap += p.per_warp ? 32 : 1) {
        const int r = tap / p.S, s = tap - r * p.S;
        const int ih = ih0 + r, iw = iw0 + s;
        if (ih < 0 || ih >= p.H || iw < 0 || iw >= p.W) continue;
        float f[8];
        unpack_bf16x8(__ldg(x + ((n * p.H + ih) * p.W + iw) * chunks + ch), f);
        cnt += 1.f;
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] = is_max ? fmaxf(acc[i], f[i]) : acc[i] + f[i];
      }
    }
    if (p.per_warp) {
#pragma unroll 1
      for (int o = 16; o > 0; o >>= 1) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const float other = __shfl_xor_sync(0xffffffffu, acc[i], o);
          acc[i] = p.mode == 0 ? fmaxf(acc[i], other) : acc[i] + other;
        }
        cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
      }
    }
    if (p.mode == 1) {
      const float inv = 1.f / (p.count_include_pad ? static_cast<float>(taps) : cnt);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] *= inv;
    }
    if (!p.per_warp || lane == 0) reinterpret_cast<uint4*>(p.y)[idx] = pack_bf16x8(acc);
  }
}

// Specialised global average pool (mean over H*W): one warp per (image,
// 8-channel chunk) group of 32 chunks... one lane per chunk, pixels split over
// the block's 4 warps, fp32 partial sums combined in shared memory.
__device__ __forceinline__ void gavg_body(const PoolParams& p) {
  __shared__ float red[4][32][8];
  pdl_wait();
  pdl_launch_dependents();
  const int chunks = p.C >> 3;
  const int lane = threadIdx.x & 31, wq = threadIdx.x >> 5;  // 4 warps
  const int ch = blockIdx.x * 32 + lane;
  const int n = blockIdx.y;
  const int hw = p.H * p.W;
  float acc[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) acc[i] = 0.f;
  if (ch < chunks) {
    const uint4* x = reinterpret_cast<const uint4*>(p.x) + static_cast<int64_t>(n) * hw * chunks + ch;
    // unrolled: four loads in flight per warp, the sum still in pixel order
#pragma unroll 4
    for (int px = wq; px < hw; px += 4) {
      float f[8];
      unpack_bf16x8(__ldg(x + static_cast<int64_t>(px) * chunks), f);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += f[i];
    }
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) red[wq][lane][i] = acc[i];
  __syncthreads();
  if (wq == 0 && ch < chunks) {
    const float inv = 1.f / static_cast<float>(hw);
#pragma unroll
    for (int i = 0; i < 8; ++i)
      acc[i] = (((red[0][lane][i] + red[1][lane][i]) + red[2][lane][i]) + red[3][lane][i]) * inv;
    reinterpret_cast<uint4*>(p.y)[static_cast<int64_t>(n) * chunks + ch] = pack_bf16x8(acc);
  }
}

// ---------------------------------------------------------------- K5 depthwise
// One thread per (output pixel, 8-channel chunk); weights RSC so each tap is
// one 16 B load of x and one of w; fused bias / residual / activation.
__device__ __forceinline__ void dw_body(const DwParams& p) {
  // 32-bit indices: the planner guarantees n*H*W*C < 2^31
  const int chunks = p.C >> 3;
  const int total = p.n * p.P * p.Q * chunks;
  const uint4* x = reinterpret_cast<const uint4*>(p.x);
  const uint4* w = reinterpret_cast<const uint4*>(p.w);
  // 3x3: the first output chunk's nine filter taps are loaded before
  // griddepcontrol.wait (weights do not depend on the previous layer), so their
  // HBM round trip overlaps the previous layer's tail.  (An L2 prefetch of the
  // same lines by every thread measured slower: MobileNetV2 0.2371 -> 0.2471 ms.)
  const bool k3 = p.R == 3 && p.S == 3 && p.dh == 1 && p.dw == 1;
  const int idx0 = blockIdx.x * blockDim.x + threadIdx.x;
  uint4 wpre[9];
  if (k3 && idx0 < total) {
    const int ch0 = idx0 % chunks;
#pragma unroll
    for (int t9 = 0; t9 < 9; ++t9) wpre[t9] = __ldg(w + t9 * chunks + ch0);
  }
  pdl_wait();
  pdl_launch_dependents();
  for (int idx = idx0; idx < total; idx += gridDim.x * blockDim.x) {
    int t = idx;
    const int ch = t % chunks;
    t /= chunks;
    const int q = t % p.Q;
    t /= p.Q;
    const int pp = t % p.P;
    const int n = t / p.P;
    float acc[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] = 0.f;
    const int ih0 = pp * p.sh - p.ph, iw0 = q * p.sw - p.pw;
    if (k3) {
      // 3x3 (MobileNetV2): all nine tap loads issued before the first FMA (one
      // memory round trip instead of nine); same taps, same order as below
      // (later grid-stride trips reload the taps in place: selecting between the
      // prefetched and fresh taps made the compiler peel the first trip, a second
      // copy of this body -- 4 KB more code to upload)
      uint4 xv[9];
      bool ok[9];
      if (idx != idx0) {
#pragma unroll
        for (int t9 = 0; t9 < 9; ++t9) wpre[t9] = __ldg(w + t9 * chunks + ch);
      }
#pragma unroll
      for (int t9 = 0; t9 < 9; ++t9) {
        const int ih = ih0 + t9 / 3, iw = iw0 + t9 % 3;
        ok[t9] = ih >= 0 && ih < p.H && iw >= 0 && iw < p.W;
        xv[t9] = ok[t9] ? __ldg(x + ((n * p.H + ih) * p.W + iw) * chunks + ch) : make_uint4(0, 0, 0, 0);
      }
#pragma unroll
      for (int t9 = 0; t9 < 9; ++t9) {
        if (!ok[t9]) continue;
        float xf[8], wf[8];
        unpack_bf16x8(xv[t9], xf);
        unpack_bf16x8(wpre[t9], wf);
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] = fmaf(xf[i], wf[i], acc[i]);
      }
    } else {
#pragma unroll 1
      for (int r = 0; r < p.R; ++r) {
        const int ih = ih0 + r * p.dh;
        if (ih < 0 || ih >= p.H) continue;
#pragma unroll 1
        for (int s = 0; s < p.S; ++s) {
          const int iw = iw0 + s * p.dw;
          if (iw < 0 || iw >= p.W) continue;
          float xf[8], wf[8];
          unpack_bf16x8(__ldg(x + ((n * p.H + ih) * p.W + iw) * chunks + ch), xf);
          unpack_bf16x8(__ldg(w + (r * p.S + s) * chunks + ch), wf);
#pragma unroll
          for (int i = 0; i < 8; ++i) acc[i] = fmaf(xf[i], wf[i], acc[i]);
        }
      }
    }
    if (p.bias) {
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += __ldg(p.bias + ch * 8 + i);
    }
    if (p.res) {
      float rf[8];
      unpack_bf16x8(__ldg(reinterpret_cast<const uint4*>(p.res) + idx), rf);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += rf[i];
    }
    act8(acc, p.act);
    reinterpret_cast<uint4*>(p.y)[idx] = pack_bf16x8(acc);
  }
}

// ---------------------------------------------------------------- K11 softmax
// One warp per row.  Pass 1: online max / sum of exp(scale*x - max) in fp32;
// pass 2: write exp(scale*x - max) / sum as bf16.
constexpr int kSmRegChunks = 4;  // 16 B chunks per lane kept in registers (rows <= 1024)
// the register-resident path for short rows (BERT's 1536 attention rows per
// layer); families variants for models with one softmax row compile it out
#ifndef PASK_SOFTMAX_REG
#define PASK_SOFTMAX_REG 1
#endif
__device__ __forceinline__ void softmax_body(const RowParams& p) {
  pdl_wait();
  pdl_launch_dependents();
  const int lane = threadIdx.x & 31;
  // a warp past the last row recomputes the last row and stores nothing (no early
  // exit: the shuffles below then need no divergent-warp fallback code)
  if (p.rows <= 0) return;
  const int wrow = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const bool live = wrow < p.rows;
  const int row = live ? wrow : p.rows - 1;
  const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(p.x) + static_cast<int64_t>(row) * p.cols;
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.y) + static_cast<int64_t>(row) * p.cols;
  const bool vec = (p.cols & 7) == 0;
  float m = -INFINITY, s = 0.f;
  if (PASK_SOFTMAX_REG && vec && p.cols <= 256 * kSmRegChunks) {
    // short rows (BERT attention: 128, classifiers: 1000): the row stays in
    // registers, one load round trip; same arithmetic order as the loop below
    float f[kSmRegChunks][8];
#pragma unroll
    for (int j = 0; j < kSmRegChunks; ++j) {
      const int c = lane * 8 + 256 * j;
      if (c < p.cols) {
        unpack_bf16x8(*reinterpret_cast<const uint4*>(x + c), f[j]);
        float lm = m;
#pragma unroll
        for (int i = 0; i < 8; ++i) lm = fmaxf(lm, f[j][i] * p.scale);
        s *= __expf(m - lm);
#pragma unroll
        for (int i = 0; i < 8; ++i) s += __expf(f[j][i] * p.scale - lm);
        m = lm;
      }
    }
    const float gm = warp_max(m);
    s = (m == -INFINITY) ? 0.f : s * __expf(m - gm);
    const float inv = 1.f / warp_sum(s);
#pragma unroll
    for (int j = 0; j < kSmRegChunks; ++j) {
      const int c = lane * 8 + 256 * j;
      if (live && c < p.cols) {
#pragma unroll
        for (int i = 0; i < 8; ++i) f[j][i] = __expf(f[j][i] * p.scale - gm) * inv;
        *reinterpret_cast<uint4*>(y + c) = pack_bf16x8(f[j]);
      }
    }
    return;
  }
  if (vec) {
#pragma unroll 1
    for (int c = lane * 8; c < p.cols; c += 256) {
      float f[8];
      unpack_bf16x8(*reinterpret_cast<const uint4*>(x + c), f);
      float lm = m;
#pragma unroll
      for (int i = 0; i < 8; ++i) lm = fmaxf(lm, f[i] * p.scale);
      s *= __expf(m - lm);
#pragma unroll
      for (int i = 0; i < 8; ++i) s += __expf(f[i] * p.scale - lm);
      m = lm;
    }
  } else {
#pragma unroll 1
    for (int c = lane; c < p.cols; c += 32) {
      const float v = __bfloat162float(x[c]) * p.scale;
      const float lm = fmaxf(m, v);
      s = s * __expf(m - lm) + __expf(v - lm);
      m = lm;
    }
  }
  const float gm = warp_max(m);
  s = (m == -INFINITY) ? 0.f : s * __expf(m - gm);
  const float inv = 1.f / warp_sum(s);
  if (!live) return;
  if (vec) {
#pragma unroll 1
    for (int c = lane * 8; c < p.cols; c += 256) {
      float f[8];
      unpack_bf16x8(*reinterpret_cast<const uint4*>(x + c), f);
#pragma unroll
      for (int i = 0; i < 8; ++i) f[i] = __expf(f[i] * p.scale - gm) * inv;
      *reinterpret_cast<uint4*>(y + c) = pack_bf16x8(f);
    }
  } else {
#pragma unroll 1
    for (int c = lane; c < p.cols; c += 32)
      y[c] = __float2bfloat16_rn(__expf(__bfloat162float(x[c]) * p.scale - gm) * inv);
  }
}

// ---------------------------------------------------------------- K11 LayerNorm
// One warp per row (cols % 8 == 0): mean, then biased variance of (x - mean)
// (two passes over the row, fp32), then the affine transform.  Rows of up to
// 1024 columns (BERT: 768) stay in registers: one load round trip instead of
// three (gamma / beta 16 B aligned: vector loads).  Both paths accumulate in
// the same order (lane's chunks ascending).
constexpr int kLnRegChunks = 4;  // 16 B chunks per lane kept in registers
__device__ __forceinline__ void layernorm_body(const RowParams& p) {
  const int lane = threadIdx.x & 31;
  // gamma / beta do not depend on the previous layer: the register path loads
  // this lane's values before griddepcontrol.wait (BERT 0.5394 -> 0.5336 ms with
  // an L2 prefetch, -> 0.5296 ms with the loads), so the affine step waits on no
  // memory after the reductions; the generic path pulls the lines into L2
  const bool gb16 = p.gamma && p.beta &&
                    ((reinterpret_cast<uintptr_t>(p.gamma) | reinterpret_cast<uintptr_t>(p.beta)) & 15) == 0;
  const bool in_regs = p.cols <= 256 * kLnRegChunks && gb16;
  float4 gq[kLnRegChunks][2], bq[kLnRegChunks][2];
  if (in_regs) {
#pragma unroll
    for (int j = 0; j < kLnRegChunks; ++j) {
      const int c = lane * 8 + 256 * j;
      if (c < p.cols) {
        const float4* g4 = reinterpret_cast<const float4*>(p.gamma + c);
        const float4* b4 = reinterpret_cast<const float4*>(p.beta + c);
        gq[j][0] = __ldg(g4);
        gq[j][1] = __ldg(g4 + 1);
        bq[j][0] = __ldg(b4);
        bq[j][1] = __ldg(b4 + 1);
      }
    }
  } else if (p.gamma && p.beta) {
#pragma unroll 1
    for (int c = lane * 8; c < p.cols; c += 256) {
      prefetch_l2(p.gamma + c);
      prefetch_l2(p.beta + c);
    }
  }
  pdl_wait();
  pdl_launch_dependents();
  if (p.rows <= 0) return;
  // a warp past the last row recomputes the last row and stores nothing (no
  // early exit before the shuffles: no divergent-warp fallback code)
  const int wrow = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const bool live = wrow < p.rows;
  const int row = live ? wrow : p.rows - 1;
  const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(p.x) + static_cast<int64_t>(row) * p.cols;
  __nv_bfloat16* y = reinterpret_cast<__nv_bfloat16*>(p.y) + static_cast<int64_t>(row) * p.cols;
  if (in_regs) {
    float f[kLnRegChunks][8];
#pragma unroll
    for (int j = 0; j < kLnRegChunks; ++j) {
      const int c = lane * 8 + 256 * j;
      if (c < p.cols) unpack_bf16x8(*reinterpret_cast<const uint4*>(x + c), f[j]);
    }
    float s = 0.f;
#pragma unroll
    for (int j = 0; j < kLnRegChunks; ++j)
      if (lane * 8 + 256 * j < p.cols) {
#pragma unroll
        for (int i = 0; i < 8; ++i) s += f[j][i];
      }
    const float mean = warp_sum(s) / static_cast<float>(p.cols);
    float v = 0.f;
#pragma unroll
    for (int j = 0; j < kLnRegChunks; ++j)
      if (lane * 8 + 256 * j < p.cols) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const float d = f[j][i] - mean;
          v = fmaf(d, d, v);
        }
      }
    const float rstd = rsqrtf(warp_sum(v) / static_cast<float>(p.cols) + p.eps);
#pragma unroll
    for (int j = 0; j < kLnRegChunks; ++j) {
      const int c = lane * 8 + 256 * j;
      if (c < p.cols) {
        const float4 g0 = gq[j][0], g1 = gq[j][1], b0 = bq[j][0], b1 = bq[j][1];
        const float g[8] = {g0.x, g0.y, g0.z, g0.w, g1.x, g1.y, g1.z, g1.w};
        const float be[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
        for (int i = 0; i < 8; ++i) f[j][i] = (f[j][i] - mean) * rstd * g[i] + be[i];
        if (live) *reinterpret_cast<uint4*>(y + c) = pack_bf16x8(f[j]);
      }
    }
    return;
  }
  float s = 0.f;
#pragma unroll 1
  for (int c = lane * 8; c < p.cols; c += 256) {
    float f[8];
    unpack_bf16x8(*reinterpret_cast<const uint4*>(x + c), f);
#pragma unroll
    for (int i = 0; i < 8; ++i) s += f[i];
  }
  const float mean = warp_sum(s) / static_cast<float>(p.cols);
  float v = 0.f;
#pragma unroll 1
  for (int c = lane * 8; c < p.cols; c += 256) {
    float f[8];
    unpack_bf16x8(*reinterpret_cast<const uint4*>(x + c), f);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const float d = f[i] - mean;
      v = fmaf(d, d, v);
    }
  }
  const float rstd = rsqrtf(warp_sum(v) / static_cast<float>(p.cols) + p.eps);
  if (!live) return;
#pragma unroll 1
  for (int c = lane * 8; c < p.cols; c += 256) {
    float f[8];
    unpack_bf16x8(*reinterpret_cast<const uint4*>(x + c), f);
#pragma unroll
    for (int i = 0; i < 8; ++i)
      f[i] = (f[i] - mean) * rstd * __ldg(p.gamma + c + i) + __ldg(p.beta + c + i);
    *reinterpret_cast<uint4*>(y + c) = pack_bf16x8(f);
  }
}

// ---------------------------------------------------------------- K13 GEMV
// FC layers at batch <= 8 and BERT's pooler (D12): every weight byte
// is read once, so the layer is one HBM stream of the [N][K] weights.  A lane
// holds up to kGemvPre 16-byte weight vectors in registers, loaded BEFORE
// griddepcontrol.wait (weights do not depend on the previous layer), so the HBM
// round trip overlaps the previous layer's tail; after the wait it reads the M
// activation rows (L2-resident) and accumulates in fp32.  Lane partials are
// combined by the fixed xor tree, the K slices of a column in slice order.
constexpr int kGemvPre = 8;
// fp32 dot of two 8 x bf16 vectors added to acc (bf16 -> fp32 is a 16-bit shift)
__device__ __forceinline__ float dot8(const uint4& a, const uint4& b, float acc) {
  const uint32_t av[4] = {a.x, a.y, a.z, a.w}, bv[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    acc = fmaf(__uint_as_float(av[i] << 16), __uint_as_float(bv[i] << 16), acc);
    acc = fmaf(__uint_as_float(av[i] & 0xffff0000u), __uint_as_float(bv[i] & 0xffff0000u), acc);
  }
  return acc;
}
__device__ __forceinline__ void gemv_body(const GemvParams& p) {
  // [slice][column in CTA][row] partials in the dynamic smem (2 KB, set by the
  // host): the family entries share one static-smem budget with the contraction
  extern __shared__ uint8_t smem_raw[];
  float (*part)[8][8] = reinterpret_cast<float (*)[8][8]>(smem_raw);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nc = 1 << p.nc_log2, slices = (blockDim.x >> 5) >> p.nc_log2;
  const int cc = warp & (nc - 1), slice = warp >> p.nc_log2;
  const int n = (blockIdx.x << p.nc_log2) + cc;
  const int per = p.per;                           // 16-byte vectors per K slice (host)
  const int v0 = slice * per + lane, v1 = min(p.K >> 3, slice * per + per);
  const bool live = n < p.N;
  const uint4* w = reinterpret_cast<const uint4*>(reinterpret_cast<const __nv_bfloat16*>(p.w) +
                                                  static_cast<int64_t>(live ? n : 0) * p.ldb) + v0;
  uint4 wv[kGemvPre];
#pragma unroll
  for (int j = 0; j < kGemvPre; ++j)
    wv[j] = (live && v0 + 32 * j < v1) ? __ldg(w + 32 * j) : make_uint4(0, 0, 0, 0);
  pdl_wait();
  pdl_launch_dependents();
  // rows one at a time (compact code: an upload costs ~1.1 us per KB of SASS)
#pragma unroll 1
  for (int m = 0; m < p.M; ++m) {
    const uint4* x = reinterpret_cast<const uint4*>(reinterpret_cast<const __nv_bfloat16*>(p.x) +
                                                    static_cast<int64_t>(m) * p.lda) + v0;
    float acc = 0.f;
    if (live) {
#pragma unroll
      for (int j = 0; j < kGemvPre; ++j)
        if (v0 + 32 * j < v1) acc = dot8(__ldg(x + 32 * j), wv[j], acc);
#pragma unroll 1
      for (int j = kGemvPre; v0 + 32 * j < v1; ++j) acc = dot8(__ldg(x + 32 * j), __ldg(w + 32 * j), acc);
    }
    acc = warp_sum(acc);
    if (lane == 0) part[slice][cc][m] = acc;
  }
  __syncthreads();
  const int t = threadIdx.x;
  if (t < 64) {
    const int c = t & 7, m = t >> 3;               // column in CTA, row
    const int col = (blockIdx.x << p.nc_log2) + c;
    if (c < nc && m < p.M && col < p.N) {
      float v = 0.f;
      for (int s = 0; s < slices; ++s) v += part[s][c][m];
      if (p.bias) v += __ldg(p.bias + col);
      const int64_t o = static_cast<int64_t>(m) * p.ldc + col;
      if (p.res) v += __bfloat162float(reinterpret_cast<const __nv_bfloat16*>(p.res)[o]);
      if (p.act == 1) v = fmaxf(v, 0.f);
      else if (p.act == 2) v = fminf(fmaxf(v, 0.f), 6.f);
      else if (p.act >= 3) v = act1_slow(v, p.act);
      reinterpret_cast<__nv_bfloat16*>(p.y)[o] = __float2bfloat16_rn(v);
    }
  }
}

}  // namespace pask
