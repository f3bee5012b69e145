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
// Structure (352 threads, one 128 x BN output tile per CTA or cluster, or a
// persistent CTA looping over tiles):
//   warps 0-7 : bias -> smem; A_GATHER: implicit im2col producer (cp.async,
//               16 B per lane, SWIZZLE_128B placement); then the epilogue, two
//               warps per TMEM lane quarter (alternate 16-column chunks)
//   warp 8    : TMA producer (B always, A in A_TMA mode, the residual tile)
//   warp 9    : TMEM allocator + single-thread tcgen05.mma issuer
//   warp 10   : store agent: TMA store of each staged tile, residual prefetch
//   smem      : ring of `stages` x {A 128x64, B BNx64} bf16 with full/empty
//               mbarriers; residual/output staging tile; bias vector
//   epilogue  : TMEM -> registers -> (+bias, +residual from smem, act) -> bf16
//               staged in smem -> TMA tensor store (clips the M / N tails)
//   split-K   : a thread-block cluster of S = 2/4/8 CTAs along z, one K range
//               each; rank r owns rows [r*128/S, (r+1)*128/S) of the tile.  Every
//               CTA pushes each fp32 row of its partial to the owner's receive
//               slot [source rank] (st.async into DSMEM, completion counted on the
//               owner's mbarrier); the owner sums its S slots in fixed rank order
//               0..S-1 -- deterministic, so a given (kernel, problem) is bitwise
//               reproducible (SURVEY.md §7 part 8) -- and runs the epilogue.
#pragma once
#include "pask_params.h"
#include "ptx.cuh"

namespace pask {

// Paths compiled into the one-tile contraction body (conv_gemm_body).  The
// operator-families objects come in variants (build.py FAMILY_VARIANTS) that
// compile only the paths their models' plans use, so a model uploads less code
// (an upload costs ~1.1 us per KB of SASS, D8 / D13); the host picks
// the smallest variant covering every contraction node, and a launch that asks
// for a path compiled out traps instead of computing something else.
enum GemmFeat : unsigned {
  GF_SPLITK = 1,    // split-K thread-block clusters (DSMEM reduction)
  GF_MN_B = 2,      // MN-major B operand (attention PV)
  GF_STAGED = 4,    // staged epilogue + TMA tensor store (c_tma = 1)
  GF_SCALAR = 8,    // scalar epilogue for unaligned rows (c_tma = 0)
  GF_SLOWACT = 16,  // GELU / tanh epilogue
  GF_GATHER = 32,   // A_GATHER implicit im2col by cp.async
  GF_IM2COL = 64,   // A_IM2COL implicit im2col by TMA
  GF_ALL = 127
};
#ifndef PASK_GEMM_FEAT
#define PASK_GEMM_FEAT 127
#endif
constexpr unsigned kGemmFeat = PASK_GEMM_FEAT;
__device__ __forceinline__ constexpr bool gfeat(unsigned f) { return (kGemmFeat & f) != 0; }

__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Activation over 16 values: ReLU / ReLU6 inline; GELU / tanh (transformer
// GEMMs) through one out-of-line routine to keep the code object small.
__device__ __noinline__ float act_slow(float v, int act) { return apply_act(v, act); }
__device__ __forceinline__ void act16(float (&v)[16], int act) {
  if (act == 1) {
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = fmaxf(v[i], 0.f);
  } else if (act == 2) {
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = fminf(fmaxf(v[i], 0.f), 6.f);
  } else if (act >= 3 && gfeat(GF_SLOWACT)) {
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = act_slow(v[i], act);
  }
}

// Layout of the residual / output staging tile: column boxes of 2^lb (16/32/64)
// columns, each 128 rows x 2^lb bf16; 64-wide boxes use the TMA SWIZZLE_128B
// pattern (16 B chunk c of row r at chunk c ^ (r & 7)).  col is a multiple of 8.
__device__ __forceinline__ uint32_t ro_addr(uint32_t ro, int lb, int row, int col) {
  const int j = col >> lb;
  const int cc = (col & ((1 << lb) - 1)) >> 3;
  const uint32_t base = ro + (static_cast<uint32_t>(j * 128 + row) << (lb + 1));
  return lb == 6 ? base + ((cc ^ (row & 7)) << 4) : base + (cc << 4);
}
// box width of the staged epilogue for an N tile of bn columns (power of two)
__device__ __forceinline__ int box_log2(int bn) { return bn >= 64 ? 6 : (bn == 32 ? 5 : 4); }

// The parameters the epilogue reads, loaded by the epilogue warps while the
// mainloop runs, so their first (cold constant-cache) reads are off the critical
// path.  Measured: ResNet-50 hot 0.2872 -> 0.2854 ms.  The epilogue itself is
// bound by TMEM reads (a 128 x 64 fp32 tile is 32 KB at 64 B/cycle per SM; the
// first 16-column chunk lands ~750 cycles after the accumulator is ready even with
// no epilogue math, DESIGN.md §6 K6).
struct EpiArgs {
  void* out;
  const void* res;
  int64_t ldc, off_c, stride_c;
  int32_t M, N, act, c_tma;
};
__device__ __forceinline__ EpiArgs load_epi_args(const GemmParams& p) {
  EpiArgs e;
  e.out = p.out;
  e.res = p.res;
  e.ldc = p.ldc;
  e.off_c = p.off_c;
  e.stride_c = p.stride_c;
  e.M = p.M;
  e.N = p.N;
  e.act = p.act;
  e.c_tma = p.c_tma;
  // consume the values here: the loads (and the constant-cache fills of their
  // lines) happen now, not at the first chunk -- ptxas may still re-read the bank
  // at the use sites, which then hit
  asm volatile("" ::"l"(e.out), "l"(e.res), "l"(e.ldc), "l"(e.off_c), "l"(e.stride_c));
  asm volatile("" ::"r"(e.M), "r"(e.N), "r"(e.act), "r"(e.c_tma));
  return e;
}

// v = act(acc + bias + res) -> bf16 (RNE) for 16 columns [cb, cb+16) of tile row
// `row`: staged in smem for the TMA tensor store (c_tma 1), stored straight from
// registers (c_tma 2) or, for unaligned output rows, stored element by element.
__device__ __forceinline__ void epi16(const EpiArgs& p, uint32_t sbias, uint32_t ro, int lb, int m0,
                                      int n0, int b, int row, int cb, float (&v)[16]) {
#pragma unroll
  for (int q4 = 0; q4 < 4; ++q4) {
    const float4 bb = lds_f4(sbias + (cb + 4 * q4) * 4);  // broadcast
    v[4 * q4] += bb.x;
    v[4 * q4 + 1] += bb.y;
    v[4 * q4 + 2] += bb.z;
    v[4 * q4 + 3] += bb.w;
  }
  if (p.c_tma || !gfeat(GF_SCALAR)) {
    const uint32_t a0 = ro_addr(ro, lb, row, cb);
    const uint32_t a1 = ro_addr(ro, lb, row, cb + 8);
    if (p.res) {  // the residual tile was TMA-loaded into the staging smem
      float f0[8], f1[8];
      unpack_bf16x8(lds_u4(a0), f0);
      unpack_bf16x8(lds_u4(a1), f1);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        v[i] += f0[i];
        v[8 + i] += f1[i];
      }
    }
    act16(v, p.act);
    const uint4 w0 = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                                pack_bf16x2(v[6], v[7]));
    const uint4 w1 = make_uint4(pack_bf16x2(v[8], v[9]), pack_bf16x2(v[10], v[11]), pack_bf16x2(v[12], v[13]),
                                pack_bf16x2(v[14], v[15]));
    if (p.c_tma == 2 || !gfeat(GF_STAGED)) {
      // direct epilogue: the 32 B of one output row in a single 256-bit store from
      // registers (N % 16 == 0, 32-byte aligned rows; one-tile kernel only)
      if (n0 + cb < p.N)
        stg_u8(reinterpret_cast<__nv_bfloat16*>(p.out) + p.off_c + static_cast<int64_t>(b) * p.stride_c +
                   static_cast<int64_t>(m0 + row) * p.ldc + n0 + cb,
               w0, w1);
      return;
    }
    sts_u4(a0, w0.x, w0.y, w0.z, w0.w);
    sts_u4(a1, w1.x, w1.y, w1.z, w1.w);
    return;
  }
  // unaligned output rows (e.g. N = 10): scalar stores, residual from global
  const int m = m0 + row, n = n0 + cb;
  if (m >= p.M || n >= p.N) return;
  const int nv = min(16, p.N - n);
  const int64_t base = p.off_c + static_cast<int64_t>(b) * p.stride_c + static_cast<int64_t>(m) * p.ldc + n;
  if (p.res) {
    const __nv_bfloat16* res = reinterpret_cast<const __nv_bfloat16*>(p.res);
#pragma unroll
    for (int i = 0; i < 16; ++i)
      if (i < nv) v[i] += __bfloat162float(res[base + i]);
  }
  act16(v, p.act);
  __nv_bfloat16* o = reinterpret_cast<__nv_bfloat16*>(p.out) + base;
#pragma unroll
  for (int i = 0; i < 16; ++i)
    if (i < nv) o[i] = __float2bfloat16_rn(v[i]);
}

// Geometry policy of the contraction body.  DynGeo reads filter size, stride,
// padding, dilation, input channels and the A-operand path from the parameter
// block (the generic, reusable kernels); FixGeo bakes them in at compile time
// (the per-problem specialised solutions of the paper's Baseline, PAPER.md:83
// Fig. 4: smaller, branch-free code that is applicable to one problem shape).
struct DynGeo {
  __device__ static int R(const GemmParams& p) { return p.R; }
  __device__ static int S(const GemmParams& p) { return p.S; }
  __device__ static int SH(const GemmParams& p) { return p.sh; }
  __device__ static int SW(const GemmParams& p) { return p.sw; }
  __device__ static int PH(const GemmParams& p) { return p.ph; }
  __device__ static int PW(const GemmParams& p) { return p.pw; }
  __device__ static int DH(const GemmParams& p) { return p.dh; }
  __device__ static int DW(const GemmParams& p) { return p.dw; }
  __device__ static int C(const GemmParams& p) { return p.C; }
  __device__ static int amode(const GemmParams& p) { return p.a_mode; }
};
template <int R_, int S_, int ST_, int PD_, int DL_, int C_>
struct FixGeo {
  __device__ static constexpr int R(const GemmParams&) { return R_; }
  __device__ static constexpr int S(const GemmParams&) { return S_; }
  __device__ static constexpr int SH(const GemmParams&) { return ST_; }
  __device__ static constexpr int SW(const GemmParams&) { return ST_; }
  __device__ static constexpr int PH(const GemmParams&) { return PD_; }
  __device__ static constexpr int PW(const GemmParams&) { return PD_; }
  __device__ static constexpr int DH(const GemmParams&) { return DL_; }
  __device__ static constexpr int DW(const GemmParams&) { return DL_; }
  __device__ static constexpr int C(const GemmParams&) { return C_; }
  __device__ static constexpr int amode(const GemmParams&) {
    return (R_ == 1 && S_ == 1 && ST_ == 1 && PD_ == 0) ? A_TMA : (C_ % 64 == 0 ? A_IM2COL : A_GATHER);
  }
};


template <bool kAllowGather, class Geo = DynGeo>
__device__ __forceinline__ void conv_gemm_body(const GemmParams& p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int t = threadIdx.x;
  const int stages = p.stages;
  const int bn = p.bn;
  // a path compiled out of this families variant (GemmFeat) must never be asked for
  if (kGemmFeat != GF_ALL &&
      ((!gfeat(GF_SPLITK) && p.splits > 1) || (!gfeat(GF_MN_B) && p.b_major != 0) ||
       (!gfeat(GF_STAGED) && p.c_tma == 1) || (!gfeat(GF_SCALAR) && p.c_tma == 0) ||
       (!gfeat(GF_SLOWACT) && p.act >= 3) || (!gfeat(GF_GATHER) && kAllowGather && p.a_mode == A_GATHER) ||
       (!gfeat(GF_IM2COL) && kAllowGather && p.a_mode == A_IM2COL)))
    __trap();
  const int splits = gfeat(GF_SPLITK) ? p.splits : 1;
  const int b_major = gfeat(GF_MN_B) ? p.b_major : 0;
  constexpr uint32_t kABytes = kBM * kBK * 2;  // 16 KB
  const uint32_t b_bytes = static_cast<uint32_t>(bn) * kBK * 2;
  const uint32_t stage_bytes = kABytes + b_bytes;
  const uint32_t a_tx = static_cast<uint32_t>(p.a_rows) * (kBK * 2);  // A bytes a TMA k-block delivers
  // ---- smem carve-up (mirrors gemm_tiling() on the host)
  const uint32_t ring_bytes = (stages * stage_bytes + 1023u) & ~1023u;
  const uint32_t recv_pitch = (bn + 4) * 4;  // fp32 split-K receive row pitch (bank spread)
  const uint32_t recv_bytes = splits > 1 ? ((128u * recv_pitch + 1023u) & ~1023u) : 0u;
  const uint32_t reg0 = ring_bytes + recv_bytes;
  const uint32_t ro_bytes = p.c_tma ? ((128u * bn * 2 + 1023u) & ~1023u) : 0u;
  float* s_bias = reinterpret_cast<float*>(smem + reg0 + ro_bytes);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + reg0 + ro_bytes + 1024);
  const uint32_t smem_base = smem_u32(smem);
  const uint32_t full0 = smem_u32(bars);
  const uint32_t empty0 = smem_u32(bars + stages);
  const uint32_t accum_bar = smem_u32(bars + 2 * stages);
  const uint32_t res_bar = smem_u32(bars + 2 * stages + 1);
  const uint32_t recv_bar = smem_u32(bars + 2 * stages + 2);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * stages + 3);
  const uint32_t ro = smem_base + reg0;
  const uint32_t recv = smem_base + ring_bytes;  // slot s: rows [s*rows_per, (s+1)*rows_per)

  const int a_mode = Geo::amode(p);
  const bool gather = kAllowGather && gfeat(GF_GATHER) && (a_mode == A_GATHER);
  const bool im2col = kAllowGather && gfeat(GF_IM2COL) && (a_mode == A_IM2COL);
  const int gR = Geo::R(p), gS = Geo::S(p), gSH = Geo::SH(p), gSW = Geo::SW(p);
  const int gPH = Geo::PH(p), gPW = Geo::PW(p), gDH = Geo::DH(p), gDW = Geo::DW(p), gC = Geo::C(p);
  (void)gR;
  const int mt = blockIdx.x, nt = blockIdx.y;
  const int b = blockIdx.z / splits;
  const int split = blockIdx.z - b * splits;
  // 32-bit: num_kb * splits < 2^31 (num_kb <= 2^25 for an int32 K, splits <= 16)
  const int kb_begin = (split * p.num_kb) / splits;
  const int kb_end = ((split + 1) * p.num_kb) / splits;
  const int nk = kb_end - kb_begin;  // >= 1 (host guarantees num_kb >= splits)
  const int m0 = mt * kBM, n0 = nt * bn;
  const int lb = box_log2(bn);
  const int box_cols = 1 << lb;
  const int rows_per = p.rows_per;
  const int r0 = splits > 1 ? static_cast<int>(cluster_ctarank()) * rows_per : 0;
  // rows of this tile inside the output, and of this rank's slice (split-K)
  const int valid_rows = min(kBM, p.M - m0);
  const int slice_rows = max(0, min(rows_per, valid_rows - r0));
  const bool res_tma = p.c_tma && p.res != nullptr;
  // the debug phase trace is compiled into the full-feature objects only (the
  // per-model families variants drop it: 1.5 KB less code to upload)
  unsigned long long* trace =
      (kGemmFeat == GF_ALL && p.trace)
          ? p.trace + 8ull * (blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z))
          : nullptr;
  // debug phase stamps: [0] start [1] prologue done [2] producer past griddepcontrol.wait
  // [3] first k-block landed [4] first accumulator chunk in registers (or split-K
  // partials pushed) [5] accumulator ready [6] epilogue math done [7] tile stored
  auto stamp = [&]() -> unsigned long long {
    if (p.trace_clock) {
      unsigned long long c;
      asm volatile("mov.u64 %0, %%clock64;" : "=l"(c));
      return c;
    }
    return globaltimer();
  };
  if (trace && t == 0) trace[0] = stamp();

  // ---------------- prologue (overlaps the previous kernel under PDL)
  if (t == 0) {
    for (int s = 0; s < stages; ++s) {
      mbar_init(full0 + 8 * s, gather ? kEpiThreads + 1u : 1u);
      mbar_init(empty0 + 8 * s, 1u);
    }
    mbar_init(accum_bar, 1u);
    mbar_init(res_bar, 1u);
    mbar_init(recv_bar, 1u);
    if (splits > 1)  // the S-1 peers push the valid rows of this rank's slice, bn fp32 each
      mbar_arrive_expect_tx(recv_bar, static_cast<uint32_t>((splits - 1) * slice_rows * bn * 4));
    fence_barrier_init();
  }
  if (warp == kEpiWarps && lane == 0) {
    if (!gather) tma_prefetch_desc(&p.tmap_a);
    tma_prefetch_desc(&p.tmap_b);
    if (p.c_tma) tma_prefetch_desc(&p.tmap_c);
    if (res_tma) tma_prefetch_desc(&p.tmap_r);
  }
  if (warp == kEpiWarps + 1) tmem_alloc(smem_u32(tmem_slot), p.tmem_cols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (splits > 1) cluster_sync_all();  // peers' receive barriers are initialised
  const uint32_t tmem_base = *tmem_slot;
  if (trace && t == 0) trace[1] = stamp();

  pdl_launch_dependents();  // let the next layer's prologue start
  // griddepcontrol.wait is per role: weights (B, bias) do not depend on the
  // previous layer, so they are fetched before it; activations after it.
  EpiArgs ea;  // epilogue warps: their parameters, in registers before the accumulator wait

  if (warp == kEpiWarps) {
    // ================= TMA producer
    if (lane == 0) {
      // im2col: the tile's first output pixel and the (tap, channel chunk) of kb_begin
      int iw = 0, ih = 0, in = 0, cc = 0, tr = 0, ts = 0;
      const int cpt = gC >> 6;  // 64-channel chunks per filter tap
      if (kAllowGather && im2col) {
        const int pq = p.P * p.Q;
        in = m0 / pq;
        const int rem = m0 - in * pq;
        const int pp = rem / p.Q;
        const int qq = rem - pp * p.Q;
        iw = qq * gSW - gPW;
        ih = pp * gSH - gPH;
        const int tap = kb_begin / cpt;
        cc = kb_begin - tap * cpt;
        tr = tap / gS;
        ts = tap - tr * gS;
      }
      // weights of the first min(nk, stages) k-blocks before griddepcontrol.wait
      // (they overlap the previous layer's tail); ring slots start empty.  An
      // activation B operand (attention QK^T / PV) must wait like A.
      const int pre = p.b_const ? min(min(nk, stages), p.pre_b > 0 ? p.pre_b : stages) : 0;
      for (int i = 0; i < pre; ++i) {
        const uint32_t sb = smem_base + i * stage_bytes + kABytes;
        const int kb = kb_begin + i;
        mbar_arrive_expect_tx(full0 + 8 * i, b_bytes + (gather ? 0u : a_tx));
        if (b_major == 0) {
          tma_load_3d(sb, &p.tmap_b, full0 + 8 * i, kb * kBK, n0, b);
        } else {
#pragma unroll 1
          for (int j = 0; j < bn / 64; ++j)
            tma_load_3d(sb + j * 8192, &p.tmap_b, full0 + 8 * i, n0 + j * 64, kb * kBK, b);
        }
      }
      pdl_wait();  // activations / residual of this layer are complete and visible
      if (trace) trace[2] = stamp();
      if (res_tma && slice_rows > 0) {  // residual rows [r0, r0 + rows_per), read by the epilogue
        mbar_arrive_expect_tx(res_bar, static_cast<uint32_t>(rows_per * bn * 2));
#pragma unroll 1
        for (int j = 0; j < bn / box_cols; ++j)
          tma_load_3d(ro + j * (128 * box_cols * 2) + r0 * (box_cols * 2), &p.tmap_r, res_bar,
                      n0 + j * box_cols, m0 + r0, b);
      }
      int s = 0;
      uint32_t ph = 0;
      for (int i = 0; i < nk; ++i) {
        const bool b_done = i < pre;
        if (!b_done) mbar_wait(empty0 + 8 * s, ph ^ 1);
        const uint32_t sa = smem_base + s * stage_bytes;
        const uint32_t sb = sa + kABytes;
        const int kb = kb_begin + i;
        if (!b_done) mbar_arrive_expect_tx(full0 + 8 * s, b_bytes + (gather ? 0u : a_tx));
        if (kAllowGather && im2col) {
          tma_load_im2col_4d(sa, &p.tmap_a, full0 + 8 * s, cc * 64, iw, ih, in,
                             static_cast<uint16_t>(ts * gDW), static_cast<uint16_t>(tr * gDH));
          if (++cc == cpt) {
            cc = 0;
            if (++ts == gS) {
              ts = 0;
              ++tr;
            }
          }
        } else if (!gather) {
          tma_load_3d(sa, &p.tmap_a, full0 + 8 * s, kb * kBK, m0, b);
        }
        if (!b_done) {
          if (b_major == 0) {
            tma_load_3d(sb, &p.tmap_b, full0 + 8 * s, kb * kBK, n0, b);
          } else {
#pragma unroll 1
            for (int j = 0; j < bn / 64; ++j)
              tma_load_3d(sb + j * 8192, &p.tmap_b, full0 + 8 * s, n0 + j * 64, kb * kBK, b);
          }
        }
        if (++s == stages) {
          s = 0;
          ph ^= 1;
        }
      }
    }
    __syncwarp();
  } else if (warp == kEpiWarps + 1) {
    // ================= MMA issuer (one thread issues for the whole CTA)
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      for (int i = 0; i < nk; ++i) {
        mbar_wait(full0 + 8 * s, ph);
        tc_fence_after();
        if (trace && i == 0) trace[3] = stamp();
        const uint32_t sa = smem_base + s * stage_bytes;
        const uint32_t sb = sa + kABytes;
#pragma unroll
        for (int k = 0; k < kBK / 16; ++k) {
          // K-major SWIZZLE_128B: +32 B per 16-element K step inside the 128 B row
          const uint64_t adesc = umma_desc_sw128(sa + k * 32, 16, 1024);
          const uint64_t bdesc = (b_major == 0)
                                     ? umma_desc_sw128(sb + k * 32, 16, 1024)
                                     // MN-major: +16 K rows of 128 B; 64-wide N chunks 8 KB apart
                                     : umma_desc_sw128(sb + k * 2048, 8192, 1024);
          umma_f16(tmem_base, adesc, bdesc, p.idesc, (i | k) != 0 ? 1u : 0u);
        }
        umma_commit(empty0 + 8 * s);  // frees the smem slot when these MMAs complete
        if (++s == stages) {
          s = 0;
          ph ^= 1;
        }
      }
      umma_commit(accum_bar);  // accumulator complete -> epilogue
    }
    __syncwarp();
  } else {
    // ================= warps 0-7: bias, (gather), epilogue
    if (t < bn) s_bias[t] = (p.bias != nullptr && n0 + t < p.N) ? __ldg(p.bias + n0 + t) : 0.f;
    ea = load_epi_args(p);
    pdl_wait();  // before reading this layer's activations (gather) or writing outputs
    if (kAllowGather && gather) {
      // implicit im2col: thread t owns 16 B chunk j = t % 8 of rows rg + kGR * ri
      constexpr int kGR = kEpiThreads / 8;  // rows per pass
      constexpr int kGI = kBM / kGR;        // passes per 128-row tile
      const int j = t & 7;
      const int rg = t >> 3;
      const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(p.x);
      int ih0[kGI], iw0[kGI], nb[kGI];
      bool rv[kGI];
      {
        // output pixel of row rg, then step kGR pixels per ri (no per-row divisions)
        const int m = m0 + rg;
        const int pq = p.P * p.Q;
        int n = m / pq;
        const int rem = m - n * pq;
        int pp = rem / p.Q;
        int qq = rem - pp * p.Q;
#pragma unroll
        for (int ri = 0; ri < kGI; ++ri) {
          rv[ri] = (m + kGR * ri) < p.M;
          ih0[ri] = pp * gSH - gPH;
          iw0[ri] = qq * gSW - gPW;
          nb[ri] = n * p.H;
          qq += kGR;
          while (qq >= p.Q) {
            qq -= p.Q;
            if (++pp == p.P) {
              pp = 0;
              ++n;
            }
          }
        }
      }
      int kk = kb_begin * kBK + 8 * j;
      int tap = kk / gC;
      int c = kk - tap * gC;
      int r = tap / gS;
      int s = tap - r * gS;
      const int lag = min(p.gather_lag, stages - 1);  // k-blocks of cp.async in flight before publishing
      int st = 0, st_lag = 0;  // ring slot being filled / being published
      uint32_t ph = 0;
      for (int i = 0; i < nk; ++i) {
        mbar_wait(empty0 + 8 * st, ph ^ 1);
        const uint32_t sa = smem_base + st * stage_bytes;
        const bool kval = kk < p.K;
        const int dih = r * gDH, diw = s * gDW;
#pragma unroll
        for (int ri = 0; ri < kGI; ++ri) {
          const int row = rg + kGR * ri;
          const uint32_t dst = sa + row * 128 + ((j ^ (row & 7)) << 4);
          const int ih = ih0[ri] + dih;
          const int iw = iw0[ri] + diw;
          const bool ok = kval && rv[ri] && ih >= 0 && ih < p.H && iw >= 0 && iw < p.W;
          const __nv_bfloat16* src =
              ok ? x + ((static_cast<int64_t>(nb[ri] + ih) * p.W + iw) * gC + c) : x;
          cp_async_16(dst, src, ok ? 16u : 0u);
        }
        cp_async_commit();
        if (i >= lag) {
          cp_async_wait_dyn(lag);
          fence_proxy_async_smem();  // generic-proxy smem writes -> tcgen05 (async proxy)
          mbar_arrive(full0 + 8 * st_lag);
          if (++st_lag == stages) st_lag = 0;
        }
        if (++st == stages) {
          st = 0;
          ph ^= 1;
        }
        kk += kBK;
        c += kBK;
        while (c >= gC) {
          c -= gC;
          if (++s == gS) {
            s = 0;
            ++r;
          }
        }
      }
      cp_async_wait<0>();
      fence_proxy_async_smem();
      for (int i = max(0, nk - lag); i < nk; ++i) {
        mbar_arrive(full0 + 8 * st_lag);
        if (++st_lag == stages) st_lag = 0;
      }
    }
    named_bar_sync(1, kEpiThreads);  // s_bias complete
    mbar_wait(accum_bar, 0);
    tc_fence_after();
    if (trace && t == 0) trace[5] = stamp();
  }

  // ---------------- epilogue: warp w (0-7) reads TMEM lanes / tile rows
  // 32*(w%4) .. +31 (the tcgen05.ld lane quarter of its warp) and the 16-column
  // chunks c with c % 2 == w / 4.  Rows at or beyond M are never read or stored.
  if (warp < kEpiWarps) {
    const int quarter = warp & 3;
    const int half = warp >> 2;  // warp group 0..kEpiGroups-1: chunks half, half + kEpiGroups, ...
    const int row = quarter * 32 + lane;
    const uint32_t taddr = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16);
    const int cpr = bn >> 4;  // 16-column chunks per row
    const uint32_t sbias = smem_u32(s_bias);
    const bool warp_live = quarter * 32 < valid_rows;  // warp-uniform: tcgen05.ld is .sync.aligned
    uint32_t r[16];
    if (splits > 1) {
      // push this split's fp32 partial rows to their owners' receive slot [my rank]
      const uint32_t owner = static_cast<uint32_t>(row / rows_per);
      const uint32_t me = cluster_ctarank();
      const uint32_t slot_row = me * rows_per + (row - owner * rows_per);
      const uint32_t local = recv + slot_row * recv_pitch;
      const uint32_t remote = mapa_cluster(local, owner);
      const uint32_t rbar = mapa_cluster(recv_bar, owner);
      const bool live = row < valid_rows;
      if (warp_live) {
        int c = half;
        if (c < cpr) {
          tmem_ld16_issue(taddr + c * 16, r);
          tmem_ld_wait(r);
        }
        // not unrolled: 4 copies of the 4 DSMEM stores were 5 KB of SASS to upload
#pragma unroll 1
        for (; c < cpr; c += kEpiGroups) {
          uint32_t u[16];
#pragma unroll
          for (int i = 0; i < 16; ++i) u[i] = r[i];
          const bool more = c + kEpiGroups < cpr;
          if (more) tmem_ld16_issue(taddr + (c + kEpiGroups) * 16, r);
          if (live) {
#pragma unroll
            for (int q4 = 0; q4 < 4; ++q4) {
              const uint32_t off = (c * 16 + 4 * q4) * 4;
              const float x0 = __uint_as_float(u[4 * q4]), x1 = __uint_as_float(u[4 * q4 + 1]);
              const float x2 = __uint_as_float(u[4 * q4 + 2]), x3 = __uint_as_float(u[4 * q4 + 3]);
              if (owner == me)
                sts_f4(local + off, x0, x1, x2, x3);
              else
                st_async_f4(remote + off, x0, x1, x2, x3, rbar);
            }
          }
          if (more) tmem_ld_wait(r);
        }
      }
      if (trace && t == 0) trace[4] = stamp();
      named_bar_sync(1, kEpiThreads);  // own-slot rows visible to all epilogue threads
      mbar_wait(recv_bar, 0);          // every peer's rows have landed
      if (res_tma && slice_rows > 0) mbar_wait(res_bar, 0);
    } else {
      if (res_tma) mbar_wait(res_bar, 0);
      if (warp_live && half < cpr) {
        tmem_ld16_issue(taddr + half * 16, r);
        tmem_ld_wait(r);
        if (trace && t == 0) trace[4] = stamp();
      }
    }
    // one epilogue loop (a single epi16 site keeps the code object small):
    //   splits == 1: this warp's chunks c = half, half + G, ... (G = kEpiGroups), TMEM
    //                reads software-pipelined (chunk c + G in flight while c is processed);
    //   splits  > 1: items (row, chunk) of this rank's slice, the S receive slots
    //                summed in fixed rank order 0..S-1 (deterministic)
    const int n_iter = splits == 1 ? (warp_live && half < cpr ? (cpr - half + kEpiGroups - 1) / kEpiGroups : 0)
                                   : max(0, (slice_rows * cpr - t + kEpiThreads - 1) / kEpiThreads);
    for (int k = 0; k < n_iter; ++k) {
      float v[16];
      int erow, cb;
      bool more = false;
      if (splits == 1) {
        const int c = half + kEpiGroups * k;
        erow = row;
        cb = c * 16;
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
        more = c + kEpiGroups < cpr;
        if (more) tmem_ld16_issue(taddr + (c + kEpiGroups) * 16, r);
      } else {
        const int it = t + k * kEpiThreads;
        const int lr = it / cpr;
        erow = r0 + lr;
        cb = (it - lr * cpr) << 4;
        const uint32_t src = recv + lr * recv_pitch + cb * 4;
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = 0.f;
        // two slots per trip: their 8 loads in flight together, half the code of
        // the compiler's 4-way unroll
#pragma unroll 2
        for (int sp = 0; sp < splits; ++sp) {
          const uint32_t a = src + sp * rows_per * recv_pitch;
#pragma unroll
          for (int q4 = 0; q4 < 4; ++q4) {
            const float4 f = lds_f4(a + 16 * q4);
            v[4 * q4] += f.x;
            v[4 * q4 + 1] += f.y;
            v[4 * q4 + 2] += f.z;
            v[4 * q4 + 3] += f.w;
          }
        }
      }
      if (erow < valid_rows) epi16(ea, sbias, ro, lb, m0, n0, b, erow, cb, v);
      if (more) tmem_ld_wait(r);
    }
    if (trace && t == 0) trace[6] = stamp();
    if (gfeat(GF_STAGED) && p.c_tma == 1) {
      fence_proxy_async_smem();  // staged bf16 tile -> TMA store (async proxy)
      named_bar_sync(1, kEpiThreads);
      if (t == 0 && slice_rows > 0) {
#pragma unroll 1
        for (int j = 0; j < bn / box_cols; ++j)
          tma_store_3d(&p.tmap_c, ro + j * (128 * box_cols * 2) + r0 * (box_cols * 2), n0 + j * box_cols,
                       m0 + r0, b);
        tma_store_commit_and_wait_read();
      }
    }
    if (trace && t == 0) trace[7] = stamp();
  }

  // ---------------- teardown
  tc_fence_before();
  __syncthreads();
  if (warp == kEpiWarps + 1) {
    tc_fence_after();
    tmem_dealloc(tmem_base, p.tmem_cols);
  }
}


// Persistent-tile variant (pask_conv_igemm_pt, DESIGN.md §6 K6-PT): when the grid
// exceeds one wave, min(tiles, #SMs) CTAs loop over the tiles with double-buffered
// TMEM accumulator / staging / bias and a store agent warp; otherwise one tile per
// CTA.  Kept separate from conv_gemm_body so the one-tile solutions keep their
// smaller, faster code (folding the loop into them cost 2-3% at batch 1).
template <bool kAllowGather>
__device__ __forceinline__ void conv_gemm_body_pt(const GemmParams& p) {
  using Geo = DynGeo;
  constexpr bool kPersistent = true;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int t = threadIdx.x;
  const int stages = p.stages;
  const int bn = p.bn;
  const int splits = p.splits;
  // kPersistent (pask_conv_igemm_pt): tiles looped by <= #SMs CTAs when the grid
  // exceeds one wave; otherwise (and in every other solution) one tile per CTA
  const bool persistent = kPersistent && p.persistent != 0;
  constexpr uint32_t kABytes = kBM * kBK * 2;  // 16 KB
  const uint32_t b_bytes = static_cast<uint32_t>(bn) * kBK * 2;
  // b_res (D18): a layer with one N tile keeps its whole B (every
  // k-block of the weights) resident after the ring, loaded once per CTA; the
  // ring then carries A only
  const bool b_res = persistent && p.b_res != 0;
  const uint32_t stage_bytes = kABytes + (b_res ? 0u : b_bytes);
  // ---- smem carve-up (mirrors gemm_tiling() on the host): ring | resident B |
  // split-K receive slots | staging tile(s) (2 when persistent) | bias vector(s) | barriers
  const uint32_t bres_off = stages * stage_bytes;
  const uint32_t ring_bytes = (bres_off + (b_res ? p.num_kb * b_bytes : 0u) + 1023u) & ~1023u;
  const uint32_t recv_pitch = (bn + 4) * 4;  // fp32 split-K receive row pitch (bank spread)
  const uint32_t recv_bytes = splits > 1 ? ((128u * recv_pitch + 1023u) & ~1023u) : 0u;
  const uint32_t reg0 = ring_bytes + recv_bytes;
  const uint32_t ro_bytes = p.c_tma ? ((128u * bn * 2 + 1023u) & ~1023u) : 0u;
  const int nbuf = persistent ? 2 : 1;
  float* s_bias = reinterpret_cast<float*>(smem + reg0 + nbuf * ro_bytes);  // nbuf x 256 floats
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + reg0 + nbuf * ro_bytes + nbuf * 1024);
  const uint32_t smem_base = smem_u32(smem);
  const uint32_t full0 = smem_u32(bars);
  const uint32_t empty0 = smem_u32(bars + stages);
  const uint32_t tfull0 = smem_u32(bars + 2 * stages);      // [2] accumulator ready
  const uint32_t tempty0 = smem_u32(bars + 2 * stages + 2);  // [2] accumulator drained
  const uint32_t res0 = smem_u32(bars + 2 * stages + 4);     // [2] residual tile landed
  const uint32_t staged0 = smem_u32(bars + 2 * stages + 6);  // [2] output tile staged (256 arrivals)
  const uint32_t rofree0 = smem_u32(bars + 2 * stages + 8);  // [2] staging buffer read by its store
  const uint32_t recv_bar = smem_u32(bars + 2 * stages + 10);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * stages + 11);
  const uint32_t bres_bar = smem_u32(bars + 2 * stages + 12);  // b_res: the resident B landed
  const uint32_t ro0 = smem_base + reg0;
  const uint32_t recv = smem_base + ring_bytes;  // slot s: rows [s*rows_per, (s+1)*rows_per)

  const int a_mode = Geo::amode(p);
  const bool gather = kAllowGather && (a_mode == A_GATHER);
  const bool im2col = kAllowGather && (a_mode == A_IM2COL);
  const int gR = Geo::R(p), gS = Geo::S(p), gSH = Geo::SH(p), gSW = Geo::SW(p);
  const int gPH = Geo::PH(p), gPW = Geo::PW(p), gDH = Geo::DH(p), gDW = Geo::DW(p), gC = Geo::C(p);
  (void)gR;
  // tiles: one per CTA (grid = m_tiles x n_tiles x batch*splits), or, persistent
  // (splits == 1, more tiles than SMs), tiles blockIdx.x, +gridDim.x, ... of the
  // n-fastest linear order: the CTAs working at the same time cover all N tiles
  // of a few M tiles, so each A tile (the activation: up to 400 MB at batch 128)
  // is read from HBM once and hit in L2 by its other N tiles, while the weights
  // (<= 4.7 MB per ResNet-50 layer) stay L2-resident either way.  (The m-fastest
  // order re-read A from HBM once per N tile.)
  const int n_tiles_total = persistent ? p.n_tiles_total : 1;
  const int tile0 = persistent ? static_cast<int>(blockIdx.x) : 0;
  const int tstep = persistent ? static_cast<int>(gridDim.x) : 1;
  auto decode = [&](int tile, int& mt, int& nt, int& bb) {
    if (persistent) {
      nt = tile % p.n_tiles;
      const int rest = tile / p.n_tiles;
      mt = rest % p.m_tiles;
      bb = rest / p.m_tiles;
    } else {
      mt = blockIdx.x;
      nt = blockIdx.y;
      bb = blockIdx.z / splits;
    }
  };
  const int split = static_cast<int>(blockIdx.z) % splits;
  const int kb_begin = static_cast<int>((static_cast<int64_t>(split) * p.num_kb) / splits);
  const int kb_end = static_cast<int>((static_cast<int64_t>(split + 1) * p.num_kb) / splits);
  const int nk = kb_end - kb_begin;  // >= 1 (host guarantees num_kb >= splits)
  const int lb = box_log2(bn);
  const int box_cols = 1 << lb;
  const int rows_per = p.rows_per;
  const int r0 = splits > 1 ? static_cast<int>(cluster_ctarank()) * rows_per : 0;
  const uint32_t acc_cols = p.tmem_cols / nbuf;
  const bool res_tma = p.c_tma && p.res != nullptr;
  unsigned long long* trace =
      p.trace ? p.trace + 8ull * (blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z)) : nullptr;
  // debug phase stamps (first tile): [0] start [1] prologue done [2] producer past
  // griddepcontrol.wait [3] first k-block landed [4] first accumulator chunk in
  // registers (or split-K partials pushed) [5] accumulator ready [6] epilogue math
  // done [7] tile stored
  auto stamp = [&]() -> unsigned long long {
    if (p.trace_clock) {
      unsigned long long c;
      asm volatile("mov.u64 %0, %%clock64;" : "=l"(c));
      return c;
    }
    return globaltimer();
  };
  if (trace && t == 0) trace[0] = stamp();
  int mt0, nt0, b0;
  decode(tile0, mt0, nt0, b0);
  // the residual tile of a given tile into staging buffer buf (rows [r0, r0 + rows_per))
  auto load_residual = [&](int buf, int mt, int nt, int bb) {
    const int vr = max(0, min(rows_per, min(kBM, p.M - mt * kBM) - r0));
    if (!res_tma || vr == 0) return;
    const uint32_t rb = res0 + 8 * buf;
    mbar_arrive_expect_tx(rb, static_cast<uint32_t>(rows_per * bn * 2));
    const uint32_t ro = ro0 + buf * ro_bytes;
#pragma unroll 1
    for (int j = 0; j < bn / box_cols; ++j)
      tma_load_3d(ro + j * (128 * box_cols * 2) + r0 * (box_cols * 2), &p.tmap_r, rb, nt * bn + j * box_cols,
                  mt * kBM + r0, bb);
  };

  // ---------------- prologue (overlaps the previous kernel under PDL)
  if (t == 0) {
    for (int s = 0; s < stages; ++s) {
      mbar_init(full0 + 8 * s, gather ? kEpiThreadsPT + 1u : 1u);
      mbar_init(empty0 + 8 * s, 1u);
    }
    for (int j = 0; j < 2; ++j) {
      mbar_init(tfull0 + 8 * j, 1u);
      mbar_init(tempty0 + 8 * j, static_cast<uint32_t>(kEpiThreadsPT));
      mbar_init(res0 + 8 * j, 1u);
      mbar_init(staged0 + 8 * j, static_cast<uint32_t>(kEpiThreadsPT));
      mbar_init(rofree0 + 8 * j, 1u);
    }
    mbar_init(recv_bar, 1u);
    mbar_init(bres_bar, 1u);
    if (splits > 1) {  // the S-1 peers push the valid rows of this rank's slice, bn fp32 each
      const int sr = max(0, min(rows_per, min(kBM, p.M - mt0 * kBM) - r0));
      mbar_arrive_expect_tx(recv_bar, static_cast<uint32_t>((splits - 1) * sr * bn * 4));
    }
    fence_barrier_init();
  }
  if (warp == kEpiWarpsPT && lane == 0) {
    if (!gather) tma_prefetch_desc(&p.tmap_a);
    tma_prefetch_desc(&p.tmap_b);
    if (p.c_tma) tma_prefetch_desc(&p.tmap_c);
    if (res_tma) tma_prefetch_desc(&p.tmap_r);
  }
  if (warp == kEpiWarpsPT + 1) tmem_alloc(smem_u32(tmem_slot), p.tmem_cols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (splits > 1) cluster_sync_all();  // peers' receive barriers are initialised
  const uint32_t tmem_base = *tmem_slot;
  if (trace && t == 0) trace[1] = stamp();

  pdl_launch_dependents();  // let the next layer's prologue start
  // griddepcontrol.wait is per role: weights (B, bias) do not depend on the
  // previous layer, so they are fetched before it; activations after it.

  if (warp == kEpiWarpsPT) {
    // ================= TMA producer
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      const int cpt = gC >> 6;  // 64-channel chunks per filter tap
      for (int tile = tile0, it = 0; tile < n_tiles_total; tile += tstep, ++it) {
        int mt, nt, bb;
        decode(tile, mt, nt, bb);
        const int m0 = mt * kBM, n0 = nt * bn;
        // im2col: the tile's first output pixel and the (tap, channel chunk) of kb_begin
        int iw = 0, ih = 0, in = 0, cc = 0, tr = 0, ts = 0;
        if (kAllowGather && im2col) {
          const int pq = p.P * p.Q;
          in = m0 / pq;
          const int rem = m0 - in * pq;
          const int pp = rem / p.Q;
          const int qq = rem - pp * p.Q;
          iw = qq * gSW - gPW;
          ih = pp * gSH - gPH;
          if (im2col) {
            const int tap = kb_begin / cpt;
            cc = kb_begin - tap * cpt;
            tr = tap / gS;
            ts = tap - tr * gS;
          }
        }
        int pre = 0;
        if (it == 0 && b_res) {
          // the resident B: every k-block once (weights before griddepcontrol.wait;
          // an activation B, or the stem fold's first-inference weights, after it)
          auto load_bres = [&]() {
            mbar_arrive_expect_tx(bres_bar, static_cast<uint32_t>(nk) * b_bytes);
#pragma unroll 1
            for (int i = 0; i < nk; ++i)
              tma_load_3d(smem_base + bres_off + i * b_bytes, &p.tmap_b, bres_bar, (kb_begin + i) * kBK, n0, bb);
          };
          if (p.b_const) load_bres();
          pdl_wait();
          if (!p.b_const) load_bres();
          if (trace) trace[2] = stamp();
        } else if (it == 0) {
          // weights of the first min(nk, stages) k-blocks before griddepcontrol.wait
          // (they overlap the previous layer's tail); ring slots start empty.  An
          // activation B operand (attention QK^T / PV) must wait like A.
          pre = p.b_const ? min(min(nk, stages), p.pre_b > 0 ? p.pre_b : stages) : 0;
          for (int i = 0; i < pre; ++i) {
            const uint32_t sb = smem_base + i * stage_bytes + kABytes;
            const int kb = kb_begin + i;
            mbar_arrive_expect_tx(full0 + 8 * i, b_bytes + (gather ? 0u : kABytes));
            if (p.b_major == 0) {
              tma_load_3d(sb, &p.tmap_b, full0 + 8 * i, kb * kBK, n0, bb);
            } else {
#pragma unroll 1
              for (int j = 0; j < bn / 64; ++j)
                tma_load_3d(sb + j * 8192, &p.tmap_b, full0 + 8 * i, n0 + j * 64, kb * kBK, bb);
            }
          }
          pdl_wait();  // activations of this layer are complete and visible
          if (trace) trace[2] = stamp();
          if (!kPersistent) load_residual(0, mt, nt, bb);  // persistent: the store agent
        }
        for (int i = 0; i < nk; ++i) {
          const bool b_done = i < pre;
          if (!b_done) mbar_wait(empty0 + 8 * s, ph ^ 1);
          const uint32_t sa = smem_base + s * stage_bytes;
          const uint32_t sb = sa + kABytes;
          const int kb = kb_begin + i;
          if (!b_done) mbar_arrive_expect_tx(full0 + 8 * s, (b_res ? 0u : b_bytes) + (gather ? 0u : kABytes));
          if (kAllowGather && im2col) {
            tma_load_im2col_4d(sa, &p.tmap_a, full0 + 8 * s, cc * 64, iw, ih, in,
                               static_cast<uint16_t>(ts * gDW), static_cast<uint16_t>(tr * gDH));
            if (++cc == cpt) {
              cc = 0;
              if (++ts == gS) {
                ts = 0;
                ++tr;
              }
            }
          } else if (!gather) {
            tma_load_3d(sa, &p.tmap_a, full0 + 8 * s, kb * kBK, m0, bb);
          }
          if (!b_done && !b_res) {
            if (p.b_major == 0) {
              tma_load_3d(sb, &p.tmap_b, full0 + 8 * s, kb * kBK, n0, bb);
            } else {
#pragma unroll 1
              for (int j = 0; j < bn / 64; ++j)
                tma_load_3d(sb + j * 8192, &p.tmap_b, full0 + 8 * s, n0 + j * 64, kb * kBK, bb);
            }
          }
          if (++s == stages) {
            s = 0;
            ph ^= 1;
          }
        }
      }
    }
    __syncwarp();
  } else if (kPersistent && warp == kEpiWarpsPT + 2) {
    if (lane == 0 && p.c_tma) {
      // ================= store agent: TMA-stores each staged output tile, frees the
      // staging buffer, and loads the residual tile two tiles ahead into it, so no
      // epilogue thread waits on a bulk copy (its own warp: a spinning lane must
      // not stall the producer's or the MMA issuer's warp)
      pdl_wait();  // residual tiles are the previous layers' outputs
      for (int j = 0; j < 2; ++j) {
        const int tl = tile0 + j * tstep;
        if (tl < n_tiles_total) {
          int mt, nt, bb;
          decode(tl, mt, nt, bb);
          load_residual(j, mt, nt, bb);
        }
      }
      for (int tile = tile0, it = 0; tile < n_tiles_total; tile += tstep, ++it) {
        int mt, nt, bb;
        decode(tile, mt, nt, bb);
        const int buf = it & 1;
        const uint32_t ro = ro0 + buf * ro_bytes;
        const int slice_rows = max(0, min(rows_per, min(kBM, p.M - mt * kBM) - r0));
        mbar_wait(staged0 + 8 * buf, (it >> 1) & 1);
        if (slice_rows > 0) {
#pragma unroll 1
          for (int j = 0; j < bn / box_cols; ++j)
            tma_store_3d(&p.tmap_c, ro + j * (128 * box_cols * 2) + r0 * (box_cols * 2), nt * bn + j * box_cols,
                         mt * kBM + r0, bb);
          tma_store_commit_and_wait_read();
        }
        if (trace && it == 0) trace[7] = stamp();
        mbar_arrive(rofree0 + 8 * buf);
        const int t2 = tile + 2 * tstep;
        if (t2 < n_tiles_total) {
          int mt2, nt2, bb2;
          decode(t2, mt2, nt2, bb2);
          load_residual(buf, mt2, nt2, bb2);
        }
      }
    }
    __syncwarp();
  } else if (warp == kEpiWarpsPT + 1) {
    // ================= MMA issuer (one thread issues for the whole CTA)
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      for (int tile = tile0, it = 0; tile < n_tiles_total; tile += tstep, ++it) {
        const int buf = it & 1;
        const uint32_t acc = tmem_base + buf * acc_cols;
        if (persistent) {  // the epilogue has drained this accumulator buffer (two tiles ago)
          mbar_wait(tempty0 + 8 * buf, ((it >> 1) & 1) ^ 1);
          tc_fence_after();
        }
        if (b_res && it == 0) mbar_wait(bres_bar, 0);
        for (int i = 0; i < nk; ++i) {
          mbar_wait(full0 + 8 * s, ph);
          tc_fence_after();
          if (trace && it == 0 && i == 0) trace[3] = stamp();
          const uint32_t sa = smem_base + s * stage_bytes;
          const uint32_t sb = b_res ? smem_base + bres_off + i * b_bytes : sa + kABytes;
#pragma unroll
          for (int k = 0; k < kBK / 16; ++k) {
            // K-major SWIZZLE_128B: +32 B per 16-element K step inside the 128 B row
            const uint64_t adesc = umma_desc_sw128(sa + k * 32, 16, 1024);
            const uint64_t bdesc = (p.b_major == 0)
                                       ? umma_desc_sw128(sb + k * 32, 16, 1024)
                                       // MN-major: +16 K rows of 128 B; 64-wide N chunks 8 KB apart
                                       : umma_desc_sw128(sb + k * 2048, 8192, 1024);
            umma_f16(acc, adesc, bdesc, p.idesc, (i | k) != 0 ? 1u : 0u);
          }
          umma_commit(empty0 + 8 * s);  // frees the smem slot when these MMAs complete
          if (++s == stages) {
            s = 0;
            ph ^= 1;
          }
        }
        umma_commit(tfull0 + 8 * buf);  // accumulator complete -> epilogue
      }
    }
    __syncwarp();
  } else {
    // ================= warps 0-7: bias, (gather), epilogue, per tile
    if (t < bn) s_bias[t] = (p.bias != nullptr && nt0 * bn + t < p.N) ? __ldg(p.bias + nt0 * bn + t) : 0.f;
    const EpiArgs ea = load_epi_args(p);
    pdl_wait();  // before reading this layer's activations (gather) or writing outputs
    const int quarter = warp & 3;
    const int half = warp >> 2;
    const int erow = quarter * 32 + lane;  // tile row == TMEM lane read by this thread
    const int cpr = bn >> 4;                // 16-column chunks per row
    // gather ring position (persists across tiles)
    const int lag = min(p.gather_lag, stages - 1);
    int gst = 0, gst_lag = 0;
    uint32_t gph = 0;
    for (int tile = tile0, it = 0; tile < n_tiles_total; tile += tstep, ++it) {
      int mt, nt, bb;
      decode(tile, mt, nt, bb);
      const int m0 = mt * kBM, n0 = nt * bn;
      const int buf = it & 1;
      const uint32_t ro = ro0 + buf * ro_bytes;
      const uint32_t sbias = smem_u32(s_bias + buf * 256);
      const int valid_rows = min(kBM, p.M - m0);
      const int slice_rows = max(0, min(rows_per, valid_rows - r0));
      // next tile (persistent): its bias into a register now (stored after this
      // tile, no exposed latency) and its residual into the other staging buffer
      // (free: that buffer's previous store finished reading before this tile)
      const int ntile = tile + tstep;
      float bias_next = 0.f;
      if (persistent && ntile < n_tiles_total) {
        int mtn, ntn, bbn;
        decode(ntile, mtn, ntn, bbn);
        if (t < bn && p.bias != nullptr && ntn * bn + t < p.N) bias_next = __ldg(p.bias + ntn * bn + t);
      }
      if (kAllowGather && gather) {
        // implicit im2col: thread t owns 16 B chunk j = t % 8 of rows rg + kGR * ri
        constexpr int kGR = kEpiThreadsPT / 8;  // rows per pass
        constexpr int kGI = kBM / kGR;        // passes per 128-row tile
        const int j = t & 7;
        const int rg = t >> 3;
        const __nv_bfloat16* x = reinterpret_cast<const __nv_bfloat16*>(p.x);
        int ih0[kGI], iw0[kGI], nb[kGI];
        bool rv[kGI];
        {
          // output pixel of row rg, then step kGR pixels per ri (no per-row divisions)
          const int m = m0 + rg;
          const int pq = p.P * p.Q;
          int n = m / pq;
          const int rem = m - n * pq;
          int pp = rem / p.Q;
          int qq = rem - pp * p.Q;
#pragma unroll
          for (int ri = 0; ri < kGI; ++ri) {
            rv[ri] = (m + kGR * ri) < p.M;
            ih0[ri] = pp * gSH - gPH;
            iw0[ri] = qq * gSW - gPW;
            nb[ri] = n * p.H;
            qq += kGR;
            while (qq >= p.Q) {
              qq -= p.Q;
              if (++pp == p.P) {
                pp = 0;
                ++n;
              }
            }
          }
        }
        int kk = kb_begin * kBK + 8 * j;
        int tap = kk / gC;
        int c = kk - tap * gC;
        int r = tap / gS;
        int s = tap - r * gS;
        for (int i = 0; i < nk; ++i) {
          mbar_wait(empty0 + 8 * gst, gph ^ 1);
          const uint32_t sa = smem_base + gst * stage_bytes;
          const bool kval = kk < p.K;
          const int dih = r * gDH, diw = s * gDW;
#pragma unroll
          for (int ri = 0; ri < kGI; ++ri) {
            const int row = rg + kGR * ri;
            const uint32_t dst = sa + row * 128 + ((j ^ (row & 7)) << 4);
            const int ih = ih0[ri] + dih;
            const int iw = iw0[ri] + diw;
            const bool ok = kval && rv[ri] && ih >= 0 && ih < p.H && iw >= 0 && iw < p.W;
            const __nv_bfloat16* src =
                ok ? x + ((static_cast<int64_t>(nb[ri] + ih) * p.W + iw) * gC + c) : x;
            cp_async_16(dst, src, ok ? 16u : 0u);
          }
          cp_async_commit();
          if (i >= lag) {
            cp_async_wait_dyn(lag);
            fence_proxy_async_smem();  // generic-proxy smem writes -> tcgen05 (async proxy)
            mbar_arrive(full0 + 8 * gst_lag);
            if (++gst_lag == stages) gst_lag = 0;
          }
          if (++gst == stages) {
            gst = 0;
            gph ^= 1;
          }
          kk += kBK;
          c += kBK;
          while (c >= gC) {
            c -= gC;
            if (++s == gS) {
              s = 0;
              ++r;
            }
          }
        }
        cp_async_wait<0>();
        fence_proxy_async_smem();
        for (int i = max(0, nk - lag); i < nk; ++i) {
          mbar_arrive(full0 + 8 * gst_lag);
          if (++gst_lag == stages) gst_lag = 0;
        }
      }
      named_bar_sync(1, kEpiThreadsPT);  // this tile's bias visible
      mbar_wait(tfull0 + 8 * buf, (it >> 1) & 1);
      tc_fence_after();
      if (kPersistent && p.c_tma) mbar_wait(rofree0 + 8 * buf, ((it >> 1) & 1) ^ 1);  // store of tile it-2 read it
      const bool first = it == 0;
      if (trace && first && t == 0) trace[5] = stamp();

      // ---------------- epilogue: warp w (0-7) reads TMEM lanes / tile rows
      // 32*(w%4) .. +31 (the tcgen05.ld lane quarter of its warp) and the 16-column
      // chunks c with c % 2 == w / 4.  Rows at or beyond M are never read or stored.
      const uint32_t taddr = tmem_base + buf * acc_cols + (static_cast<uint32_t>(quarter * 32) << 16);
      const bool warp_live = quarter * 32 < valid_rows;  // warp-uniform: tcgen05.ld is .sync.aligned
      uint32_t r[16];
      if (splits > 1) {
        // push this split's fp32 partial rows to their owners' receive slot [my rank]
        const uint32_t owner = static_cast<uint32_t>(erow / rows_per);
        const uint32_t me = cluster_ctarank();
        const uint32_t slot_row = me * rows_per + (erow - owner * rows_per);
        const uint32_t local = recv + slot_row * recv_pitch;
        const uint32_t remote = mapa_cluster(local, owner);
        const uint32_t rbar = mapa_cluster(recv_bar, owner);
        const bool live = erow < valid_rows;
        if (warp_live) {
          int c = half;
          if (c < cpr) {
            tmem_ld16_issue(taddr + c * 16, r);
            tmem_ld_wait(r);
          }
          for (; c < cpr; c += 2) {
            uint32_t u[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) u[i] = r[i];
            const bool more = c + 2 < cpr;
            if (more) tmem_ld16_issue(taddr + (c + 2) * 16, r);
            if (live) {
#pragma unroll
              for (int q4 = 0; q4 < 4; ++q4) {
                const uint32_t off = (c * 16 + 4 * q4) * 4;
                const float x0 = __uint_as_float(u[4 * q4]), x1 = __uint_as_float(u[4 * q4 + 1]);
                const float x2 = __uint_as_float(u[4 * q4 + 2]), x3 = __uint_as_float(u[4 * q4 + 3]);
                if (owner == me)
                  sts_f4(local + off, x0, x1, x2, x3);
                else
                  st_async_f4(remote + off, x0, x1, x2, x3, rbar);
              }
            }
            if (more) tmem_ld_wait(r);
          }
        }
        if (trace && t == 0) trace[4] = stamp();
        named_bar_sync(1, kEpiThreadsPT);  // own-slot rows visible to all epilogue threads
        mbar_wait(recv_bar, 0);          // every peer's rows have landed
        if (res_tma && slice_rows > 0) mbar_wait(res0 + 8 * buf, (it >> 1) & 1);
      } else {
        if (res_tma) mbar_wait(res0 + 8 * buf, (it >> 1) & 1);
        if (warp_live && half < cpr) {
          tmem_ld16_issue(taddr + half * 16, r);
          tmem_ld_wait(r);
          if (trace && first && t == 0) trace[4] = stamp();
        }
      }
      // one epilogue loop (a single epi16 site keeps the code object small):
      //   splits == 1: this warp's chunks c = half, half + 2, ..., TMEM reads software-
      //                pipelined (chunk c + 2 in flight while c is processed);
      //   splits  > 1: items (row, chunk) of this rank's slice, the S receive slots
      //                summed in fixed rank order 0..S-1 (deterministic)
      const int n_iter = splits == 1 ? (warp_live && half < cpr ? (cpr - half + 1) >> 1 : 0)
                                     : max(0, (slice_rows * cpr - t + kEpiThreadsPT - 1) / kEpiThreadsPT);
      for (int k = 0; k < n_iter; ++k) {
        float v[16];
        int row, cb;
        bool more = false;
        if (splits == 1) {
          const int c = half + 2 * k;
          row = erow;
          cb = c * 16;
#pragma unroll
          for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
          more = c + 2 < cpr;
          if (more) tmem_ld16_issue(taddr + (c + 2) * 16, r);
        } else {
          const int item = t + k * kEpiThreadsPT;
          const int lr = item / cpr;
          row = r0 + lr;
          cb = (item - lr * cpr) << 4;
          const uint32_t src = recv + lr * recv_pitch + cb * 4;
#pragma unroll
          for (int i = 0; i < 16; ++i) v[i] = 0.f;
          for (int sp = 0; sp < splits; ++sp) {
            const uint32_t a = src + sp * rows_per * recv_pitch;
#pragma unroll
            for (int q4 = 0; q4 < 4; ++q4) {
              const float4 f = lds_f4(a + 16 * q4);
              v[4 * q4] += f.x;
              v[4 * q4 + 1] += f.y;
              v[4 * q4 + 2] += f.z;
              v[4 * q4 + 3] += f.w;
            }
          }
        }
        if (row < valid_rows) epi16(ea, sbias, ro, lb, m0, n0, bb, row, cb, v);
        if (more) tmem_ld_wait(r);
      }
      if (kPersistent) {  // this accumulator buffer may be overwritten by the MMA of tile it + 2
        tc_fence_before();
        mbar_arrive(tempty0 + 8 * buf);
      }
      if (trace && first && t == 0) trace[6] = stamp();
      if (p.c_tma) {
        fence_proxy_async_smem();  // staged bf16 tile -> TMA store (async proxy)
        if (kPersistent) {
          mbar_arrive(staged0 + 8 * buf);  // the store agent issues the TMA store
        } else {
          named_bar_sync(1, kEpiThreadsPT);
          if (t == 0 && slice_rows > 0) {
#pragma unroll 1
            for (int j = 0; j < bn / box_cols; ++j)
              tma_store_3d(&p.tmap_c, ro + j * (128 * box_cols * 2) + r0 * (box_cols * 2), n0 + j * box_cols,
                           m0 + r0, bb);
            tma_store_commit_and_wait_read();
          }
          if (trace && t == 0) trace[7] = stamp();
        }
      }
      if (persistent && ntile < n_tiles_total && t < bn) s_bias[(buf ^ 1) * 256 + t] = bias_next;
    }
  }

  // ---------------- teardown
  tc_fence_before();
  __syncthreads();
  if (warp == kEpiWarpsPT + 1) {
    tc_fence_after();
    tmem_dealloc(tmem_base, p.tmem_cols);
  }
}

}  // namespace pask
