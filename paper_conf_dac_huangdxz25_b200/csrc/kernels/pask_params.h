// Launch-parameter blocks shared by the host runtime (C++) and the sm_100a
// kernels.  Each kernel takes exactly one of these by value as a
// __grid_constant__ parameter; the CUtensorMaps inside are encoded on the host
// at pask_load_model time (overlapping the proactive loads).
#pragma once
#include <cuda.h>
#include <stddef.h>
#include <stdint.h>

namespace pask {

constexpr int kBM = 128;       // UMMA M (cta_group::1): one TMEM lane per tile row
constexpr int kBK = 64;        // 64 bf16 = 128 B = one SWIZZLE_128B row
#ifndef PASK_EPI_WARPS
#define PASK_EPI_WARPS 8
#endif
// one-tile contraction kernel: warps 0..kEpiWarps-1 load the bias, gather
// (A_GATHER) and run the epilogue, kEpiGroups warps per TMEM lane quarter
constexpr int kEpiWarps = PASK_EPI_WARPS;
static_assert(kEpiWarps % 4 == 0, "epilogue warps cover the four TMEM lane quarters");
constexpr int kEpiGroups = kEpiWarps / 4;
constexpr int kEpiThreads = 32 * kEpiWarps;
constexpr int kGemmThreads = kEpiThreads + 64;  // + TMA producer warp, TMEM / MMA warp
// persistent-tile kernel: 8 epilogue warps (its 157 registers per thread do not
// fit more), + TMA producer, TMEM / MMA and store / residual agent warps
constexpr int kEpiWarpsPT = 8;
constexpr int kEpiThreadsPT = 32 * kEpiWarpsPT;
constexpr int kGemmThreadsPT = kEpiThreadsPT + 96;

// pask_config.timeline (GPU busy during the cold start, Fig. 6(b)): node i's
// kernel atomically lowers tl[i] to its first CTA's start and raises
// tl[i + kTimelineStride] to its last CTA's end (%globaltimer ns).  The buffer
// (2 x kTimelineStride u64) is owned by the ctx; graphs longer than
// kTimelineStride nodes run without stamps.
constexpr int kTimelineStride = 4096;

// A-operand source of the contraction kernel.
enum AMode : int32_t {
  A_TMA = 0,     // A is a plain K-major matrix: TMA tiled load (GEMM, 1x1 s1 p0 conv)
  A_GATHER = 1,  // implicit im2col: cp.async gather with runtime pad/stride/dilation (any C % 8)
  A_IM2COL = 2,  // implicit im2col by TMA im2col mode (C % 64 == 0): one load per (tap, 64 ch)
};

struct alignas(64) GemmParams {
  CUtensorMap tmap_a;  // A_TMA: 3-D {K, M, batch}, box {64, 128, 1}, SWIZZLE_128B
                       // A_IM2COL: 4-D im2col {C, W, H, N}, 64 ch x 128 px, corners -pad / pad-(R-1)dil
  CUtensorMap tmap_b;  // K-major: {K, N, batch} box {64, BN, 1}; MN-major: {N, K, batch} box {64, 64, 1}
  CUtensorMap tmap_c;  // c_tma: output {N, M, batch} (ldc), box {64, rows_per, 1}, SWIZZLE_128B
  CUtensorMap tmap_r;  // c_tma && res: residual, same geometry as tmap_c with box {64, 128, 1}
  const void* x;       // A_GATHER: NHWC bf16 input
  void* out;           // bf16 output (row i of tile at out + off_c + b*stride_c + i*ldc)
  const void* res;     // bf16 residual, same indexing as out (nullable)
  const float* bias;   // fp32 [N] (nullable)
  int32_t trace_clock;  // debug: 1 = trace stamps are SM clock64 cycles instead of %globaltimer ns
  int32_t pre_b;        // weight k-blocks fetched before griddepcontrol.wait (0 = the whole ring)
  int32_t persistent;   // 1: grid of <= #SMs CTAs loops over the tiles, TMEM double-buffered
  int32_t n_tiles_total;  // m_tiles * n_tiles * batch (persistent)
  unsigned long long* trace;  // debug: per-CTA phase stamps (null in production)
  unsigned long long* tl;     // pask_config.timeline: this node's [start, end] slots (null = off)
  int64_t ldc, off_c, stride_c;
  int32_t M, N, K, batch;
  int32_t num_kb;        // ceil(K / 64)
  int32_t kb_per_split;  // k-blocks per split
  int32_t splits;        // grid.z = batch * splits
  int32_t bn;            // N tile: 16..256, multiple of 16
  int32_t stages;        // smem pipeline depth
  int32_t a_mode;        // AMode
  int32_t b_major;       // 0 K-major, 1 MN-major
  int32_t b_const;       // 1: B is weights (fetched before griddepcontrol.wait); 0: B is an activation
  int32_t act;           // pask_act
  int32_t m_tiles, n_tiles;
  int32_t c_tma;         // 1: output (and residual) through TMA + smem staging
  int32_t rows_per;      // rows reduced / stored per cluster rank = 128 / splits
  int32_t gather_lag;    // A_GATHER: k-blocks of cp.async kept in flight before a slot is published
  int32_t a_rows;        // A rows TMA-loaded per k-block: 128, or 64 when the whole M fits
                         // in 64 rows (one m-tile; rows 64-127 of the operand are never
                         // stored, so their stale smem contents only reach unread TMEM lanes)
  // implicit-GEMM geometry (A_GATHER): input [n][H][W][C], output pixel m -> (n, p, q)
  int32_t H, W, C, P, Q, R, S;
  int32_t sh, sw, ph, pw, dh, dw;
  uint32_t idesc;      // tcgen05 instruction descriptor (kind::f16, bf16 x bf16 -> f32)
  uint32_t tmem_cols;  // power of two >= max(32, bn)
  uint32_t smem_bytes;
  int32_t family;      // pask_all (packaging 3): 0 = this block, 1 = the MemParams overlaid at offset 0
  int32_t b_res;       // persistent, one N tile: B resident in smem after the ring (D18)
};

struct alignas(16) LayoutParams {
  const float* x;  // NCHW fp32
  void* y;         // NHWC bf16, c_out channels (c_out % 8 == 0)
  int32_t n, c, h, w, c_out;
  unsigned long long* tl;  // pask_config.timeline slots (null = off)
  // Stem fold (D16; null yf = off; persistent CTAs over n * fT rows): the consuming conv (R x S, stride
  // fsh x fsw, pad fph / fpw, P x Q output) is re-expressed as an fR2 x 1
  // stride-1 conv over 64 channels, which the contraction kernel loads by TMA
  // im2col.  Also written, from the same input:
  //   yf[n][t][q][j*S*c + s*c + ci] = x[n][ci][fsh*t - fph + j][fsw*q - fpw + s]
  //     (0 outside the image and for channels >= fsh*S*c),  t < fT = P + fR2 - 1
  //   wf[k][r2][j*S*c + s*c + ci]   = wsrc[k][fsh*r2 + j][s][ci]  (KRSC, fcw channels;
  //     0 where fsh*r2 + j >= R or the channel is padding)
  void* yf;              // bf16 [n][fT][fQ][64] (workspace)
  const void* wsrc;      // bf16 [fK][fR][fS][fcw], the conv's weights; null: wf already
                         // written (the first inference writes it, later ones skip it)
  void* wf;              // bf16 [fK][fR2][64] (workspace)
  int32_t fT, fQ, fsh, fsw, fph, fpw, fR, fS, fR2, fK, fcw;
  int32_t fWp;           // smem row pitch of the staged input rows
  int32_t frow_ctas;     // CTAs [0, frow_ctas) walk the folded rows; the rest write wf
  uint16_t foff[64];     // smem element offset of folded channel cc in a staged row
                         // buffer ((j*c + ci) * fWp + s), 0xffff for a padding channel
  uint16_t fwoff[64];    // weights: source offset of folded channel cc within the
                         // (k, fsh*r2) filter rows (j*fS*fcw + s*fcw + ci)
  uint8_t fwj[64];       // ... its j (0xff for a padding channel)
};

struct alignas(16) PoolParams {
  const void* x;  // NHWC bf16 [n][H][W][C]
  void* y;        // NHWC bf16 [n][P][Q][C]
  int32_t n, H, W, C, P, Q, R, S, sh, sw, ph, pw;
  int32_t mode;   // 0 max, 1 avg
  int32_t count_include_pad;
  int32_t per_warp;  // 1: one warp per output chunk, lanes split the window (large windows)
  unsigned long long* tl;  // pask_config.timeline slots (null = off)
};

struct alignas(16) DwParams {
  const void* x;       // NHWC bf16 [n][H][W][C]
  const void* w;       // RSC bf16 [R][S][C]
  const float* bias;   // [C] or null
  const void* res;     // NHWC bf16 [n][P][Q][C] or null
  void* y;             // NHWC bf16 [n][P][Q][C]
  int32_t n, H, W, C, P, Q, R, S, sh, sw, ph, pw, dh, dw;
  int32_t act;
  unsigned long long* tl;  // pask_config.timeline slots (null = off)
};

// Fused attention (PASK_K_ATTENTION): one CTA per (128-query tile, head, sequence).
struct alignas(64) AttnParams {
  CUtensorMap tmap_qkv;  // 3-D {3H, S, batch} bf16, box {64, 64, 1}, SWIZZLE_128B
  void* out;             // bf16 [batch][S][H]
  int32_t S, heads, batch, H;
  int32_t s_pad;         // S rounded up to 64 (key blocks; TMA zero-fills the tail)
  float scale_log2e;     // softmax scale * log2(e) (exp2 form)
  uint32_t idesc_qk;     // M=128, N=s_pad, A/B K-major
  uint32_t idesc_pv;     // M=128, N=64, A K-major, B MN-major
  uint32_t tmem_cols;    // power of two >= s_pad + 64
  uint32_t smem_bytes;
  unsigned long long* tl;  // pask_config.timeline slots (null = off)
};

struct alignas(16) RowParams {
  const void* x;  // bf16 [rows][cols]
  void* y;        // bf16 [rows][cols]
  const float* gamma;
  const float* beta;
  int32_t rows, cols;
  float scale;  // softmax
  float eps;    // layernorm
  unsigned long long* tl;  // pask_config.timeline slots (null = off)
};

// Weight-streaming GEMV (PASK_K_GEMV, D12): y[m][n] = act(sum_k
// x[m][k] w[n][k] + bias[n] + res[m][n]) for m < M <= 8.  A CTA of 8 warps owns
// `nc` consecutive columns; warp w takes column w % nc and K slice w / nc of
// 8 / nc slices; the slices are summed in fixed order (deterministic).
constexpr int kGemvThreads = 256;
constexpr unsigned kGemvSmem = 8 * 8 * 8 * 4;  // partials [slice][column][row], dynamic smem
struct alignas(16) GemvParams {
  const void* x;      // bf16, row m at x + m * lda (offset applied)
  const void* w;      // bf16 [N][ldb] (offset applied)
  const float* bias;  // [N] or null
  const void* res;    // bf16, same indexing as y, or null
  void* y;            // bf16, y[m * ldc + n] (offset applied)
  int64_t lda, ldb, ldc;
  int32_t M, N, K;
  int32_t nc_log2;    // columns per CTA: 1 << nc_log2 (1, 2, 4 or 8)
  int32_t per;        // 16-byte K vectors per slice: ceil(K / 8 / slices)
  int32_t act;
  unsigned long long* tl;  // pask_config.timeline slots (null = off)
};

// Operator-family entry (pask_config.packaging = 2): the memory-bound solutions
// (layout, depthwise conv, pooling, softmax, LayerNorm) share ONE CUfunction,
// `pask_mem`, so one code upload makes all of them resident.  The solution's
// own parameter block sits at offset 0; `kind` selects its body.
enum MemKind : int32_t { MEM_LAYOUT = 0, MEM_DW, MEM_POOL, MEM_GAVG, MEM_SOFTMAX, MEM_LAYERNORM, MEM_GEMV };
// bit of a families variant's memory mask (PASK_MEM_MASK) beyond the MemKind
// cases: the layout kernel's stem-fold path (D16)
constexpr int MEM_FOLD_BIT = 7;
struct alignas(16) MemParams {
  union {
    LayoutParams l;
    PoolParams p;
    DwParams d;
    RowParams r;
    GemvParams v;
  };
  int32_t kind;  // MemKind
};

// pask_create's driver primer (primer.cuh; not a solution, D11).
struct alignas(64) PrimerParams {
  CUtensorMap tmap_a;  // 3-D {64, 128, 1} bf16, SWIZZLE_128B
  CUtensorMap tmap_b;  // 3-D {64, 64, 1} bf16, SWIZZLE_128B
  float* out;          // [128][64] fp32
  int32_t run;         // 0: return at once (how pask_create launches it)
};

// Single-function entry (pask_config.packaging = 3): the contraction body and the
// memory-bound family in ONE CUfunction, `pask_all`, so a model's whole catalog
// becomes resident with one code upload.  g.family 0 runs g, 1 runs m (m lies at
// offset 0, below g.family, so a contraction launch passes the same bytes as in
// the other packagings).
union alignas(64) AllParams {
  GemmParams g;
  MemParams m;
};
static_assert(sizeof(MemParams) <= offsetof(GemmParams, family), "family flag outside the memory block");

}  // namespace pask
