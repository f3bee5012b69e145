// libpask.so: the C ABI of include/pask.h.
//
// Threads (§III-A "PASK spawns two extra host threads to handle
// code loading and kernel issuing"; :164 §III-D SPSC channels):
//   * caller thread = parser + planner (pask_load_model) and issuer (pask_infer);
//   * one loader thread per context, fed a FIFO of kernel ids in first-use order
//     (single producer: the planner; single consumer: the loader), publishing each
//     loaded CUfunction through a per-kernel atomic ready flag that the issuer
//     acquires right before the launch that needs it.
#include <immintrin.h>
#include <pthread.h>
#include <stdint.h>
#include <string.h>

#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstdio>
#include <cstdlib>
#include <deque>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../kernels/pask_params.h"
#include "driver.h"
#include "plan.h"

#define PASK_API extern "C" __attribute__((visibility("default")))

// Code objects embedded by build.py (fatbins.S): the whole catalog, and one
// SASS-only fatbin per catalog kernel.
extern "C" const unsigned char pask_fatbin_start[];
extern "C" const unsigned char pask_fatbin_end[];
#define PASK_FB(k)                                    \
  extern "C" const unsigned char pask_fb_##k##_start[]; \
  extern "C" const unsigned char pask_fb_##k##_end[];
PASK_FB(pask_layout)
PASK_FB(pask_conv_igemm)
PASK_FB(pask_conv_1x1)
PASK_FB(pask_conv_dw)
PASK_FB(pask_pool)
PASK_FB(pask_pool_gavg)
PASK_FB(pask_gemm)
PASK_FB(pask_softmax)
PASK_FB(pask_layernorm)
#undef PASK_FB

namespace pask {

namespace {

thread_local std::string t_err;

int set_err(int code, const std::string& m) {
  t_err = m;
  return code;
}

uint64_t now_ns() {
  return static_cast<uint64_t>(
      std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now().time_since_epoch())
          .count());
}

union alignas(64) AnyParams {
  GemmParams g;
  LayoutParams l;
  PoolParams p;
  DwParams d;
  RowParams r;
};

struct Launch {
  int32_t kernel = -1;
  unsigned grid[3] = {1, 1, 1};
  unsigned block[3] = {1, 1, 1};
  unsigned smem = 0;
  unsigned cluster_z = 1;  // split-K cluster size (thread-block cluster along z)
  std::unique_ptr<AnyParams> params;
};

struct Image {
  const unsigned char* begin;
  const unsigned char* end;
};
#define PASK_IMG(k) {pask_fb_##k##_start, pask_fb_##k##_end}
const Image kKernelImage[PASK_NUM_KERNELS] = {
    PASK_IMG(pask_layout),    PASK_IMG(pask_conv_igemm), PASK_IMG(pask_conv_1x1),
    PASK_IMG(pask_conv_dw),   PASK_IMG(pask_pool),       PASK_IMG(pask_pool_gavg),
    PASK_IMG(pask_gemm),      PASK_IMG(pask_softmax),    PASK_IMG(pask_layernorm)};
#undef PASK_IMG

bool is_gemm_kernel(int32_t k) {
  return k == PASK_K_CONV_IGEMM || k == PASK_K_CONV_1X1 || k == PASK_K_GEMM;
}

}  // namespace

struct Ctx {
  const Driver* d = nullptr;
  int device = 0;
  CUcontext cuctx = nullptr;
  pask_config cfg{};

  // ---- loader (proactive code loading)
  std::thread loader;
  std::mutex mu;
  std::condition_variable cv;
  std::deque<int32_t> fifo;
  bool stop = false;
  std::mutex lib_mu;  // serialises library/function loads (loader vs reactive issuer)
  CUlibrary lib = nullptr;                     // packaging 1: the whole catalog
  CUlibrary klib[PASK_NUM_KERNELS] = {};       // packaging 0: one code object per kernel
  std::atomic<int32_t> ready[PASK_NUM_KERNELS];
  CUfunction fn[PASK_NUM_KERNELS] = {};
  CUresult kerr[PASK_NUM_KERNELS] = {};
  bool requested[PASK_NUM_KERNELS] = {};
  std::atomic<uint64_t> load_ns{0};
  std::atomic<int32_t> code_objects{0};
  std::atomic<uint64_t> code_bytes{0};
  std::atomic<int32_t> kernels_loaded{0};
  // Issue priority: a code-object load holds the driver for 30-90 us and stalls
  // concurrent cuLaunchKernelEx calls (measured: 32 us per launch during a
  // load burst vs 2.4 us).  The loader therefore starts a load only while the
  // issuer is not issuing (blocked on a missing kernel, or between inferences);
  // the GPU keeps executing the already-queued layers meanwhile.
  std::atomic<int32_t> issuing{0};
  // proactive = 2: the helper thread encodes launch parameters (job kEncodeJob)
  // while the caller thread uploads the planned kernels
  std::atomic<int32_t> encode_state{0};  // 0 idle, 1 queued/running, 2 done
  int encode_rc = 0;
  uint64_t encode_job_ns = 0;
  std::string encode_err;
  uint64_t k_load_ns[PASK_NUM_KERNELS] = {};   // per-kernel cold timeline
  uint64_t k_ready_at[PASK_NUM_KERNELS] = {};  // absolute steady-clock ns
  uint64_t k_lib_ns[PASK_NUM_KERNELS] = {};

  // ---- model
  bool have_model = false;
  std::vector<pask_tensor> tensors;
  std::vector<pask_node> nodes;
  std::vector<int32_t> inputs, outputs;
  void* ws = nullptr;
  uint64_t ws_bytes = 0;
  std::vector<Problem> probs;
  PlanResult plan;
  std::vector<Launch> launches;

  // ---- timing / stats
  pask_stats_t st{};
  uint64_t t_entry = 0;
  bool first_done = false;
  bool pending = false;
  CUevent ev0 = nullptr, ev1 = nullptr;
  std::vector<CUevent> node_ev;
  CUgraph graph = nullptr;          // cfg.graph: captured hot launch sequence
  CUgraphExec graph_exec = nullptr;
  CUstream capture_stream = nullptr;  // private non-blocking stream (legacy streams cannot capture)
  std::vector<uint64_t> node_ns;

  Ctx() {
    for (auto& r : ready) r.store(0);
  }
};

namespace {

constexpr int32_t kEncodeJob = -1;
int encode_all(Ctx* c, std::string* err);

std::string cu_err(const Driver* d, CUresult r, const char* what) {
  const char* name = nullptr;
  if (d && d->cuGetErrorName) d->cuGetErrorName(r, &name);
  return std::string(what) + " failed: " + (name ? name : "CUDA_ERROR_?") + " (" + std::to_string(r) + ")";
}

// Load one catalog kernel into the context: library once, then
// cuLibraryGetKernel -> cuKernelGetFunction -> cuFuncLoad (A13 of SURVEY.md §2).
void load_kernel(Ctx* c, int32_t k) {
  std::lock_guard<std::mutex> g(c->lib_mu);
  if (c->ready[k].load(std::memory_order_acquire) != 0) return;
  const uint64_t t0 = now_ns();
  const Driver* d = c->d;
  CUresult r = CUDA_SUCCESS;
  // the embedded image stays valid for the life of the process: no driver copy
  CUlibraryOption opt[1] = {CU_LIBRARY_BINARY_IS_PRESERVED};
  void* optv[1] = {reinterpret_cast<void*>(1)};
  CUlibrary* lib = c->cfg.packaging == 1 ? &c->lib : &c->klib[k];
  if (!*lib) {
    const unsigned char* img = c->cfg.packaging == 1 ? pask_fatbin_start : kKernelImage[k].begin;
    const unsigned char* end = c->cfg.packaging == 1 ? pask_fatbin_end : kKernelImage[k].end;
    r = d->cuLibraryLoadData(lib, img, nullptr, nullptr, 0, opt, optv, 1);
    c->k_lib_ns[k] = now_ns() - t0;
    if (r == CUDA_SUCCESS) {
      c->code_objects.fetch_add(1);
      c->code_bytes.fetch_add(static_cast<uint64_t>(end - img));
    }
  }
  CUkernel kern = nullptr;
  CUfunction f = nullptr;
  if (r == CUDA_SUCCESS) r = d->cuLibraryGetKernel(&kern, *lib, catalog(k).name);
  if (r == CUDA_SUCCESS) r = d->cuKernelGetFunction(&f, kern);
  if (r == CUDA_SUCCESS) r = d->cuFuncLoad(f);
  if (r == CUDA_SUCCESS && is_gemm_kernel(k))
    r = d->cuFuncSetAttribute(f, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, static_cast<int>(kMaxDynSmem));
  if (r == CUDA_SUCCESS && is_gemm_kernel(k))  // one fixed L1/smem split: no per-launch reconfiguration
    r = d->cuFuncSetAttribute(f, CU_FUNC_ATTRIBUTE_PREFERRED_SHARED_MEMORY_CARVEOUT, 100);
  c->fn[k] = f;
  c->kerr[k] = r;
  if (r == CUDA_SUCCESS) c->kernels_loaded.fetch_add(1);
  const uint64_t t1 = now_ns();
  c->k_load_ns[k] = t1 - t0;
  c->k_ready_at[k] = t1;
  c->load_ns.fetch_add(t1 - t0);
  c->ready[k].store(r == CUDA_SUCCESS ? 1 : -1, std::memory_order_release);
}

// The loader polls for work (keeping its core awake) for a bounded window after
// each wake-up -- a load started on a just-woken, down-clocked core measured up
// to 7x slower -- then sleeps on the condition variable.
void loader_main(Ctx* c) {
  pthread_setname_np(pthread_self(), "pask-loader");
  c->d->cuCtxSetCurrent(c->cuctx);
  constexpr uint64_t kSpinNs = 20ull * 1000 * 1000;  // 20 ms
  uint64_t spin_until = now_ns() + kSpinNs;
  for (;;) {
    int32_t k = 0;
    bool got = false;
    while (!got) {
      {
        std::unique_lock<std::mutex> lk(c->mu);
        if (c->stop && c->fifo.empty()) return;
        if (!c->fifo.empty()) {
          k = c->fifo.front();
          c->fifo.pop_front();
          got = true;
          break;
        }
        if (now_ns() > spin_until) {
          c->cv.wait(lk, [&] { return c->stop || !c->fifo.empty(); });
          spin_until = now_ns() + kSpinNs;
          continue;
        }
      }
      for (int i = 0; i < 64; ++i) _mm_pause();
    }
    if (k == kEncodeJob) {
      const uint64_t e0 = now_ns();
      c->encode_rc = encode_all(c, &c->encode_err);
      c->encode_job_ns = now_ns() - e0;
      c->encode_state.store(2, std::memory_order_release);
      spin_until = now_ns() + kSpinNs;
      continue;
    }
    if (c->cfg.interleave)
      while (c->issuing.load(std::memory_order_acquire) && !c->stop) _mm_pause();
    load_kernel(c, k);
    spin_until = now_ns() + kSpinNs;
  }
}

// ------------------------------------------------------------------ tensor maps
int encode_3d(Ctx* c, CUtensorMap* m, const void* base, uint64_t d0, uint64_t d1, uint64_t d2,
              uint64_t s1_bytes, uint64_t s2_bytes, uint32_t b0, uint32_t b1, std::string* err,
              CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  if (d2 <= 1) s2_bytes = s1_bytes * d1;
  cuuint64_t dims[3] = {d0, d1, std::max<uint64_t>(d2, 1)};
  cuuint64_t strides[2] = {s1_bytes, s2_bytes};
  cuuint32_t box[3] = {b0, b1, 1};
  cuuint32_t es[3] = {1, 1, 1};
  CUresult r = c->d->cuTensorMapEncodeTiled(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(base), dims,
                                            strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                            swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    *err = cu_err(c->d, r, "cuTensorMapEncodeTiled");
    return PASK_ECUDA;
  }
  return PASK_OK;
}

uint32_t make_idesc(int bn, int b_major) {
  uint32_t d = 0;
  d |= 1u << 4;                              // D format f32
  d |= 1u << 7;                              // A bf16
  d |= 1u << 10;                             // B bf16
  d |= static_cast<uint32_t>(b_major) << 16;  // B major (A is always K-major)
  d |= static_cast<uint32_t>(bn >> 3) << 17;  // N >> 3
  d |= static_cast<uint32_t>(128 >> 4) << 24;  // M >> 4
  return d;
}

unsigned grid_1d(int64_t total, int threads) {
  int64_t b = (total + threads - 1) / threads;
  if (b < 1) b = 1;
  if (b > 148 * 16) b = 148 * 16;  // grid-stride beyond 16 waves of 1 CTA/SM
  return static_cast<unsigned>(b);
}

// Build the launch (grid, block, smem, parameter block) of node i for its bound kernel.
int lower_node(Ctx* c, int32_t i, std::string* err) {
  const pask_node& nd = c->nodes[i];
  const Problem& p = c->probs[i];
  Launch& L = c->launches[i];
  L.kernel = c->plan.bindings[i].bound_kernel;
  if (!L.params) L.params.reset(new AnyParams);
  memset(L.params.get(), 0, sizeof(AnyParams));
  const pask_tensor& x = c->tensors[nd.in0];
  const pask_tensor& y = c->tensors[nd.out];
  const void* res = nd.res >= 0 ? c->tensors[nd.res].dptr : nullptr;
  L.block[0] = 256;
  L.block[1] = L.block[2] = 1;
  L.grid[1] = L.grid[2] = 1;
  L.smem = 0;
  L.cluster_z = 1;
  switch (L.kernel) {
    case PASK_K_LAYOUT: {
      LayoutParams& q = L.params->l;
      q.x = static_cast<const float*>(x.dptr);
      q.y = y.dptr;
      q.n = p.n; q.c = p.c; q.h = p.h; q.w = p.w; q.c_out = p.k;
      L.grid[0] = grid_1d(static_cast<int64_t>(p.n) * p.h * p.w * (p.k / 8), 256);
      return PASK_OK;
    }
    case PASK_K_CONV_DW: {
      DwParams& q = L.params->d;
      q.x = x.dptr; q.w = nd.w; q.bias = nd.bias; q.res = res; q.y = y.dptr;
      q.n = p.n; q.H = p.h; q.W = p.w; q.C = p.c; q.P = p.p; q.Q = p.q; q.R = p.r; q.S = p.s;
      q.sh = p.stride_h; q.sw = p.stride_w; q.ph = p.pad_h; q.pw = p.pad_w; q.dh = p.dil_h; q.dw = p.dil_w;
      q.act = nd.act;
      L.grid[0] = grid_1d(static_cast<int64_t>(p.n) * p.p * p.q * (p.c / 8), 256);
      return PASK_OK;
    }
    case PASK_K_POOL:
    case PASK_K_POOL_GAVG: {
      PoolParams& q = L.params->p;
      q.x = x.dptr; q.y = y.dptr;
      q.n = p.n; q.H = p.h; q.W = p.w; q.C = p.c; q.P = p.p; q.Q = p.q; q.R = p.r; q.S = p.s;
      q.sh = p.stride_h; q.sw = p.stride_w; q.ph = p.pad_h; q.pw = p.pad_w;
      q.mode = p.pool_mode; q.count_include_pad = nd.count_include_pad;
      if (L.kernel == PASK_K_POOL_GAVG) {
        L.block[0] = 128;
        L.grid[0] = static_cast<unsigned>((p.c / 8 + 31) / 32);
        L.grid[1] = static_cast<unsigned>(p.n);
      } else {
        const int64_t outs = static_cast<int64_t>(p.n) * p.p * p.q * (p.c / 8);
        q.per_warp = (p.r * p.s > 16) ? 1 : 0;
        L.grid[0] = grid_1d(q.per_warp ? outs * 32 : outs, 256);
      }
      return PASK_OK;
    }
    case PASK_K_SOFTMAX:
    case PASK_K_LAYERNORM: {
      RowParams& q = L.params->r;
      q.x = x.dptr; q.y = y.dptr; q.gamma = nd.gamma; q.beta = nd.beta;
      q.rows = p.rows; q.cols = p.cols; q.scale = nd.scale; q.eps = nd.eps;
      L.grid[0] = static_cast<unsigned>((p.rows + 7) / 8);
      return PASK_OK;
    }
    case PASK_K_CONV_IGEMM:
    case PASK_K_CONV_1X1:
    case PASK_K_GEMM: {
      GemmParams& q = L.params->g;
      int32_t M, N, K, batch, b_major;
      contraction_shape(p, nd, &M, &N, &K, &batch, &b_major);
      const int64_t ldc = p.op == OC_CONV ? p.k : nd.ldc;
      const int64_t off_c = p.op == OC_CONV ? 0 : nd.off_c;
      const int64_t stride_c = p.op == OC_CONV ? 0 : nd.stride_c;
      auto al16 = [](const void* ptr) { return (reinterpret_cast<uintptr_t>(ptr) & 15) == 0; };
      // staged TMA epilogue needs 16-byte row pitch / offsets (not e.g. the N = 10 FC)
      const int32_t c_tma = (ldc % 8 == 0) && (off_c % 8 == 0) && (batch == 1 || stride_c % 8 == 0) &&
                            al16(y.dptr) && (!res || al16(res));
      const GemmTiling t = gemm_tiling(M, N, K, batch, b_major, c_tma);
      q.M = M; q.N = N; q.K = K; q.batch = batch;
      q.num_kb = t.num_kb; q.kb_per_split = (t.num_kb + t.splits - 1) / t.splits; q.splits = t.splits;
      q.rows_per = t.rows_per; q.c_tma = c_tma;
      q.bn = t.bn; q.stages = t.stages; q.b_major = b_major; q.act = nd.act;
      q.b_const = (p.op == OC_CONV || nd.w != nullptr) ? 1 : 0;
      q.m_tiles = t.m_tiles; q.n_tiles = t.n_tiles;
      q.idesc = make_idesc(t.bn, b_major);
      q.tmem_cols = t.tmem_cols;
      q.smem_bytes = t.smem_bytes;
      q.out = y.dptr; q.res = res; q.bias = nd.bias;
      q.ldc = ldc; q.off_c = off_c; q.stride_c = stride_c;
      int rc;
      if (c_tma) {
        const uint32_t box_cols = t.bn < 64 ? static_cast<uint32_t>(t.bn) : 64u;
        const CUtensorMapSwizzle swz = box_cols == 64 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE;
        const char* cbase = static_cast<const char*>(y.dptr) + off_c * 2;
        rc = encode_3d(c, &q.tmap_c, cbase, static_cast<uint64_t>(N), static_cast<uint64_t>(M),
                       static_cast<uint64_t>(batch), static_cast<uint64_t>(ldc) * 2,
                       static_cast<uint64_t>(stride_c) * 2, box_cols, static_cast<uint32_t>(t.rows_per), err, swz);
        if (rc) return rc;
        if (res) {
          const char* rbase = static_cast<const char*>(res) + off_c * 2;
          rc = encode_3d(c, &q.tmap_r, rbase, static_cast<uint64_t>(N), static_cast<uint64_t>(M),
                         static_cast<uint64_t>(batch), static_cast<uint64_t>(ldc) * 2,
                         static_cast<uint64_t>(stride_c) * 2, box_cols, static_cast<uint32_t>(t.rows_per), err, swz);
          if (rc) return rc;
        }
      }
      if (p.op == OC_CONV) {
        const bool plain = (p.r == 1 && p.s == 1 && p.stride_h == 1 && p.stride_w == 1 && p.pad_h == 0 &&
                            p.pad_w == 0);
        // TMA im2col needs whole 64-channel chunks per tap and its corner ranges
        const int lw = -p.pad_w, lh = -p.pad_h;
        const int uw = p.pad_w - (p.s - 1) * p.dil_w, uh = p.pad_h - (p.r - 1) * p.dil_h;
        const bool im2col_ok = (p.c % 64 == 0) && lw >= -128 && lh >= -128 && uw >= -128 && uh >= -128 &&
                               uw <= 127 && uh <= 127 && (p.s - 1) * p.dil_w < 65536 && (p.r - 1) * p.dil_h < 65536 &&
                               !getenv("PASK_NO_IM2COL");
        q.a_mode = (L.kernel == PASK_K_CONV_1X1 || plain) ? A_TMA : (im2col_ok ? A_IM2COL : A_GATHER);
        q.x = x.dptr;
        q.H = p.h; q.W = p.w; q.C = p.c; q.P = p.p; q.Q = p.q; q.R = p.r; q.S = p.s;
        q.sh = p.stride_h; q.sw = p.stride_w; q.ph = p.pad_h; q.pw = p.pad_w; q.dh = p.dil_h; q.dw = p.dil_w;
        if (q.a_mode == A_TMA) {
          rc = encode_3d(c, &q.tmap_a, x.dptr, static_cast<uint64_t>(K), static_cast<uint64_t>(M), 1,
                         static_cast<uint64_t>(p.c) * 2, 0, 64, 128, err);
          if (rc) return rc;
        } else if (q.a_mode == A_IM2COL) {
          cuuint64_t dims[4] = {static_cast<cuuint64_t>(p.c), static_cast<cuuint64_t>(p.w),
                                static_cast<cuuint64_t>(p.h), static_cast<cuuint64_t>(p.n)};
          cuuint64_t strides[3] = {static_cast<cuuint64_t>(p.c) * 2, static_cast<cuuint64_t>(p.w) * p.c * 2,
                                   static_cast<cuuint64_t>(p.h) * p.w * p.c * 2};
          int lower[2] = {lw, lh}, upper[2] = {uw, uh};  // {W, H} (innermost spatial first)
          cuuint32_t es[4] = {1, static_cast<cuuint32_t>(p.stride_w), static_cast<cuuint32_t>(p.stride_h), 1};
          CUresult r = c->d->cuTensorMapEncodeIm2col(&q.tmap_a, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, x.dptr, dims,
                                                     strides, lower, upper, 64, 128, es,
                                                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
          if (r != CUDA_SUCCESS) {
            *err = cu_err(c->d, r, "cuTensorMapEncodeIm2col");
            return PASK_ECUDA;
          }
        }
        // weights KRSC = [N][K] K-major
        rc = encode_3d(c, &q.tmap_b, nd.w, static_cast<uint64_t>(K), static_cast<uint64_t>(N), 1,
                       static_cast<uint64_t>(K) * 2, 0, 64, static_cast<uint32_t>(t.bn), err);
        if (rc) return rc;
      } else {
        q.a_mode = A_TMA;
        const char* abase = static_cast<const char*>(x.dptr) + nd.off_a * 2;
        rc = encode_3d(c, &q.tmap_a, abase, static_cast<uint64_t>(K), static_cast<uint64_t>(M),
                       static_cast<uint64_t>(batch), static_cast<uint64_t>(nd.lda) * 2,
                       static_cast<uint64_t>(nd.stride_a) * 2, 64, 128, err);
        if (rc) return rc;
        const void* bsrc = nd.w ? nd.w : c->tensors[nd.in1].dptr;
        const char* bbase = static_cast<const char*>(bsrc) + nd.off_b * 2;
        if (b_major == 0)
          rc = encode_3d(c, &q.tmap_b, bbase, static_cast<uint64_t>(K), static_cast<uint64_t>(N),
                         static_cast<uint64_t>(batch), static_cast<uint64_t>(nd.ldb) * 2,
                         static_cast<uint64_t>(nd.stride_b) * 2, 64, static_cast<uint32_t>(t.bn), err);
        else
          rc = encode_3d(c, &q.tmap_b, bbase, static_cast<uint64_t>(N), static_cast<uint64_t>(K),
                         static_cast<uint64_t>(batch), static_cast<uint64_t>(nd.ldb) * 2,
                         static_cast<uint64_t>(nd.stride_b) * 2, 64, 64, err);
        if (rc) return rc;
      }
      {  // debug-only phase trace (PASK_TRACE_NODE=i or -1 for all; PASK_TRACE_PTR=<device
         // address>; node i writes 8 stamps per CTA at PTR + i * 8 * 4096 words)
        const char* tn = getenv("PASK_TRACE_NODE");
        const char* tp = getenv("PASK_TRACE_PTR");
        if (tn && tp && (atoi(tn) == i || atoi(tn) == -1))
          q.trace = reinterpret_cast<unsigned long long*>(strtoull(tp, nullptr, 0)) +
                    (atoi(tn) == -1 ? static_cast<size_t>(i) * 8 * 4096 : 0);
      }
      L.block[0] = kGemmThreads;
      L.grid[0] = static_cast<unsigned>(t.m_tiles);
      L.grid[1] = static_cast<unsigned>(t.n_tiles);
      L.grid[2] = static_cast<unsigned>(batch * t.splits);
      L.cluster_z = static_cast<unsigned>(t.splits);
      L.smem = t.smem_bytes;
      return PASK_OK;
    }
  }
  *err = "node " + std::to_string(i) + ": no lowering for kernel";
  return PASK_EINVAL;
}

int encode_all(Ctx* c, std::string* err) {
  for (int32_t i = 0; i < static_cast<int32_t>(c->nodes.size()); ++i) {
    int rc = lower_node(c, i, err);
    if (rc) return rc;
  }
  return PASK_OK;
}

int plan_graph(const pask_graph* g, const pask_config& cfg, std::vector<Problem>* probs, PlanResult* plan) {
  std::string err;
  int rc = extract_problems(g, probs, &err);
  if (rc) return set_err(rc, err);
  std::vector<int32_t> desired(probs->size());
  for (size_t i = 0; i < probs->size(); ++i) {
    const int32_t sol = g->nodes[i].solution;
    desired[i] = (sol >= 0) ? sol : static_choice((*probs)[i]);
  }
  rc = execution_plan(*probs, desired, cfg, plan, &err);
  if (rc) return set_err(rc, err);
  return PASK_OK;
}

// Wait until kernel k is loaded.  A blocked issuer does not idle: it pops the
// next queued load (first-use order) and performs it itself -- its core is
// already running, while the loader thread may be waking on a cold core.
int wait_kernel(Ctx* c, int32_t k) {
  int32_t s = c->ready[k].load(std::memory_order_acquire);
  if (s == 0) {
    const uint64_t t0 = now_ns();
    c->issuing.store(0, std::memory_order_release);  // blocked: the loader may take the driver
    if (!c->cfg.proactive) {
      load_kernel(c, k);  // reactive: load at launch, on the issue thread (A1 baseline)
    } else {
      for (;;) {
        if ((s = c->ready[k].load(std::memory_order_acquire)) != 0) break;
        int32_t next = -1;
        {
          std::lock_guard<std::mutex> lk(c->mu);
          if (!c->requested[k]) {  // not planned for loading (e.g. rebinding) -> queue it now
            c->requested[k] = true;
            c->fifo.push_back(k);
          }
          if (!c->fifo.empty()) {
            next = c->fifo.front();
            c->fifo.pop_front();
          }
        }
        if (next >= 0)
          load_kernel(c, next);  // work stealing; lib_mu keeps loads serialised
        else
          _mm_pause();  // the loader thread holds the last pending load
      }
    }
    c->issuing.store(1, std::memory_order_release);
    c->st.load_exposed_ns += now_ns() - t0;
    s = c->ready[k].load(std::memory_order_acquire);
  }
  if (s < 0)
    return set_err(PASK_ECUDA, cu_err(c->d, c->kerr[k], (std::string("loading ") + catalog(k).name).c_str()));
  return PASK_OK;
}

int rebind(Ctx* c, int32_t tidx, void* ptr) {
  if (c->tensors[tidx].dptr == ptr) return PASK_OK;
  c->tensors[tidx].dptr = ptr;
  std::string err;
  for (size_t i = 0; i < c->nodes.size(); ++i) {
    const pask_node& nd = c->nodes[i];
    if (nd.in0 == tidx || nd.in1 == tidx || nd.res == tidx || nd.out == tidx) {
      int rc = lower_node(c, static_cast<int32_t>(i), &err);
      if (rc) return set_err(rc, err);
    }
  }
  return PASK_OK;
}

size_t tensor_bytes(const pask_tensor& t) {
  return static_cast<size_t>(t.n) * t.h * t.w * t.c * (t.dtype == PASK_F32 ? 4 : 2);
}

}  // namespace
}  // namespace pask

using namespace pask;

struct pask_ctx : pask::Ctx {};

// ====================================================================== API
PASK_API int pask_version(void) { return PASK_VERSION; }

PASK_API const char* pask_last_error(void) { return t_err.c_str(); }

PASK_API int32_t pask_num_kernels(void) { return PASK_NUM_KERNELS; }

PASK_API const char* pask_kernel_name(int32_t id) {
  if (id < 0 || id >= PASK_NUM_KERNELS) return "";
  return catalog(id).name;
}

PASK_API int pask_plan(const pask_graph* g, const pask_config* cfg, pask_binding* plan_out,
                       pask_stats_t* stats_out) {
  t_err.clear();
  const uint64_t t0 = now_ns();
  pask_config c = cfg ? *cfg : default_config();
  std::vector<Problem> probs;
  PlanResult plan;
  int rc = plan_graph(g, c, &probs, &plan);
  if (rc) return rc;
  if (plan_out) memcpy(plan_out, plan.bindings.data(), plan.bindings.size() * sizeof(pask_binding));
  if (stats_out) {
    memset(stats_out, 0, sizeof(*stats_out));
    stats_out->n_nodes = g->n_nodes;
    stats_out->kernels_loaded = static_cast<int32_t>(plan.loaded.size());
    stats_out->queries = plan.queries;
    stats_out->hits = plan.hits;
    stats_out->lookups = plan.lookups;
    stats_out->plan_ns = now_ns() - t0;
  }
  return PASK_OK;
}

PASK_API int pask_workspace_bytes(const pask_graph* g, uint64_t* bytes) {
  t_err.clear();
  if (!bytes) return set_err(PASK_EINVAL, "bytes is null");
  std::vector<Problem> probs;
  std::string err;
  int rc = extract_problems(g, &probs, &err);
  if (rc) return set_err(rc, err);
  // split-K partials are reduced on chip (cluster DSMEM): no global scratch today
  *bytes = 0;
  return PASK_OK;
}

PASK_API int pask_create(pask_ctx** out, int device, const pask_config* cfg) {
  t_err.clear();
  if (!out) return set_err(PASK_EINVAL, "ctx out-pointer is null");
  *out = nullptr;
  const char* why = "";
  const Driver* d = driver(&why);
  if (!d) return set_err(PASK_ECUDA, std::string("CUDA driver unavailable: ") + why);
  CUresult r = d->cuInit(0);
  if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuInit"));
  std::unique_ptr<pask_ctx> c(new pask_ctx);
  c->d = d;
  c->device = device;
  c->cfg = cfg ? *cfg : default_config();
  CUcontext cur = nullptr;
  d->cuCtxGetCurrent(&cur);
  if (!cur) {
    CUdevice dev;
    r = d->cuDeviceGet(&dev, device);
    if (r == CUDA_SUCCESS) r = d->cuDevicePrimaryCtxRetain(&cur, dev);
    if (r == CUDA_SUCCESS) r = d->cuCtxSetCurrent(cur);
    if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "primary context"));
  }
  c->cuctx = cur;
  r = d->cuEventCreate(&c->ev0, CU_EVENT_DEFAULT);
  if (r == CUDA_SUCCESS) r = d->cuEventCreate(&c->ev1, CU_EVENT_DEFAULT);
  if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuEventCreate"));
  pask_ctx* raw = c.get();
  raw->loader = std::thread(loader_main, raw);
  *out = c.release();
  return PASK_OK;
}

PASK_API int pask_load_model(pask_ctx* c, const pask_graph* g, pask_binding* plan_out) {
  t_err.clear();
  if (!c || !g) return set_err(PASK_EINVAL, "null ctx or graph");
  if (c->have_model) return set_err(PASK_ESTATE, "a model is already loaded in this context");
  c->t_entry = now_ns();
  // ---- parse + plan (Algorithm 1)
  int rc = plan_graph(g, c->cfg, &c->probs, &c->plan);
  if (rc) return rc;
  const uint64_t t_plan = now_ns();
  // ---- copy the graph (the library keeps its own arrays)
  c->tensors.assign(g->tensors, g->tensors + g->n_tensors);
  c->nodes.assign(g->nodes, g->nodes + g->n_nodes);
  c->inputs.assign(g->inputs, g->inputs + g->n_inputs);
  c->outputs.assign(g->outputs, g->outputs + g->n_outputs);
  for (int32_t t : c->inputs)
    if (t < 0 || t >= g->n_tensors) return set_err(PASK_EINVAL, "graph input index out of range");
  for (int32_t t : c->outputs)
    if (t < 0 || t >= g->n_tensors) return set_err(PASK_EINVAL, "graph output index out of range");
  c->ws = g->workspace;
  c->ws_bytes = g->workspace_bytes;
  c->launches.clear();
  c->launches.resize(g->n_nodes);
  std::string err;
  uint64_t t_loads = 0;
  if (c->cfg.proactive == 2) {
    // the caller thread uploads the planned kernels in first-use order while
    // the helper thread encodes the per-node launch parameters
    c->encode_state.store(1, std::memory_order_release);
    {
      std::lock_guard<std::mutex> lk(c->mu);
      c->fifo.push_back(kEncodeJob);
      c->cv.notify_one();
    }
    for (int32_t k : c->plan.loaded) {
      {
        std::lock_guard<std::mutex> lk(c->mu);
        c->requested[k] = true;
      }
      load_kernel(c, k);
    }
    t_loads = now_ns();
    while (c->encode_state.load(std::memory_order_acquire) != 2) _mm_pause();
    c->encode_state.store(0, std::memory_order_release);
    if (c->encode_rc) return set_err(c->encode_rc, c->encode_err);
    for (int32_t k : c->plan.loaded)
      if (c->ready[k].load(std::memory_order_acquire) < 0)
        return set_err(PASK_ECUDA, cu_err(c->d, c->kerr[k], (std::string("loading ") + catalog(k).name).c_str()));
  } else {
    // ---- proactive loading: hand the bound kernels to the loader, first-use order
    if (c->cfg.proactive) {
      std::lock_guard<std::mutex> lk(c->mu);
      for (const pask_binding& b : c->plan.bindings) {
        const int32_t k = b.bound_kernel;
        if (!c->requested[k]) {
          c->requested[k] = true;
          c->fifo.push_back(k);
        }
      }
      c->cv.notify_one();
    }
    // ---- lower every node while loading proceeds
    rc = encode_all(c, &err);
    if (rc) return set_err(rc, err);
  }
  if (c->cfg.instrument) {
    c->node_ev.resize(2 * g->n_nodes);
    for (auto& e : c->node_ev) {
      CUresult r = c->d->cuEventCreate(&e, CU_EVENT_DEFAULT);
      if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(c->d, r, "cuEventCreate"));
    }
  }
  const uint64_t t_enc = now_ns();
  memset(&c->st, 0, sizeof(c->st));
  c->st.n_nodes = g->n_nodes;
  c->st.queries = c->plan.queries;
  c->st.hits = c->plan.hits;
  c->st.lookups = c->plan.lookups;
  c->st.plan_ns = t_plan - c->t_entry;
  // proactive 2 encodes on the helper thread concurrently with the uploads
  c->st.encode_ns = c->cfg.proactive == 2 ? c->encode_job_ns : t_enc - t_plan;
  c->st.load_done_ns = t_loads ? t_loads - c->t_entry : 0;
  if (plan_out) memcpy(plan_out, c->plan.bindings.data(), c->plan.bindings.size() * sizeof(pask_binding));
  c->have_model = true;
  c->first_done = false;
  return PASK_OK;
}

namespace pask {
namespace {
// Issue every node's launch on stream s (the issue loop, PAPER.md:95 I_i).
int issue_all(Ctx* c, CUstream s, bool first) {
  const Driver* d = c->d;
  int rc;
  CUlaunchAttribute attr[2];
  for (size_t i = 0; i < c->launches.size(); ++i) {
    Launch& L = c->launches[i];
    if ((rc = wait_kernel(c, L.kernel))) return rc;
    if (c->cfg.instrument) d->cuEventRecord(c->node_ev[2 * i], s);
    CUlaunchConfig cfg{};
    cfg.gridDimX = L.grid[0];
    cfg.gridDimY = L.grid[1];
    cfg.gridDimZ = L.grid[2];
    cfg.blockDimX = L.block[0];
    cfg.blockDimY = L.block[1];
    cfg.blockDimZ = L.block[2];
    cfg.sharedMemBytes = L.smem;
    cfg.hStream = s;
    unsigned na = 0;
    if (c->cfg.pdl && !c->cfg.instrument && i > 0) {
      attr[na].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
      attr[na].value.programmaticStreamSerializationAllowed = 1;
      ++na;
    }
    if (L.cluster_z > 1) {
      attr[na].id = CU_LAUNCH_ATTRIBUTE_CLUSTER_DIMENSION;
      attr[na].value.clusterDim.x = 1;
      attr[na].value.clusterDim.y = 1;
      attr[na].value.clusterDim.z = L.cluster_z;
      ++na;
    }
    cfg.attrs = attr;
    cfg.numAttrs = na;
    void* args[1] = {L.params.get()};
    const uint64_t t0 = now_ns();
    CUresult r = d->cuLaunchKernelEx(&cfg, c->fn[L.kernel], args, nullptr);
    c->st.issue_ns += now_ns() - t0;
    if (r != CUDA_SUCCESS)
      return set_err(PASK_ECUDA, cu_err(d, r, ("launch of node " + std::to_string(i) + " (" +
                                               catalog(L.kernel).name + ")").c_str()));
    if (c->cfg.instrument) d->cuEventRecord(c->node_ev[2 * i + 1], s);
    c->st.launches++;
    if (first && i == 0) c->st.first_launch_ns = now_ns() - c->t_entry;
  }
  return PASK_OK;
}

void drop_graph(Ctx* c) {
  if (c->graph_exec) c->d->cuGraphExecDestroy(c->graph_exec);
  if (c->graph) c->d->cuGraphDestroy(c->graph);
  c->graph_exec = nullptr;
  c->graph = nullptr;
}

// Capture the launch sequence into a CUDA graph (hot path) on the private
// capture stream; the executable graph is then launched on the caller's stream.
int capture_graph(Ctx* c) {
  const Driver* d = c->d;
  drop_graph(c);
  CUresult r;
  if (!c->capture_stream) {
    r = d->cuStreamCreate(&c->capture_stream, CU_STREAM_NON_BLOCKING);
    if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuStreamCreate"));
  }
  CUstream s = c->capture_stream;
  r = d->cuStreamBeginCapture(s, CU_STREAM_CAPTURE_MODE_THREAD_LOCAL);
  if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuStreamBeginCapture"));
  const uint64_t launches = c->st.launches;
  int rc = issue_all(c, s, false);
  c->st.launches = launches;  // captured, not launched
  CUgraph g = nullptr;
  r = d->cuStreamEndCapture(s, &g);
  if (rc) {
    if (g) d->cuGraphDestroy(g);
    return rc;
  }
  if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuStreamEndCapture"));
  CUgraphExec ge = nullptr;
  r = d->cuGraphInstantiateWithFlags(&ge, g, 0);
  if (r != CUDA_SUCCESS) {
    d->cuGraphDestroy(g);
    return set_err(PASK_ECUDA, cu_err(d, r, "cuGraphInstantiateWithFlags"));
  }
  c->graph = g;
  c->graph_exec = ge;
  return PASK_OK;
}
}  // namespace
}  // namespace pask

PASK_API int pask_infer(pask_ctx* c, void* const* inputs, void* const* outputs, void* stream) {
  t_err.clear();
  if (!c) return set_err(PASK_EINVAL, "null ctx");
  if (!c->have_model) return set_err(PASK_ESTATE, "pask_infer before pask_load_model");
  int rc;
  const bool first = c->st.infer_count == 0;
  if (first) c->st.infer_entry_ns = now_ns() - c->t_entry;
  bool rebound = false;
  for (size_t i = 0; inputs && i < c->inputs.size(); ++i)
    if (inputs[i] && c->tensors[c->inputs[i]].dptr != inputs[i]) {
      if ((rc = rebind(c, c->inputs[i], inputs[i]))) return rc;
      rebound = true;
    }
  for (size_t i = 0; outputs && i < c->outputs.size(); ++i)
    if (outputs[i] && c->tensors[c->outputs[i]].dptr != outputs[i]) {
      if ((rc = rebind(c, c->outputs[i], outputs[i]))) return rc;
      rebound = true;
    }
  const Driver* d = c->d;
  CUstream s = static_cast<CUstream>(stream);
  if (c->cfg.proactive && !c->cfg.interleave) {
    // load-first: every planned kernel uploaded before the first launch (uploads
    // wait for running GPU work, so interleaving them with launches only
    // serialises each upload behind the layers already queued)
    for (int32_t k : c->plan.loaded)
      if ((rc = wait_kernel(c, k))) return rc;
  }
  c->issuing.store(1, std::memory_order_release);
  struct Idle {  // the loader may run again once this inference is issued (or fails)
    std::atomic<int32_t>& f;
    ~Idle() { f.store(0, std::memory_order_release); }
  } idle{c->issuing};
  const bool use_graph = c->cfg.graph && !c->cfg.instrument && !first;
  if (use_graph && (rebound || !c->graph_exec)) {
    if ((rc = capture_graph(c))) return rc;
  }
  d->cuEventRecord(c->ev0, s);
  if (use_graph) {
    const uint64_t t0 = now_ns();
    CUresult r = d->cuGraphLaunch(c->graph_exec, s);
    c->st.issue_ns += now_ns() - t0;
    if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuGraphLaunch"));
    c->st.launches += c->launches.size();
  } else if ((rc = issue_all(c, s, first))) {
    return rc;
  }
  if (first) {
    c->st.last_launch_ns = now_ns() - c->t_entry;
    if (!c->st.load_done_ns) c->st.load_done_ns = c->st.first_launch_ns;
  }
  d->cuEventRecord(c->ev1, s);
  c->st.infer_count++;
  c->pending = true;
  return PASK_OK;
}

PASK_API int pask_sync(pask_ctx* c) {
  t_err.clear();
  if (!c) return set_err(PASK_EINVAL, "null ctx");
  if (!c->pending) return PASK_OK;
  const Driver* d = c->d;
  CUresult r = d->cuEventSynchronize(c->ev1);
  if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuEventSynchronize"));
  const uint64_t t1 = now_ns();
  if (!c->first_done) {
    c->st.cold_wall_ns = t1 - c->t_entry;
    c->first_done = true;
  }
  float ms = 0.f;
  if (d->cuEventElapsedTime(&ms, c->ev0, c->ev1) == CUDA_SUCCESS)
    c->st.gpu_span_ns = static_cast<uint64_t>(ms * 1e6);
  if (c->cfg.instrument) {
    uint64_t busy = 0;
    c->node_ns.assign(c->node_ev.size() / 2, 0);
    for (size_t i = 0; i + 1 < c->node_ev.size(); i += 2) {
      float e = 0.f;
      if (d->cuEventElapsedTime(&e, c->node_ev[i], c->node_ev[i + 1]) == CUDA_SUCCESS) {
        c->node_ns[i / 2] = static_cast<uint64_t>(e * 1e6);
        busy += c->node_ns[i / 2];
      }
    }
    c->st.gpu_busy_ns = busy;
  }
  c->pending = false;
  return PASK_OK;
}

PASK_API int pask_infer_host(pask_ctx* c, const void* const* host_inputs, void* const* host_outputs,
                             void* stream) {
  t_err.clear();
  if (!c) return set_err(PASK_EINVAL, "null ctx");
  if (!c->have_model) return set_err(PASK_ESTATE, "pask_infer_host before pask_load_model");
  const Driver* d = c->d;
  CUstream s = static_cast<CUstream>(stream);
  for (size_t i = 0; host_inputs && i < c->inputs.size(); ++i) {
    const pask_tensor& t = c->tensors[c->inputs[i]];
    CUresult r = d->cuMemcpyHtoDAsync(reinterpret_cast<CUdeviceptr>(t.dptr), host_inputs[i], tensor_bytes(t), s);
    if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuMemcpyHtoDAsync"));
  }
  int rc = pask_infer(c, nullptr, nullptr, stream);
  if (rc) return rc;
  for (size_t i = 0; host_outputs && i < c->outputs.size(); ++i) {
    const pask_tensor& t = c->tensors[c->outputs[i]];
    CUresult r = d->cuMemcpyDtoHAsync(host_outputs[i], reinterpret_cast<CUdeviceptr>(t.dptr), tensor_bytes(t), s);
    if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuMemcpyDtoHAsync"));
  }
  CUresult r = d->cuStreamSynchronize(s);
  if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(d, r, "cuStreamSynchronize"));
  return pask_sync(c);
}

PASK_API int pask_stats(const pask_ctx* c, pask_stats_t* out) {
  t_err.clear();
  if (!c || !out) return set_err(PASK_EINVAL, "null ctx or out");
  *out = c->st;
  out->kernels_loaded = c->kernels_loaded.load();
  out->code_objects_loaded = c->code_objects.load();
  out->code_bytes_loaded = c->code_bytes.load();
  out->load_ns = c->load_ns.load();
  return PASK_OK;
}

PASK_API int pask_kernel_is_loaded(const pask_ctx* c, int32_t k, int32_t* state) {
  t_err.clear();
  if (!c || !state || k < 0 || k >= PASK_NUM_KERNELS) return set_err(PASK_EINVAL, "bad argument");
  *state = 0;
  if (c->ready[k].load(std::memory_order_acquire) != 1 || !c->fn[k]) return PASK_OK;
  CUfunctionLoadingState ls;
  CUresult r = c->d->cuFuncIsLoaded(&ls, c->fn[k]);
  if (r != CUDA_SUCCESS) return set_err(PASK_ECUDA, cu_err(c->d, r, "cuFuncIsLoaded"));
  *state = (ls == CU_FUNCTION_LOADING_STATE_LOADED) ? 1 : 0;
  return PASK_OK;
}

PASK_API int pask_kernel_timeline(const pask_ctx* c, int32_t k, uint64_t* load_ns, uint64_t* ready_ns,
                                  uint64_t* lib_ns) {
  t_err.clear();
  if (!c || k < 0 || k >= PASK_NUM_KERNELS) return set_err(PASK_EINVAL, "bad argument");
  const bool done = c->ready[k].load(std::memory_order_acquire) == 1;
  if (load_ns) *load_ns = done ? c->k_load_ns[k] : 0;
  if (ready_ns) *ready_ns = (done && c->k_ready_at[k] > c->t_entry) ? c->k_ready_at[k] - c->t_entry : 0;
  if (lib_ns) *lib_ns = done ? c->k_lib_ns[k] : 0;
  return PASK_OK;
}

PASK_API int pask_node_times(const pask_ctx* c, uint64_t* ns_out, int32_t n) {
  t_err.clear();
  if (!c || !ns_out) return set_err(PASK_EINVAL, "null argument");
  if (!c->cfg.instrument) return set_err(PASK_ESTATE, "context not created with instrument = 1");
  if (n != static_cast<int32_t>(c->node_ns.size())) return set_err(PASK_EINVAL, "n_nodes mismatch (sync first)");
  for (int32_t i = 0; i < n; ++i) ns_out[i] = c->node_ns[i];
  return PASK_OK;
}

PASK_API int pask_destroy(pask_ctx* c) {
  t_err.clear();
  if (!c) return PASK_OK;
  {
    std::lock_guard<std::mutex> lk(c->mu);
    c->stop = true;
    c->cv.notify_one();
  }
  if (c->loader.joinable()) c->loader.join();
  const Driver* d = c->d;
  if (c->pending) d->cuEventSynchronize(c->ev1);
  for (auto e : c->node_ev)
    if (e) d->cuEventDestroy(e);
  if (c->ev0) d->cuEventDestroy(c->ev0);
  if (c->ev1) d->cuEventDestroy(c->ev1);
  drop_graph(c);
  if (c->capture_stream) d->cuStreamDestroy(c->capture_stream);
  if (c->lib) d->cuLibraryUnload(c->lib);
  for (CUlibrary l : c->klib)
    if (l) d->cuLibraryUnload(l);
  delete c;
  return PASK_OK;
}
