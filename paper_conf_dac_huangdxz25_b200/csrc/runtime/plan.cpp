// Host planner: catalog, IsApplicable, static choice s*, Algorithm 1.
// The catalog table and predicates are DESIGN.md "Kernel catalog"; the
// algorithm follows PAPER.md:105-132 (Algorithm 1) and :135-141 (§III-C).
#include "plan.h"

#include <algorithm>
#include <cstdio>
#include <list>
#include <map>

namespace pask {

namespace {
// (op class, dtype, layout) per kernel id; dtype 0 = bf16 path, 1 = f32 input.
const CatalogEntry kCatalog[PASK_NUM_KERNELS] = {
    {PASK_K_LAYOUT, "pask_layout", OC_LAYOUT, 1, PASK_NCHW},
    {PASK_K_CONV_IGEMM, "pask_conv_igemm", OC_CONV, 0, PASK_NHWC},
    {PASK_K_CONV_1X1, "pask_conv_1x1", OC_CONV, 0, PASK_NHWC},
    {PASK_K_CONV_DW, "pask_conv_dw", OC_DWCONV, 0, PASK_NHWC},
    {PASK_K_POOL, "pask_pool", OC_POOL, 0, PASK_NHWC},
    {PASK_K_POOL_GAVG, "pask_pool_gavg", OC_POOL, 0, PASK_NHWC},
    {PASK_K_GEMM, "pask_gemm", OC_GEMM, 0, PASK_ROWMAJOR},
    {PASK_K_SOFTMAX, "pask_softmax", OC_SOFTMAX, 0, PASK_ROWMAJOR},
    {PASK_K_LAYERNORM, "pask_layernorm", OC_LAYERNORM, 0, PASK_ROWMAJOR},
};

std::string fmt(const char* f, long long a = 0, long long b = 0, long long c = 0) {
  char buf[256];
  snprintf(buf, sizeof buf, f, a, b, c);
  return buf;
}

int64_t numel(const pask_tensor& t) {
  return static_cast<int64_t>(t.n) * t.h * t.w * t.c;
}
}  // namespace

const CatalogEntry& catalog(int32_t id) { return kCatalog[id]; }

int64_t category_key(int32_t id) {
  const CatalogEntry& e = kCatalog[id];
  return (static_cast<int64_t>(e.op_class) << 16) | (e.dtype << 8) | e.layout;
}

pask_config default_config() {
  pask_config c{};
  c.reuse = 1;
  c.search = 0;
  c.milestone = 0;
  c.proactive = 2;
  c.pdl = 1;
  c.instrument = 0;
  c.packaging = 0;
  c.interleave = 0;
  c.graph = 0;
  return c;
}

// ------------------------------------------------------------------ IsApplicable
bool is_applicable(int32_t id, const Problem& p, std::string* why) {
  auto fail = [&](const char* m) {
    if (why) *why = m;
    return false;
  };
  switch (id) {
    case PASK_K_LAYOUT:
      if (p.op != OC_LAYOUT) return fail("not a layout op");
      if (static_cast<int64_t>(p.n) * p.h * p.w * std::max(p.c, p.k) >= (1ll << 31)) return fail("tensor too large for 32-bit indexing");
      if (p.k % 8 != 0) return fail("padded channels % 8 != 0");
      if (p.c > p.k) return fail("input channels exceed padded channels");
      return true;
    case PASK_K_CONV_IGEMM:
      if (p.op != OC_CONV || p.groups != 1) return fail("not a dense conv");
      if (p.c % 8 != 0 || p.k % 8 != 0) return fail("C % 8 or K % 8 != 0 (16-byte TMA/vector strides)");
      if (p.r < 1 || p.r > 16 || p.s < 1 || p.s > 16) return fail("filter size outside [1,16]");
      if (p.stride_h < 1 || p.stride_h > 8 || p.stride_w < 1 || p.stride_w > 8) return fail("stride outside [1,8]");
      if (p.pad_h < 0 || p.pad_h > 64 || p.pad_w < 0 || p.pad_w > 64) return fail("pad outside [0,64]");
      if (p.dil_h < 1 || p.dil_h > 8 || p.dil_w < 1 || p.dil_w > 8) return fail("dilation outside [1,8]");
      if (p.p < 1 || p.q < 1) return fail("empty output");
      return true;
    case PASK_K_CONV_1X1:
      if (p.op != OC_CONV || p.groups != 1) return fail("not a dense conv");
      if (p.r != 1 || p.s != 1) return fail("filter is not 1x1");
      if (p.stride_h != 1 || p.stride_w != 1) return fail("stride != 1");
      if (p.pad_h != 0 || p.pad_w != 0) return fail("pad != 0");
      if (p.c % 8 != 0 || p.k % 8 != 0) return fail("C % 8 or K % 8 != 0");
      return true;
    case PASK_K_CONV_DW:
      if (p.op != OC_DWCONV) return fail("not a depthwise conv");
      if (static_cast<int64_t>(p.n) * p.h * p.w * p.c >= (1ll << 31)) return fail("tensor too large for 32-bit indexing");
      if (p.c % 8 != 0) return fail("C % 8 != 0");
      if (p.r < 1 || p.r > 15 || p.s < 1 || p.s > 15) return fail("filter size outside [1,15]");
      if (p.stride_h < 1 || p.stride_h > 8 || p.stride_w < 1 || p.stride_w > 8) return fail("stride outside [1,8]");
      if (p.dil_h < 1 || p.dil_h > 8 || p.dil_w < 1 || p.dil_w > 8) return fail("dilation outside [1,8]");
      if (p.p < 1 || p.q < 1) return fail("empty output");
      return true;
    case PASK_K_POOL:
      if (p.op != OC_POOL) return fail("not a pool");
      if (static_cast<int64_t>(p.n) * p.h * p.w * p.c >= (1ll << 31)) return fail("tensor too large for 32-bit indexing");
      if (p.c % 8 != 0) return fail("C % 8 != 0");
      if (static_cast<int64_t>(p.r) * p.s > 1024) return fail("window larger than 1024 taps");
      if (p.stride_h < 1 || p.stride_w < 1) return fail("stride < 1");
      if (p.pad_h >= p.r || p.pad_w >= p.s) return fail("pad >= window");
      return true;
    case PASK_K_POOL_GAVG:
      if (p.op != OC_POOL) return fail("not a pool");
      if (p.global != 1 || p.pool_mode != 1) return fail("not a global average pool");
      if (p.c % 8 != 0) return fail("C % 8 != 0");
      return true;
    case PASK_K_GEMM:
      if (p.op != OC_GEMM) return fail("not a GEMM");
      if (p.gk % 8 != 0) return fail("K % 8 != 0 (16-byte TMA strides)");
      if (p.lda % 8 != 0 || p.ldb % 8 != 0) return fail("lda/ldb % 8 != 0");
      if (p.off_a % 8 != 0 || p.off_b % 8 != 0) return fail("operand offsets % 8 != 0");
      if (p.gm < 1 || p.gn < 1 || p.batch < 1) return fail("empty GEMM");
      return true;
    case PASK_K_SOFTMAX:
      if (p.op != OC_SOFTMAX) return fail("not a softmax");
      if (p.cols < 1 || p.cols > 16384) return fail("row length outside [1,16384]");
      return true;
    case PASK_K_LAYERNORM:
      if (p.op != OC_LAYERNORM) return fail("not a LayerNorm");
      if (p.cols % 8 != 0 || p.cols < 8 || p.cols > 8192) return fail("row length not a multiple of 8 in [8,8192]");
      return true;
    default:
      return fail("unknown kernel id");
  }
}

int32_t static_choice(const Problem& p) {
  switch (p.op) {
    case OC_LAYOUT: return PASK_K_LAYOUT;
    case OC_DWCONV: return PASK_K_CONV_DW;
    case OC_CONV:
      if (p.r == 1 && p.s == 1 && p.stride_h == 1 && p.stride_w == 1 && p.pad_h == 0 && p.pad_w == 0)
        return PASK_K_CONV_1X1;
      return PASK_K_CONV_IGEMM;
    case OC_POOL: return (p.global == 1 && p.pool_mode == 1) ? PASK_K_POOL_GAVG : PASK_K_POOL;
    case OC_GEMM: return PASK_K_GEMM;
    case OC_SOFTMAX: return PASK_K_SOFTMAX;
    case OC_LAYERNORM: return PASK_K_LAYERNORM;
  }
  return -1;
}

// ------------------------------------------------------------------ parse
int extract_problems(const pask_graph* g, std::vector<Problem>* out, std::string* err) {
  if (!g || g->n_nodes < 0 || g->n_tensors < 0 || (g->n_nodes > 0 && !g->nodes) ||
      (g->n_tensors > 0 && !g->tensors)) {
    *err = "null or malformed graph";
    return PASK_EINVAL;
  }
  out->clear();
  out->reserve(g->n_nodes);
  auto T = [&](int32_t i) -> const pask_tensor* {
    return (i >= 0 && i < g->n_tensors) ? &g->tensors[i] : nullptr;
  };
  for (int32_t i = 0; i < g->n_nodes; ++i) {
    const pask_node& nd = g->nodes[i];
    Problem p;
    const pask_tensor* x = T(nd.in0);
    const pask_tensor* y = T(nd.out);
    auto bad = [&](const std::string& m) {
      *err = fmt("node %lld: ", i) + m;
      return PASK_EINVAL;
    };
    if (!x || !y) return bad("in0/out tensor index out of range");
    if (nd.res >= 0 && !T(nd.res)) return bad("res tensor index out of range");
    switch (nd.op) {
      case PASK_OP_LAYOUT:
        if (x->dtype != PASK_F32 || x->layout != PASK_NCHW) return bad("layout input must be f32 NCHW");
        if (y->dtype != PASK_BF16 || y->layout != PASK_NHWC) return bad("layout output must be bf16 NHWC");
        if (y->n != x->n || y->h != x->h || y->w != x->w) return bad("layout output dims mismatch");
        p.op = OC_LAYOUT;
        p.n = x->n; p.h = x->h; p.w = x->w; p.c = x->c; p.k = y->c;
        break;
      case PASK_OP_CONV2D: {
        if (x->dtype != PASK_BF16 || x->layout != PASK_NHWC || y->dtype != PASK_BF16 || y->layout != PASK_NHWC)
          return bad("conv tensors must be bf16 NHWC");
        if (!nd.w) return bad("conv weights missing");
        if (nd.r < 1 || nd.s < 1 || nd.stride[0] < 1 || nd.stride[1] < 1 || nd.dil[0] < 1 || nd.dil[1] < 1 ||
            nd.pad[0] < 0 || nd.pad[1] < 0 || nd.groups < 1 || nd.k < 1)
          return bad("bad conv geometry");
        const int32_t P = (x->h + 2 * nd.pad[0] - nd.dil[0] * (nd.r - 1) - 1) / nd.stride[0] + 1;
        const int32_t Q = (x->w + 2 * nd.pad[1] - nd.dil[1] * (nd.s - 1) - 1) / nd.stride[1] + 1;
        if (y->n != x->n || y->h != P || y->w != Q || y->c != nd.k) return bad("conv output dims mismatch");
        if (x->c % nd.groups != 0 || nd.k % nd.groups != 0) return bad("groups must divide C and K");
        if (nd.res >= 0) {
          const pask_tensor* r = T(nd.res);
          if (r->n != y->n || r->h != y->h || r->w != y->w || r->c != y->c || r->dtype != PASK_BF16)
            return bad("residual dims mismatch");
        }
        p.n = x->n; p.h = x->h; p.w = x->w; p.c = x->c; p.k = nd.k; p.r = nd.r; p.s = nd.s;
        p.stride_h = nd.stride[0]; p.stride_w = nd.stride[1]; p.pad_h = nd.pad[0]; p.pad_w = nd.pad[1];
        p.dil_h = nd.dil[0]; p.dil_w = nd.dil[1]; p.groups = nd.groups; p.p = P; p.q = Q;
        p.op = (nd.groups > 1 && nd.groups == x->c && nd.k == x->c) ? OC_DWCONV : OC_CONV;
        break;
      }
      case PASK_OP_POOL: {
        if (x->dtype != PASK_BF16 || x->layout != PASK_NHWC || y->dtype != PASK_BF16 || y->layout != PASK_NHWC)
          return bad("pool tensors must be bf16 NHWC");
        if (y->c != x->c || y->n != x->n) return bad("pool channel/batch mismatch");
        p.op = OC_POOL;
        p.n = x->n; p.h = x->h; p.w = x->w; p.c = x->c; p.k = x->c;
        p.pool_mode = nd.pool_mode; p.global = nd.global_pool ? 1 : 0;
        if (nd.pool_mode != 0 && nd.pool_mode != 1) return bad("pool_mode must be 0 (max) or 1 (avg)");
        if (p.global) {
          p.r = x->h; p.s = x->w; p.stride_h = p.stride_w = 1; p.pad_h = p.pad_w = 0; p.p = p.q = 1;
          if (y->h != 1 || y->w != 1) return bad("global pool output must be 1x1");
        } else {
          if (nd.r < 1 || nd.s < 1 || nd.stride[0] < 1 || nd.stride[1] < 1 || nd.pad[0] < 0 || nd.pad[1] < 0)
            return bad("bad pool geometry");
          p.r = nd.r; p.s = nd.s; p.stride_h = nd.stride[0]; p.stride_w = nd.stride[1];
          p.pad_h = nd.pad[0]; p.pad_w = nd.pad[1];
          p.p = (x->h + 2 * nd.pad[0] - nd.r) / nd.stride[0] + 1;
          p.q = (x->w + 2 * nd.pad[1] - nd.s) / nd.stride[1] + 1;
          if (y->h != p.p || y->w != p.q) return bad("pool output dims mismatch");
        }
        break;
      }
      case PASK_OP_GEMM: {
        if (x->dtype != PASK_BF16 || y->dtype != PASK_BF16) return bad("GEMM tensors must be bf16");
        if (nd.m < 1 || nd.n < 1 || nd.kk < 1 || nd.batch < 1) return bad("empty GEMM");
        if (nd.trans_b != 0 && nd.trans_b != 1) return bad("trans_b must be 0 or 1");
        if (!nd.w && !T(nd.in1)) return bad("GEMM B operand missing (w and in1)");
        if (nd.lda < nd.kk || nd.ldc < nd.n || nd.ldb < (nd.trans_b ? nd.kk : nd.n)) return bad("leading dimension too small");
        if (nd.off_a < 0 || nd.off_b < 0 || nd.off_c < 0 || nd.stride_a < 0 || nd.stride_b < 0 || nd.stride_c < 0)
          return bad("negative offset/stride");
        const int64_t need_a = nd.off_a + (nd.batch - 1) * nd.stride_a + (int64_t)(nd.m - 1) * nd.lda + nd.kk;
        const int64_t need_c = nd.off_c + (nd.batch - 1) * nd.stride_c + (int64_t)(nd.m - 1) * nd.ldc + nd.n;
        if (need_a > numel(*x)) return bad("A extent exceeds tensor in0");
        if (need_c > numel(*y)) return bad("C extent exceeds tensor out");
        if (nd.res >= 0 && need_c > numel(*T(nd.res))) return bad("residual extent exceeds tensor res");
        if (!nd.w) {
          const int64_t need_b = nd.off_b + (nd.batch - 1) * nd.stride_b +
                                 (int64_t)((nd.trans_b ? nd.n : nd.kk) - 1) * nd.ldb + (nd.trans_b ? nd.kk : nd.n);
          if (need_b > numel(*T(nd.in1))) return bad("B extent exceeds tensor in1");
        }
        p.op = OC_GEMM;
        p.gm = nd.m; p.gn = nd.n; p.gk = nd.kk; p.batch = nd.batch;
        p.lda = nd.lda; p.ldb = nd.ldb; p.off_a = nd.off_a; p.off_b = nd.off_b;
        break;
      }
      case PASK_OP_SOFTMAX:
      case PASK_OP_LAYERNORM:
        if (x->dtype != PASK_BF16 || y->dtype != PASK_BF16) return bad("row-op tensors must be bf16");
        if (numel(*x) != numel(*y) || x->c != y->c) return bad("row-op output dims mismatch");
        if (nd.op == PASK_OP_LAYERNORM && (!nd.gamma || !nd.beta)) return bad("LayerNorm gamma/beta missing");
        p.op = nd.op == PASK_OP_SOFTMAX ? OC_SOFTMAX : OC_LAYERNORM;
        p.rows = static_cast<int32_t>(static_cast<int64_t>(x->n) * x->h * x->w);
        p.cols = x->c;
        break;
      default:
        return bad("unknown op");
    }
    out->push_back(p);
  }
  return PASK_OK;
}

// ------------------------------------------------------------------ Algorithm 1
int execution_plan(const std::vector<Problem>& probs, const std::vector<int32_t>& desired,
                   const pask_config& cfg, PlanResult* out, std::string* err) {
  out->bindings.clear();
  out->loaded.clear();
  out->queries = out->hits = out->lookups = 0;
  bool loaded[PASK_NUM_KERNELS] = {};
  std::map<int64_t, std::list<int32_t>> mru;  // category -> kernels, head = most recent

  auto touch = [&](int32_t k) {  // insert / move to head
    auto& l = mru[category_key(k)];
    l.remove(k);
    l.push_front(k);
  };
  auto load = [&](int32_t k) {  // "wait for s*_i loading; add s*_i to S_m" (Alg. 1 l.10-11)
    loaded[k] = true;
    out->loaded.push_back(k);
    touch(k);
  };

  const int32_t n = static_cast<int32_t>(probs.size());
  for (int32_t i = 0; i < n; ++i) {
    const Problem& p = probs[i];
    const int32_t want = desired[i];
    std::string why;
    if (want < 0 || want >= PASK_NUM_KERNELS || !is_applicable(want, p, &why)) {
      *err = fmt("node %lld: desired solution ", i) +
             (want >= 0 && want < PASK_NUM_KERNELS ? kCatalog[want].name : "?") + " not applicable: " + why;
      return PASK_EUNSUPPORTED;
    }
    pask_binding b{i, want, want, PASK_HOW_DIRECT, 0};
    const int32_t layer_no = i + 1;
    if (layer_no <= cfg.milestone || !cfg.reuse) {  // before the milestone: load s* unconditionally
      if (loaded[want]) {
        touch(want);
      } else {
        load(want);
        b.how = PASK_HOW_LOADED;
      }
      out->bindings.push_back(b);
      continue;
    }
    if (loaded[want]) {  // Alg. 1 l.3-4
      touch(want);
      out->bindings.push_back(b);
      continue;
    }
    // Alg. 1 l.6: GETSUBSOLUTION(S, s*, p) -- l.12-18
    out->queries++;
    std::vector<int32_t> cand;
    if (cfg.search == 0) {
      auto it = mru.find(category_key(want));
      if (it != mru.end()) cand.assign(it->second.begin(), it->second.end());  // MRU -> LRU
    } else {
      cand = out->loaded;  // naive (PaSK-R): every loaded solution, load order
    }
    int32_t found = -1, nl = 0;
    for (int32_t k : cand) {
      ++nl;
      if (is_applicable(k, p)) {
        found = k;
        break;
      }
    }
    out->lookups += nl;
    b.lookups = nl;
    if (found >= 0) {  // l.7-8 reuse, l.16 lru.update
      out->hits++;
      touch(found);
      b.bound_kernel = found;
      b.how = PASK_HOW_REUSED;
    } else {  // l.9-11
      load(want);
      b.how = PASK_HOW_LOADED;
    }
    out->bindings.push_back(b);
  }
  return PASK_OK;
}

// ------------------------------------------------------------------ tiling
bool contraction_shape(const Problem& p, const pask_node& nd, int32_t* M, int32_t* N, int32_t* K,
                       int32_t* batch, int32_t* b_major) {
  if (p.op == OC_CONV) {
    *M = p.n * p.p * p.q;
    *N = p.k;
    *K = p.r * p.s * p.c;
    *batch = 1;
    *b_major = 0;
    return true;
  }
  if (p.op == OC_GEMM) {
    *M = p.gm;
    *N = p.gn;
    *K = p.gk;
    *batch = p.batch;
    *b_major = nd.trans_b ? 0 : 1;
    return true;
  }
  return false;
}

GemmTiling gemm_tiling(int32_t M, int32_t N, int32_t K, int32_t batch, int32_t b_major, int32_t c_tma) {
  GemmTiling t{};
  t.M = M; t.N = N; t.K = K; t.batch = batch;
  constexpr int kSMs = 148;
  // N tile: 16/32/48 for narrow outputs, else multiples of 64 (whole 128 B
  // TMA boxes for the staged epilogue); MN-major B needs whole 64-wide boxes.
  if (b_major) {
    t.bn = std::min(256, (N + 63) / 64 * 64);
  } else if (N <= 48) {
    t.bn = (N + 15) / 16 * 16;
  } else {
    t.bn = std::min(128, (N + 63) / 64 * 64);
  }
  t.m_tiles = (M + 127) / 128;
  t.n_tiles = (N + t.bn - 1) / t.bn;
  // more CTAs for small-M layers: halve a 128-wide N tile while far below one wave
  if (!b_major && t.bn == 128 && static_cast<int64_t>(t.m_tiles) * t.n_tiles * batch < kSMs / 2) {
    t.bn = 64;
    t.n_tiles = (N + 63) / 64;
  }
  t.num_kb = (K + 63) / 64;
  // split-K as a cluster of 2 / 4 / 8 CTAs (DSMEM reduction) when the grid is
  // well below one wave and each split keeps >= 4 k-blocks: a k-block streams
  // in ~0.3 us per SM while the cluster reduction costs ~1.5 us (measured), so
  // shorter splits lose
  const int64_t tiles = static_cast<int64_t>(t.m_tiles) * t.n_tiles * batch;
  int32_t splits = 1;
  while (splits < 8 && tiles * splits * 2 <= kSMs && t.num_kb >= 8 * splits && t.bn <= 128) splits *= 2;
  t.splits = splits;
  t.rows_per = 128 / splits;
  const int32_t kb_per = (t.num_kb + splits - 1) / splits;
  const uint32_t stage_bytes = 16384u + static_cast<uint32_t>(t.bn) * 128u;
  const uint32_t recv = splits > 1 ? ((128u * (t.bn + 4) * 4 + 1023u) & ~1023u) : 0u;
  const uint32_t ro = c_tma ? ((128u * t.bn * 2 + 1023u) & ~1023u) : 0u;
  const uint32_t fixed = recv + ro + 1024u /*bias*/ + 256u /*barriers*/ + 1024u /*align slack*/;
  const uint32_t budget = kMaxDynSmem - fixed;  // ring gets what is left, at most 8 stages
  int32_t stages = static_cast<int32_t>(budget / stage_bytes);
  stages = std::min(stages, 8);
  stages = std::min(stages, std::max(2, kb_per));
  t.stages = std::max(2, stages);
  const uint32_t ring = (t.stages * stage_bytes + 1023u) & ~1023u;
  t.smem_bytes = ring + fixed;
  uint32_t cols = 32;
  while (cols < static_cast<uint32_t>(t.bn)) cols <<= 1;
  t.tmem_cols = cols;
  return t;
}

}  // namespace pask
