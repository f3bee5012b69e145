// Host-only planning: problem extraction (parse step P_i), the
// kernel catalog with IsApplicable predicates, the static choice
// s*_i and Algorithm 1 over the categorical MRU cache
// (PAPER.md:105-141).  Pure integer code; no CUDA.
#pragma once
#include <stdint.h>

#include <string>
#include <vector>

#include "../../../include/pask.h"

namespace pask {

enum OpClass : int32_t { OC_LAYOUT = 0, OC_CONV, OC_DWCONV, OC_POOL, OC_GEMM, OC_SOFTMAX, OC_LAYERNORM, OC_ATTENTION };

struct Problem {
  int32_t op = 0;
  int32_t n = 0, h = 0, w = 0, c = 0, k = 0, r = 0, s = 0;
  int32_t stride_h = 0, stride_w = 0, pad_h = 0, pad_w = 0, dil_h = 0, dil_w = 0;
  int32_t groups = 0, p = 0, q = 0, pool_mode = 0, global = 0;
  int32_t gm = 0, gn = 0, gk = 0, batch = 0;
  int64_t lda = 0, ldb = 0, off_a = 0, off_b = 0;
  int32_t trans_b = 0, b_weights = 0;  // GEMM: B stored [n][k]; B is the weight operand (w)
  int32_t rows = 0, cols = 0;
};

struct CatalogEntry {
  int32_t id;
  const char* name;    // extern "C" kernel symbol in the embedded cubin
  int32_t op_class;    // category key = (op class, dtype, layout)
  int32_t dtype;
  int32_t layout;
};

int32_t num_kernels();                 // generic + specialised
const CatalogEntry& catalog(int32_t id);
int64_t category_key(int32_t kernel_id);
bool is_spec_kernel(int32_t kernel_id);  // a per-problem specialised conv solution

bool is_applicable(int32_t kernel_id, const Problem& p, std::string* why = nullptr);
int32_t static_choice(const Problem& p, int32_t catalog_mode = 0);

// Validate the graph and extract problems.  Returns PASK_OK or an error with *err set.
int extract_problems(const pask_graph* g, std::vector<Problem>* out, std::string* err);

struct PlanResult {
  std::vector<pask_binding> bindings;
  std::vector<int32_t> loaded;  // kernel ids in load (= first-use) order
  int32_t queries = 0, hits = 0, lookups = 0;
};

// Algorithm 1 (EXECUTIONPLAN / GETSUBSOLUTION).  desired[i] = s*_i.
int execution_plan(const std::vector<Problem>& probs, const std::vector<int32_t>& desired,
                   const pask_config& cfg, PlanResult* out, std::string* err);

// Tiling of the contraction kernel for a GEMM-view problem (pure function of
// the problem, so reuse stays bitwise reproducible).
struct GemmTiling {
  int32_t M, N, K, batch;
  int32_t bn, m_tiles, n_tiles, num_kb, splits, rows_per, stages;
  uint32_t smem_bytes, tmem_cols;
  int32_t persistent;  // 1: grid of min(tiles, #SMs) CTAs looping over tiles (splits == 1)
  int32_t grid_x;      // persistent grid size
  int32_t b_res;       // persistent with one N tile: the whole B resident in smem (D18)
};
// Dynamic shared memory the contraction kernels may request (attribute set at load).
constexpr uint32_t kMaxDynSmem = 220u * 1024u;
// c_tma: output / residual go through smem staging + TMA (changes the smem size)
// max_cluster: largest split-K cluster the device co-schedules (16 on a full B200)
GemmTiling gemm_tiling(int32_t M, int32_t N, int32_t K, int32_t batch, int32_t b_major, int32_t c_tma,
                       int32_t persistent_kernel = 0, int32_t max_cluster = 16);
// s* rule: a GEMM of at most kGemvMaxRows rows with a [N][K] weight operand takes
// the GEMV solution (PASK_K_GEMV, D12)
constexpr int32_t kGemvMaxRows = 8;
// s* rule: a dense conv with more output rows than 148 SMs x 128-row tiles takes
// the persistent-tile solution (PASK_K_CONV_IGEMM_PT)
constexpr int64_t kPersistentRows = 148 * 128;

// Contraction view of a conv / GEMM problem (M, N, K, batch, b_major).
bool contraction_shape(const Problem& p, const pask_node& node, int32_t* M, int32_t* N, int32_t* K,
                       int32_t* batch, int32_t* b_major);

pask_config default_config();

}  // namespace pask
