// Tiling and issue constants of the runtime, and the experiment switches used
// to measure the alternatives DESIGN.md reports.
//
// The PASK_* environment variables are read ONCE -- the first tuning() call,
// from pask_create / pask_plan on the caller's thread, never from the helper
// thread -- and every value is clamped to the range the kernels support (e.g.
// splits <= min(16, num_kb) holds in gemm_tiling whatever PASK_SPLIT_MAX says).
// The device phase trace (PASK_TRACE_PTR: a device address the kernels write
// to) is honoured only in builds with -DPASK_EXPERIMENTS
// (PASK_NVCC_DEFINES="-DPASK_EXPERIMENTS" python -m paper_conf_dac_huangdxz25_b200.build).
#pragma once
#include <stdint.h>

namespace pask {

struct Tuning {
  // gemm_tiling (plan.cpp)
  int tile_target = 74;   // halve the N tile while the grid has fewer tiles than this
  int bn_min = 64;        // ... but not below this N tile
  int split_min_kb = 8;   // k-blocks each split-K slice keeps at least
  int split_max = 8;      // largest portable split-K cluster
  int split_fill = 2;     // tiles * splits * fill <= #SMs
  int bn32_tiles = 8;     // unsplittable layers with <= this many tiles take 32-wide N tiles
  int fine_ctas = 32;     // grids below this many CTAs with K <= fine_max_k retile finer (0: off)
  int fine_max_k = 1024;
  int fine_max_mtiles = 8;
  int smem_budget_kb = 220;  // dynamic smem a contraction CTA may use (ring = what is left)
  // lowering (pask.cpp)
  int gather_lag = 2;     // A_GATHER: k-blocks of cp.async in flight before publishing a slot
  int pre_b = 0;          // weight k-blocks fetched before griddepcontrol.wait (0 = whole ring)
  bool staged_store = false;  // stage every epilogue tile for a TMA store (c_tma = 1)
  bool no_a64 = false;        // never use 64-row A boxes
  bool no_im2col = false;     // A_GATHER instead of TMA im2col
  int stem_fold = 1;          // D16: 0 off; 1 fold a stem conv that then needs fewer k-blocks; 2 ... no more
  bool no_b_res = false;      // D18 off: persistent one-N-tile layers stream B per k-block
  // issue / loading (pask.cpp)
  bool encode_first = false;       // proactive 2: encode, then upload (instead of concurrently)
  bool debug_cold = false;         // print per-launch host times of the cold inference
  bool fork_no_pdl = false;        // branches: drop PDL after a fork record
  bool join_no_pdl = false;        // branches: drop PDL after a join wait
  bool direct_one_stream = false;  // branches: direct issue on one stream
  bool no_event_warm = false;      // pask_create: do not pre-record the timing events
  bool parallel_upload = false;    // packaging 2: helper uploads the contraction family concurrently
  bool keep_primer = false;        // keep the driver primer's code object loaded until destroy
  // device phase trace (experiment builds only)
  int trace_node = -2;             // node index, -1 = all, -2 = off
  uint64_t trace_ptr = 0;          // device address of the trace buffer
  bool trace_clock = false;        // SM clock64 cycles instead of %globaltimer
};

const Tuning& tuning();

}  // namespace pask
