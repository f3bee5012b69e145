/*
 * pask.h -- C ABI of libpask.so, the B200-native hot path of PASK
 * ("PASK: Cold Start Mitigation for Inference with Proactive and Selective
 * Kernel Loading on GPUs", Huang, Du, Xiao, Zhang, DAC'25).  Citations are
 * lines of /root/reference/PAPER.md ("PAPER.md:N") with their section.
 *
 * Problem statement (§III, Fig. 5): PASK "receives the lowered
 * model (a sequence of n solutions) as input, and then proactively parses,
 * loads, issues the DNN layer ... Upon absent solution, PASK seeks the
 * opportunities to reuse the loaded solutions and organizes them based on
 * their patterns".  Here the lowered model is a pask_graph, a "solution" is
 * one kernel of the catalog below (PASK_K_*), and the library:
 *   - plans (pask_plan / pask_load_model): Algorithm 1 EXECUTIONPLAN with the
 *     categorical MRU cache (§III-B/C);
 *   - loads proactively on a loader thread (PAPER.md:95, §III-A; :164 §III-D):
 *     cuLibraryLoadData once, then cuLibraryGetKernel -> cuKernelGetFunction ->
 *     cuFuncLoad per bound kernel, in first-use order;
 *   - issues (pask_infer) on the caller's thread, each launch waiting only for
 *     its own kernel's ready flag ("starts the kernels at the earliest feasible
 *     time right after the loading").
 *
 * Conventions for every entry point:
 *   - Returns PASK_OK (0) or a negative pask_status.  No C++ exception crosses
 *     the ABI.  On error, pask_last_error() returns a thread-local message that
 *     names the failing node / predicate / CUresult.
 *   - There is no CPU fallback: a node with no applicable kernel fails with
 *     PASK_EUNSUPPORTED; a driver failure returns PASK_ECUDA.
 *   - Device memory (weights, every tensor, the workspace) is owned by the
 *     caller and must stay alive until pask_destroy.  The library owns its host
 *     structures, the CUlibrary/CUfunction handles, encoded CUtensorMaps and
 *     the loader thread.
 *   - A pask_ctx is not thread-safe: use one ctx per thread.
 *   - The CUDA driver is loaded at run time (dlopen "libcuda.so.1"); the
 *     host-only entry points (pask_plan, pask_workspace_bytes, pask_kernel_*)
 *     work without a GPU.
 */
#ifndef PASK_H
#define PASK_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PASK_VERSION 100

typedef struct pask_ctx pask_ctx; /* opaque, library-owned */

typedef enum {
  PASK_OK = 0,
  PASK_EINVAL = -1,      /* malformed graph / argument                                  */
  PASK_EUNSUPPORTED = -2, /* a node's chosen solution s* is not applicable (no fallback)  */
  PASK_ECUDA = -3,       /* driver call failed; message carries the CUresult name        */
  PASK_ENOMEM = -4,      /* host allocation / workspace too small                        */
  PASK_ESTATE = -5       /* call order violated (e.g. infer before load_model)           */
} pask_status;

typedef enum { PASK_BF16 = 0, PASK_F32 = 1 } pask_dtype;

/* Memory order of a 4-D tensor with logical dims (n, h, w, c):
 *   PASK_NCHW     : n, c, h, w (only the fp32 model input)
 *   PASK_NHWC     : n, h, w, c (activations; c contiguous)
 *   PASK_ROWMAJOR : a matrix of rows = n*h*w and cols = c (same bytes as NHWC) */
typedef enum { PASK_NCHW = 0, PASK_NHWC = 1, PASK_ROWMAJOR = 2 } pask_layout;

/* Operator classes of the lowered model ("PASK implements the
 * reuse logic for the common convolution, pooling and activation primitives";
 * PAPER.md:238 §VI extends it to GEMM). */
typedef enum {
  PASK_OP_LAYOUT = 0,   /* NCHW fp32 -> NHWC bf16, C zero-padded (PAPER.md:73 fn. 2)  */
  PASK_OP_CONV2D = 1,   /* dense (groups = 1) or depthwise (groups = C = K)           */
  PASK_OP_GEMM = 2,     /* batched C = act(A op(B) + bias + res)                      */
  PASK_OP_POOL = 3,     /* max / avg, windowed or global                              */
  PASK_OP_SOFTMAX = 4,  /* row softmax of scale * x                                   */
  PASK_OP_LAYERNORM = 5, /* row LayerNorm, biased variance                            */
  PASK_OP_ATTENTION = 6  /* fused multi-head scaled dot-product attention (QK^T ->
                            softmax -> PV in one kernel)      */
} pask_op;

/* Activations are fused epilogues of conv / GEMM (the activation primitive of
 * PAPER.md:166; no standalone kernel). */
typedef enum {
  PASK_ACT_NONE = 0,
  PASK_ACT_RELU = 1,
  PASK_ACT_RELU6 = 2,
  PASK_ACT_GELU_ERF = 3, /* 0.5 x (1 + erf(x / sqrt 2)) */
  PASK_ACT_TANH = 4
} pask_act;

/* The kernel catalog ("solutions", PAPER.md:69, :73 fn. 2, :83 §II-B).  All of
 * them live in ONE SASS-only code object embedded in libpask.so. */
typedef enum {
  PASK_K_LAYOUT = 0,     /* category (LAYOUT, f32, NCHW)                                */
  PASK_K_CONV_IGEMM = 1, /* generic implicit-GEMM conv, tcgen05/TMEM; cat (CONV, bf16, NHWC) */
  PASK_K_CONV_1X1 = 2,   /* specialised 1x1 s1 p0 conv (TMA-only A); cat (CONV, bf16, NHWC) */
  PASK_K_CONV_DW = 3,    /* depthwise direct conv; cat (DWCONV, bf16, NHWC)             */
  PASK_K_POOL = 4,       /* windowed max/avg pool; cat (POOL, bf16, NHWC)               */
  PASK_K_POOL_GAVG = 5,  /* specialised global average pool; cat (POOL, bf16, NHWC)     */
  PASK_K_GEMM = 6,       /* batched GEMM, tcgen05/TMEM; cat (GEMM, bf16, ROWMAJOR)      */
  PASK_K_SOFTMAX = 7,    /* cat (SOFTMAX, bf16, ROWMAJOR)                               */
  PASK_K_LAYERNORM = 8,  /* cat (LAYERNORM, bf16, ROWMAJOR)                             */
  PASK_K_ATTENTION = 9,  /* fused attention, tcgen05/TMEM; cat (ATTENTION, bf16, ROWMAJOR) */
  PASK_K_CONV_IGEMM_PT = 10, /* implicit-GEMM conv as persistent tiles (large M); cat (CONV, bf16, NHWC) */
  PASK_K_GEMV = 11,      /* weight-streaming GEMV for GEMMs of <= 8 rows with a weight operand
                            [N][K] (FC layers at batch <= 8, BERT's pooler); cat (GEMM, bf16,
                            ROWMAJOR); D12                                       */
  PASK_NUM_KERNELS = 12  /* size of the generic catalog; ids >= 12 are the per-problem
                            specialised conv solutions of the tuned catalog (one per
                            (R, S, stride, pad, dilation, C) of configs C1-C3, category
                            (CONV, bf16, NHWC), applicable to exactly that problem
                            shape); pask_num_kernels() returns the total            */
} pask_kernel_id;

#define PASK_MAX_KERNELS 64

/* A tensor: logical dims (n, h, w, c), element type, memory order, and a
 * caller-owned device pointer (16-byte aligned). */
typedef struct {
  int32_t dtype;  /* pask_dtype  */
  int32_t layout; /* pask_layout */
  int32_t n, h, w, c;
  void *dptr;
} pask_tensor;

/* One lowered layer.  Fields not used by an op are ignored.
 *
 * LAYOUT   : in0 (NCHW f32, c <= out.c) -> out (NHWC bf16); channels c..out.c-1 = 0.
 * CONV2D   : out[n,p,q,k] = act(bias[k] + res[n,p,q,k] +
 *              sum_{c,r,s} in0[n, p*stride0 - pad0 + r*dil0, q*stride1 - pad1 + s*dil1, c]
 *                          * w[k, r, s, c])                     (PAPER.md:83 patterns)
 *            in0/out/res NHWC bf16; w KRSC bf16 (dense) or RSC bf16 (depthwise,
 *            groups = C = K); bias fp32 [K] or NULL; res tensor index or -1.
 * GEMM     : for b < batch, i < m, j < n:
 *              C_b[i,j] = act( sum_{t<kk} A_b[i,t] * B_b[t,j] + bias[j] + R_b[i,j] )
 *            A_b[i,t] = A[off_a + b*stride_a + i*lda + t]          (A = tensor in0)
 *            B_b[t,j] = B[off_b + b*stride_b + j*ldb + t]  if trans_b (B stored [n][kk])
 *                     = B[off_b + b*stride_b + t*ldb + j]  otherwise (B stored [kk][n])
 *            B = w when w != NULL (weights), else tensor in1 (activation x activation)
 *            C_b[i,j] = out[off_c + b*stride_c + i*ldc + j]; R uses res with the same
 *            indexing.  All operands bf16; bias fp32 [n] or NULL.
 * POOL     : pool_mode 0 = max (padding = -inf), 1 = avg (count_include_pad);
 *            window (r, s), stride, pad; global_pool = 1 means window = (h, w).
 * SOFTMAX  : rows = n*h*w of in0, cols = c: y = softmax(scale * x) per row.
 * LAYERNORM: rows of in0: y = (x - mean) / sqrt(var + eps) * gamma + beta, var biased.
 * ATTENTION: in0 = packed QKV rows [batch * m][3 * n * kk] (Q | K | V, head h at
 *            columns h*kk of each third), out = [batch * m][n * kk]; m = sequence
 *            length, n = heads, kk = head dim, scale = softmax scale.  For b, head h,
 *            query i:  out[b*m + i][h*kk + d] =
 *              sum_j softmax_j(scale * sum_e Q[b*m+i][h*kk+e] K[b*m+j][h*kk+e]) V[b*m+j][h*kk+d]
 *            (no mask), the composition of the qk -> softmax -> pv layers.
 *
 * solution: the statically chosen kernel s*_i carried by the lowered model
 * (".mgx ... the determined optimal solutions for each layer"),
 * or -1 to let the library apply its own static choice. */
typedef struct {
  int32_t op;       /* pask_op */
  int32_t in0, in1, res, out; /* tensor indices; -1 = none */
  const void *w;    /* device weights (see op)                  */
  const float *bias, *gamma, *beta; /* device fp32 vectors or NULL */
  int32_t k, r, s;
  int32_t stride[2], pad[2], dil[2];
  int32_t groups;
  int32_t m, n, kk, batch, trans_b;
  int64_t lda, ldb, ldc;
  int64_t off_a, off_b, off_c;
  int64_t stride_a, stride_b, stride_c;
  int32_t pool_mode, count_include_pad, global_pool;
  float eps, scale;
  int32_t act;      /* pask_act */
  int32_t solution; /* pask_kernel_id or -1 */
} pask_node;

typedef struct {
  int32_t n_tensors;
  const pask_tensor *tensors;
  int32_t n_nodes;
  const pask_node *nodes;
  int32_t n_inputs;
  const int32_t *inputs;  /* tensor indices fed by pask_infer(inputs)  */
  int32_t n_outputs;
  const int32_t *outputs; /* tensor indices read by pask_infer(outputs) */
  void *workspace;        /* caller-owned device scratch, zero-filled before
                             pask_load_model; >= pask_workspace_bytes()      */
  uint64_t workspace_bytes;
} pask_graph;

typedef struct {
  int32_t reuse;      /* 1 = Algorithm 1 reuse (PaSK); 0 = always load s* (PaSK-I / Baseline) */
  int32_t search;     /* 0 = categorical MRU lists; 1 = naive scan (PaSK-R, :186) */
  int32_t milestone;  /* m of PAPER.md:97; layers 1..m load s* unconditionally (default 0)    */
  int32_t proactive;  /* 1 = loader thread started at parse time;
                         2 = the caller thread uploads every planned kernel inside
                             pask_load_model, right after planning (a hot core; fastest
                             measured on B200, D5);
                         0 = reactive: each kernel loaded at its first launch (A1 baseline) */
  int32_t pdl;        /* 1 = programmatic dependent launch between consecutive kernels        */
  int32_t instrument; /* 1 = per-node CUDA events for gpu_busy_ns (perturbs timing)           */
  int32_t packaging;  /* 0 = one code object per catalog kernel (default: a load costs ~0.9 us
                         per KB of image, so only the bound kernels' code is parsed);
                         1 = the whole catalog as one code object;
                         2 = operator families (D8): the memory-bound solutions
                             (layout, dw, pool, gavg, softmax, LayerNorm) share one
                             CUfunction `pask_mem`, and conv_1x1 / gemm run on the generic
                             implicit-GEMM function -- one upload makes a whole family
                             resident; the plan (Algorithm 1) is unchanged, kernels_loaded
                             counts the uploaded functions; the families object is loaded
                             in the smallest variant whose memory cases cover every
                             solution the plan binds and whose contraction entry compiles
                             every path the plan's contraction nodes take (D13);
                         3 = one CUfunction `pask_all` for both families (D10:
                             one upload for the cold start, in the same per-model variants;
                             slower on the hot path until pask_promote repacks the model
                             into the two family entries, D15) */
  int32_t interleave; /* 0 = load-first (default): the first inference launches once every
                         planned kernel is uploaded -- on this driver a code upload waits for
                         all running GPU work, so
                         uploads are done while the GPU is idle anyway;
                         1 = Fig. 5 interleaving: launch each layer as soon as its kernel is
                         ready (the loader yields to the issuer)                             */
  int32_t graph;      /* 1 = hot inferences replay a CUDA graph captured on the second call
                         (PDL edges kept); the cold first inference always issues directly   */
  int32_t catalog;    /* 0 = generic catalog; 1 = tuned catalog: s* of a dense conv is its
                         per-problem specialised solution when one exists (the library
                         behaviour PASK starts from; the Baseline scheme)       */
  int32_t branches;   /* 1 = a node that does not read its predecessor's output (ResNet's
                         downsample conv) runs on a second stream, forked after its last
                         producer and joined before its first consumer, so it overlaps the
                         main chain (D9); 0 = one stream, node order.  Ignored
                         with instrument = 1.  Same kernels and parameters either way:
                         outputs are bitwise identical                                       */
  int32_t timeline;   /* 1 = every kernel stamps its first-CTA start / last-CTA end (%globaltimer)
                         into a ctx-owned device buffer, so pask_sync can report the GPU busy
                         time of an inference without events between the layers (PDL kept):
                         gpu_busy_ns = union of the node intervals, the cold start's GPU
                         utilisation of Fig. 6(b).  Two atomics per CTA   */
  int32_t no_prefault; /* 1 = pask_create does not touch the host pages of the embedded code
                         objects, so the first library parse inside the cold window also pays
                         the page faults of reading the image (the Baseline's ELF read,
                         PAPER.md:29); 0 (default) = prefault at create (D8)        */
  int32_t no_prime;   /* 1 = pask_create does not prime the driver; 0 (default) = it loads,
                         launches once and unloads a trivial kernel of its own (not a catalog
                         solution), so the context's one-time module-loader / launch state
                         exists before the first model load, as in any framework process that
                         has already run a kernel (D11)                            */
} pask_config;

typedef enum { PASK_HOW_DIRECT = 0, PASK_HOW_REUSED = 1, PASK_HOW_LOADED = 2 } pask_how;

typedef struct {
  int32_t node;
  int32_t desired_kernel; /* s*_i                                     */
  int32_t bound_kernel;   /* s*_i or the substitute \hat{s}_i           */
  int32_t how;            /* pask_how                                 */
  int32_t lookups;        /* IsApplicable calls spent on this node    */
} pask_binding;

typedef struct {
  int32_t n_nodes;
  int32_t kernels_loaded;      /* distinct CUfunctions loaded for this model      */
  int32_t code_objects_loaded; /* CUlibrary loads (1: single fatbin)              */
  int32_t queries;             /* GETSUBSOLUTION calls (Alg. 1 l.6)               */
  int32_t hits;                /* queries that returned a substitute              */
  int32_t lookups;             /* IsApplicable calls inside queries              */
  uint64_t code_bytes_loaded;  /* bytes of the code object handed to the driver  */
  uint64_t plan_ns;            /* validation + problem extraction + Algorithm 1  */
  uint64_t load_ns;            /* loader thread busy time (library + functions)  */
  uint64_t load_exposed_ns;    /* issue thread blocked on not-yet-ready kernels  */
  uint64_t issue_ns;           /* time inside cuLaunchKernelEx calls             */
  uint64_t encode_ns;          /* CUtensorMap encoding + parameter packing        */
  uint64_t gpu_span_ns;        /* first launch -> last kernel end of the last timed
                                  inference: the first (cold) one, or every one
                                  under timeline / instrument (a hot inference
                                  otherwise records no timing event)            */
  uint64_t gpu_busy_ns;        /* GPU busy time of the last synced inference: the
                                  union of the kernels' [start, end] intervals
                                  (timeline = 1), or the sum of per-kernel event
                                  times (instrument = 1); 0 otherwise               */
  uint64_t cold_wall_ns;       /* pask_load_model entry -> first inference done   */
  uint64_t infer_count;
  uint64_t launches;           /* kernel launches issued so far                   */
  uint64_t load_done_ns;       /* cold timeline, ns after pask_load_model entry:  */
  uint64_t infer_entry_ns;     /*   last planned kernel uploaded, first pask_infer */
  uint64_t first_launch_ns;    /*   entry, its first and last launch              */
  uint64_t last_launch_ns;
  uint64_t encode_begin_ns;    /* launch-parameter encoding window, ns after      */
  uint64_t encode_end_ns;      /*   pask_load_model entry                         */
  uint64_t kernel_span_ns;     /* timeline = 1: first kernel start -> last kernel end
                                  (%globaltimer) of the last synced inference       */
  uint64_t prefault_ns;        /* pask_create's host page touch of the code objects
                                  (outside the cold window; 0 with no_prefault)     */
  uint64_t prefault_bytes;
  int32_t max_cluster;         /* largest split-K cluster this device can co-schedule
                                  (cuOccupancyMaxActiveClusters; 16 or 8)           */
  int32_t reserved0;
  uint64_t prime_ns;           /* pask_create's driver primer (outside the cold
                                  window; 0 with no_prime)                          */
} pask_stats_t;

/* Library version (PASK_VERSION). */
int pask_version(void);

/* Create a context for `device` and start the (idle) helper / loader thread --
 * the "two extra host threads" PASK spawns for loading and issuing
 * (PAPER.md:95, §III-A; :164, §III-D).  The ctx retains the device's primary
 * context (the one PyTorch uses) and releases it in pask_destroy; if the
 * calling thread has a current context on ANOTHER device (or a non-primary
 * context) the call fails with PASK_EINVAL instead of binding the wrong one.
 * The ctx makes its context current on the calling thread of every later entry
 * point.  Outside the cold window it also touches the host pages of the
 * embedded code objects this packaging may load (host residency of the library
 * image, D8; cfg.no_prefault skips it; nothing is uploaded to the
 * GPU) and, with cfg.timeline, allocates the 64 KB stamp buffer.  cfg may be
 * NULL for defaults {reuse 1, search 0, milestone 0, proactive 2, pdl 1,
 * instrument 0, packaging 0, interleave 0, graph 0, catalog 0, branches 0,
 * timeline 0, no_prefault 0}.  Errors: PASK_ECUDA (driver missing / failing),
 * PASK_EINVAL (null out-pointer, device mismatch). */
int pask_create(pask_ctx **ctx, int device, const pask_config *cfg);

/* Host-only planning (no GPU needed): the parse step P_i and
 * Algorithm 1 EXECUTIONPLAN over the categorical cache (PAPER.md:105-141,
 * §III-B/C): validate g, extract problems p_i, apply the static choice s*_i
 * (the library's "find") and Algorithm 1.  plan_out: caller-allocated
 * [g->n_nodes]; stats_out (may be NULL) receives n_nodes, kernels_loaded
 * (planned), queries, hits, lookups, plan_ns.  Deterministic: a pure function
 * of (graph shapes, cfg). */
int pask_plan(const pask_graph *g, const pask_config *cfg, pask_binding *plan_out,
              pask_stats_t *stats_out);

/* Bytes of device workspace the graph needs; host-only, a pure function of the
 * graph's shapes (and the PASK_STEM_FOLD switch).  Today: the stem fold of
 * DESIGN.md D16 -- a conv fed by a layout node over few input channels (the
 * ResNet-50 7x7 s2 stem) reads a regrouped copy of its input and weights that
 * the layout kernel writes here each inference.  0 when no node needs any.
 * pask_load_model fails with PASK_ENOMEM if g->workspace is null or smaller. */
int pask_workspace_bytes(const pask_graph *g, uint64_t *bytes);

/* Plan g (Algorithm 1), then load the bound kernels in first-use order while
 * the per-node launch parameters are encoded concurrently:
 *   proactive 2 (default): the caller thread uploads, the helper thread encodes,
 *                          and the call returns with every kernel resident;
 *   proactive 1: the loader thread uploads asynchronously, the
 *                caller encodes and returns; pask_infer waits for / steals loads;
 *   proactive 0: nothing is loaded here (reactive baseline).
 * plan_out may be NULL.  The graph arrays are copied; the device buffers they
 * point to are not. */
int pask_load_model(pask_ctx *ctx, const pask_graph *g, pask_binding *plan_out);

/* Issue one inference on cuda_stream (a CUstream / cudaStream_t; NULL = legacy
 * default stream): the issue step I_i of every layer, each launched "at the
 * earliest feasible time right after the loading" of its solution
 * (Fig. 5; the hot path afterwards is the paper's Ideal,
 * PAPER.md:178).  inputs / outputs: device pointers, one per graph input /
 * output, or NULL to use the tensors' bound dptr; a pointer different from the
 * bound one rebinds that tensor (re-encoding the affected launch parameters).
 * Blocks only while a needed kernel is still loading; returns after the last
 * launch (asynchronous w.r.t. the GPU). */
int pask_infer(pask_ctx *ctx, void *const *inputs, void *const *outputs, void *cuda_stream);

/* End-to-end inference from host buffers: every graph input from
 * host_inputs[i], pask_infer, every graph output into host_outputs[i], then
 * stream synchronisation; sizes follow the tensors' dims and dtype.  A pinned,
 * device-mapped host buffer (cuMemHostAlloc / cudaHostAlloc under unified
 * addressing) whose tensor only memory-family kernels touch (plain loads and
 * stores: the layout / LayerNorm reading an input, the softmax / LayerNorm
 * writing an output) is bound into the graph directly -- the kernel reads the
 * input over the host link and writes the output there (zero copy; the launch
 * parameters of those nodes are re-encoded on the first such call).  Any other
 * buffer (pageable memory, or a tensor a TMA kernel touches) goes through an
 * H2D / D2H copy into the graph's own device buffer. */
int pask_infer_host(pask_ctx *ctx, const void *const *host_inputs, void *const *host_outputs,
                    void *cuda_stream);

/* Idle-interval loading (§VI "Loading desired solutions"): upload
 * the solutions Algorithm 1 skipped and rebind those nodes to them.
 *   target_catalog < 0: the model's own catalog -- every reused node goes back
 *                       to its s*_i;
 *   target_catalog 0/1: re-run the static choice under that catalog (1 = the
 *                       tuned per-problem solutions) and bind every node whose
 *                       choice differs from its current kernel.
 * Synchronous and meant for the gap between requests: it first waits for the
 * in-flight inference (uploads wait for running GPU work, D3).
 * Results stay within tolerance; a graph captured for hot replay is re-captured.
 * *promoted (may be NULL) = number of nodes rebound.
 * Under packaging 3 the call only repacks (D15): it uploads the two
 * family entries of the variant with the same cases and paths as the loaded
 * single entry, moves every node served by pask_all onto them (same bodies:
 * outputs bitwise equal) and switches the context to packaging 2 -- the cold
 * start pays one upload, the hot path gets per-entry register allocation and
 * the memory solutions' small parameter block; *promoted = nodes moved, the
 * plan is unchanged.  A later call promotes as above. */
int pask_promote(pask_ctx *ctx, int32_t target_catalog, int32_t *promoted);

/* Wait for the last issued inference and finalise its timing statistics
 * (gpu_span_ns if it was timed; cold_wall_ns after the first inference). */
int pask_sync(pask_ctx *ctx);

/* Copy the statistics (host only; call pask_sync first for GPU times): the
 * quantities of the paper's cold-start breakdown -- code loading, issue, GPU
 * execution (Fig. 1(b); Fig. 7, :212-216), GPU busy for the
 * utilisation of Fig. 6(b) (:208, :214) and the cache statistics of Fig. 9
 * (queries, hits, lookups; :226-234).  Errors: PASK_EINVAL on null arguments. */
int pask_stats(const pask_ctx *ctx, pask_stats_t *out);

/* Cross-check with the driver: *state = 1 if kernel_id's CUfunction is loaded
 * in this context (cuFuncIsLoaded), 0 if not or never requested. */
int pask_kernel_is_loaded(const pask_ctx *ctx, int32_t kernel_id, int32_t *state);

/* Cold-start timeline of one catalog kernel in this context (host clock, ns
 * relative to the last pask_load_model entry; 0 when not loaded):
 *   load_ns     time spent loading it (cuLibraryGetKernel + cuKernelGetFunction
 *               + cuFuncLoad + attributes; the first load also includes
 *               cuLibraryLoadData, reported separately in lib_ns),
 *   ready_ns    when its ready flag was published,
 *   lib_ns      cuLibraryLoadData time if this kernel's load performed it. */
int pask_kernel_timeline(const pask_ctx *ctx, int32_t kernel_id, uint64_t *load_ns,
                         uint64_t *ready_ns, uint64_t *lib_ns);

/* Per-node GPU durations (ns) of the last inference issued with
 * cfg.instrument = 1 (call pask_sync first).  ns_out: caller array of
 * n_nodes entries; PASK_ESTATE if the context is not instrumented. */
int pask_node_times(const pask_ctx *ctx, uint64_t *ns_out, int32_t n_nodes);

/* Per-node GPU intervals of the last synced inference of a timeline = 1 ctx:
 * start_ns[i] / end_ns[i] = node i's first CTA start / last CTA end, ns after
 * the inference's first kernel start (%globaltimer, ~0.25 us resolution); a
 * node that did not run reports 0 / 0.  PASK_ESTATE without timeline. */
int pask_node_intervals(const pask_ctx *ctx, uint64_t *start_ns, uint64_t *end_ns, int32_t n_nodes);

/* Join the loader thread, unload the library and free host state. */
int pask_destroy(pask_ctx *ctx);

/* Thread-local description of the last error on this thread ("" if none). */
const char *pask_last_error(void);

/* Catalog introspection (host only): total kernels (generic + specialised). */
int32_t pask_num_kernels(void);
const char *pask_kernel_name(int32_t kernel_id);
/* Name of the CUfunction entry that serves catalog solution kernel_id under
 * code-object packaging `packaging` (pask_config.packaging): its own entry for
 * packaging 0 / 1; for packaging 2 the operator family's entry ("pask_mem" for
 * layout / dw / pool / gavg / softmax / LayerNorm, "pask_conv_igemm" for
 * igemm / conv_1x1 / gemm, D8); for packaging 3 "pask_all" for all of
 * those (D10).  "" for a bad id.  Host only. */
const char *pask_kernel_function(int32_t kernel_id, int32_t packaging);

#ifdef __cplusplus
}
#endif

#endif /* PASK_H */
