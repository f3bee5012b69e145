// pask_cold -- one cold start of a lowered model in a fresh native process
// (SURVEY.md §8(d) cold protocol; the paper's cold start).
//
//   pask_cold MODEL.pmodel [--cfg key=value,...] [--device D] [--wait]
//             [--sleep-ms MS] [--promote] [--hot N] [--flush-mb MB] [--dump PATH]
//
// MODEL is a model image written by DeviceModel.save_image() (model.py): the
// pask_graph's tensors and nodes, with every weight / bias / gamma / beta and
// the graph inputs' data as blobs.  The process
//   1. creates the device's primary context, allocates every tensor and blob,
//      uploads the blobs and the input, and synchronises;
//   2. pask_create(cfg)                          -- outside the cold window;
//   3. with --wait prints "ready" and blocks until a line arrives on stdin (the
//      replica harness releases N processes together), then idles --sleep-ms;
//   4. t0 = pask_load_model entry, first pask_infer, pask_sync = t1 (the
//      library's cold_wall_ns), and prints one JSON line with the statistics,
//      the per-kernel load timeline and, with cfg timeline=1, the per-node GPU
//      intervals; --hot N then times N more inferences (CUDA events, L2 flushed
//      by a --flush-mb memset before each when MB > 0); --dump writes every
//      tensor's bytes, in tensor order, after the cold inference; --promote
//      calls pask_promote (idle-interval loading; packaging 3: the repack into
//      the two family entries, D15) before the hot inferences.
// No PyTorch, no Python: the whole process is native, so a sample costs
// milliseconds of process start instead of seconds of interpreter start.
#include <dlfcn.h>
#include <malloc.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <thread>
#include <chrono>
#include <string>
#include <type_traits>
#include <vector>

#include <cuda.h>

#include "../../../include/pask.h"

namespace {

struct Cu {
  decltype(&::cuInit) init;
  decltype(&::cuDeviceGet) device_get;
  decltype(&::cuDevicePrimaryCtxRetain) primary_retain;
  decltype(&::cuCtxSetCurrent) ctx_set;
  decltype(&::cuCtxSynchronize) ctx_sync;
  decltype(&::cuMemAlloc_v2) mem_alloc;
  decltype(&::cuMemcpyHtoD_v2) h2d;
  decltype(&::cuMemcpyDtoH_v2) d2h;
  decltype(&::cuMemsetD8_v2) memset_d8;
  decltype(&::cuMemsetD8Async) memset_d8_async;
  decltype(&::cuEventCreate) event_create;
  decltype(&::cuEventRecord) event_record;
  decltype(&::cuEventSynchronize) event_sync;
  decltype(&::cuEventElapsedTime) event_elapsed;
  decltype(&::cuGetErrorName) err_name;
};

[[noreturn]] void die(const std::string& m) {
  fprintf(stderr, "pask_cold: %s\n", m.c_str());
  exit(2);
}

Cu resolve() {
  void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_LOCAL);
  if (!h) die("libcuda.so.1 not found (no NVIDIA driver)");
  using GetProc = CUresult (*)(const char*, void**, int, cuuint64_t, CUdriverProcAddressQueryResult*);
  auto gp = reinterpret_cast<GetProc>(dlsym(h, "cuGetProcAddress_v2"));
  if (!gp) die("cuGetProcAddress_v2 missing");
  Cu c{};
  auto get = [&](const char* name, auto* slot) {
    void* fn = nullptr;
    CUdriverProcAddressQueryResult q;
    if (gp(name, &fn, CUDA_VERSION, CU_GET_PROC_ADDRESS_DEFAULT, &q) != CUDA_SUCCESS || !fn)
      die(std::string("cannot resolve ") + name);
    *slot = reinterpret_cast<std::remove_reference_t<decltype(*slot)>>(fn);
  };
  get("cuInit", &c.init);
  get("cuDeviceGet", &c.device_get);
  get("cuDevicePrimaryCtxRetain", &c.primary_retain);
  get("cuCtxSetCurrent", &c.ctx_set);
  get("cuCtxSynchronize", &c.ctx_sync);
  get("cuMemAlloc", &c.mem_alloc);
  get("cuMemcpyHtoD", &c.h2d);
  get("cuMemcpyDtoH", &c.d2h);
  get("cuMemsetD8", &c.memset_d8);
  get("cuMemsetD8Async", &c.memset_d8_async);
  get("cuEventCreate", &c.event_create);
  get("cuEventRecord", &c.event_record);
  get("cuEventSynchronize", &c.event_sync);
  get("cuEventElapsedTime", &c.event_elapsed);
  get("cuGetErrorName", &c.err_name);
  return c;
}

const Cu* g_cu = nullptr;

void ck(CUresult r, const char* what) {
  if (r == CUDA_SUCCESS) return;
  const char* n = nullptr;
  if (g_cu) g_cu->err_name(r, &n);
  die(std::string(what) + ": " + (n ? n : "?"));
}

void pk(int rc, const char* what) {
  if (rc != PASK_OK) die(std::string(what) + " failed (" + std::to_string(rc) + "): " + pask_last_error());
}

// ---------------------------------------------------------------- model image
struct Image {
  std::vector<pask_tensor> tensors;
  std::vector<pask_node> nodes;
  std::vector<int32_t> inputs, outputs, input_blob;
  std::vector<uint64_t> blob_bytes, blob_off;
  std::vector<unsigned char> data;  // blob payloads
  uint64_t ws_bytes = 0;
};

Image read_image(const char* path) {
  FILE* f = fopen(path, "rb");
  if (!f) die(std::string("cannot open ") + path);
  auto rd = [&](void* p, size_t n) {
    if (n && fread(p, 1, n, f) != n) die("truncated model image");
  };
  char magic[8];
  rd(magic, 8);
  if (memcmp(magic, "PASKMDL1", 8) != 0) die("not a pask model image");
  int32_t hdr[6];
  rd(hdr, sizeof hdr);
  uint64_t sizes[3];
  rd(sizes, sizeof sizes);
  if (hdr[0] != 1) die("model image version mismatch");
  if (sizes[0] != sizeof(pask_tensor) || sizes[1] != sizeof(pask_node))
    die("model image struct sizes differ from include/pask.h");
  Image im;
  im.ws_bytes = sizes[2];
  im.tensors.resize(hdr[1]);
  im.nodes.resize(hdr[2]);
  im.inputs.resize(hdr[3]);
  im.outputs.resize(hdr[4]);
  im.input_blob.resize(hdr[3]);
  im.blob_bytes.resize(hdr[5]);
  rd(im.tensors.data(), im.tensors.size() * sizeof(pask_tensor));
  rd(im.nodes.data(), im.nodes.size() * sizeof(pask_node));
  rd(im.inputs.data(), im.inputs.size() * 4);
  rd(im.outputs.data(), im.outputs.size() * 4);
  rd(im.input_blob.data(), im.input_blob.size() * 4);
  rd(im.blob_bytes.data(), im.blob_bytes.size() * 8);
  uint64_t total = 0;
  for (uint64_t b : im.blob_bytes) {
    im.blob_off.push_back(total);
    total += (b + 255) / 256 * 256;
  }
  im.data.resize(total);
  rd(im.data.data(), total);
  fclose(f);
  return im;
}

size_t tensor_bytes(const pask_tensor& t) {
  return static_cast<size_t>(t.n) * t.h * t.w * t.c * (t.dtype == PASK_F32 ? 4 : 2);
}

void set_cfg(pask_config* c, const std::string& kv) {
  const size_t eq = kv.find('=');
  if (eq == std::string::npos) die("--cfg expects key=value: " + kv);
  const std::string k = kv.substr(0, eq);
  const int v = atoi(kv.c_str() + eq + 1);
#define F(name) \
  if (k == #name) { c->name = v; return; }
  F(reuse) F(search) F(milestone) F(proactive) F(pdl) F(instrument) F(packaging) F(interleave) F(graph)
  F(catalog) F(branches) F(timeline) F(no_prefault) F(no_prime)
#undef F
  die("unknown pask_config field " + k);
}

uint64_t now_ns() {
  return static_cast<uint64_t>(std::chrono::duration_cast<std::chrono::nanoseconds>(
                                   std::chrono::steady_clock::now().time_since_epoch())
                                   .count());
}

}  // namespace

int main(int argc, char** argv) {
  const uint64_t t_proc = now_ns();
  if (argc < 2) {
    fprintf(stderr,
            "usage: pask_cold MODEL.pmodel [--cfg k=v,...] [--device D] [--wait] [--sleep-ms MS] "
            "[--promote] [--hot N] [--flush-mb MB] [--dump PATH]\n");
    return 1;
  }
  const char* model = argv[1];
  pask_config cfg{1, 0, 0, 2, 1, 0, 0, 0, 0, 0, 0, 0, 0, 0};  // the library defaults (pask.h)
  int device = 0, hot = 0, flush_mb = 256, warm_heap_mb = 0;
  bool promote = false;
  bool wait = false, plan_only = false, bg_spin = false, cudart = false;
  double sleep_ms = 50, spin_ms = 0;
  const char* dump = nullptr;
  std::string pre_image;  // experiment: PATH:function loaded, uploaded and unloaded before pask_create
  for (int i = 2; i < argc; ++i) {
    const std::string a = argv[i];
    auto next = [&]() -> const char* {
      if (i + 1 >= argc) die("missing value for " + a);
      return argv[++i];
    };
    if (a == "--cfg") {
      std::string s = next();
      size_t p = 0;
      while (p <= s.size()) {
        const size_t q = s.find(',', p);
        const std::string kv = s.substr(p, q == std::string::npos ? std::string::npos : q - p);
        if (!kv.empty()) set_cfg(&cfg, kv);
        if (q == std::string::npos) break;
        p = q + 1;
      }
    } else if (a == "--device") {
      device = atoi(next());
    } else if (a == "--wait") {
      wait = true;
    } else if (a == "--plan-only") {  // host only: parse the image, print pask_plan's bindings
      plan_only = true;
    } else if (a == "--sleep-ms") {
      sleep_ms = atof(next());
    } else if (a == "--warm-heap-mb") {  // experiment: a warm malloc arena, as in a long-lived server
      warm_heap_mb = atoi(next());
    } else if (a == "--pre-image") {
      pre_image = next();
    } else if (a == "--cudart") {  // experiment: initialise the CUDA runtime first, as a framework does
      cudart = true;
    } else if (a == "--bg-spin") {  // experiment: a second thread busy through the cold window
      bg_spin = true;
    } else if (a == "--spin-ms") {  // busy-wait (core kept awake) instead of sleeping before t0
      spin_ms = atof(next());
      sleep_ms = 0;
    } else if (a == "--promote") {
      promote = true;
    } else if (a == "--hot") {
      hot = atoi(next());
    } else if (a == "--flush-mb") {
      flush_mb = atoi(next());
    } else if (a == "--dump") {
      dump = next();
    } else {
      die("unknown argument " + a);
    }
  }
  if (warm_heap_mb > 0) {
    mallopt(M_MMAP_THRESHOLD, 512 << 20);
    mallopt(M_TRIM_THRESHOLD, 1 << 30);
    mallopt(M_TOP_PAD, 64 << 20);
    void* h = malloc(static_cast<size_t>(warm_heap_mb) << 20);
    memset(h, 1, static_cast<size_t>(warm_heap_mb) << 20);
    free(h);
  }
  Image im = read_image(model);
  if (plan_only) {  // no GPU: check the image round trip through the host planner
    pask_graph g{};
    for (size_t i = 0; i < im.tensors.size(); ++i) im.tensors[i].dptr = reinterpret_cast<void*>((i + 1) << 20);
    g.n_tensors = static_cast<int32_t>(im.tensors.size());
    g.tensors = im.tensors.data();
    g.n_nodes = static_cast<int32_t>(im.nodes.size());
    g.nodes = im.nodes.data();
    g.n_inputs = static_cast<int32_t>(im.inputs.size());
    g.inputs = im.inputs.data();
    g.n_outputs = static_cast<int32_t>(im.outputs.size());
    g.outputs = im.outputs.data();
    std::vector<pask_binding> plan(im.nodes.size());
    pask_stats_t st;
    pk(pask_plan(&g, &cfg, plan.data(), &st), "pask_plan");
    uint64_t blob_total = 0;
    for (uint64_t b : im.blob_bytes) blob_total += b;
    printf("{\"n_nodes\": %d, \"n_tensors\": %d, \"n_blobs\": %zu, \"blob_bytes\": %llu, \"bindings\": [",
           g.n_nodes, g.n_tensors, im.blob_bytes.size(), static_cast<unsigned long long>(blob_total));
    for (size_t i = 0; i < plan.size(); ++i)
      printf("%s[%d, %d, %d, %d, %d]", i ? ", " : "", plan[i].node, plan[i].desired_kernel, plan[i].bound_kernel,
             plan[i].how, plan[i].lookups);
    printf("]}\n");
    return 0;
  }
  const Cu cu = resolve();
  g_cu = &cu;
  // ---- outside the cold window: context, memory, weights, input
  if (cudart) {
    void* rt = dlopen("libcudart.so.12", RTLD_NOW | RTLD_GLOBAL);
    if (!rt) die("libcudart.so.12 not found");
    using FreeFn = int (*)(void*);
    using MallocFn = int (*)(void**, size_t);
    auto cfree = reinterpret_cast<FreeFn>(dlsym(rt, "cudaFree"));
    auto cmalloc = reinterpret_cast<MallocFn>(dlsym(rt, "cudaMalloc"));
    void* p0 = nullptr;
    if (!cfree || !cmalloc || cfree(nullptr) != 0 || cmalloc(&p0, 1 << 21) != 0) die("cudart init failed");
  }
  ck(cu.init(0), "cuInit");
  CUdevice dev;
  ck(cu.device_get(&dev, device), "cuDeviceGet");
  CUcontext ctx;
  ck(cu.primary_retain(&ctx, dev), "cuDevicePrimaryCtxRetain");
  ck(cu.ctx_set(ctx), "cuCtxSetCurrent");
  const uint64_t t_ctx = now_ns();
  uint64_t arena = 0;
  std::vector<uint64_t> t_off(im.tensors.size()), b_off(im.blob_bytes.size());
  for (size_t i = 0; i < im.tensors.size(); ++i) {
    t_off[i] = arena;
    arena += (tensor_bytes(im.tensors[i]) + 255) / 256 * 256;
  }
  for (size_t i = 0; i < im.blob_bytes.size(); ++i) {
    b_off[i] = arena;
    arena += (im.blob_bytes[i] + 255) / 256 * 256;
  }
  const uint64_t ws_off = arena;
  arena += (im.ws_bytes + 255) / 256 * 256;
  CUdeviceptr base;
  ck(cu.mem_alloc(&base, arena ? arena : 256), "cuMemAlloc");
  ck(cu.memset_d8(base, 0, arena), "cuMemsetD8");
  for (size_t i = 0; i < im.blob_bytes.size(); ++i)
    ck(cu.h2d(base + b_off[i], im.data.data() + im.blob_off[i], im.blob_bytes[i]), "upload weights");
  for (size_t i = 0; i < im.tensors.size(); ++i) im.tensors[i].dptr = reinterpret_cast<void*>(base + t_off[i]);
  auto blob_ptr = [&](const void* enc) -> uint64_t {
    const uint64_t id = reinterpret_cast<uint64_t>(enc);
    if (!id) return 0;
    if (id > im.blob_bytes.size()) die("bad blob reference in model image");
    return base + b_off[id - 1];
  };
  for (pask_node& nd : im.nodes) {
    nd.w = reinterpret_cast<const void*>(blob_ptr(nd.w));
    nd.bias = reinterpret_cast<const float*>(blob_ptr(nd.bias));
    nd.gamma = reinterpret_cast<const float*>(blob_ptr(nd.gamma));
    nd.beta = reinterpret_cast<const float*>(blob_ptr(nd.beta));
  }
  for (size_t i = 0; i < im.inputs.size(); ++i) {  // the graph inputs' data
    const int32_t b = im.input_blob[i];
    if (b >= static_cast<int32_t>(im.blob_bytes.size()) || im.inputs[i] < 0 ||
        im.inputs[i] >= static_cast<int32_t>(im.tensors.size()))
      die("bad input reference in model image");
    const pask_tensor& t = im.tensors[im.inputs[i]];
    if (b >= 0 && im.blob_bytes[b] < tensor_bytes(t)) die("input blob smaller than its tensor");
    if (b >= 0) ck(cu.h2d(base + t_off[im.inputs[i]], im.data.data() + im.blob_off[b], tensor_bytes(t)), "upload input");
  }
  CUdeviceptr flush = 0;
  if (hot > 0 && flush_mb > 0) ck(cu.mem_alloc(&flush, static_cast<size_t>(flush_mb) << 20), "cuMemAlloc flush");
  ck(cu.ctx_sync(), "cuCtxSynchronize");
  pask_graph g{};
  g.n_tensors = static_cast<int32_t>(im.tensors.size());
  g.tensors = im.tensors.data();
  g.n_nodes = static_cast<int32_t>(im.nodes.size());
  g.nodes = im.nodes.data();
  g.n_inputs = static_cast<int32_t>(im.inputs.size());
  g.inputs = im.inputs.data();
  g.n_outputs = static_cast<int32_t>(im.outputs.size());
  g.outputs = im.outputs.data();
  g.workspace = im.ws_bytes ? reinterpret_cast<void*>(base + ws_off) : nullptr;
  g.workspace_bytes = im.ws_bytes;
  std::atomic<bool> bg_stop{false};
  std::thread bg;
  if (bg_spin)
    bg = std::thread([&] {
      volatile uint64_t x = 0;
      while (!bg_stop.load(std::memory_order_relaxed)) x = x + 1;
    });
  if (!pre_image.empty()) {
    const size_t colon = pre_image.rfind(':');
    const std::string path = pre_image.substr(0, colon), fn = pre_image.substr(colon + 1);
    FILE* f = fopen(path.c_str(), "rb");
    if (!f) die("cannot open " + path);
    std::vector<unsigned char> img;
    unsigned char buf[65536];
    size_t nrd;
    while ((nrd = fread(buf, 1, sizeof buf, f)) > 0) img.insert(img.end(), buf, buf + nrd);
    fclose(f);
    void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_LOCAL);
    auto lload = reinterpret_cast<decltype(&::cuLibraryLoadData)>(dlsym(h, "cuLibraryLoadData"));
    auto lget = reinterpret_cast<decltype(&::cuLibraryGetKernel)>(dlsym(h, "cuLibraryGetKernel"));
    auto kfn = reinterpret_cast<decltype(&::cuKernelGetFunction)>(dlsym(h, "cuKernelGetFunction"));
    auto fload = reinterpret_cast<decltype(&::cuFuncLoad)>(dlsym(h, "cuFuncLoad"));
    auto lunload = reinterpret_cast<decltype(&::cuLibraryUnload)>(dlsym(h, "cuLibraryUnload"));
    CUlibrary lib;
    CUkernel k;
    CUfunction fnc;
    ck(lload(&lib, img.data(), nullptr, nullptr, 0, nullptr, nullptr, 0), "pre-image load");
    ck(lget(&k, lib, fn.c_str()), "pre-image kernel");
    ck(kfn(&fnc, k), "pre-image function");
    ck(fload(fnc), "pre-image upload");
    ck(lunload(lib), "pre-image unload");
  }
  pask_ctx* pc = nullptr;
  pk(pask_create(&pc, device, &cfg), "pask_create");
  const uint64_t t_ready = now_ns();
  if (wait) {  // replica harness: all processes are released into the cold window together
    printf("ready\n");
    fflush(stdout);
    char line[64];
    if (!fgets(line, sizeof line, stdin)) die("stdin closed before go");
  }
  if (sleep_ms > 0) usleep(static_cast<useconds_t>(sleep_ms * 1000));  // idle before the window
  if (spin_ms > 0) {
    const uint64_t until = now_ns() + static_cast<uint64_t>(spin_ms * 1e6);
    while (now_ns() < until) {
    }
  }
  ck(cu.ctx_sync(), "cuCtxSynchronize");
  // ---- the cold window: pask_load_model entry -> first inference complete
  const uint64_t t0 = now_ns();
  std::vector<pask_binding> plan(im.nodes.size());
  pk(pask_load_model(pc, &g, plan.data()), "pask_load_model");
  pk(pask_infer(pc, nullptr, nullptr, nullptr), "pask_infer");
  pk(pask_sync(pc), "pask_sync");
  const uint64_t t1 = now_ns();
  bg_stop.store(true);
  if (bg.joinable()) bg.join();
  pask_stats_t st;
  pk(pask_stats(pc, &st), "pask_stats");
  std::string js = "{";
  auto kv = [&](const char* k, double v) {
    char b[96];
    snprintf(b, sizeof b, "\"%s\": %.3f, ", k, v);
    js += b;
  };
  kv("cold_us", st.cold_wall_ns / 1e3);
  kv("cold_proc_clock_us", (t1 - t0) / 1e3);
  kv("setup_us", (t_ready - t_ctx) / 1e3);
  kv("ctx_create_us", (t_ctx - t_proc) / 1e3);
  kv("kernels_loaded", st.kernels_loaded);
  kv("code_objects", st.code_objects_loaded);
  kv("code_bytes", static_cast<double>(st.code_bytes_loaded));
  kv("queries", st.queries);
  kv("hits", st.hits);
  kv("lookups", st.lookups);
  kv("plan_us", st.plan_ns / 1e3);
  kv("encode_us", st.encode_ns / 1e3);
  kv("load_us", st.load_ns / 1e3);
  kv("load_exposed_us", st.load_exposed_ns / 1e3);
  kv("issue_us", st.issue_ns / 1e3);
  kv("gpu_span_us", st.gpu_span_ns / 1e3);
  kv("gpu_busy_us", st.gpu_busy_ns / 1e3);
  kv("kernel_span_us", st.kernel_span_ns / 1e3);
  kv("t_load_done_us", st.load_done_ns / 1e3);
  kv("t_infer_entry_us", st.infer_entry_ns / 1e3);
  kv("t_first_launch_us", st.first_launch_ns / 1e3);
  kv("t_last_launch_us", st.last_launch_ns / 1e3);
  kv("t_encode_begin_us", st.encode_begin_ns / 1e3);
  kv("t_encode_end_us", st.encode_end_ns / 1e3);
  kv("launches", static_cast<double>(st.launches));
  kv("prefault_us", st.prefault_ns / 1e3);
  kv("prime_us", st.prime_ns / 1e3);
  kv("max_cluster", st.max_cluster);
  {  // per-kernel load timeline [lib_us, load_us, ready_at_us]
    js += "\"timeline\": {";
    bool firstk = true;
    for (int32_t k = 0; k < pask_num_kernels(); ++k) {
      uint64_t ld = 0, rd = 0, lb = 0;
      if (pask_kernel_timeline(pc, k, &ld, &rd, &lb) == PASK_OK && ld) {
        char b[160];
        snprintf(b, sizeof b, "%s\"%s\": [%.1f, %.1f, %.1f]", firstk ? "" : ", ", pask_kernel_name(k), lb / 1e3,
                 ld / 1e3, rd / 1e3);
        js += b;
        firstk = false;
      }
    }
    js += "}, ";
  }
  if (cfg.timeline) {
    std::vector<uint64_t> s(im.nodes.size()), e(im.nodes.size());
    if (pask_node_intervals(pc, s.data(), e.data(), static_cast<int32_t>(s.size())) == PASK_OK) {
      js += "\"node_intervals_us\": [";
      for (size_t i = 0; i < s.size(); ++i) {
        char b[64];
        snprintf(b, sizeof b, "%s[%.2f, %.2f]", i ? ", " : "", s[i] / 1e3, e[i] / 1e3);
        js += b;
      }
      js += "], ";
    }
  }
  js += "\"bindings\": [";
  for (size_t i = 0; i < plan.size(); ++i) {
    char b[64];
    snprintf(b, sizeof b, "%s[%d, %d, %d, %d]", i ? ", " : "", plan[i].desired_kernel, plan[i].bound_kernel,
             plan[i].how, plan[i].lookups);
    js += b;
  }
  js += "], ";
  if (dump) {  // every tensor's bytes after the cold inference
    FILE* f = fopen(dump, "wb");
    if (!f) die(std::string("cannot write ") + dump);
    std::vector<unsigned char> h;
    for (size_t i = 0; i < im.tensors.size(); ++i) {
      h.resize(tensor_bytes(im.tensors[i]));
      ck(cu.d2h(h.data(), base + t_off[i], h.size()), "dump");
      fwrite(h.data(), 1, h.size(), f);
    }
    fclose(f);
  }
  if (promote) {
    int32_t n = 0;
    pk(pask_promote(pc, -1, &n), "pask_promote");
    kv("promoted", n);
  }
  if (hot > 0) {  // hot inferences in the same process (CUDA events on the stream)
    CUevent e0, e1;
    ck(cu.event_create(&e0, CU_EVENT_DEFAULT), "cuEventCreate");
    ck(cu.event_create(&e1, CU_EVENT_DEFAULT), "cuEventCreate");
    for (int w = 0; w < 5; ++w) pk(pask_infer(pc, nullptr, nullptr, nullptr), "pask_infer");
    pk(pask_sync(pc), "pask_sync");
    std::vector<float> ms(hot);
    for (int it = 0; it < hot; ++it) {
      if (flush) ck(cu.memset_d8_async(flush, static_cast<unsigned char>(it), static_cast<size_t>(flush_mb) << 20, nullptr), "flush");
      ck(cu.event_record(e0, nullptr), "cuEventRecord");
      pk(pask_infer(pc, nullptr, nullptr, nullptr), "pask_infer");
      ck(cu.event_record(e1, nullptr), "cuEventRecord");
      ck(cu.event_sync(e1), "cuEventSynchronize");
      ck(cu.event_elapsed(&ms[it], e0, e1), "cuEventElapsedTime");
    }
    std::vector<float> srt = ms;
    std::sort(srt.begin(), srt.end());
    double sum = 0;
    for (float v : ms) sum += v;
    kv("hot_median_us", 1e3 * srt[srt.size() / 2]);
    kv("hot_mean_us", 1e3 * sum / hot);
    kv("hot_n", hot);
    kv("hot_flushed", flush ? 1 : 0);
  }
  pk(pask_destroy(pc), "pask_destroy");
  js += "\"ok\": 1}";
  printf("%s\n", js.c_str());
  return 0;
}
