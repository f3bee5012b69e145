// Test-only fake CUDA driver (include/pask_testing.h): exercises the loader /
// issuer host logic without a GPU.  Handles are small integers disguised as
// pointers; a CUfunction encodes its catalog kernel id (found from the name).
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <atomic>
#include <mutex>
#include <thread>
#include <vector>

#include "../../../include/pask_testing.h"
#include "driver.h"
#include "plan.h"

#define PASK_API extern "C" __attribute__((visibility("default")))

namespace pask {
namespace {

std::mutex g_mu;
int g_load_us = 0;
int g_fail_kernel = -1;
std::vector<int32_t> g_ids, g_kinds;
bool g_loaded[PASK_MAX_KERNELS] = {};
constexpr int32_t kFakeMemFamilyId = PASK_MAX_KERNELS - 1;  // id logged for the `pask_mem` entry
constexpr int32_t kFakeAllId = PASK_MAX_KERNELS - 2;        // id logged for the `pask_all` entry
constexpr int32_t kFakePrimerId = PASK_MAX_KERNELS - 3;     // pask_create's primer: never logged
std::atomic<int32_t> g_primer_loads{0};

int32_t kernel_of_name(const char* name) {
  for (int32_t k = 0; k < num_kernels(); ++k)
    if (strcmp(catalog(k).name, name) == 0) return k;
  if (strcmp(name, "pask_mem") == 0) return kFakeMemFamilyId;  // packaging-2 family entry
  if (strcmp(name, "pask_all") == 0) return kFakeAllId;        // packaging-3 single entry
  if (strcmp(name, "pask_primer") == 0) return kFakePrimerId;  // driver primer (pask_create)
  return -1;
}
void sleep_us(int us) {
  if (us > 0) std::this_thread::sleep_for(std::chrono::microseconds(us));
}
void log_event(int32_t id, int32_t kind) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_ids.push_back(id);
  g_kinds.push_back(kind);
}
template <class T>
T fake_handle(uintptr_t v) {
  return reinterpret_cast<T>(v);
}
constexpr uintptr_t kFnBase = 0x1000;

CUresult f_ok_init(unsigned int) { return CUDA_SUCCESS; }
CUresult f_err_name(CUresult r, const char** s) {
  *s = r == CUDA_SUCCESS ? "CUDA_SUCCESS" : (r == CUDA_ERROR_INVALID_IMAGE ? "CUDA_ERROR_INVALID_IMAGE" : "CUDA_ERROR_FAKE");
  return CUDA_SUCCESS;
}
CUresult f_dev_get(CUdevice* d, int o) {
  *d = o;
  return CUDA_SUCCESS;
}
// contexts: device d's primary context is 0x10 + d; "current" is process-wide
// here (device 0's primary by default, as after torch.cuda.set_device(0))
std::atomic<uintptr_t> g_current{0x10};
std::atomic<int32_t> g_occupancy{1};      // cuOccupancyMaxActiveClusters result
std::atomic<int32_t> g_max_cluster_z{0};  // largest cluster launched
CUresult f_ctx_get(CUcontext* c) {
  *c = fake_handle<CUcontext>(g_current.load());
  return CUDA_SUCCESS;
}
CUresult f_ctx_set(CUcontext c) {
  g_current.store(reinterpret_cast<uintptr_t>(c));
  return CUDA_SUCCESS;
}
CUresult f_primary_retain(CUcontext* c, CUdevice d) {
  *c = fake_handle<CUcontext>(0x10 + static_cast<uintptr_t>(d));
  return CUDA_SUCCESS;
}
CUresult f_primary_release(CUdevice) { return CUDA_SUCCESS; }
CUresult f_ctx_get_device(CUdevice* d) {
  *d = static_cast<CUdevice>(g_current.load() - 0x10);
  return CUDA_SUCCESS;
}
CUresult f_occupancy_clusters(int* n, CUfunction, const CUlaunchConfig*) {
  *n = g_occupancy.load();
  return CUDA_SUCCESS;
}
// device memory of the fake: host memory (only the timeline buffer uses it)
CUresult f_mem_alloc(CUdeviceptr* p, size_t bytes) {
  void* h = calloc(1, bytes);
  if (!h) return CUDA_ERROR_OUT_OF_MEMORY;
  *p = reinterpret_cast<CUdeviceptr>(h);
  return CUDA_SUCCESS;
}
CUresult f_mem_free(CUdeviceptr p) {
  free(reinterpret_cast<void*>(p));
  return CUDA_SUCCESS;
}
CUresult f_memset_d8(CUdeviceptr p, unsigned char v, size_t n) {
  memset(reinterpret_cast<void*>(p), v, n);
  return CUDA_SUCCESS;
}
CUresult f_memcpy_dtoh(void* dst, CUdeviceptr src, size_t n) {
  memcpy(dst, reinterpret_cast<const void*>(src), n);
  return CUDA_SUCCESS;
}
CUresult f_lib_load(CUlibrary* lib, const void*, CUjit_option*, void**, unsigned int, CUlibraryOption*, void**,
                    unsigned int) {
  sleep_us(g_load_us);
  *lib = fake_handle<CUlibrary>(0x20);
  return CUDA_SUCCESS;
}
CUresult f_lib_unload(CUlibrary) { return CUDA_SUCCESS; }
CUresult f_lib_get_kernel(CUkernel* k, CUlibrary, const char* name) {
  const int32_t id = kernel_of_name(name);
  if (id < 0) return CUDA_ERROR_NOT_FOUND;
  *k = fake_handle<CUkernel>(kFnBase + id);
  return CUDA_SUCCESS;
}
CUresult f_kernel_get_fn(CUfunction* f, CUkernel k) {
  const int32_t id = static_cast<int32_t>(reinterpret_cast<uintptr_t>(k) - kFnBase);
  sleep_us(g_load_us);
  if (id == g_fail_kernel) return CUDA_ERROR_INVALID_IMAGE;
  *f = fake_handle<CUfunction>(kFnBase + id);
  return CUDA_SUCCESS;
}
CUresult f_func_load(CUfunction f) {
  const int32_t id = static_cast<int32_t>(reinterpret_cast<uintptr_t>(f) - kFnBase);
  if (id == kFakePrimerId) {
    g_primer_loads.fetch_add(1);
    return CUDA_SUCCESS;
  }
  {
    std::lock_guard<std::mutex> lk(g_mu);
    if (id >= 0 && id < PASK_MAX_KERNELS) g_loaded[id] = true;
  }
  log_event(id, 0);
  return CUDA_SUCCESS;
}
CUresult f_func_is_loaded(CUfunctionLoadingState* s, CUfunction f) {
  const int32_t id = static_cast<int32_t>(reinterpret_cast<uintptr_t>(f) - kFnBase);
  std::lock_guard<std::mutex> lk(g_mu);
  *s = (id >= 0 && id < PASK_MAX_KERNELS && g_loaded[id]) ? CU_FUNCTION_LOADING_STATE_LOADED
                                                          : CU_FUNCTION_LOADING_STATE_UNLOADED;
  return CUDA_SUCCESS;
}
CUresult f_func_set_attr(CUfunction, CUfunction_attribute, int) { return CUDA_SUCCESS; }
// the stream the last capture began on: "main" like the caller's stream (0)
std::atomic<uintptr_t> g_capture_stream{0};
CUresult f_launch(const CUlaunchConfig* cfg, CUfunction f, void**, void**) {
  const int32_t id = static_cast<int32_t>(reinterpret_cast<uintptr_t>(f) - kFnBase);
  if (id == kFakePrimerId) return CUDA_SUCCESS;
  bool loaded;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    loaded = id >= 0 && id < PASK_MAX_KERNELS && g_loaded[id];
  }
  // 1: launch on the caller's stream, 3: on another stream (the branches side
  // stream, D9), 2: kernel not loaded (must never happen)
  for (unsigned a = 0; a < cfg->numAttrs; ++a)
    if (cfg->attrs[a].id == CU_LAUNCH_ATTRIBUTE_CLUSTER_DIMENSION)
      g_max_cluster_z.store(std::max<int32_t>(g_max_cluster_z.load(), cfg->attrs[a].value.clusterDim.z));
  const uintptr_t sh = reinterpret_cast<uintptr_t>(cfg->hStream);
  const bool main_stream = sh == 0 || sh == g_capture_stream.load();
  log_event(id, !loaded ? 2 : (main_stream ? 1 : 3));
  return CUDA_SUCCESS;
}
CUresult f_tmap_tiled(CUtensorMap* m, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                      const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                      CUtensorMapL2promotion, CUtensorMapFloatOOBfill) {
  memset(m, 0, sizeof(*m));
  return CUDA_SUCCESS;
}
CUresult f_tmap_im2col(CUtensorMap* m, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                       const int*, const int*, cuuint32_t, cuuint32_t, const cuuint32_t*, CUtensorMapInterleave,
                       CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill) {
  memset(m, 0, sizeof(*m));
  return CUDA_SUCCESS;
}
CUresult f_event_create(CUevent* e, unsigned int) {
  *e = fake_handle<CUevent>(0x30);
  return CUDA_SUCCESS;
}
CUresult f_event_destroy(CUevent) { return CUDA_SUCCESS; }
CUresult f_event_record(CUevent, CUstream) { return CUDA_SUCCESS; }
CUresult f_event_sync(CUevent) { return CUDA_SUCCESS; }
CUresult f_event_elapsed(float* ms, CUevent, CUevent) {
  *ms = 0.f;
  return CUDA_SUCCESS;
}
CUresult f_h2d(CUdeviceptr, const void*, size_t, CUstream) { return CUDA_SUCCESS; }
CUresult f_d2h(void*, CUdeviceptr, size_t, CUstream) { return CUDA_SUCCESS; }
// host buffers are never device-mapped here: pask_infer_host takes the copy path
CUresult f_ptr_attr(void*, CUpointer_attribute, CUdeviceptr) { return CUDA_ERROR_INVALID_VALUE; }
CUresult f_stream_sync(CUstream) { return CUDA_SUCCESS; }
// streams get handles 0x40, 0x41, ... in creation order; launches on the
// caller's stream (0) or on the capture stream are "main" (kind 1), on any other
// (the branches side streams) kind 3
std::atomic<uintptr_t> g_next_stream{0x40};
CUresult f_stream_create(CUstream* s, unsigned int) {
  *s = fake_handle<CUstream>(g_next_stream.fetch_add(1));
  return CUDA_SUCCESS;
}
CUresult f_stream_destroy(CUstream) { return CUDA_SUCCESS; }
// graph capture: launches during a capture are logged like direct launches (the
// issue order is what the tests check); replaying the fake graph launches nothing
CUresult f_begin_capture(CUstream s, CUstreamCaptureMode) {
  g_capture_stream.store(reinterpret_cast<uintptr_t>(s));
  return CUDA_SUCCESS;
}
CUresult f_end_capture(CUstream, CUgraph* g) {
  *g = fake_handle<CUgraph>(0x50);
  return CUDA_SUCCESS;
}
CUresult f_graph_instantiate(CUgraphExec* ge, CUgraph, unsigned long long) {
  *ge = fake_handle<CUgraphExec>(0x60);
  return CUDA_SUCCESS;
}
CUresult f_graph_launch(CUgraphExec, CUstream) { return CUDA_SUCCESS; }
CUresult f_graph_destroy(CUgraph) { return CUDA_SUCCESS; }
CUresult f_graph_exec_destroy(CUgraphExec) { return CUDA_SUCCESS; }
CUresult f_stream_wait_event(CUstream, CUevent, unsigned int) { return CUDA_SUCCESS; }

Driver make_fake() {
  Driver d;
  d.cuInit = f_ok_init;
  d.cuGetErrorName = f_err_name;
  d.cuDeviceGet = f_dev_get;
  d.cuCtxGetCurrent = f_ctx_get;
  d.cuCtxSetCurrent = f_ctx_set;
  d.cuDevicePrimaryCtxRetain = f_primary_retain;
  d.cuDevicePrimaryCtxRelease = f_primary_release;
  d.cuCtxGetDevice = f_ctx_get_device;
  d.cuOccupancyMaxActiveClusters = f_occupancy_clusters;
  d.cuMemAlloc = f_mem_alloc;
  d.cuMemFree = f_mem_free;
  d.cuMemsetD8 = f_memset_d8;
  d.cuMemcpyDtoH = f_memcpy_dtoh;
  d.cuLibraryLoadData = f_lib_load;
  d.cuLibraryUnload = f_lib_unload;
  d.cuLibraryGetKernel = f_lib_get_kernel;
  d.cuKernelGetFunction = f_kernel_get_fn;
  d.cuFuncLoad = f_func_load;
  d.cuFuncIsLoaded = f_func_is_loaded;
  d.cuFuncSetAttribute = f_func_set_attr;
  d.cuLaunchKernelEx = f_launch;
  d.cuTensorMapEncodeTiled = f_tmap_tiled;
  d.cuTensorMapEncodeIm2col = f_tmap_im2col;
  d.cuEventCreate = f_event_create;
  d.cuEventDestroy = f_event_destroy;
  d.cuEventRecord = f_event_record;
  d.cuEventSynchronize = f_event_sync;
  d.cuEventElapsedTime = f_event_elapsed;
  d.cuMemcpyHtoDAsync = f_h2d;
  d.cuMemcpyDtoHAsync = f_d2h;
  d.cuPointerGetAttribute = f_ptr_attr;
  d.cuStreamSynchronize = f_stream_sync;
  d.cuStreamCreate = f_stream_create;
  d.cuStreamDestroy = f_stream_destroy;
  d.cuStreamBeginCapture = f_begin_capture;
  d.cuStreamEndCapture = f_end_capture;
  d.cuGraphInstantiateWithFlags = f_graph_instantiate;
  d.cuGraphLaunch = f_graph_launch;
  d.cuGraphDestroy = f_graph_destroy;
  d.cuGraphExecDestroy = f_graph_exec_destroy;
  d.cuStreamWaitEvent = f_stream_wait_event;
  d.ok = true;
  return d;
}
Driver g_fake;

}  // namespace
}  // namespace pask

PASK_API int pask_test_fake_driver(int32_t enable, int32_t load_us, int32_t fail_kernel) {
  using namespace pask;
  std::lock_guard<std::mutex> lk(g_mu);
  g_load_us = load_us;
  g_fail_kernel = fail_kernel;
  g_ids.clear();
  g_kinds.clear();
  memset(g_loaded, 0, sizeof(g_loaded));
  g_next_stream.store(0x40);
  g_capture_stream.store(0);
  g_current.store(0x10);
  g_occupancy.store(1);
  g_max_cluster_z.store(0);
  g_primer_loads.store(0);
  if (enable) {
    g_fake = make_fake();
    driver_override(&g_fake);
  } else {
    driver_override(nullptr);
  }
  return 0;
}

PASK_API int32_t pask_test_fake_knob(int32_t knob, int32_t value) {
  using namespace pask;
  switch (knob) {
    case PASK_FAKE_OCCUPANCY: g_occupancy.store(value); return 0;
    case PASK_FAKE_CURRENT_DEVICE: g_current.store(0x10 + static_cast<uintptr_t>(value)); return 0;
    case PASK_FAKE_MAX_CLUSTER_LAUNCHED: return g_max_cluster_z.load();
    case PASK_FAKE_PRIMER_LOADS: return g_primer_loads.load();
    default: return -1;
  }
}

PASK_API int32_t pask_test_fake_log(int32_t* out, int32_t* kinds, int32_t cap) {
  using namespace pask;
  std::lock_guard<std::mutex> lk(g_mu);
  const int32_t n = static_cast<int32_t>(g_ids.size());
  for (int32_t i = 0; i < n && i < cap; ++i) {
    if (out) out[i] = g_ids[i];
    if (kinds) kinds[i] = g_kinds[i];
  }
  return n;
}
