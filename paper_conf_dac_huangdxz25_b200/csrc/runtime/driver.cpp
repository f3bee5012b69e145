#include "driver.h"

#include <dlfcn.h>

#include <mutex>

namespace pask {

namespace {
Driver g_real;
const Driver* g_override = nullptr;
const char* g_why = "not initialised";
std::once_flag g_once;

using GetProc = CUresult (*)(const char*, void**, int, cuuint64_t, CUdriverProcAddressQueryResult*);

void resolve() {
  void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_LOCAL);
  if (!h) h = dlopen("libcuda.so", RTLD_NOW | RTLD_LOCAL);
  if (!h) {
    g_why = "libcuda.so.1 not found (no NVIDIA driver on this machine)";
    return;
  }
  auto gp = reinterpret_cast<GetProc>(dlsym(h, "cuGetProcAddress_v2"));
  if (!gp) {
    g_why = "cuGetProcAddress_v2 missing from libcuda";
    return;
  }
  bool all = true;
#define PASK_RESOLVE(name)                                                                    \
  {                                                                                         \
    void* fn = nullptr;                                                                     \
    CUdriverProcAddressQueryResult q;                                                       \
    if (gp(#name, &fn, CUDA_VERSION, CU_GET_PROC_ADDRESS_DEFAULT, &q) != CUDA_SUCCESS || !fn) \
      all = false;                                                                          \
    g_real.name = reinterpret_cast<decltype(g_real.name)>(fn);                              \
  }
  PASK_RESOLVE(cuInit)
  PASK_RESOLVE(cuGetErrorName)
  PASK_RESOLVE(cuDeviceGet)
  PASK_RESOLVE(cuDeviceGetAttribute)
  PASK_RESOLVE(cuDevicePrimaryCtxRetain)
  PASK_RESOLVE(cuDevicePrimaryCtxRelease)
  PASK_RESOLVE(cuCtxGetCurrent)
  PASK_RESOLVE(cuCtxSetCurrent)
  PASK_RESOLVE(cuLibraryLoadData)
  PASK_RESOLVE(cuLibraryUnload)
  PASK_RESOLVE(cuLibraryGetKernel)
  PASK_RESOLVE(cuKernelGetFunction)
  PASK_RESOLVE(cuFuncLoad)
  PASK_RESOLVE(cuFuncIsLoaded)
  PASK_RESOLVE(cuFuncSetAttribute)
  PASK_RESOLVE(cuLaunchKernelEx)
  PASK_RESOLVE(cuTensorMapEncodeTiled)
  PASK_RESOLVE(cuTensorMapEncodeIm2col)
  PASK_RESOLVE(cuEventCreate)
  PASK_RESOLVE(cuEventDestroy)
  PASK_RESOLVE(cuEventRecord)
  PASK_RESOLVE(cuEventSynchronize)
  PASK_RESOLVE(cuEventElapsedTime)
  PASK_RESOLVE(cuMemcpyHtoDAsync)
  PASK_RESOLVE(cuMemcpyDtoHAsync)
  PASK_RESOLVE(cuStreamSynchronize)
  PASK_RESOLVE(cuStreamCreate)
  PASK_RESOLVE(cuStreamDestroy)
  PASK_RESOLVE(cuStreamWaitEvent)
  PASK_RESOLVE(cuStreamBeginCapture)
  PASK_RESOLVE(cuStreamEndCapture)
  PASK_RESOLVE(cuGraphInstantiateWithFlags)
  PASK_RESOLVE(cuGraphLaunch)
  PASK_RESOLVE(cuGraphDestroy)
  PASK_RESOLVE(cuGraphExecDestroy)
  PASK_RESOLVE(cuCtxGetDevice)
  PASK_RESOLVE(cuOccupancyMaxActiveClusters)
  PASK_RESOLVE(cuMemAlloc)
  PASK_RESOLVE(cuMemFree)
  PASK_RESOLVE(cuMemsetD8)
  PASK_RESOLVE(cuMemcpyDtoH)
  PASK_RESOLVE(cuPointerGetAttribute)
#undef PASK_RESOLVE
  if (!all) {
    g_why = "a required CUDA driver entry point could not be resolved (driver too old?)";
    return;
  }
  g_real.ok = true;
  g_why = "";
}
}  // namespace

const Driver* driver(const char** why) {
  if (g_override) return g_override;
  std::call_once(g_once, resolve);
  if (!g_real.ok) {
    if (why) *why = g_why;
    return nullptr;
  }
  return &g_real;
}

void driver_override(const Driver* fake) { g_override = fake; }

}  // namespace pask
