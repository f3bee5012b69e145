// CUDA driver API resolved at run time (dlopen("libcuda.so.1") +
// cuGetProcAddress), so libpask.so loads on machines without a GPU driver
// (the host-only planner entry points then still work) and so tests can
// substitute a fake driver table for the loader / issuer logic.
#pragma once
#include <cuda.h>

namespace pask {

struct Driver {
#define PASK_DRV_FN(name) decltype(&::name) name = nullptr;
  PASK_DRV_FN(cuInit)
  PASK_DRV_FN(cuGetErrorName)
  PASK_DRV_FN(cuDeviceGet)
  PASK_DRV_FN(cuDeviceGetAttribute)
  PASK_DRV_FN(cuDevicePrimaryCtxRetain)
  PASK_DRV_FN(cuDevicePrimaryCtxRelease)
  PASK_DRV_FN(cuCtxGetCurrent)
  PASK_DRV_FN(cuCtxSetCurrent)
  PASK_DRV_FN(cuLibraryLoadData)
  PASK_DRV_FN(cuLibraryUnload)
  PASK_DRV_FN(cuLibraryGetKernel)
  PASK_DRV_FN(cuKernelGetFunction)
  PASK_DRV_FN(cuFuncLoad)
  PASK_DRV_FN(cuFuncIsLoaded)
  PASK_DRV_FN(cuFuncSetAttribute)
  PASK_DRV_FN(cuLaunchKernelEx)
  PASK_DRV_FN(cuTensorMapEncodeTiled)
  PASK_DRV_FN(cuTensorMapEncodeIm2col)
  PASK_DRV_FN(cuEventCreate)
  PASK_DRV_FN(cuEventDestroy)
  PASK_DRV_FN(cuEventRecord)
  PASK_DRV_FN(cuEventSynchronize)
  PASK_DRV_FN(cuEventElapsedTime)
  PASK_DRV_FN(cuMemcpyHtoDAsync)
  PASK_DRV_FN(cuMemcpyDtoHAsync)
  PASK_DRV_FN(cuStreamSynchronize)
  PASK_DRV_FN(cuStreamCreate)
  PASK_DRV_FN(cuStreamDestroy)
  PASK_DRV_FN(cuStreamWaitEvent)
  PASK_DRV_FN(cuStreamBeginCapture)
  PASK_DRV_FN(cuStreamEndCapture)
  PASK_DRV_FN(cuGraphInstantiateWithFlags)
  PASK_DRV_FN(cuGraphLaunch)
  PASK_DRV_FN(cuGraphDestroy)
  PASK_DRV_FN(cuGraphExecDestroy)
  PASK_DRV_FN(cuCtxGetDevice)
  PASK_DRV_FN(cuOccupancyMaxActiveClusters)
  PASK_DRV_FN(cuMemAlloc)
  PASK_DRV_FN(cuMemFree)
  PASK_DRV_FN(cuMemsetD8)
  PASK_DRV_FN(cuMemcpyDtoH)
  PASK_DRV_FN(cuPointerGetAttribute)
#undef PASK_DRV_FN
  bool ok = false;
};

// Resolve the driver once (thread-safe).  Returns nullptr and sets *why when
// libcuda is unavailable.
const Driver* driver(const char** why);

// Tests: replace the resolved driver table (nullptr restores the real one).
void driver_override(const Driver* fake);

}  // namespace pask
