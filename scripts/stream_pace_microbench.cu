// GPU-side pacing of chained launches (not part of the product): how long does
// the GPU take per kernel when 58 tiny PDL-chained kernels are queued behind a
// 2 ms spin kernel (so the host is never the bottleneck), by parameter-block
// size, PDL attribute, and stream launch vs CUDA-graph replay?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o spm stream_pace_microbench.cu -lcuda
#include <cuda.h>
#include <stdio.h>
#include <stdlib.h>

#include <vector>

#define CK(x)                                                          \
  do {                                                                 \
    CUresult r_ = (x);                                                 \
    if (r_ != CUDA_SUCCESS) {                                          \
      const char* s_;                                                  \
      cuGetErrorName(r_, &s_);                                         \
      fprintf(stderr, "%s:%d %s -> %s\n", __FILE__, __LINE__, #x, s_); \
      exit(1);                                                         \
    }                                                                  \
  } while (0)

struct Small { int a[4]; };
struct alignas(64) Big { CUtensorMap m[4]; long long x[24]; };

__device__ __forceinline__ void pdl() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  asm volatile("griddepcontrol.wait;" ::: "memory");
}
extern "C" __global__ void k_small(const __grid_constant__ Small p) {
  pdl();
  if (p.a[0] == 12345 && threadIdx.x == 0) printf("x");
}
extern "C" __global__ void k_big(const __grid_constant__ Big p) {
  pdl();
  if (p.x[0] == 12345 && threadIdx.x == 0) printf("x");
}
extern "C" __global__ void k_spin(long long cycles) {
  long long t0 = clock64();
  while (clock64() - t0 < cycles) {
  }
}

int main() {
  CK(cuInit(0));
  CUdevice dev;
  CK(cuDeviceGet(&dev, 0));
  CUcontext ctx;
  CK(cuDevicePrimaryCtxRetain(&ctx, dev));
  CK(cuCtxSetCurrent(ctx));
  CUmodule mod;
  CUfunction fs, fb, fspin;
  // this file's own kernels through the runtime-registered fatbin are not
  // reachable from the driver API; load them from the side-built cubin
  CK(cuModuleLoad(&mod, "spm.cubin"));
  CK(cuModuleGetFunction(&fs, mod, "k_small"));
  CK(cuModuleGetFunction(&fb, mod, "k_big"));
  CK(cuModuleGetFunction(&fspin, mod, "k_spin"));
  CUstream s;
  CK(cuStreamCreate(&s, CU_STREAM_NON_BLOCKING));
  CUevent e0, e1;
  CK(cuEventCreate(&e0, 0));
  CK(cuEventCreate(&e1, 0));
  Small ps{};
  Big pb{};
  const int n = 58;
  auto chain = [&](CUfunction f, void* par, bool pdl_attr, unsigned grid, unsigned block) {
    for (int i = 0; i < n; ++i) {
      CUlaunchAttribute a[1];
      a[0].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
      a[0].value.programmaticStreamSerializationAllowed = 1;
      CUlaunchConfig c{};
      c.gridDimX = grid;
      c.gridDimY = c.gridDimZ = 1;
      c.blockDimX = block;
      c.blockDimY = c.blockDimZ = 1;
      c.hStream = s;
      c.attrs = a;
      c.numAttrs = (pdl_attr && i > 0) ? 1 : 0;
      void* args[1] = {par};
      CK(cuLaunchKernelEx(&c, f, args, nullptr));
    }
  };
  long long spin = 4000000;  // ~2 ms
  void* sargs[1] = {&spin};
  for (int big = 0; big < 2; ++big)
    for (int pdl_attr = 0; pdl_attr < 2; ++pdl_attr)
      for (unsigned grid : {1u, 64u, 148u}) {
        CUfunction f = big ? fb : fs;
        void* par = big ? static_cast<void*>(&pb) : static_cast<void*>(&ps);
        // stream launches, GPU-paced: queued behind the spin kernel
        float best_stream = 1e9f, best_graph = 1e9f;
        for (int rep = 0; rep < 5; ++rep) {
          CK(cuLaunchKernel(fspin, 1, 1, 1, 32, 1, 1, 0, s, sargs, nullptr));
          CK(cuEventRecord(e0, s));
          chain(f, par, pdl_attr, grid, 352);
          CK(cuEventRecord(e1, s));
          CK(cuStreamSynchronize(s));
          float ms;
          CK(cuEventElapsedTime(&ms, e0, e1));
          if (ms < best_stream) best_stream = ms;
        }
        // the same chain captured in a graph
        CUgraph g;
        CUgraphExec ge;
        CK(cuStreamBeginCapture(s, CU_STREAM_CAPTURE_MODE_THREAD_LOCAL));
        chain(f, par, pdl_attr, grid, 352);
        CK(cuStreamEndCapture(s, &g));
        CK(cuGraphInstantiateWithFlags(&ge, g, 0));
        for (int rep = 0; rep < 5; ++rep) {
          CK(cuLaunchKernel(fspin, 1, 1, 1, 32, 1, 1, 0, s, sargs, nullptr));
          CK(cuEventRecord(e0, s));
          CK(cuGraphLaunch(ge, s));
          CK(cuEventRecord(e1, s));
          CK(cuStreamSynchronize(s));
          float ms;
          CK(cuEventElapsedTime(&ms, e0, e1));
          if (ms < best_graph) best_graph = ms;
        }
        CK(cuGraphExecDestroy(ge));
        CK(cuGraphDestroy(g));
        printf("params %4zu B  pdl %d  grid %3u x 352 : stream %.3f us/kernel  graph %.3f us/kernel\n",
               big ? sizeof(Big) : sizeof(Small), pdl_attr, grid, 1e3f * best_stream / n, 1e3f * best_graph / n);
      }
  return 0;
}
