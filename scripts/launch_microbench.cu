// Driver-level microbenchmark for the cold path (not part of the product):
//   1. host cost of cuLaunchKernelEx vs parameter size and launch attributes
//   2. code-object load cost alone, concurrently with a launch burst, and with
//      two loader threads in parallel (driver-lock contention)
//   3. CUDA-graph replay cost of a 58-kernel chain
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o lmb launch_microbench.cu -lcuda -lpthread
#include <cuda.h>
#include <stdio.h>
#include <stdlib.h>

#include <atomic>
#include <chrono>
#include <fstream>
#include <iterator>
#include <thread>
#include <vector>

#define CK(x)                                                              \
  do {                                                                     \
    CUresult r_ = (x);                                                     \
    if (r_ != CUDA_SUCCESS) {                                              \
      const char* s_;                                                      \
      cuGetErrorName(r_, &s_);                                             \
      fprintf(stderr, "%s:%d %s -> %s\n", __FILE__, __LINE__, #x, s_);     \
      exit(1);                                                             \
    }                                                                      \
  } while (0)

struct Small { int a[4]; };
struct alignas(64) Big { CUtensorMap m[4]; long long x[24]; };

extern "C" __global__ void k_small(const __grid_constant__ Small p) {
  if (p.a[0] == 12345 && threadIdx.x == 0) printf("x");
}
extern "C" __global__ void k_spin(long long cycles) {
  long long t0 = clock64();
  while (clock64() - t0 < cycles) {
  }
}
extern "C" __global__ void k_big(const __grid_constant__ Big p) {
  if (p.x[0] == 12345 && threadIdx.x == 0) printf("x");
}

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

std::vector<char> readf(const char* p) {
  std::ifstream f(p, std::ios::binary);
  return std::vector<char>(std::istreambuf_iterator<char>(f), {});
}

int main(int argc, char** argv) {
  const char* dir = argc > 1 ? argv[1] : "paper_conf_dac_huangdxz25_b200/_build";
  CK(cuInit(0));
  CUdevice dev;
  CK(cuDeviceGet(&dev, 0));
  CUcontext ctx;
  CK(cuDevicePrimaryCtxRetain(&ctx, dev));
  CK(cuCtxSetCurrent(ctx));
  CUstream s;
  CK(cuStreamCreate(&s, CU_STREAM_NON_BLOCKING));
  // self module for k_small / k_big: obtain via runtime-less path: the kernels are in this
  // executable's fatbin; use cuModuleGetFunction through cudaGetFuncBySymbol equivalent:
  CUfunction fs, fb, fspin;
  {
    CUmodule m;
    std::string me = std::string(argv[0]);
    // load the microbench's own cubin (built alongside as lmb.cubin)
    std::vector<char> img = readf((me + ".cubin").c_str());
    CK(cuModuleLoadData(&m, img.data()));
    CK(cuModuleGetFunction(&fs, m, "k_small"));
    CK(cuModuleGetFunction(&fb, m, "k_big"));
    CK(cuModuleGetFunction(&fspin, m, "k_spin"));
  }
  Small sp{};
  Big bp{};
  void* as[1] = {&sp};
  void* ab[1] = {&bp};
  CUlaunchAttribute at[2];
  at[0].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
  at[0].value.programmaticStreamSerializationAllowed = 1;
  at[1].id = CU_LAUNCH_ATTRIBUTE_CLUSTER_DIMENSION;
  at[1].value.clusterDim.x = 1;
  at[1].value.clusterDim.y = 1;
  at[1].value.clusterDim.z = 2;
  auto bench_launch = [&](CUfunction f, void** args, int nattr, unsigned gz, const char* name) {
    CUlaunchConfig c{};
    c.gridDimX = 4;
    c.gridDimY = 1;
    c.gridDimZ = gz;
    c.blockDimX = 128;
    c.blockDimY = c.blockDimZ = 1;
    c.hStream = s;
    c.attrs = at;
    c.numAttrs = nattr;
    for (int i = 0; i < 200; ++i) CK(cuLaunchKernelEx(&c, f, args, nullptr));
    CK(cuStreamSynchronize(s));
    const int n = 2000;
    double t0 = now_us();
    for (int i = 0; i < n; ++i) CK(cuLaunchKernelEx(&c, f, args, nullptr));
    double t1 = now_us();
    CK(cuStreamSynchronize(s));
    double t2 = now_us();
    printf("launch %-28s host %.2f us/launch   gpu-paced %.2f us/launch\n", name, (t1 - t0) / n, (t2 - t0) / n);
  };
  bench_launch(fs, as, 0, 1, "small params");
  bench_launch(fb, ab, 0, 1, "640B params");
  bench_launch(fb, ab, 1, 1, "640B params + PDL");
  bench_launch(fb, ab, 2, 2, "640B params + PDL + cluster");

  // ---- graph of 58 launches
  {
    CUlaunchConfig c{};
    c.gridDimX = 4;
    c.gridDimY = c.gridDimZ = 1;
    c.blockDimX = 128;
    c.blockDimY = c.blockDimZ = 1;
    c.hStream = s;
    c.attrs = at;
    c.numAttrs = 1;
    CUgraph g;
    CK(cuStreamBeginCapture(s, CU_STREAM_CAPTURE_MODE_THREAD_LOCAL));
    for (int i = 0; i < 58; ++i) CK(cuLaunchKernelEx(&c, fb, ab, nullptr));
    CK(cuStreamEndCapture(s, &g));
    CUgraphExec ge;
    double t0 = now_us();
    CK(cuGraphInstantiate(&ge, g, 0));
    double t1 = now_us();
    for (int i = 0; i < 20; ++i) CK(cuGraphLaunch(ge, s));
    CK(cuStreamSynchronize(s));
    const int n = 200;
    double t2 = now_us();
    for (int i = 0; i < n; ++i) CK(cuGraphLaunch(ge, s));
    double t3 = now_us();
    CK(cuStreamSynchronize(s));
    double t4 = now_us();
    printf("graph(58) instantiate %.1f us, launch host %.2f us, gpu-paced %.2f us per graph\n", t1 - t0,
           (t3 - t2) / n, (t4 - t2) / n);
  }

  // ---- code-object loads
  const char* names[] = {"pask_layout", "pask_conv_igemm", "pask_pool", "pask_gemm", "pask_softmax",
                         "pask_conv_dw", "pask_pool_gavg", "pask_layernorm", "pask_conv_1x1"};
  std::vector<std::vector<char>> imgs;
  for (auto n : names) imgs.push_back(readf((std::string(dir) + "/" + n + ".fatbin").c_str()));
  auto load = [&](int i, double* lib_us, double* fn_us) {
    CUlibrary lib;
    CUkernel k;
    CUfunction f;
    CUlibraryOption o[1] = {CU_LIBRARY_BINARY_IS_PRESERVED};
    void* ov[1] = {(void*)1};
    double t0 = now_us();
    CK(cuLibraryLoadData(&lib, imgs[i].data(), nullptr, nullptr, 0, o, ov, 1));
    double t1 = now_us();
    CK(cuLibraryGetKernel(&k, lib, names[i]));
    CK(cuKernelGetFunction(&f, k));
    CK(cuFuncLoad(f));
    double t2 = now_us();
    *lib_us = t1 - t0;
    *fn_us = t2 - t1;
  };
  // (a) alone, sequential: kernels 0..4
  {
    double tot = 0;
    for (int i = 0; i < 5; ++i) {
      double a, b;
      load(i, &a, &b);
      tot += a + b;
      printf("load alone   %-16s lib %7.1f  fn %7.1f us\n", names[i], a, b);
    }
    printf("load alone total %.1f us\n", tot);
  }
  // (b) two loader threads in parallel: kernels 5,6 vs 7,8 (fresh objects)
  {
    double r[4][2];
    double t0 = now_us();
    std::thread th([&] {
      CK(cuCtxSetCurrent(ctx));
      load(5, &r[0][0], &r[0][1]);
      load(6, &r[1][0], &r[1][1]);
    });
    load(7, &r[2][0], &r[2][1]);
    load(8, &r[3][0], &r[3][1]);
    th.join();
    double t1 = now_us();
    printf("two loader threads: wall %.1f us; per load (lib+fn): %.1f %.1f | %.1f %.1f\n", t1 - t0,
           r[0][0] + r[0][1], r[1][0] + r[1][1], r[2][0] + r[2][1], r[3][0] + r[3][1]);
  }
  // (c) loading while another thread launches a burst
  {
    std::atomic<bool> go{false}, done{false};
    double burst_us = 0;
    int launched = 0;
    std::thread th([&] {
      CK(cuCtxSetCurrent(ctx));
      CUlaunchConfig c{};
      c.gridDimX = 4;
      c.gridDimY = c.gridDimZ = 1;
      c.blockDimX = 128;
      c.blockDimY = c.blockDimZ = 1;
      c.hStream = s;
      c.attrs = at;
      c.numAttrs = 1;
      while (!go.load()) {
      }
      double t0 = now_us();
      while (!done.load()) {
        CK(cuLaunchKernelEx(&c, fb, ab, nullptr));
        ++launched;
      }
      burst_us = now_us() - t0;
    });
    // reload images 0..4 into new libraries while launching
    go.store(true);
    double tot = 0;
    for (int i = 0; i < 5; ++i) {
      double a, b;
      load(i, &a, &b);
      tot += a + b;
      printf("load+launch  %-16s lib %7.1f  fn %7.1f us\n", names[i], a, b);
    }
    done.store(true);
    th.join();
    CK(cuStreamSynchronize(s));
    printf("load during launch burst total %.1f us; launcher did %d launches in %.1f us (%.2f us each)\n", tot,
           launched, burst_us, burst_us / launched);
  }
  // (d) loading while the GPU is busy (a ~2 ms spin kernel on 148 CTAs)
  {
    long long cyc = 4000000;
    void* sa[1] = {&cyc};
    CUlaunchConfig c{};
    c.gridDimX = 148;
    c.gridDimY = c.gridDimZ = 1;
    c.blockDimX = 128;
    c.blockDimY = c.blockDimZ = 1;
    c.hStream = s;
    c.numAttrs = 0;
    CK(cuLaunchKernelEx(&c, fspin, sa, nullptr));
    double t0 = now_us();
    double tot = 0;
    // fresh libraries of kernels 0..4 again
    for (int i = 0; i < 5; ++i) {
      double a, b;
      load(i, &a, &b);
      tot += a + b;
      printf("load busyGPU %-16s lib %7.1f  fn %7.1f us\n", names[i], a, b);
    }
    double t1 = now_us();
    CK(cuStreamSynchronize(s));
    double t2 = now_us();
    printf("loads while GPU busy: %.1f us (GPU finished %.1f us after launch)\n", t1 - t0, t2 - t0);
  }
  // (d2) variants: 1-CTA spin on the same stream; 148-CTA spin on ANOTHER stream
  for (int variant = 0; variant < 2; ++variant) {
    long long cyc = 2000000;
    void* sa[1] = {&cyc};
    CUstream s2;
    CK(cuStreamCreate(&s2, CU_STREAM_NON_BLOCKING));
    CUlaunchConfig c{};
    c.gridDimX = variant == 0 ? 1 : 148;
    c.gridDimY = c.gridDimZ = 1;
    c.blockDimX = 128;
    c.blockDimY = c.blockDimZ = 1;
    c.hStream = variant == 0 ? s : s2;
    CK(cuLaunchKernelEx(&c, fspin, sa, nullptr));
    // a fresh library of kernel 5 / 6
    double a, b;
    double t0 = now_us();
    load(5 + variant, &a, &b);
    double t1 = now_us();
    CK(cuCtxSynchronize());
    double t2 = now_us();
    printf("load while %s: lib %.1f fn %.1f us (spin done %.1f us after)\n",
           variant == 0 ? "1-CTA spin, same stream" : "148-CTA spin, other stream", a, b, t2 - t0);
  }
  // (e) launch cost while the GPU is busy (queueing behind the spin kernel)
  {
    long long cyc = 4000000;
    void* sa[1] = {&cyc};
    CUlaunchConfig c{};
    c.gridDimX = 148;
    c.gridDimY = c.gridDimZ = 1;
    c.blockDimX = 128;
    c.blockDimY = c.blockDimZ = 1;
    c.hStream = s;
    CK(cuLaunchKernelEx(&c, fspin, sa, nullptr));
    CUlaunchConfig c2 = c;
    c2.gridDimX = 4;
    c2.attrs = at;
    c2.numAttrs = 1;
    double t0 = now_us();
    for (int i = 0; i < 100; ++i) CK(cuLaunchKernelEx(&c2, fb, ab, nullptr));
    double t1 = now_us();
    CK(cuStreamSynchronize(s));
    printf("100 PDL launches queued behind a busy GPU: %.2f us each\n", (t1 - t0) / 100);
  }
  return 0;
}
