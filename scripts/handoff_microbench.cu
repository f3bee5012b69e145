// Layer hand-off microbenchmark (not part of the product): how long does a
// chain of L dependent kernels take per link when the dependency is carried by
//   (a) plain stream order,
//   (b) PDL: griddepcontrol.launch_dependents early + griddepcontrol.wait,
//   (c) PDL launch + a device-scope completion counter (release/acquire) that
//       the next kernel's CTAs poll instead of griddepcontrol.wait?
// Each kernel: G CTAs x 256 threads; every CTA reads one value of the previous
// layer's output, writes its own 16 KB, then (c) bumps the layer counter.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o hmb handoff_microbench.cu
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <time.h>

#define CK(x)                                                                     \
  do {                                                                            \
    cudaError_t e_ = (x);                                                         \
    if (e_ != cudaSuccess) {                                                      \
      fprintf(stderr, "%s:%d %s -> %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
      exit(1);                                                                    \
    }                                                                             \
  } while (0)

struct P {
  const float* in;
  float* out;
  unsigned* cnt_prev;  // null: first layer
  unsigned* cnt_mine;
  unsigned target;     // value cnt_prev reaches when the previous layer is complete
  int mode;            // 0 stream, 1 pdl wait, 2 flag
  int work;            // extra per-thread loop iterations (simulated compute)
};

__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__global__ void __launch_bounds__(256) k_layer(const __grid_constant__ P p) {
  if (p.mode >= 1) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (p.mode == 1) asm volatile("griddepcontrol.wait;" ::: "memory");
  if (p.mode == 2 && p.cnt_prev) {
    if (threadIdx.x == 0)
      while (ld_acquire(p.cnt_prev) < p.target) {
      }
    __syncthreads();
  }
  float v = p.in[(blockIdx.x * 256 + threadIdx.x) % 4096];
  for (int i = 0; i < p.work; ++i) v = v * 1.0001f + 0.5f;
  float4* o = reinterpret_cast<float4*>(p.out) + blockIdx.x * 1024;
#pragma unroll
  for (int i = 0; i < 4; ++i) o[threadIdx.x + 256 * i] = make_float4(v, v, v, v);
  if (p.mode == 2) {
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(p.cnt_mine) : "memory");
    }
  }
}

// Same layer with a 640 B parameter block (four 128 B tensor maps + scalars, like
// GemmParams): does the parameter size cost host issue time or GPU launch latency?
struct alignas(64) PB {
  unsigned char maps[512];
  P p;
};
__global__ void __launch_bounds__(256) k_layer_big(const __grid_constant__ PB b) {
  const P& p = b.p;
  if (p.mode >= 1) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (p.mode == 1) asm volatile("griddepcontrol.wait;" ::: "memory");
  float v = p.in[(blockIdx.x * 256 + threadIdx.x) % 4096] + (b.maps[threadIdx.x] == 7 ? 1.f : 0.f);
  for (int i = 0; i < p.work; ++i) v = v * 1.0001f + 0.5f;
  float4* o = reinterpret_cast<float4*>(p.out) + blockIdx.x * 1024;
#pragma unroll
  for (int i = 0; i < 4; ++i) o[threadIdx.x + 256 * i] = make_float4(v, v, v, v);
}

// direct issue (no graph): host time per launch and GPU time per link, small vs big params
void direct_issue(cudaStream_t s, float** buf, int L, int G, bool big, cudaEvent_t e0, cudaEvent_t e1) {
  float best = 1e30f, host_best = 1e30f;
  for (int it = 0; it < 30; ++it) {
    CK(cudaStreamSynchronize(s));
    CK(cudaEventRecord(e0, s));
    auto t0 = clock();
    struct timespec a, z;
    clock_gettime(CLOCK_MONOTONIC, &a);
    for (int l = 0; l < L; ++l) {
      P p{buf[l], buf[l + 1], nullptr, nullptr, 0u, 1, 0};
      cudaLaunchConfig_t cfg{};
      cfg.gridDim = dim3(G);
      cfg.blockDim = dim3(256);
      cfg.stream = s;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      at[0].val.programmaticStreamSerializationAllowed = 1;
      cfg.attrs = at;
      cfg.numAttrs = l > 0 ? 1 : 0;
      if (big) {
        PB b{};
        b.p = p;
        CK(cudaLaunchKernelEx(&cfg, k_layer_big, b));
      } else {
        CK(cudaLaunchKernelEx(&cfg, k_layer, p));
      }
    }
    clock_gettime(CLOCK_MONOTONIC, &z);
    (void)t0;
    CK(cudaEventRecord(e1, s));
    CK(cudaEventSynchronize(e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    const float host_us = (z.tv_sec - a.tv_sec) * 1e6f + (z.tv_nsec - a.tv_nsec) / 1e3f;
    if (it >= 5) {
      if (ms < best) best = ms;
      if (host_us < host_best) host_best = host_us;
    }
  }
  printf("direct issue grid %3d params %4d B: host %.2f us/launch, GPU %.3f us/link (best of 25)\n", G,
         big ? (int)sizeof(PB) : (int)sizeof(P), host_best / L, 1e3f * best / L);
}

int main(int argc, char** argv) {
  const int L = 50;
  const int iters = 50;
  int grids[] = {16, 64, 148};
  float* buf[L + 1];
  for (int i = 0; i <= L; ++i) {
    CK(cudaMalloc(&buf[i], 148 * 1024 * 16));
    CK(cudaMemset(buf[i], 0, 148 * 1024 * 16));
  }
  unsigned* cnt;
  CK(cudaMalloc(&cnt, (L + 1) * sizeof(unsigned)));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  for (int G : {16, 64}) {
    direct_issue(s, buf, L, G, false, e0, e1);
    direct_issue(s, buf, L, G, true, e0, e1);
  }
  for (int work : {0, 2000}) {
    for (int G : grids) {
      for (int mode = 0; mode < 4; ++mode) {  // 3: pdl-wait with the 640 B parameter block
        // one CUDA graph per configuration: counter reset + the L-kernel chain
        cudaGraph_t g;
        cudaGraphExec_t ge;
        CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
        CK(cudaMemsetAsync(cnt, 0, (L + 1) * sizeof(unsigned), s));
        for (int l = 0; l < L; ++l) {
          P p{buf[l], buf[l + 1], l ? cnt + l - 1 : nullptr, cnt + l, (unsigned)G, mode == 3 ? 1 : mode, work};
          cudaLaunchConfig_t cfg{};
          cfg.gridDim = dim3(G);
          cfg.blockDim = dim3(256);
          cfg.stream = s;
          cudaLaunchAttribute at[1];
          at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
          at[0].val.programmaticStreamSerializationAllowed = 1;
          cfg.attrs = at;
          cfg.numAttrs = (mode >= 1 && l > 0) ? 1 : 0;
          if (mode == 3) {
            PB bp{};
            bp.p = p;
            CK(cudaLaunchKernelEx(&cfg, k_layer_big, bp));
          } else {
            CK(cudaLaunchKernelEx(&cfg, k_layer, p));
          }
        }
        CK(cudaStreamEndCapture(s, &g));
        CK(cudaGraphInstantiate(&ge, g, 0));
        float best = 1e30f, sum = 0.f;
        for (int it = 0; it < iters + 5; ++it) {
          CK(cudaEventRecord(e0, s));
          CK(cudaGraphLaunch(ge, s));
          CK(cudaEventRecord(e1, s));
          CK(cudaEventSynchronize(e1));
          float ms;
          CK(cudaEventElapsedTime(&ms, e0, e1));
          if (it >= 5) {
            sum += ms;
            if (ms < best) best = ms;
          }
        }
        CK(cudaGraphExecDestroy(ge));
        CK(cudaGraphDestroy(g));
        const char* nm[] = {"stream", "pdl-wait", "pdl-flag", "pdl-big"};
        printf("work %4d grid %3d %-9s  per link: mean %.3f us  best %.3f us\n", work, G, nm[mode],
               1e3f * sum / iters / L, 1e3f * best / L);
      }
    }
  }
  return 0;
}
