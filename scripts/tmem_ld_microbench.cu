// TMEM read microbenchmark (not part of the product): how long do the epilogue
// warps of the contraction kernel take to read a 128-lane x 64-column fp32
// accumulator back from TMEM, by tcgen05.ld shape / batching / warp count?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o tlm tmem_ld_microbench.cu
#include <cuda.h>
#include <stdint.h>
#include <stdio.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

template <int N>
__device__ __forceinline__ void ld32x32b(uint32_t taddr, uint32_t* r);
template <>
__device__ __forceinline__ void ld32x32b<16>(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr)
      : "memory");
}
template <>
__device__ __forceinline__ void ld32x32b<32>(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
        "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
        "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr)
      : "memory");
}
__device__ __forceinline__ void ld_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// mode 0: each of 8 warps reads 2 chunks of 16 columns (x16, wait after each)
// mode 1: each of 8 warps reads its 32 columns with one x32
// mode 2: 4 warps (one per lane quarter) read 64 columns as 2 x32 + one wait
// mode 3: each of 8 warps issues its 2 x16 then one wait
// mode 4: 4 warps read 64 columns as 4 x16, wait after each
// mode 5: 8 warps, the contraction epilogue's pipelined pattern
extern "C" __global__ void __launch_bounds__(256, 1) tlm(int mode, unsigned long long* out, float* sink) {
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(smem_u32(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = slot;
  const int quarter = warp & 3, half = warp >> 2;
  const uint32_t taddr = tmem + (static_cast<uint32_t>(quarter * 32) << 16);
  uint32_t r[64];
  float acc = 0.f;
  __syncthreads();
  long long t0 = clock64();
  if (mode == 0) {
    for (int c = half; c < 4; c += 2) {
      ld32x32b<16>(taddr + c * 16, r);
      ld_wait();
      for (int i = 0; i < 16; ++i) acc += __uint_as_float(r[i]);
    }
  } else if (mode == 1) {
    ld32x32b<32>(taddr + half * 32, r);
    ld_wait();
    for (int i = 0; i < 32; ++i) acc += __uint_as_float(r[i]);
  } else if (mode == 2) {
    if (half == 0) {
      ld32x32b<32>(taddr, r);
      ld32x32b<32>(taddr + 32, r + 32);
      ld_wait();
      for (int i = 0; i < 64; ++i) acc += __uint_as_float(r[i]);
    }
  } else if (mode == 3) {
    ld32x32b<16>(taddr + half * 16, r);
    ld32x32b<16>(taddr + (half + 2) * 16, r + 16);
    ld_wait();
    for (int i = 0; i < 32; ++i) acc += __uint_as_float(r[i]);
  } else if (mode == 5) {
    // the contraction kernel's epilogue pattern: chunk c + 2 loaded while chunk c
    // is processed (copy, issue next, math, wait)
    ld32x32b<16>(taddr + half * 16, r);
    ld_wait();
    asm volatile("" : "+r"(r[0]), "+r"(r[1]), "+r"(r[15]));
    for (int c = half; c < 4; c += 2) {
      float v[16];
      for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
      const bool more = c + 2 < 4;
      if (more) ld32x32b<16>(taddr + (c + 2) * 16, r);
      for (int i = 0; i < 16; ++i) acc += fmaxf(v[i] + 1.f, 0.f);
      if (more) {
        ld_wait();
        asm volatile("" : "+r"(r[0]), "+r"(r[1]), "+r"(r[15]));
      }
    }
  } else {
    if (half == 0)
      for (int c = 0; c < 4; ++c) {
        ld32x32b<16>(taddr + c * 16, r);
        ld_wait();
        for (int i = 0; i < 16; ++i) acc += __uint_as_float(r[i]);
      }
  }
  long long t1 = clock64();
  if (lane == 0) out[blockIdx.x * 8 + warp] = static_cast<unsigned long long>(t1 - t0);
  if (acc == 12345.f) sink[threadIdx.x] = acc;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
}

#define CK(x)                                                          \
  do {                                                                 \
    CUresult r_ = (x);                                                 \
    if (r_ != CUDA_SUCCESS) {                                          \
      const char* s_;                                                  \
      cuGetErrorName(r_, &s_);                                         \
      fprintf(stderr, "%s:%d %s -> %s\n", __FILE__, __LINE__, #x, s_); \
      return 1;                                                        \
    }                                                                  \
  } while (0)

int main() {
  CK(cuInit(0));
  CUdevice dev;
  CK(cuDeviceGet(&dev, 0));
  CUcontext ctx;
  CK(cuDevicePrimaryCtxRetain(&ctx, dev));
  CK(cuCtxSetCurrent(ctx));
  CUmodule mod;
  CK(cuModuleLoad(&mod, "tlm.cubin"));
  CUfunction f;
  CK(cuModuleGetFunction(&f, mod, "tlm"));
  const int blocks = 148;
  CUdeviceptr out, sink;
  CK(cuMemAlloc(&out, blocks * 8 * 8));
  CK(cuMemAlloc(&sink, 256 * 4));
  const char* names[6] = {"8 warps, 2 x16 chunks, wait each", "8 warps, 1 x32", "4 warps, 2 x32 + one wait",
                          "8 warps, 2 x16 + one wait", "4 warps, 4 x16, wait each",
                          "8 warps, kernel's pipelined pattern"};
  for (int mode = 0; mode < 6; ++mode) {
    unsigned long long h[blocks * 8];
    unsigned long long best = ~0ull, worst_med = 0;
    for (int rep = 0; rep < 5; ++rep) {
      void* args[3] = {&mode, &out, &sink};
      CK(cuLaunchKernel(f, blocks, 1, 1, 256, 1, 1, 0, nullptr, args, nullptr));
      CK(cuCtxSynchronize());
      CK(cuMemcpyDtoH(h, out, sizeof(h)));
      unsigned long long mx = 0;
      for (int b = 0; b < blocks; ++b)
        for (int w = 0; w < 8; ++w) {
          const bool live = (mode == 2 || mode == 4) ? w < 4 : true;  // modes 0, 1, 3, 5: all 8
          if (live && h[b * 8 + w] > mx) mx = h[b * 8 + w];
        }
      if (mx < best) best = mx;
      worst_med = h[0];
    }
    printf("mode %d (%s): slowest warp %llu cycles (best of 5), block 0 warp 0 %llu\n", mode, names[mode], best,
           worst_med);
  }
  return 0;
}
