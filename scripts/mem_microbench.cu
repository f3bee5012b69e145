// Per-SM memory-path microbenchmark (B200, sm_100a): cycles for one CTA to
//   (1) write B bytes with coalesced 16-byte STG, (2) write B bytes with one bulk
//   async copy smem->global (TMA engine), waiting for the smem read / the global
//   write, (3) read B bytes global->smem with bulk async copies (TMA ingest),
//   as a function of the number of concurrently active CTAs (one per SM).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mem_microbench mem_microbench.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ unsigned long long clk() { unsigned long long c; asm volatile("mov.u64 %0, %%clock64;" : "=l"(c)); return c; }

__global__ void k_stg(uint4* out, int bytes, unsigned long long* cyc) {
  unsigned long long t0 = clk();
  uint4* o = out + (size_t)blockIdx.x * (bytes / 16);
  for (int i = threadIdx.x; i < bytes / 16; i += blockDim.x) o[i] = make_uint4(i, 1, 2, 3);
  __syncthreads();
  unsigned long long t1 = clk();
  asm volatile("fence.acq_rel.gpu;" ::: "memory");  // writes globally performed
  __syncthreads();
  unsigned long long t2 = clk();
  if (threadIdx.x == 0) { cyc[blockIdx.x * 4] = t1 - t0; cyc[blockIdx.x * 4 + 1] = t2 - t0; }
}

__global__ void k_bulk_store(char* out, int bytes, unsigned long long* cyc) {
  extern __shared__ __align__(1024) unsigned char sm[];
  for (int i = threadIdx.x * 16; i < bytes; i += blockDim.x * 16) *(uint4*)(sm + i) = make_uint4(i, 1, 2, 3);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t0 = clk();
    char* dst = out + (size_t)blockIdx.x * bytes;
    for (int off = 0; off < bytes; off += 16384) {
      int n = bytes - off < 16384 ? bytes - off : 16384;
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + off), "r"(smem_u32(sm + off)), "r"(n) : "memory");
    }
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
    unsigned long long t1 = clk();
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    unsigned long long t2 = clk();
    cyc[blockIdx.x * 4] = t1 - t0;
    cyc[blockIdx.x * 4 + 1] = t2 - t0;
  }
}

__global__ void k_bulk_load(const char* in, int bytes, unsigned long long* cyc) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ __align__(8) unsigned long long bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t0 = clk();
    const char* src = in + (size_t)blockIdx.x * bytes;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar)), "r"(bytes) : "memory");
    for (int off = 0; off < bytes; off += 16384) {
      int n = bytes - off < 16384 ? bytes - off : 16384;
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(smem_u32(sm + off)), "l"(src + off), "r"(n), "r"(smem_u32(&bar)) : "memory");
    }
    uint32_t ok = 0;
    while (!ok) {
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(ok) : "r"(smem_u32(&bar)) : "memory");
    }
    unsigned long long t1 = clk();
    cyc[blockIdx.x * 4] = t1 - t0;
  }
}

static double med(std::vector<unsigned long long>& v, int n, int k) {
  std::vector<unsigned long long> a;
  for (int i = 0; i < n; ++i) a.push_back(v[i * 4 + k]);
  std::sort(a.begin(), a.end());
  return (double)a[a.size() / 2];
}

#include <algorithm>
int main() {
  const int maxb = 200 * 1024;
  char *buf, *src;
  unsigned long long* cyc;
  cudaMalloc(&buf, (size_t)148 * maxb);
  cudaMalloc(&src, (size_t)148 * maxb);
  cudaMemset(src, 1, (size_t)148 * maxb);
  cudaMalloc(&cyc, 148 * 4 * 8);
  cudaFuncSetAttribute(k_bulk_store, cudaFuncAttributeMaxDynamicSharedMemorySize, maxb);
  cudaFuncSetAttribute(k_bulk_load, cudaFuncAttributeMaxDynamicSharedMemorySize, maxb);
  std::vector<unsigned long long> h(148 * 4);
  int ctas_list[] = {1, 16, 64, 148};
  int bytes_list[] = {8192, 16384, 32768, 65536, 131072};
  printf("%-10s %5s %7s | %10s %10s | B/cyc(issue) B/cyc(done)\n", "kind", "ctas", "bytes", "issue_cyc", "done_cyc");
  for (int ctas : ctas_list)
    for (int bytes : bytes_list) {
      for (int rep = 0; rep < 3; ++rep) {  // warm: L2 resident source / TLB
        k_stg<<<ctas, 256>>>((uint4*)buf, bytes, cyc);
        cudaDeviceSynchronize();
      }
      cudaMemcpy(h.data(), cyc, 148 * 32, cudaMemcpyDeviceToHost);
      double a = med(h, ctas, 0), b = med(h, ctas, 1);
      printf("%-10s %5d %7d | %10.0f %10.0f | %6.1f %6.1f\n", "stg", ctas, bytes, a, b, bytes / a, bytes / b);
      for (int rep = 0; rep < 3; ++rep) {
        k_bulk_store<<<ctas, 256, bytes>>>(buf, bytes, cyc);
        cudaDeviceSynchronize();
      }
      cudaMemcpy(h.data(), cyc, 148 * 32, cudaMemcpyDeviceToHost);
      a = med(h, ctas, 0); b = med(h, ctas, 1);
      printf("%-10s %5d %7d | %10.0f %10.0f | %6.1f %6.1f\n", "bulk_st", ctas, bytes, a, b, bytes / a, bytes / b);
      for (int rep = 0; rep < 3; ++rep) {
        k_bulk_load<<<ctas, 32, bytes>>>(src, bytes, cyc);
        cudaDeviceSynchronize();
      }
      cudaMemcpy(h.data(), cyc, 148 * 32, cudaMemcpyDeviceToHost);
      a = med(h, ctas, 0);
      printf("%-10s %5d %7d | %10.0f %10s | %6.1f\n", "bulk_ld", ctas, bytes, a, "-", bytes / a);
    }
  cudaError_t e = cudaGetLastError();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
