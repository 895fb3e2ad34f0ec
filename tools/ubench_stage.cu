// Single-SM staging throughput on sm_100a: copy B bytes from an L2-resident
// buffer into shared memory with (a) LDG.128 -> STS.128, (b) cp.async.cg 16 B,
// (c) cp.async.bulk (TMA 1D, one 4 KB chunk per elected thread).  One CTA of
// 512 threads; cycles per copy via clock64, averaged over reps.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int BYTES = 64 * 1024;

__global__ void __launch_bounds__(512) k_ldg(const int4* src, int reps, long long* out, int* sink) {
  extern __shared__ int4 sm4[];
  const int n = BYTES / 16;
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
    const int4* s = src + (r & 7) * n;
#pragma unroll 8
    for (int i = threadIdx.x; i < n; i += blockDim.x) sm4[i] = __ldg(s + i);
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) { out[0] = (t1 - t0) / reps; *sink = sm4[5].x; }
}

__global__ void __launch_bounds__(512) k_cpasync(const int4* src, int reps, long long* out, int* sink) {
  extern __shared__ int4 sm4[];
  const int n = BYTES / 16;
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
    const int4* s = src + (r & 7) * n;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
      uint32_t d = (uint32_t)__cvta_generic_to_shared(sm4 + i);
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(d), "l"(s + i));
    }
    asm volatile("cp.async.commit_group;\n" ::);
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) { out[0] = (t1 - t0) / reps; *sink = sm4[5].x; }
}

__global__ void __launch_bounds__(512) k_bulk(const int4* src, int reps, long long* out, int* sink) {
  extern __shared__ __align__(128) int4 sm4[];
  __shared__ __align__(8) unsigned long long bar;
  const int n = BYTES / 16;
  const int chunk = 4096;  // bytes per bulk copy
  const int nchunks = BYTES / chunk;
  uint32_t bar_s = (uint32_t)__cvta_generic_to_shared(&bar);
  if (threadIdx.x == 0) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(bar_s));
  __syncthreads();
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
    const char* s = reinterpret_cast<const char*>(src + (r & 7) * n);
    if (threadIdx.x == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(bar_s), "r"(BYTES));
    __syncthreads();
    if (threadIdx.x < nchunks) {
      uint32_t d = (uint32_t)__cvta_generic_to_shared(reinterpret_cast<char*>(sm4) + threadIdx.x * chunk);
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(d), "l"(s + threadIdx.x * chunk), "r"(chunk), "r"(bar_s) : "memory");
    }
    // wait phase r&1
    uint32_t done = 0;
    while (!done) {
      asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                   : "=r"(done) : "r"(bar_s), "r"(r & 1) : "memory");
    }
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) { out[0] = (t1 - t0) / reps; *sink = sm4[5].x; }
}

// transpose 64 KB smem row layout [1024][16] -> column layout [16][1025]
__global__ void __launch_bounds__(512) k_transpose(int reps, long long* out, int* sink) {
  extern __shared__ int sm[];
  int* a = sm;                 // [1024][16]
  int* b = sm + 1024 * 16;     // [16][1025]
  for (int i = threadIdx.x; i < 1024 * 16; i += blockDim.x) a[i] = i;
  __syncthreads();
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
#pragma unroll 8
    for (int f = threadIdx.x; f < 1024 * 16; f += blockDim.x) {
      const int x = f >> 4, j = f & 15;
      b[j * 1025 + x] = a[x * 16 + j] + r;
    }
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) { out[0] = (t1 - t0) / reps; *sink = b[77]; }
}

int main() {
  int4* src; long long* out; int* sink;
  cudaMalloc(&src, BYTES * 8); cudaMemset(src, 1, BYTES * 8);
  cudaMalloc(&out, 64); cudaMalloc(&sink, 4);
  long long r;
  cudaFuncSetAttribute(k_ldg, cudaFuncAttributeMaxDynamicSharedMemorySize, BYTES);
  cudaFuncSetAttribute(k_cpasync, cudaFuncAttributeMaxDynamicSharedMemorySize, BYTES);
  cudaFuncSetAttribute(k_bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, BYTES);
  cudaFuncSetAttribute(k_transpose, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * 1025 * 16 * 4 + 64);
  for (int w = 0; w < 2; ++w) {
    k_ldg<<<1, 512, BYTES>>>(src, 200, out, sink); cudaMemcpy(&r, out, 8, cudaMemcpyDeviceToHost);
    if (w) printf("LDG.128->STS.128  64 KB: %lld cycles (%.1f B/cycle)\n", r, (double)BYTES / r);
    k_cpasync<<<1, 512, BYTES>>>(src, 200, out, sink); cudaMemcpy(&r, out, 8, cudaMemcpyDeviceToHost);
    if (w) printf("cp.async.cg 16 B  64 KB: %lld cycles (%.1f B/cycle)\n", r, (double)BYTES / r);
    k_bulk<<<1, 512, BYTES>>>(src, 200, out, sink); cudaMemcpy(&r, out, 8, cudaMemcpyDeviceToHost);
    if (w) printf("cp.async.bulk 4KB 64 KB: %lld cycles (%.1f B/cycle)\n", r, (double)BYTES / r);
    k_transpose<<<1, 512, 2 * 1025 * 16 * 4 + 64>>>(200, out, sink); cudaMemcpy(&r, out, 8, cudaMemcpyDeviceToHost);
    if (w) printf("smem transpose 16K ints: %lld cycles\n", r);
  }
  printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
