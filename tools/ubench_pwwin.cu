// Quiet-round skeleton of PAIRWIN (S = 1024, 512 pairs, 1 CTA): per window of
// K = 16 classes: wait for this window's TU/TV rows (cp.async, double buffer),
// issue the next window's rows, test all K classes of the thread's fixed pair
// column (2 LDS + add + compare each), atomicMin, barrier.  Cycles per window.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int NPR = 512, K = 16, NWIN = 64 * 20, NCLS = 1023;

__device__ __forceinline__ void cp16(int* s, const int* g) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(s);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(d), "l"(g));
}

template <int VAR>
__global__ void __launch_bounds__(512, 1) k_pw(const int* __restrict__ TU, const int* __restrict__ TV, long long* out, int* sink) {
  extern __shared__ __align__(16) int sm[];
  int* buf = sm;                       // [2][2][K][NPR]
  int* ctl = sm + 4 * K * NPR;
  const int tid = threadIdx.x, T = blockDim.x;
  const int tsz = K * NPR;
  auto issue = [&](int wb, int b) {
    const int n16 = K * NPR / 4;
    for (int i = tid; i < n16; i += T) {
      cp16(buf + (2 * b) * tsz + 4 * i, TU + (size_t)wb * NPR + 4 * i);
      cp16(buf + (2 * b + 1) * tsz + 4 * i, TV + (size_t)wb * NPR + 4 * i);
    }
    asm volatile("cp.async.commit_group;\n" ::);
  };
  if (tid < 4) ctl[tid] = 0x7fffffff;
  issue(0, 0);
  int acc = 0;
  long long tw = 0, ts = 0;
  long long t00 = clock64();
  for (int w = 0; w < NWIN; ++w) {
    const int b = w & 1;
    long long t0 = clock64();
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    __syncthreads();
    long long t1 = clock64();
    issue(((w + 1) * K) % (NCLS - K), b ^ 1);
    const int* U = buf + (2 * b) * tsz;
    const int* V = U + tsz;
    unsigned hits = 0;
#pragma unroll
    for (int t = 0; t < K; ++t) {
      const int tu = U[t * NPR + tid], tv = V[t * NPR + tid];
      if (VAR == 0) hits |= ((long long)tu + tv < 0 ? 1u : 0u) << t;
      else hits |= (tu + tv < 0 ? 1u : 0u) << t;
    }
    if (hits) atomicMin(ctl + (w % 3), __ffs(hits) - 1);
    if (tid == 0) ctl[(w + 1) % 3] = 0x7fffffff;
    __syncthreads();
    acc += ctl[w % 3];
    long long t2 = clock64();
    tw += t1 - t0; ts += t2 - t1;
  }
  long long t3 = clock64();
  if (tid == 0) { out[0] = tw / NWIN; out[1] = ts / NWIN; out[2] = (t3 - t00) / NWIN; *sink = acc; }
}

int main() {
  int *TU, *TV; long long* out; int* sink; long long r[3];
  cudaMalloc(&TU, (size_t)NCLS * NPR * 4); cudaMalloc(&TV, (size_t)NCLS * NPR * 4);
  cudaMemset(TU, 1, (size_t)NCLS * NPR * 4); cudaMemset(TV, 1, (size_t)NCLS * NPR * 4);
  cudaMalloc(&out, 64); cudaMalloc(&sink, 4);
  const size_t smem = (4 * K * NPR + 8) * 4;
  const char* names[2] = {"int64 compare", "int32 compare"};
#define RUN(V) cudaFuncSetAttribute(k_pw<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); \
  for (int w = 0; w < 2; ++w) { k_pw<V><<<1, 512, smem>>>(TU, TV, out, sink); cudaMemcpy(r, out, 24, cudaMemcpyDeviceToHost); } \
  printf("%-16s wait %5lld  scan+issue %5lld  total %5lld cycles/window -> %.0f cycles/class\n", names[V], r[0], r[1], r[2], r[2] / 16.0);
  RUN(0) RUN(1)
  printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
