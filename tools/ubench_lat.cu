// Latency probes for the local-search design on sm_100a (B200):
//  (1) dependent global-load chain (pointer chase) in an L2-resident / L1-resident buffer
//  (2) __syncthreads() round trip at 128..1024 threads
//  (3) cp.async 4B + wait_all round trip (L2-resident source)
//  (4) smem read -> dependent global load -> smem write -> barrier (one "class step")
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__global__ void chase(const int* __restrict__ nxt, int hops, long long* out, int* sink) {
  int p = 0;
  long long t0 = clock64();
  for (int i = 0; i < hops; ++i) p = __ldcg(nxt + p);   // L2 (bypass L1)
  long long t1 = clock64();
  int q = 0;
  long long t2 = clock64();
  for (int i = 0; i < hops; ++i) q = __ldca(nxt + q);   // L1-cacheable
  long long t3 = clock64();
  out[0] = (t1 - t0) / hops; out[1] = (t3 - t2) / hops; *sink = p + q;
}

__global__ void bar_loop(int iters, long long* out) {
  __shared__ int s[1024];
  s[threadIdx.x] = threadIdx.x;
  __syncthreads();
  long long t0 = clock64();
  int acc = 0;
  for (int i = 0; i < iters; ++i) {
    acc += s[(threadIdx.x + i) & 1023];
    s[threadIdx.x] = acc;
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (t1 - t0) / iters;
  if (acc == 12345) out[1] = acc;
}

__global__ void cpasync_loop(const int* __restrict__ src, int iters, long long* out) {
  __shared__ int s[1024];
  long long t0 = clock64();
  int off = 0;
  for (int i = 0; i < iters; ++i) {
    uint32_t d = (uint32_t)__cvta_generic_to_shared(&s[threadIdx.x]);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(d), "l"(src + ((off + threadIdx.x * 97) & ((1 << 20) - 1))));
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    off += s[threadIdx.x] & 7;
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) { out[0] = (t1 - t0) / iters; out[1] = off; }
}

// one "class step": s_r read -> dependent global gather -> smem write -> barrier
__global__ void step_loop(const int* __restrict__ E, int n, int iters, long long* out) {
  extern __shared__ int sr[];
  for (int i = threadIdx.x; i < n; i += blockDim.x) sr[i] = (i * 7919) % n;
  __syncthreads();
  long long t0 = clock64();
  for (int c = 0; c < iters; ++c) {
    int u = (threadIdx.x + c) % n;
    int a = sr[u];
    int e = __ldg(E + (long)a * n + u);
    sr[u] = (a + (e & 1)) % n;
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (t1 - t0) / iters;
}

int main() {
  const int N = 1 << 20;   // 4 MB
  std::vector<int> h(N);
  // random cycle with stride > line
  for (int i = 0; i < N; ++i) h[i] = (int)(((long long)i * 1000003LL + 12345) % N);
  int *d, *sink; long long* o;
  cudaMalloc(&d, N * 4); cudaMalloc(&sink, 4); cudaMalloc(&o, 64);
  cudaMemcpy(d, h.data(), N * 4, cudaMemcpyHostToDevice);
  long long r[2];
  for (int w = 0; w < 2; ++w) chase<<<1, 1>>>(d, 20000, o, sink);
  cudaMemcpy(r, o, 16, cudaMemcpyDeviceToHost);
  printf("pointer chase 4MB: ldcg(L2) %lld cyc/hop, ldca %lld cyc/hop\n", r[0], r[1]);
  for (int t : {128, 256, 512, 1024}) {
    bar_loop<<<1, t>>>(100000, o);
    cudaMemcpy(r, o, 16, cudaMemcpyDeviceToHost);
    printf("smem rd/wr + __syncthreads at %4d threads: %lld cyc/iter\n", t, r[0]);
  }
  for (int t : {128, 512, 1024}) {
    cpasync_loop<<<1, t>>>(d, 20000, o);
    cudaMemcpy(r, o, 16, cudaMemcpyDeviceToHost);
    printf("cp.async 4B + wait_all + bar at %4d threads: %lld cyc/iter\n", t, r[0]);
  }
  for (int n : {256, 1024}) {
    int* E; cudaMalloc(&E, (size_t)n * n * 4); cudaMemset(E, 0, (size_t)n * n * 4);
    for (int t : {128, 512}) {
      step_loop<<<1, t, n * 4>>>(E, n, 20000, o);
      cudaMemcpy(r, o, 16, cudaMemcpyDeviceToHost);
      printf("class-step probe n=%d threads=%d: %lld cyc/step\n", n, t, r[0]);
    }
    cudaFree(E);
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
