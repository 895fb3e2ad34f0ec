// Per-class-step cost of the single-CTA local-search skeleton on sm_100a
// (512 pairs per class = S 1024).  Each class every thread evaluates PPT pairs
// (u0+k, u0-k) mod m from shared-memory t-value windows, then the CTA
// synchronises.  VAR 0: plain __syncthreads + smem any-flag; VAR 1:
// __syncthreads_or; VAR 2: VAR 0 + swap path (warp exchange) taken by
// one lane in ~1/swap_every of the pair evaluations.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int NCLS = 20000, NPAIRS = 512, K = 20, SP = 1025;

template <int VAR, int PPT>
__global__ void k_class(int m, long long* out, int* sink, int swap_every) {
  extern __shared__ int sm[];
  int* W = sm;                    // [K][SP]
  int* R = sm + K * SP;           // [1024]
  int* flag = R + 1024;           // [2]
  const int tid = threadIdx.x, T = blockDim.x, lane = tid & 31;
  for (int i = tid; i < K * SP; i += T) W[i] = (i * 7919) % 1000 + 10;
  for (int i = tid; i < 1024; i += T) R[i] = i;
  if (tid < 2) flag[tid] = 0;
  __syncthreads();
  int u[PPT], v[PPT];
#pragma unroll
  for (int q = 0; q < PPT; ++q) { const int k = tid + q * T; u[q] = (k + 1) % m; v[q] = (m - k - 1 + m) % m; }
  int acc = 0;
  long long t0 = clock64();
  for (int c = 0; c < NCLS; ++c) {
    const int j = c % (K - 4);
    int fire = 0;
#pragma unroll
    for (int q = 0; q < PPT; ++q) {
      const int tu = W[j * SP + u[q]], tv = W[j * SP + v[q]];
      int f = tu + tv < 0;
      if (VAR == 2) f |= (((c * 131 + (tid + q * T) * 7) * 2654435761u) & (unsigned)swap_every) == 0u;   // swap_every = 2^k - 1
      if (VAR == 2) {
        if (f) { const int a = R[u[q]], b = R[v[q]]; R[u[q]] = b; R[v[q]] = a; }
        unsigned mask = __ballot_sync(0xffffffffu, f);
        while (mask) {
          const int sl = __ffs(mask) - 1; mask &= mask - 1;
          const int su = __shfl_sync(0xffffffffu, u[q], sl), sv = __shfl_sync(0xffffffffu, v[q], sl);
          for (int jj = j + 1 + lane; jj < K - 4; jj += 32) {
            int* Wu = W + jj * SP + su; int* Wv = W + jj * SP + sv;
            const int a = *Wu, b = *Wv; *Wu = b; *Wv = a;
          }
        }
      }
      fire |= f;
    }
    if (VAR == 1) {
      acc += __syncthreads_or(fire);
    } else {
      if (fire) flag[c & 1] = 1;
      __syncthreads();
      acc += flag[c & 1];
      if (tid == 0) flag[(c + 1) & 1] = 0;
    }
#pragma unroll
    for (int q = 0; q < PPT; ++q) { u[q] = (u[q] + 1 == m) ? 0 : u[q] + 1; v[q] = (v[q] + 1 == m) ? 0 : v[q] + 1; }
  }
  long long t1 = clock64();
  if (tid == 0) { out[0] = (t1 - t0) / NCLS; *sink = acc; }
}

template <int VAR, int PPT>
long long run(int se) {
  long long* out; int* sink; long long r = 0;
  cudaMalloc(&out, 64); cudaMalloc(&sink, 4);
  const size_t smem = (K * SP + 1024 + 8) * 4;
  cudaFuncSetAttribute(k_class<VAR, PPT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  for (int w = 0; w < 2; ++w) {
    k_class<VAR, PPT><<<1, NPAIRS / PPT, smem>>>(1023, out, sink, se);
    cudaMemcpy(&r, out, 8, cudaMemcpyDeviceToHost);
  }
  cudaFree(out); cudaFree(sink);
  return r;
}

int main() {
  printf("PPT threads | syncthreads+flag | syncthreads_or | +swap path never | 1/4096 | 1/512 | 1/128\n");
#define ROW(P) printf("%3d %5d     | %6lld           | %6lld         | %6lld           | %6lld | %6lld | %6lld\n", P, NPAIRS / P, \
    run<0, P>(1), run<1, P>(1), run<2, P>(-1), run<2, P>(4095), run<2, P>(511), run<2, P>(127));
  ROW(1) ROW(2) ROW(4) ROW(8) ROW(16)
  printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
