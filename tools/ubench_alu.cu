// Issue-rate microbenchmark for the byte-SAD candidates on sm_100a (B200).
// Measures per-SM throughput of VABSDIFF4.U8.ACC (vabsdiff4...add), the
// two-instruction __vabsdiffu4 + IDP.4A form, IDP.4A alone and IADD3 as a
// reference ALU op.  Whole-grid, 148*k CTAs, CUDA-event timed; prints
// ops/clk/SM using the SM clock read from the device during the run.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define ITERS 4096
#define CH 16

template <int KIND>
__global__ void __launch_bounds__(256) k_alu(const uint32_t* __restrict__ in, uint32_t* out, long long* clk) {
  uint32_t a[CH], b = in[threadIdx.x & 31] ^ 0x5a5a5a5a;
#pragma unroll
  for (int i = 0; i < CH; ++i) a[i] = in[(threadIdx.x + i) & 63];
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) {
      if (KIND == 0) {
        asm volatile("vabsdiff4.u32.u32.u32.add %0, %1, %2, %0;" : "+r"(a[i]) : "r"(b), "r"(a[(i + 1) % CH]));
      } else if (KIND == 1) {
        uint32_t t = __vabsdiffu4(b, a[(i + 1) % CH]);
        a[i] = __dp4a(t, 0x01010101u, a[i]);
      } else if (KIND == 2) {
        asm volatile("dp4a.u32.u32 %0, %1, %2, %0;" : "+r"(a[i]) : "r"(b), "r"(a[(i + 1) % CH]));
      } else {
        asm volatile("add.u32 %0, %0, %1;" : "+r"(a[i]) : "r"(b));
      }
    }
  }
  long long t1 = clock64();
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += a[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0 && blockIdx.x == 0) *clk = t1 - t0;
}

int main() {
  int dev = 0; cudaDeviceProp p; cudaGetDeviceProperties(&p, dev);
  int sms = p.multiProcessorCount;
  uint32_t *in, *out; long long* clk;
  cudaMalloc(&in, 256 * 4); cudaMemset(in, 0x37, 256 * 4);
  cudaMalloc(&out, sizeof(uint32_t) * 256 * sms * 8);
  cudaMalloc(&clk, 8);
  const char* names[4] = {"vabsdiff4.add (VABSDIFF4.U8.ACC)", "__vabsdiffu4+__dp4a (2 instr)", "dp4a (IDP.4A)", "add.u32 (IADD3)"};
  for (int kind = 0; kind < 4; ++kind) {
    for (int occ : {4, 8}) {
      int grid = sms * occ;
      cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
      for (int w = 0; w < 2; ++w) {
        cudaEventRecord(e0);
        if (kind == 0) k_alu<0><<<grid, 256>>>(in, out, clk);
        if (kind == 1) k_alu<1><<<grid, 256>>>(in, out, clk);
        if (kind == 2) k_alu<2><<<grid, 256>>>(in, out, clk);
        if (kind == 3) k_alu<3><<<grid, 256>>>(in, out, clk);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
      }
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      long long c; cudaMemcpy(&c, clk, 8, cudaMemcpyDeviceToHost);
      double instr = (double)grid * 256 * ITERS * CH * (kind == 1 ? 2 : 1);
      double ops_per_s = (double)grid * 256 * ITERS * CH / (ms * 1e-3);
      // clock-normalised: one CTA's clock64 span; occ CTAs per SM run concurrently
      double per_clk_sm = (double)occ * 256 * ITERS * CH / (double)c;
      printf("%-34s occ=%d  %.3f ms  %.3e ops/s  ~%.1f ops/clk/SM (clock64)  eff_MHz=%.0f  instr=%.2e\n",
             names[kind], occ, ms, ops_per_s, per_clk_sm,
             (double)c / (ms * 1e-3) / 1e6, instr);
    }
  }
  printf("SMs=%d clockRate(kHz)=%d\n", sms, p.clockRate);
  return 0;
}
