// k_hist.cu -- adjusting the input image's intensity distribution to the
// target's before Step 1 (Sec. II; reading R12): per channel, level k
// of the input becomes the smallest level z with C_T(z) >= C_I(k), C_I and
// C_T the cumulative pixel counts of the two images (histogram
// specification of the paper's ref. [10] on counts: exact integers).
//
// Three launches, all HBM-bound on the 2 N^2 C image bytes:
//   k_hist_count -- both histograms per channel: shared-memory counters per
//                   CTA (16-byte loads, channel = byte index mod C), one
//                   64-bit global atomic per non-empty bin per CTA;
//   k_hist_map   -- one CTA per channel: block prefix sums of the two
//                   histograms, then each level's target by binary search
//                   over C_T (monotone);
//   k_hist_apply -- out = map[channel][in], 16-byte loads/stores.
#include <cuda_runtime.h>

#include "pm_internal.cuh"

namespace pm {

constexpr int kHistThreads = 256;
constexpr int kHistMaxC = 4;

__global__ void __launch_bounds__(kHistThreads) k_hist_count(const uint8_t* __restrict__ I,
                                                            const uint8_t* __restrict__ T, int64_t nbytes,
                                                            int32_t C, unsigned long long* __restrict__ hist) {
  __shared__ unsigned int s_h[2 * kHistMaxC * 256];
  for (int i = threadIdx.x; i < 2 * C * 256; i += blockDim.x) s_h[i] = 0;
  __syncthreads();
  const bool vec = ((reinterpret_cast<uintptr_t>(I) | reinterpret_cast<uintptr_t>(T)) & 15) == 0;
  const int64_t nvec = vec ? nbytes / 16 : 0;
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += (int64_t)gridDim.x * blockDim.x) {
    const uint4 a = __ldg(reinterpret_cast<const uint4*>(I) + v);
    const uint4 b = __ldg(reinterpret_cast<const uint4*>(T) + v);
    const uint32_t wa[4] = {a.x, a.y, a.z, a.w}, wb[4] = {b.x, b.y, b.z, b.w};
    int c = (int)((v * 16) % C);
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      atomicAdd(&s_h[c * 256 + ((wa[q >> 2] >> (8 * (q & 3))) & 0xff)], 1u);
      atomicAdd(&s_h[(C + c) * 256 + ((wb[q >> 2] >> (8 * (q & 3))) & 0xff)], 1u);
      c = (c + 1 == C) ? 0 : c + 1;
    }
  }
  for (int64_t i = nvec * 16 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nbytes;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(i % C);
    atomicAdd(&s_h[c * 256 + I[i]], 1u);
    atomicAdd(&s_h[(C + c) * 256 + T[i]], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 2 * C * 256; i += blockDim.x)
    if (s_h[i]) atomicAdd(hist + i, (unsigned long long)s_h[i]);
}

__global__ void __launch_bounds__(256) k_hist_map(const unsigned long long* __restrict__ hist, int32_t C,
                                                  uint8_t* __restrict__ map) {
  __shared__ unsigned long long s_cI[256], s_cT[256];
  const int c = blockIdx.x, k = threadIdx.x;
  // inclusive prefix sums (Hillis-Steele over 256 entries)
  s_cI[k] = hist[c * 256 + k];
  s_cT[k] = hist[(C + c) * 256 + k];
  __syncthreads();
  for (int o = 1; o < 256; o <<= 1) {
    const unsigned long long a = k >= o ? s_cI[k - o] : 0ull, b = k >= o ? s_cT[k - o] : 0ull;
    __syncthreads();
    s_cI[k] += a;
    s_cT[k] += b;
    __syncthreads();
  }
  // smallest z with C_T(z) >= C_I(k) (C_T(255) = N^2 >= C_I(k): always found)
  const unsigned long long need = s_cI[k];
  int lo = 0, hi = 255;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (s_cT[mid] >= need) hi = mid;
    else lo = mid + 1;
  }
  map[c * 256 + k] = (uint8_t)lo;
}

__global__ void __launch_bounds__(kHistThreads) k_hist_apply(const uint8_t* I, int64_t nbytes, int32_t C,
                                                            const uint8_t* __restrict__ map, uint8_t* out) {
  __shared__ uint8_t s_map[kHistMaxC * 256];
  for (int i = threadIdx.x; i < C * 256; i += blockDim.x) s_map[i] = map[i];
  __syncthreads();
  const bool vec = ((reinterpret_cast<uintptr_t>(I) | reinterpret_cast<uintptr_t>(out)) & 15) == 0;
  const int64_t nvec = vec ? nbytes / 16 : 0;
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += (int64_t)gridDim.x * blockDim.x) {
    const uint4 a = reinterpret_cast<const uint4*>(I)[v];   // (out may alias I: element-wise)
    uint32_t w[4] = {a.x, a.y, a.z, a.w}, r[4] = {0u, 0u, 0u, 0u};
    int c = (int)((v * 16) % C);
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      r[q >> 2] |= (uint32_t)s_map[c * 256 + ((w[q >> 2] >> (8 * (q & 3))) & 0xff)] << (8 * (q & 3));
      c = (c + 1 == C) ? 0 : c + 1;
    }
    reinterpret_cast<uint4*>(out)[v] = make_uint4(r[0], r[1], r[2], r[3]);
  }
  for (int64_t i = nvec * 16 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nbytes;
       i += (int64_t)gridDim.x * blockDim.x)
    out[i] = s_map[(int)(i % C) * 256 + I[i]];
}

int32_t hist_max_channels() { return kHistMaxC; }

pm_status_t run_histogram_match(const uint8_t* I, const uint8_t* T, int32_t N, int32_t C, uint8_t* out,
                                cudaStream_t st) {
  if (C < 1 || C > kHistMaxC) return PM_ERR_UNSUPPORTED;
  const int64_t nbytes = (int64_t)N * N * C;
  ScopedScratch buf(st);
  const size_t hb = sizeof(unsigned long long) * 2 * C * 256;
  PM_CUDA_TRY(scratch_alloc(&buf.p, hb + 256 * C, st));
  unsigned long long* hist = buf.as<unsigned long long>();
  uint8_t* map = reinterpret_cast<uint8_t*>(buf.as<char>() + hb);
  PM_CUDA_TRY(cudaMemsetAsync(hist, 0, hb, st));
  int64_t blocks = (nbytes / 16 + kHistThreads - 1) / kHistThreads;
  if (blocks > 148 * 4) blocks = 148 * 4;
  if (blocks < 1) blocks = 1;
  k_hist_count<<<(unsigned)blocks, kHistThreads, 0, st>>>(I, T, nbytes, C, hist);
  k_hist_map<<<C, 256, 0, st>>>(hist, C, map);
  k_hist_apply<<<(unsigned)blocks, kHistThreads, 0, st>>>(I, nbytes, C, map, out);
  note_launch(3);
  PM_CUDA_TRY(cudaGetLastError());
  return PM_OK;
}

}  // namespace pm
