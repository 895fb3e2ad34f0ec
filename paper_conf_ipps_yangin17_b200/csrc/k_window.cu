// k_window.cu -- PM_LS_WINDOW: Algorithm 2 in one CTA whose
// E reads are streamed, coalesced, into a shared-memory window instead of
// gathered one entry per pair.
//
// Why: a pair (u, v) of class c needs O_c(u) = E[r[u]][p_c(u)] and O_c(v)
// (p_c = partner in class c; slot-indexed reading R5); it fires iff
// d[u] + d[v] > O_c(u) + O_c(v).  Gathering the two entries costs one L1tex
// wavefront each, so one SM spends ~S cycles per class on gathers alone
// (measured: 1071 cycles/class at S = 1024 for k_ls_cta).
//
// Observation: for a regular slot x (not the class's fixed point, not the
// special slot L = S-1 of even S) the partner is p_c(x) = (2c + 1 - x) mod m,
// so with sigma(q) = q * (m+1)/2 mod m (the inverse of 2 mod the odd m),
//   sigma(p_c(x)) = (c + sigma(1 - x)) mod m.
// Storing each row of E with its columns permuted by sigma,
//   Ep[t][pos] = E[t][2 pos mod m],
// makes slot x's entries for consecutive classes CONSECUTIVE in row r[x] of
// Ep.  A window of K classes is then one contiguous K-entry segment per slot:
// the CTA streams S*K entries per K classes with coalesced loads.  The
// remaining cases: the fixed point u0(c) of even S pairs with L and needs
// E[r[u0]][L] -> s_last[tile] = column L of E, kept in smem; slot L's partner
// u0(c) = (c + (m+1)/2) mod m walks the plain row E[r[L]][.] contiguously.
//
// Swaps move rows between slots: the two swapped slots reload the rest of
// their window segment (the only gathers on the critical path).
//
// Exact speculation: classes [c, c+B) are evaluated at once on the current
// state; if none fires, all B classes are done (their evaluation was exact,
// the state did not change); otherwise the first firing class c* was also
// evaluated exactly, is applied, and the search continues at c*+1.  B adapts
// (1 while swaps are dense, doubling while classes stay quiet), so late
// rounds cost ~1/K of a class step per class.  Results are bit-identical to
// the serial replay.
#include "pm_internal.cuh"

namespace pm {

constexpr int kWinThreads = 1024;

// Ep[t][pos] = E[t][(2 pos) mod m], pos in [0, m).
__global__ void k_permute_cols(const int32_t* __restrict__ E, int64_t ld, int32_t* __restrict__ Ep, int64_t ldp,
                               int32_t S, int32_t m) {
  const int64_t total = (int64_t)S * m;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t = i / m;
    const int32_t pos = (int32_t)(i - t * m);
    int32_t q = 2 * pos;
    if (q >= m) q -= m;
    Ep[t * ldp + pos] = __ldg(E + t * ld + q);
  }
}

template <int K>
struct WinSmem {
  static constexpr int KP = K + 1;  // padded row (conflict-free column access)
  static size_t bytes(int32_t S) { return sizeof(int32_t) * ((size_t)S * (4 + KP) + 64); }
};

template <int K>
__global__ void __launch_bounds__(kWinThreads, 1)
k_ls_window(const int32_t* __restrict__ E, int64_t ld, const int32_t* __restrict__ Ep, int64_t ldp, int32_t S,
            int32_t* __restrict__ perm, int32_t max_rounds, LsResult* out, int64_t* per_round, int32_t max_log) {
  constexpr int KP = K + 1;
  extern __shared__ int32_t sm[];
  int32_t* s_r = sm;               // r[x]: tile at slot x
  int32_t* s_d = s_r + S;          // d[x] = E[r[x]][x]
  int32_t* s_last = s_d + S;       // E[t][L] per tile t (even S)
  int32_t* s_p0 = s_last + S;      // sigma(1 - x) per regular slot
  int32_t* s_W = s_p0 + S;         // window [S][KP]
  int32_t* s_ctl = s_W + (size_t)S * KP;   // [0..2] first-fire slots, [8..40] reduction
  const Classes cl(S);
  const int32_t m = cl.m, H = cl.half;
  const bool even = (S % 2) == 0;
  const int32_t L = S - 1;
  const int tid = threadIdx.x, T = blockDim.x;

  // ---- permutation check, then d, s_last, s_p0 ----
  for (int32_t x = tid; x < S; x += T) s_d[x] = 0;
  __syncthreads();
  int bad = 0;
  for (int32_t u = tid; u < S; u += T) {
    const int32_t t = perm[u];
    s_r[u] = t;
    if (t < 0 || t >= S) bad = 1;
    else atomicAdd(&s_d[t], 1);
  }
  __syncthreads();
  for (int32_t x = tid; x < S; x += T)
    if (s_d[x] != 1) bad = 1;
  if (__syncthreads_or(bad)) {
    if (tid == 0) { out->status = PM_ERR_NOT_PERMUTATION; out->rounds = 0; out->swaps = 0; }
    return;
  }
  for (int32_t x = tid; x < S; x += T) {
    s_d[x] = __ldg(E + (int64_t)s_r[x] * ld + x);
    if (even) s_last[x] = __ldg(E + (int64_t)x * ld + L);
    int32_t q = 1 - x;
    q %= m; if (q < 0) q += m;
    s_p0[x] = (int32_t)(((int64_t)q * H) % m);
  }
  if (tid < 3) s_ctl[tid] = INT32_MAX;
  __syncthreads();

  // entry of slot x at class (wb + j), tile t
  auto win_src = [&](int32_t x, int32_t t, int32_t wb, int32_t j) -> const int32_t* {
    if (even && x == L) {
      int32_t col = wb + j + H;
      col %= m;
      return E + (int64_t)t * ld + col;
    }
    int32_t pos = wb + j + s_p0[x];
    pos %= m;
    return Ep + (int64_t)t * ldp + pos;
  };
  // reload slot x's window entries j in [j0, K) (after a swap gave it tile t)
  auto refresh = [&](int32_t x, int32_t t, int32_t wb, int32_t j0, int32_t jmax) {
    constexpr int CH = K < 8 ? K : 8;     // loads in flight per chunk
#pragma unroll
    for (int jc = 0; jc < K; jc += CH) {
      if (jc + CH <= j0 || jc >= jmax) continue;
      int32_t v[CH];
#pragma unroll
      for (int q = 0; q < CH; ++q) {
        const int j = jc + q;
        if (j >= j0 && j < jmax) v[q] = __ldg(win_src(x, t, wb, j));
      }
#pragma unroll
      for (int q = 0; q < CH; ++q) {
        const int j = jc + q;
        if (j >= j0 && j < jmax) s_W[x * KP + j] = v[q];
      }
    }
  };
  // evaluate pair k of class cc (window offset j); returns fire
  auto eval = [&](int32_t cc, int32_t k, int32_t j, int32_t& u, int32_t& v, int32_t& ou, int32_t& ov) -> bool {
    cl.pair(cc, k, u, v);
    if (even && k == 0) ou = s_last[s_r[u]];       // u = u0(cc), partner L
    else ou = s_W[u * KP + j];
    ov = s_W[v * KP + j];
    return (int64_t)s_d[u] + s_d[v] > (int64_t)ou + ov;
  };

  int32_t rounds = 0;
  int64_t total = 0;
  int status = PM_OK;
  uint32_t batch = 0;
  int32_t B = 1;
  for (;;) {                                           // Alg. 2 line 1
    int mysw = 0;
    int32_t c = 0;
    int32_t wb = INT32_MIN / 2;
    while (c < cl.ncls) {                              // line 3, classes in order
      if (c >= wb + K) {                               // stream the next window
        wb = c;
        const int32_t jmax = min(K, cl.ncls - wb);
        __syncthreads();
        for (int32_t f = tid; f < S * K; f += T) {
          const int32_t x = f / K, j = f - x * K;
          if (j < jmax) s_W[x * KP + j] = __ldg(win_src(x, s_r[x], wb, j));
        }
        __syncthreads();
      }
      const int32_t jmax = min(K, cl.ncls - wb);
      int32_t* first_slot = s_ctl + (batch % 3);
      if (tid == 0) s_ctl[(batch + 1) % 3] = INT32_MAX;
      ++batch;
      const int32_t cend = min(c + B, wb + jmax);
      int32_t cc = c;
      bool apply = true;
      if (cend - c > 1) {
        // speculative: all pairs of classes [c, cend) on the current state
        const int32_t nb = cend - c;
        const int32_t items = nb * cl.npairs;
        for (int32_t it = tid; it < items; it += T) {
          const int32_t jj = it / cl.npairs, k = it - jj * cl.npairs;
          int32_t u, v, ou, ov;
          if (eval(c + jj, k, c + jj - wb, u, v, ou, ov)) atomicMin(first_slot, jj);
        }
        __syncthreads();
        const int32_t first = *first_slot;
        if (first == INT32_MAX) {
          c = cend;
          B = min(2 * B, K);
          apply = false;
        } else {
          cc = c + first;
          B = first == 0 ? 1 : first;
        }
      }
      if (apply) {
        // exact step of class cc: evaluate, swap (line 6), refresh windows
        const int32_t j = cc - wb;
        int fired = 0;
        for (int32_t k = tid; k < cl.npairs; k += T) {
          int32_t u, v, ou, ov;
          if (eval(cc, k, j, u, v, ou, ov)) {
            const int32_t a = s_r[u], b = s_r[v];
            s_r[u] = b; s_r[v] = a;
            s_d[u] = ov; s_d[v] = ou;      // d[u] = E[b][u] = O(v), d[v] = E[a][v] = O(u)
            ++mysw;
            fired = 1;
            if (j + 1 < jmax) {
              refresh(u, b, wb, j + 1, jmax);
              refresh(v, a, wb, j + 1, jmax);
            }
          }
        }
        const int any = __syncthreads_or(fired);
        if (cend - c <= 1 && !any) B = 2;               // quiet class: start speculating
        c = cc + 1;
      }
    }
    // round end: count swaps (line 7 / 11)
    int sw = mysw;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) sw += __shfl_xor_sync(0xffffffffu, sw, o);
    int* red = s_ctl + 8;
    __syncthreads();
    if ((tid & 31) == 0) red[tid >> 5] = sw;
    __syncthreads();
    int rs = 0;
    for (int w = 0; w < (T >> 5); ++w) rs += red[w];
    if (tid == 0 && rounds < max_log) per_round[rounds] = rs;
    rounds += 1;
    total += rs;
    if (rs == 0) break;
    if (max_rounds > 0 && rounds >= max_rounds) { status = PM_ERR_NOT_CONVERGED; break; }
    B = 1;
  }
  __syncthreads();
  for (int32_t u = tid; u < S; u += T) perm[u] = s_r[u];
  if (tid == 0) { out->status = status; out->rounds = rounds; out->swaps = total; }
}

int32_t ls_window_max_S() { return 4096; }

template <int K>
static pm_status_t launch_window_k(const int32_t* E, int64_t ldE, const int32_t* Ep, int64_t ldp, int32_t S,
                                   int32_t* perm, int32_t max_rounds, LsResult* dev_out, int64_t* dev_per_round,
                                   int32_t max_log, cudaStream_t st) {
  const size_t smem = WinSmem<K>::bytes(S);
  int dev = 0, optin = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  if (smem > (size_t)optin) return PM_ERR_UNSUPPORTED;
  PM_CUDA_TRY(cudaFuncSetAttribute(k_ls_window<K>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int threads = kWinThreads;
  while (threads > 64 && threads / 2 >= S / 2) threads /= 2;
  k_ls_window<K><<<1, threads, smem, st>>>(E, ldE, Ep, ldp, S, perm, max_rounds, dev_out, dev_per_round, max_log);
  note_launch();
  PM_CUDA_TRY(cudaGetLastError());
  return PM_OK;
}

pm_status_t run_window(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                       LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st) {
  if (S > ls_window_max_S()) return PM_ERR_UNSUPPORTED;
  const Classes cl(S);
  const int32_t m = cl.m;
  const int64_t ldp = ((int64_t)m + 31) / 32 * 32;
  int32_t* Ep = nullptr;
  PM_CUDA_TRY(cudaMallocAsync(&Ep, sizeof(int32_t) * (size_t)S * (size_t)ldp, st));
  {
    const int64_t total = (int64_t)S * m;
    int64_t blocks = (total + 255) / 256;
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    k_permute_cols<<<(unsigned)blocks, 256, 0, st>>>(E, ldE, Ep, ldp, S, m);
    note_launch();
    PM_CUDA_TRY(cudaGetLastError());
  }
  pm_status_t s;
  if (S <= 1024) s = launch_window_k<32>(E, ldE, Ep, ldp, S, perm, max_rounds, dev_out, dev_per_round, max_log, st);
  else if (S <= 2048) s = launch_window_k<16>(E, ldE, Ep, ldp, S, perm, max_rounds, dev_out, dev_per_round, max_log, st);
  else s = launch_window_k<8>(E, ldE, Ep, ldp, S, perm, max_rounds, dev_out, dev_per_round, max_log, st);
  PM_CUDA_TRY(cudaFreeAsync(Ep, st));
  return s;
}

}  // namespace pm
