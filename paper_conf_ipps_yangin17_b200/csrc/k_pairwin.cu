// k_pairwin.cu -- PM_LS_PAIRWIN: Algorithm 2 with pair-indexed
// tables, one round per (grid kernel + single-CTA kernel), rounds looped on the
// device by a CUDA-graph WHILE node.
//
// Per round, with r and the diagonal d[x] = E[r[x]][x] as they are at the
// round's start, a grid-wide kernel (all SMs) writes for every class c and
// pair k = (u, v) of c (Classes::pair):
//   TU[c][k] = E[r[u]][v] - d[u]        TV[c][k] = E[r[v]][u] - d[v]
// so pair k of class c fires (line 5, strict) iff TU[c][k] + TV[c][k] < 0.
// Class rows are contiguous: one CTA streams them K classes at a time into a
// double-buffered shared-memory window with cp.async (no gathers), and a
// pair's test is two conflict-free LDS and one add.
//
// Swaps make the round-start tables stale for the two slots involved, and
// only for them.  Where slot x sits in class c is a closed form: with
// delta = (x - u0(c)) mod m, x is the u-side of pair col(delta) if
// delta <= (m-1)/2 (delta = 0: the fixed point, pair 0 of even S), else the
// v-side of pair col(m - delta).  So (i) inside the current window a swap of
// (u, v) at class c rewrites the two slots' later entries in shared memory
// from the diagonal window SW[x][i] = E[r[x]][x + 2(i+1)] (since
// p_{c+i}(u) = v + 2i:  E[b][p_{c+i}(u)] = SW[v][i-1], and SW'[u][i-1] =
// E[b][u+2i] = v's old entry at c+i), and (ii) every later window re-derives
// the entries of the round's swapped slots from their (new) rows of the
// sigma-permuted E (Ep, k_window.cu), before any class of that window runs.
// Exact speculation over classes of a window as in k_window.cu.  Results are
// bit-identical to the serial replay (tests/test_gpu_parity.py).
#include <cuda_runtime.h>

#include <map>
#include <mutex>
#include <tuple>

#include "pm_internal.cuh"

namespace pm {

struct PwParams {
  const int32_t* E;
  int64_t ld;
  const int32_t* Ep;     // sigma-permuted rows, extended (k_window.cu)
  int64_t ldp;
  int32_t* r;            // [S] current rearrangement (caller's d_perm)
  int32_t* d;            // [S] diagonal
  int32_t* seen;         // [S] permutation check
  int32_t* TU;           // [ncls][npr]
  int32_t* TV;           // [ncls][npr]
  int32_t* SWg;          // [S][K]
  int32_t S, npr, K, max_rounds, max_log, pad;
  unsigned long long round_swaps;
  LsResult* out;
  int64_t* per_round;
  unsigned long long* launches;   // device-side launch counter (graph kernels)
};

__global__ void k_pw_set_params(PwParams* dst, PwParams src) { *dst = src; }

__global__ void k_pw_check_init(PwParams* p) {
  const int32_t S = p->S;
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < S; u += gridDim.x * blockDim.x) {
    const int32_t t = p->r[u];
    if (t < 0 || t >= S) { p->out->status = PM_ERR_NOT_PERMUTATION; continue; }
    atomicAdd(p->seen + t, 1);
    p->d[u] = p->E[(int64_t)t * p->ld + u];
  }
}

__global__ void k_pw_check_seen(PwParams* p) {
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < p->S; u += gridDim.x * blockDim.x)
    if (p->seen[u] != 1) p->out->status = PM_ERR_NOT_PERMUTATION;
}

__device__ __forceinline__ int32_t pw_sigma(int32_t x, int32_t m, int32_t H) {
  return (int32_t)(((int64_t)x * H) % m);
}

// Round-start tables (grid-wide).
__global__ void __launch_bounds__(256) k_pw_tables(const PwParams* __restrict__ p) {
  if (blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(p->launches, 1ull);
  if (p->out->status != PM_OK) return;
  const Classes cl(p->S);
  const int32_t S = p->S, npr = p->npr, K = p->K, m = cl.m, H = cl.half;
  const int32_t* __restrict__ E = p->E;
  const int32_t* __restrict__ r = p->r;
  const int32_t* __restrict__ d = p->d;
  const int64_t total = (int64_t)cl.ncls * cl.npairs;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = (int32_t)(i / cl.npairs), k = (int32_t)(i - (int64_t)c * cl.npairs);
    int32_t u, v;
    cl.pair(c, k, u, v);
    const int32_t ru = __ldg(r + u), rv = __ldg(r + v);
    p->TU[(int64_t)c * npr + k] = __ldg(E + (int64_t)ru * p->ld + v) - __ldg(d + u);
    p->TV[(int64_t)c * npr + k] = __ldg(E + (int64_t)rv * p->ld + u) - __ldg(d + v);
  }
  const bool even = (S % 2) == 0;
  const int64_t tot2 = (int64_t)S * K;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < tot2; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t x = (int32_t)(i / K), q = (int32_t)(i - (int64_t)x * K);
    if (even && x == S - 1) continue;
    p->SWg[i] = __ldg(p->Ep + (int64_t)__ldg(r + x) * p->ldp + pw_sigma(x, m, H) + 1 + q);
  }
}

// Alg. 2 line 11 (+ the max_rounds cap): decide whether the while-node loops.
__global__ void k_pw_round_end(PwParams* p, cudaGraphConditionalHandle h) {
  atomicAdd(p->launches, 1ull);
  LsResult* o = p->out;
  unsigned cont = 0;
  if (o->status == PM_OK) {
    const int64_t sw = (int64_t)p->round_swaps;
    p->round_swaps = 0;
    if (o->rounds < p->max_log) p->per_round[o->rounds] = sw;
    o->rounds += 1;
    o->swaps += sw;
    if (sw > 0) {
      if (p->max_rounds > 0 && o->rounds >= p->max_rounds) o->status = PM_ERR_NOT_CONVERGED;
      else cont = 1;
    }
  }
  cudaGraphSetConditional(h, cont);
}

__device__ __forceinline__ void pw_cp16(int32_t* smem, const int32_t* gmem) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem));
}

template <int K>
struct PwSmem {
  static size_t bytes(int32_t S, int32_t npr) {
    return sizeof(int32_t) * (((((size_t)S * 6 + 3) / 4 * 4) + (size_t)S * K + 3) / 4 * 4 + (size_t)4 * K * npr + 64);
  }
};

// One round of Algorithm 2 in one CTA (lines 2-10).
template <int K, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) k_pw_round(PwParams* __restrict__ p) {
  if (threadIdx.x == 0) atomicAdd(p->launches, 1ull);
  __shared__ int s_status;                      // block-uniform early exit (no divergent barrier)
  if (threadIdx.x == 0) s_status = (int)p->out->status;
  __syncthreads();
  if (s_status != PM_OK) return;
  extern __shared__ __align__(16) int32_t sm[];
  const int32_t S = p->S, npr = p->npr;
  const Classes cl(S);
  const int32_t m = cl.m, H = cl.half, half = (m - 1) / 2;
  const bool even = (S % 2) == 0;
  const int32_t L = S - 1;
  const int32_t nreg = even ? S - 1 : S;
  const int tid = threadIdx.x, T = blockDim.x, lane = tid & 31;
  const int32_t* __restrict__ E = p->E;
  const int32_t* __restrict__ Ep = p->Ep;
  const int64_t ld = p->ld, ldp = p->ldp;

  int32_t* s_r = sm;                     // r[x]
  int32_t* s_d = s_r + S;                // d[x]
  int32_t* s_last = s_d + S;             // E[t][L]
  int32_t* s_sig = s_last + S;           // sigma(x)
  int32_t* s_gen = s_sig + S;            // window id of x's last swap this round (-1: none)
  int32_t* s_dl = s_gen + S;             // this window's list of slots swapped earlier this round
  int32_t* s_SW = sm + ((size_t)S * 6 + 3) / 4 * 4;                  // [S][K], 16-B aligned
  int32_t* s_T = sm + ((((size_t)S * 6 + 3) / 4 * 4) + (size_t)S * K + 3) / 4 * 4;   // [2 buf][2 (U,V)][K][npr], 16-B aligned
  int32_t* s_ctl = s_T + (size_t)4 * K * npr;
  const int32_t tsz = K * npr;           // one array of one buffer

#ifdef PM_LS_PROFILE
  long long t_start = clock64(), t_patch = 0, t_cls = 0, t_wait = 0;
  unsigned long long g_start;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g_start));
#endif
  for (int32_t x = tid; x < S; x += T) {
    s_r[x] = p->r[x];
    s_d[x] = p->d[x];
    if (even) s_last[x] = __ldg(E + (int64_t)x * ld + L);
    s_sig[x] = x < m ? pw_sigma(x, m, H) : 0;
    s_gen[x] = -1;
  }
  {                                            // SW: 16-byte cp.async (S*K ints, 16-B aligned)
    const int32_t n16 = S * K / 4;
    for (int32_t i = tid; i < n16; i += T) pw_cp16(s_SW + 4 * i, p->SWg + 4 * i);
    for (int32_t i = n16 * 4 + tid; i < S * K; i += T) s_SW[i] = p->SWg[i];
    asm volatile("cp.async.commit_group;\n" ::);
  }
  if (tid < 4) s_ctl[tid] = INT32_MAX;
  if (tid == 4 || tid == 5) s_ctl[tid] = 0;    // [4]: swapped since last compaction, [5]: dirty-list size

  auto wrap = [&](int32_t q) -> int32_t { if (q < 0) q += m; if (q >= m) q -= m; return q; };
  // (array, column) of regular slot x at class c; returns -1 if it idles (odd S)
  auto where = [&](int32_t x, int32_t c, bool& isU) -> int32_t {
    const int32_t delta = wrap(x - cl.fixed_point(c));
    if (delta == 0) { isU = true; return even ? 0 : -1; }
    if (delta <= half) { isU = true; return even ? delta : delta - 1; }
    isU = false;
    return even ? m - delta : m - delta - 1;
  };
  auto issue_window = [&](int32_t wb, int32_t buf) {   // rows [wb, wb + K) of TU / TV
    const int32_t rows = min(K, cl.ncls - wb);
    const int32_t n16 = rows * npr / 4;
    const int32_t* gU = p->TU + (int64_t)wb * npr;
    const int32_t* gV = p->TV + (int64_t)wb * npr;
    int32_t* dU = s_T + (size_t)(2 * buf) * tsz;
    int32_t* dV = dU + tsz;
    for (int32_t i = tid; i < n16; i += T) {
      pw_cp16(dU + 4 * i, gU + 4 * i);
      pw_cp16(dV + 4 * i, gV + 4 * i);
    }
    asm volatile("cp.async.commit_group;\n" ::);
  };

  __syncthreads();
  issue_window(0, 0);
  int mysw = 0;
  int32_t B = 1;
  uint32_t batch = 0;
  int32_t w = 0;
  for (int32_t wb = 0; wb < cl.ncls; wb += K, ++w) {
    const int32_t buf = w & 1;
    const int32_t jmax = min(K, cl.ncls - wb);
    int32_t* TUw = s_T + (size_t)(2 * buf) * tsz;
    int32_t* TVw = TUw + tsz;
#ifdef PM_LS_PROFILE
    const long long tw0 = clock64();
#endif
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    __syncthreads();
#ifdef PM_LS_PROFILE
    const long long tp0 = clock64();
    t_wait += tp0 - tw0;
#endif
    // ---- slots swapped earlier this round: re-derive their entries (and SW
    // for those swapped in the previous window) from their current rows
    // compact the round-dirty regular slots into s_dl (warp ballots + prefix),
    // only if some slot swapped since the last compaction (block-uniform flag)
    int32_t tot = s_ctl[5];
    if (s_ctl[4]) {
      const int nw = T >> 5, wid_ = tid >> 5;
      const int32_t chunk = (nreg + nw - 1) / nw;
      const int32_t x0 = wid_ * chunk, x1 = min(nreg, x0 + chunk);
      int32_t cnt = 0;
      for (int32_t xb = x0; xb < x1; xb += 32) {
        const int32_t x = xb + lane;
        cnt += __popc(__ballot_sync(0xffffffffu, x < x1 && s_gen[x] >= 0));
      }
      int* red = s_ctl + 8;
      if (lane == 0) red[wid_] = cnt;
      __syncthreads();
      int32_t off = 0;
      tot = 0;
      for (int i = 0; i < nw; ++i) { const int32_t ci = red[i]; off += i < wid_ ? ci : 0; tot += ci; }
      for (int32_t xb = x0; xb < x1; xb += 32) {
        const int32_t x = xb + lane;
        const bool dirty = x < x1 && s_gen[x] >= 0;
        const unsigned bm = __ballot_sync(0xffffffffu, dirty);
        if (dirty) s_dl[off + __popc(bm & ((1u << lane) - 1))] = x;
        off += __popc(bm);
      }
      __syncthreads();
      if (tid == 0) { s_ctl[4] = 0; s_ctl[5] = tot; }
    }
    {
      // ---- re-derive their entries (and SW for those swapped in the previous window)
      constexpr int U = 8;                     // loads in flight per thread
      const int32_t items = tot * K;
      for (int32_t f0 = 0; f0 < items; f0 += U * T) {
        int32_t val[U], dst[U], sw[U], swd[U], dx[U];
#pragma unroll
        for (int uu = 0; uu < U; ++uu) {
          const int32_t f = f0 + uu * T + tid;
          dst[uu] = -1;
          swd[uu] = -1;
          if (f >= items) continue;
          const int32_t i = f / K, j = f - i * K;
          const int32_t x = s_dl[i];
          dx[uu] = x;
          const int32_t t = s_r[x];
          if (j < jmax) {
            bool isU;
            const int32_t col = where(x, wb + j, isU);
            if (col >= 0) {
              dst[uu] = (isU ? 0 : tsz) + j * npr + col;
              val[uu] = (even && col == 0 && isU) ? s_last[t]                                   // x = u0(c)
                                                   : __ldg(Ep + (int64_t)t * ldp + wrap(wb + H - s_sig[x]) + j);
            }
          }
          if (s_gen[x] == w - 1) { swd[uu] = x * K + j; sw[uu] = __ldg(Ep + (int64_t)t * ldp + s_sig[x] + 1 + j); }
        }
#pragma unroll
        for (int uu = 0; uu < U; ++uu) {
          if (dst[uu] >= 0) TUw[dst[uu]] = val[uu] - s_d[dx[uu]];
          if (swd[uu] >= 0) s_SW[swd[uu]] = sw[uu];
        }
      }
    }
    if (even && s_gen[L] >= 0)
      for (int32_t j = tid; j < jmax; j += T)
        TVw[j * npr] = __ldg(E + (int64_t)s_r[L] * ld + wrap(wb + j + H)) - s_d[L];
    __syncthreads();
#ifdef PM_LS_PROFILE
    const long long tc0 = clock64();
    t_patch += tc0 - tp0;
#endif
    if (wb + K < cl.ncls) issue_window(wb + K, buf ^ 1);

    int32_t c = wb;
    while (c < wb + jmax) {
      int32_t* first_slot = s_ctl + (batch % 3);
      if (tid == 0) s_ctl[(batch + 1) % 3] = INT32_MAX;
      ++batch;
      const int32_t cend = min(c + B, wb + jmax);
      int32_t cc = c;
      if (cend - c > 1) {
        // speculative: classes [c, cend) on the current state
        const int32_t j0 = c - wb, nb = cend - c;
        for (int32_t k = tid; k < cl.npairs; k += T) {
          int32_t hit = INT32_MAX;
#pragma unroll
          for (int32_t jj = K - 1; jj >= 0; --jj) {     // all loads issued before the tests
            if (jj < nb) {
              const int32_t tu = TUw[(j0 + jj) * npr + k], tv = TVw[(j0 + jj) * npr + k];
              if ((int64_t)tu + tv < 0) hit = jj;
            }
          }
          if (hit != INT32_MAX) atomicMin(first_slot, hit);
        }
        __syncthreads();
        const int32_t first = *first_slot;
        if (first == INT32_MAX) { c = cend; B = min(2 * B, K); continue; }
        cc = c + first;
        B = first == 0 ? 1 : first;
      }
      // exact step of class cc
      const int32_t j = cc - wb;
      int fired = 0;
      for (int32_t kb = 0; kb < cl.npairs; kb += T) {      // warp-uniform trip count
        const int32_t k = kb + tid;
        bool f = false;
        int32_t u = 0, v = 0, a = 0, b = 0, du = 0, dv = 0, Ou = 0, Ov = 0;
        if (k < cl.npairs) {
          const int32_t tu = TUw[j * npr + k], tv = TVw[j * npr + k];
          if ((int64_t)tu + tv < 0) {
            cl.pair(cc, k, u, v);
            a = s_r[u]; b = s_r[v]; du = s_d[u]; dv = s_d[v];
            Ou = tu + du;                  // E[a][v]
            Ov = tv + dv;                  // E[b][u]
            s_r[u] = b; s_r[v] = a;        // line 6
            s_d[u] = Ov; s_d[v] = Ou;
            s_gen[u] = w; s_gen[v] = w;
            ++mysw;
            fired = 1;
            f = true;
          }
        }
        unsigned mask = __ballot_sync(0xffffffffu, f);
        while (mask) {
          const int sl = __ffs(mask) - 1;
          mask &= mask - 1;
          const int32_t sk = __shfl_sync(0xffffffffu, k, sl);
          const int32_t su = __shfl_sync(0xffffffffu, u, sl), sv = __shfl_sync(0xffffffffu, v, sl);
          const int32_t sa = __shfl_sync(0xffffffffu, a, sl), sb = __shfl_sync(0xffffffffu, b, sl);
          const int32_t sdu = __shfl_sync(0xffffffffu, du, sl), sdv = __shfl_sync(0xffffffffu, dv, sl);
          const int32_t sOu = __shfl_sync(0xffffffffu, Ou, sl), sOv = __shfl_sync(0xffffffffu, Ov, sl);
          if (!(even && sk == 0)) {
            // regular pair: shared-memory exchange for classes cc+1 .. window end
            for (int32_t i = 1 + lane; j + i < jmax; i += 32) {
              const int32_t ci = cc + i;
              bool uU, vU;
              const int32_t cu = where(su, ci, uU);
              const int32_t cv = where(sv, ci, vU);          // v is regular at ci (m >= 2K)
              int32_t* pu_ = cu >= 0 ? (uU ? TUw : TVw) + (j + i) * npr + cu : nullptr;
              int32_t* pv_ = (vU ? TUw : TVw) + (j + i) * npr + cv;
              const bool ufixed = cu < 0 || (even && cu == 0 && uU);
              const int32_t old_u = pu_ ? *pu_ : 0, old_v = *pv_;
              const int32_t swu = s_SW[su * K + i - 1], swv = s_SW[sv * K + i - 1];
              if (pu_) *pu_ = (ufixed ? s_last[sb] : swv) - sOv;   // u now holds b, d'[u] = Ov
              *pv_ = swu - sOu;                                    // v now holds a, d'[v] = Ou
              s_SW[su * K + i - 1] = old_v + sdv;                  // E[b][u + 2i]
              s_SW[sv * K + i - 1] = ufixed ? __ldg(Ep + (int64_t)sa * ldp + s_sig[sv] + i)
                                            : old_u + sdu;         // E[a][v + 2i]
            }
          } else {
            // fixed pair (u0, L): u0 now holds b (walks E[b][u0 + 2i], the v-side
            // of pair i), L holds a (walks E[a][u0 + i]); reload from global
            const int32_t sg = s_sig[su];
            for (int32_t i = 1 + lane; j + i < jmax; i += 32) {
              const int32_t e1 = __ldg(Ep + (int64_t)sb * ldp + sg + i);
              TVw[(j + i) * npr + i] = e1 - sOv;
              TVw[(j + i) * npr] = __ldg(E + (int64_t)sa * ld + wrap(su + i)) - sOu;
              s_SW[su * K + i - 1] = e1;
            }
          }
        }
      }
      const int any = __syncthreads_or(fired);
      if (any && tid == 0) s_ctl[4] = 1;
      if (cend - c <= 1 && !any) B = 2;
      c = cc + 1;
    }
#ifdef PM_LS_PROFILE
    t_cls += clock64() - tc0;
#endif
  }
  // ---- round end: swaps, state back to global
  int sw = mysw;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) sw += __shfl_xor_sync(0xffffffffu, sw, o);
  int* red = s_ctl + 8;
  __syncthreads();
  if (lane == 0) red[tid >> 5] = sw;
  for (int32_t x = tid; x < S; x += T) { p->r[x] = s_r[x]; p->d[x] = s_d[x]; }
  __syncthreads();
  if (tid == 0) {
    int rs = 0;
    for (int i = 0; i < (T >> 5); ++i) rs += red[i];
    p->round_swaps = (unsigned long long)rs;
#ifdef PM_LS_PROFILE
    const int64_t R = p->out->rounds;
    unsigned long long g_end;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g_end));
    if (p->max_log >= 1024 && R < 64) {
      p->per_round[512 + R] = clock64() - t_start;
      p->per_round[576 + R] = t_patch;
      p->per_round[640 + R] = t_cls;
      p->per_round[704 + R] = t_wait;
      p->per_round[768 + R] = (int64_t)g_start;
      p->per_round[832 + R] = (int64_t)g_end;
    }
#endif
  }
}

template <int K>
static int32_t pw_threads(int32_t S) {
  int t = (S / 2 + 31) / 32 * 32;
  return t < 32 ? 32 : t;
}

static int32_t pw_K(int32_t S) { return S <= 1024 ? 16 : 6; }

int32_t ls_pairwin_min_S() { return 40; }
int32_t ls_pairwin_max_S() { return 2048; }

struct PwGraph {
  PwParams* dparams = nullptr;
  cudaGraphExec_t exec = nullptr;
};
static std::mutex g_pw_mu;
static std::map<std::tuple<int, int32_t, cudaStream_t>, PwGraph> g_pw_graphs;

template <int K>
static cudaError_t pw_build_graph(int32_t S, int32_t npr, PwGraph& out) {
  cudaError_t e = cudaMalloc(&out.dparams, sizeof(PwParams));
  if (e != cudaSuccess) return e;
  const size_t smem = PwSmem<K>::bytes(S, npr);
  constexpr int MAXT = K == 16 ? 512 : 1024;       // S <= 1024 runs 512 threads: 128 registers, no spills
  if ((e = cudaFuncSetAttribute(k_pw_round<K, MAXT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) != cudaSuccess)
    return e;
  cudaGraph_t g = nullptr;
  if ((e = cudaGraphCreate(&g, 0)) != cudaSuccess) return e;
  cudaGraphConditionalHandle h;
  if ((e = cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault)) != cudaSuccess) return e;
  cudaGraphNodeParams cp = {};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = h;
  cp.conditional.type = cudaGraphCondTypeWhile;
  cp.conditional.size = 1;
  cudaGraphNode_t node;
  if ((e = cudaGraphAddNode(&node, g, nullptr, 0, &cp)) != cudaSuccess) return e;
  cudaGraph_t body = cp.conditional.phGraph_out[0];
  cudaStream_t cs;
  if ((e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking)) != cudaSuccess) return e;
  if ((e = cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed)) != cudaSuccess)
    return e;
  const Classes cl(S);
  int64_t work = (int64_t)cl.ncls * cl.npairs;
  int blocks = (int)((work + 255) / 256);
  if (blocks > 148 * 8) blocks = 148 * 8;
  if (blocks < 1) blocks = 1;
  k_pw_tables<<<blocks, 256, 0, cs>>>(out.dparams);
  k_pw_round<K, MAXT><<<1, pw_threads<K>(S), smem, cs>>>(out.dparams);
  k_pw_round_end<<<1, 1, 0, cs>>>(out.dparams, h);
  cudaGraph_t captured = body;
  e = cudaStreamEndCapture(cs, &captured);
  cudaStreamDestroy(cs);
  if (e != cudaSuccess) return e;
  e = cudaGraphInstantiate(&out.exec, g, 0);
  cudaGraphDestroy(g);
  return e;
}

pm_status_t run_pairwin(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                        LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st) {
  if (S < ls_pairwin_min_S() || S > ls_pairwin_max_S()) return PM_ERR_UNSUPPORTED;
  const Classes cl(S);
  const int32_t K = pw_K(S);
  const int32_t npr = (cl.npairs + 3) / 4 * 4;
  const size_t smem = K == 16 ? PwSmem<16>::bytes(S, npr) : PwSmem<6>::bytes(S, npr);
  int dev = 0, optin = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  if (smem > (size_t)optin) return PM_ERR_UNSUPPORTED;
  PwGraph pg;
  {
    std::lock_guard<std::mutex> lk(g_pw_mu);
    auto key = std::make_tuple(dev, S, st);
    auto it = g_pw_graphs.find(key);
    if (it == g_pw_graphs.end()) {
      PwGraph ng;
      PM_CUDA_TRY(K == 16 ? pw_build_graph<16>(S, npr, ng) : pw_build_graph<6>(S, npr, ng));
      it = g_pw_graphs.emplace(key, ng).first;
    }
    pg = it->second;
  }
  const int32_t m = cl.m;
  const int32_t ext = 24;
  const int64_t ldp = ((int64_t)m + ext + 31) / 32 * 32;
  const size_t nEp = (size_t)S * ldp, nT = (size_t)cl.ncls * npr, nSW = (size_t)S * K;
  int32_t* scratch = nullptr;
  PM_CUDA_TRY(scratch_alloc(&scratch, sizeof(int32_t) * (nEp + 2 * nT + nSW + 2 * (size_t)S + 16), st));
  int32_t* Ep = scratch;
  int32_t* TU = Ep + nEp;
  int32_t* TV = TU + nT;
  int32_t* SWg = TV + nT;
  int32_t* d = SWg + nSW;
  int32_t* seen = d + S;
  PM_CUDA_TRY(cudaMemsetAsync(seen, 0, sizeof(int32_t) * (size_t)S, st));
  PM_CUDA_TRY(launch_permute_cols(E, ldE, Ep, ldp, S, m, ext, st));
  PwParams hp = {};
  hp.E = E; hp.ld = ldE; hp.Ep = Ep; hp.ldp = ldp; hp.r = perm; hp.d = d; hp.seen = seen;
  hp.TU = TU; hp.TV = TV; hp.SWg = SWg; hp.S = S; hp.npr = npr; hp.K = K;
  hp.max_rounds = max_rounds; hp.max_log = max_log; hp.round_swaps = 0;
  hp.out = dev_out; hp.per_round = dev_per_round;
  hp.launches = device_launch_counter();
  if (!hp.launches) return PM_ERR_CUDA;
  k_pw_set_params<<<1, 1, 0, st>>>(pg.dparams, hp);
  const int blocks = (S + 255) / 256;
  k_pw_check_init<<<blocks, 256, 0, st>>>(pg.dparams);
  k_pw_check_seen<<<blocks, 256, 0, st>>>(pg.dparams);
  note_launch(3);
  PM_CUDA_TRY(cudaGetLastError());
  PM_CUDA_TRY(cudaGraphLaunch(pg.exec, st));
  PM_CUDA_TRY(cudaFreeAsync(scratch, st));
  return PM_OK;
}

}  // namespace pm
