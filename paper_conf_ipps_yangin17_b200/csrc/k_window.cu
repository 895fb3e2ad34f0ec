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

__device__ __forceinline__ void cp_async4(int32_t* smem, const int32_t* gmem) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(d), "l"(gmem));
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// Ep[t][pos] = E[t][(2 pos) mod m] for pos in [0, m + ext): the sigma-permuted
// row, extended cyclically by `ext` entries so that any window segment
// [pos, pos + K + 4) can be read without wrapping.
__global__ void k_permute_cols(const int32_t* __restrict__ E, int64_t ld, int32_t* __restrict__ Ep, int64_t ldp,
                               int32_t S, int32_t m, int32_t ext) {
  // rows along y (grid-stride), four consecutive outputs per thread: the
  // inputs of a warp are 256 consecutive even (or odd) columns of the row,
  // so every sector is read from DRAM once (its other half by the other
  // half of the row, from L2) and the outputs are written as 16-byte stores
  const int32_t w = m + ext;
  const int32_t q0 = 4 * (blockIdx.x * blockDim.x + threadIdx.x);
  if (q0 >= w) return;
  const bool vec4 = (ldp % 4 == 0) && ((reinterpret_cast<uintptr_t>(Ep) & 15) == 0);
  for (int64_t t = blockIdx.y; t < S; t += gridDim.y) {
    const int32_t* __restrict__ row = E + t * ld;
    int32_t v[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      int32_t pos = q0 + i;
      if (pos >= w) { v[i] = 0; continue; }
      while (pos >= m) pos -= m;
      int32_t q = 2 * pos;
      if (q >= m) q -= m;
      v[i] = __ldg(row + q);
    }
    int32_t* dst = Ep + t * ldp + q0;
    if (vec4 && q0 + 4 <= w) {
      *reinterpret_cast<int4*>(dst) = make_int4(v[0], v[1], v[2], v[3]);
    } else {
      for (int i = 0; i < 4 && q0 + i < w; ++i) dst[i] = v[i];
    }
  }
}

__host__ __device__ inline int32_t win_stride(int32_t S) { return S + ((1 - S % 32) + 32) % 32; }  // == 1 mod 32

template <int K>
struct WinSmem {
  static constexpr int KS = K + 4;   // stored entries per slot: an aligned superset of K
  static size_t bytes(int32_t S) {
    return sizeof(int32_t) * ((size_t)S * 8 + (size_t)2 * KS * win_stride(S) + 64);
  }
};

// Per regular slot x, two windows in shared memory, stored transposed
// (entry-major, stride SP == 1 mod 32: the slots of one class are read
// conflict-free).  Each holds a 16-byte-aligned superset of K entries of a
// sigma-permuted row, loaded with unconditional LDG.128 / 4 x STS; woff[x]
// (kept next to d[x]) / swoff[x] = (sigma(x)+1) & 3 locate the first wanted
// entry inside the superset:
//   W [woff[x] + j][x]  = E[r[x]][p_{wb+j}(x)]  = Ep[r[x]][sigma(1-x) + wb + j]  (class window)
//   SW[swoff[x] + i][x] = E[r[x]][x + 2(i+1)]   = Ep[r[x]][sigma(x) + i + 1]     (diagonal window)
// Swap of regular slots (u, v) in class c = wb + j, a = r[u], b = r[v]: since
// p_{c+i}(u) = v + 2i and p_{c+i}(v) = u + 2i,
//   W'[j+i][u] = E[b][v+2i] = SW[i-1][v]     SW'[i-1][u] = E[b][u+2i] = W[j+i][v]
// (and symmetrically for v): the swap is an exchange of shared-memory entries
// with no global access.  SW' entries beyond the window are stale; the slot is
// put on the dirty list of its window and its SW is reloaded at the next
// window, and they are never read before: a later swap at class c'' > c needs
// offsets < jmax - (c'' - wb).  SW does not depend on the class, so clean
// slots keep theirs across windows and rounds.  Slot L = S-1 walks the plain
// row E[r[L]][u0(c)] (u0(c) = c + (m+1)/2 advances by one per class); the rare
// swap of the fixed pair (u0, L) reloads from global.
template <int K, int PPT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1)
k_ls_window(const int32_t* __restrict__ E, int64_t ld, const int32_t* __restrict__ Ep, int64_t ldp, int32_t S,
            int32_t* __restrict__ perm, int32_t max_rounds, LsResult* out, int64_t* per_round, int32_t max_log,
            int32_t* handoff, int32_t sparse_T) {
  static_assert(K % 4 == 0, "K multiple of 4");
  constexpr int KS = K + 4;
  constexpr int NP = KS / 4;       // 16-byte pieces per window
  extern __shared__ __align__(16) int32_t sm[];
  const int32_t SP = win_stride(S);
  int2* s_do = reinterpret_cast<int2*>(sm);   // {d[x] = E[r[x]][x], woff[x]}
  int32_t* s_r = sm + 2 * S;       // r[x]: tile at slot x
  int32_t* s_last = s_r + S;       // E[t][L] per tile t (even S)
  int32_t* s_sig = s_last + S;     // sigma(x)
  int32_t* s_src = s_sig + S;      // element offset of x's W superset in Ep (current window)
  int32_t* s_dgen = s_src + S;     // window id of x's last swap (its SW is reloaded at the next window)
  int32_t* s_W = s_dgen + 2 * S;   // [KS][SP]
  int32_t* s_SW = s_W + (size_t)KS * SP;     // [KS][SP]
  int32_t* s_ctl = s_SW + (size_t)KS * SP;   // [0..2] first-fire, [4..5] dirty counts, [8..40] reduction
  const Classes cl(S);
  const int32_t m = cl.m, H = cl.half;
  const bool even = (S % 2) == 0;
  const int32_t L = S - 1;
  const int32_t nreg = even ? S - 1 : S;       // regular slots 0..m-1
  const int tid = threadIdx.x, T = blockDim.x;
  const int lane = tid & 31;

  // ---- permutation check, then d, s_last, s_sig ----
  for (int32_t x = tid; x < S; x += T) s_sig[x] = 0;
  __syncthreads();
  int bad = 0;
  for (int32_t u = tid; u < S; u += T) {
    const int32_t t = perm[u];
    s_r[u] = t;
    if (t < 0 || t >= S) bad = 1;
    else atomicAdd(&s_sig[t], 1);
  }
  __syncthreads();
  for (int32_t x = tid; x < S; x += T)
    if (s_sig[x] != 1) bad = 1;
  if (__syncthreads_or(bad)) {
    if (tid == 0) { out->status = PM_ERR_NOT_PERMUTATION; out->rounds = 0; out->swaps = 0; }
    return;
  }
  for (int32_t x = tid; x < S; x += T) {
    s_do[x] = make_int2(__ldg(E + (int64_t)s_r[x] * ld + x), 0);
    if (even) s_last[x] = __ldg(E + (int64_t)x * ld + L);
    s_sig[x] = (x < m) ? (int32_t)(((int64_t)x * H) % m) : 0;
    s_dgen[x] = -1;
  }
  if (tid < 8) s_ctl[tid] = (tid < 3) ? INT32_MAX : 0;
  __syncthreads();

  auto wrap = [&](int32_t q) -> int32_t {   // q in (-m, 2m)
    if (q < 0) q += m;
    if (q >= m) q -= m;
    return q;
  };
  // Window w for classes [wb, wb + jmax): W of every slot; SW of the slots
  // swapped during window w-1 (every slot at w = 0 or after a list overflow).
  auto fill = [&](int32_t wb, int32_t jmax, int32_t w) {
    constexpr int U = MAXT <= 512 ? 4 : 2;   // 16-byte loads in flight per thread
    __syncthreads();
    for (int32_t x = tid; x < nreg; x += T) {
      const int32_t pos = wrap(wb + H - s_sig[x]);
      const int32_t base = pos & ~3;
      s_src[x] = s_r[x] * (int32_t)ldp + base;
      s_do[x].y = (pos - base) | (((s_sig[x] + 1) & 3) << 2);   // woff | swoff << 2
    }
    __syncthreads();
    const int32_t totW = nreg * NP;
    for (int32_t f0 = 0; f0 < totW; f0 += U * T) {
      int4 val[U];
#pragma unroll
      for (int uu = 0; uu < U; ++uu) {
        const int32_t f = f0 + uu * T + tid;
        if (f < totW) {
          const int32_t x = f / NP, q = f - x * NP;
          val[uu] = __ldg(reinterpret_cast<const int4*>(Ep + s_src[x]) + q);
        }
      }
#pragma unroll
      for (int uu = 0; uu < U; ++uu) {
        const int32_t f = f0 + uu * T + tid;
        if (f < totW) {
          const int32_t x = f / NP, q = f - x * NP;
          int32_t* d = s_W + (4 * q) * SP + x;
          d[0] = val[uu].x; d[SP] = val[uu].y; d[2 * SP] = val[uu].z; d[3 * SP] = val[uu].w;
        }
      }
    }
    // SW of slots swapped during window w-1 (all slots at w = 0): one thread per slot
    for (int32_t x = tid; x < nreg; x += T) {
      if (w != 0 && s_dgen[x] != w - 1) continue;
      const int4* src = reinterpret_cast<const int4*>(Ep + s_r[x] * (int32_t)ldp + ((s_sig[x] + 1) & ~3));
      int4 val[NP];
#pragma unroll
      for (int q = 0; q < NP; ++q) val[q] = __ldg(src + q);
#pragma unroll
      for (int q = 0; q < NP; ++q) {
        int32_t* d = s_SW + (4 * q) * SP + x;
        d[0] = val[q].x; d[SP] = val[q].y; d[2 * SP] = val[q].z; d[3 * SP] = val[q].w;
      }
    }
    if (even) {
      for (int32_t j = tid; j < jmax; j += T) s_W[j * SP + L] = __ldg(E + (int64_t)s_r[L] * ld + wrap(wb + j + H));
      if (tid == 0) s_do[L].y = 0;
    }
    __syncthreads();
  };

  // this thread's pairs k = tid + q*T; (u, v) tracked for the current class
  int32_t pu[PPT] = {}, pv[PPT] = {};
  auto set_class = [&](int32_t c) {
#pragma unroll
    for (int q = 0; q < PPT; ++q) {
      const int32_t k = tid + q * T;
      if (k < cl.npairs) cl.pair(c, k, pu[q], pv[q]);
    }
  };
  auto advance = [&](int32_t delta) {   // consecutive classes: u0 + k, u0 - k, u0 all shift by +1
#pragma unroll
    for (int q = 0; q < PPT; ++q) {
      const int32_t k = tid + q * T;
      int32_t a = pu[q] + delta; if (a >= m) a -= m;
      pu[q] = a;
      if (!(even && k == 0)) { int32_t b = pv[q] + delta; if (b >= m) b -= m; pv[q] = b; }
    }
  };
  // O(u), O(v) at window offset j; fire iff d[u] + d[v] > O(u) + O(v)
  auto eval = [&](bool special, int32_t u, int32_t v, int32_t j, int32_t& ou, int32_t& ov) -> bool {
    const int2 du = s_do[u];
    const int2 dv = s_do[v];
    ou = special ? s_last[s_r[u]] : s_W[(j + (du.y & 3)) * SP + u];   // special: u = u0(c), partner L
    ov = s_W[(j + (dv.y & 3)) * SP + v];
    return (int64_t)du.x + dv.x > (int64_t)ou + ov;
  };

  int32_t rounds = 0;
  int64_t total = 0;
  int status = PM_OK;
  uint32_t batch = 0;
  int32_t wid = -1;
  bool dense = true;        // round 0, and rounds after one with > ncls/2 swaps (measured: B = 1 wins there)
#ifdef PM_LS_PROFILE
  long long t_round = clock64();
  int32_t n_apply = 0, n_spec = 0;
  long long t_fill = 0, t_spec = 0, t_apply = 0;
  long long t_ph[3] = {0, 0, 0};
  long long tA = 0, tB = 0;
#endif
  int32_t B = 1;
  for (;;) {                                           // Alg. 2 line 1
    int mysw = 0;
    int32_t c = 0;
    int32_t wb = INT32_MIN / 2;
    set_class(0);
    while (c < cl.ncls) {                              // line 3, classes in order
      if (c >= wb + K) {
        wb = c;
        ++wid;
#ifdef PM_LS_PROFILE
        const long long tf0 = clock64();
#endif
        fill(wb, min(K, cl.ncls - wb), wid);
#ifdef PM_LS_PROFILE
        t_fill += clock64() - tf0;
#endif
      }
      const int32_t jmax = min(K, cl.ncls - wb);
      int32_t* first_slot = s_ctl + (batch % 3);
      if (tid == 0) s_ctl[(batch + 1) % 3] = INT32_MAX;
      ++batch;
      if (dense) B = 1;                                // dense round: speculation only wastes work
      const int32_t cend = min(c + B, wb + jmax);
      int32_t cc = c;
#ifdef PM_LS_PROFILE
      const long long ts0 = clock64();
#endif
      if (cend - c > 1) {
        // speculative: all pairs of classes [c, cend) on the current state
        const int32_t nb = cend - c;
#pragma unroll
        for (int q = 0; q < PPT; ++q) {
          const int32_t k = tid + q * T;
          if (k >= cl.npairs) continue;
          const bool special = even && k == 0;
          int32_t u = pu[q], v = pv[q];
          // 4 classes per step: all shared-memory loads issued before any test
          for (int32_t jj0 = 0; jj0 < nb; jj0 += 4) {
            int32_t us[4], vs[4];
            int2 du[4], dv[4];
            int32_t ou[4], ov[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) {
              us[t] = u; vs[t] = v;
              u = (u + 1 == m) ? 0 : u + 1;
              if (!special) v = (v + 1 == m) ? 0 : v + 1;
            }
#pragma unroll
            for (int t = 0; t < 4; ++t) { du[t] = s_do[us[t]]; dv[t] = s_do[vs[t]]; }
            const int32_t j0 = c + jj0 - wb;
#pragma unroll
            for (int t = 0; t < 4; ++t) {
              // entries past the window end are read but never used (j < KS always)
              ou[t] = special ? s_last[s_r[us[t]]] : s_W[(j0 + t + (du[t].y & 3)) * SP + us[t]];
              ov[t] = s_W[(j0 + t + (dv[t].y & 3)) * SP + vs[t]];
            }
            int hit = -1;
#pragma unroll
            for (int t = 3; t >= 0; --t)
              if (jj0 + t < nb && (int64_t)du[t].x + dv[t].x > (int64_t)ou[t] + ov[t]) hit = t;
            if (hit >= 0) { atomicMin(first_slot, jj0 + hit); break; }
          }
        }
        __syncthreads();
        const int32_t first = *first_slot;
#ifdef PM_LS_PROFILE
        ++n_spec;
        t_spec += clock64() - ts0;
#endif
        if (first == INT32_MAX) {
          advance(nb);
          c = cend;
          B = min(2 * B, K);
          continue;
        }
        advance(first);
        cc = c + first;
        B = first == 0 ? 1 : first;
      }
      // exact step of class cc: evaluate, swap (line 6), exchange windows
      const int32_t j = cc - wb;
      int fired = 0;
#pragma unroll
      for (int q = 0; q < PPT; ++q) {                  // warp-uniform
        const int32_t k = tid + q * T;
        const int32_t u = pu[q], v = pv[q];
        const bool special = even && k == 0;
        int32_t a = 0, b = 0, yu = 0, yv = 0;
        bool f = false;
        if (k < cl.npairs) {
          const int2 du = s_do[u];
          const int2 dv = s_do[v];
          yu = du.y; yv = dv.y;
          const int32_t ou = special ? s_last[s_r[u]] : s_W[(j + (yu & 3)) * SP + u];
          const int32_t ov = s_W[(j + (yv & 3)) * SP + v];
          if ((int64_t)du.x + dv.x > (int64_t)ou + ov) {
            a = s_r[u]; b = s_r[v];
            s_r[u] = b; s_r[v] = a;
            s_do[u].x = ov; s_do[v].x = ou;  // d[u] = E[b][u] = O(v), d[v] = E[a][v] = O(u)
            s_dgen[u] = wid; s_dgen[v] = wid;
            ++mysw;
            fired = 1;
            f = true;
          }
        }
#ifdef PM_LS_PROFILE
        tA = clock64();
#endif
        unsigned mask = __ballot_sync(0xffffffffu, f);
        while (mask) {
          const int sl = __ffs(mask) - 1;
          mask &= mask - 1;
          const int32_t su = __shfl_sync(0xffffffffu, u, sl), sv = __shfl_sync(0xffffffffu, v, sl);
          const int32_t syu = __shfl_sync(0xffffffffu, yu, sl), syv = __shfl_sync(0xffffffffu, yv, sl);
          const bool sfixed = __shfl_sync(0xffffffffu, special, sl);
          const int32_t ofu = syu & 3, ofv = syv & 3;
          if (!sfixed) {
            const int32_t swu = syu >> 2, swv = syv >> 2;
            for (int32_t jj = j + 1 + lane; jj < jmax; jj += 32) {
              const int32_t i = jj - j - 1;
              int32_t* Wu = s_W + (jj + ofu) * SP + su;
              int32_t* Wv = s_W + (jj + ofv) * SP + sv;
              int32_t* Xu = s_SW + (i + swu) * SP + su;
              int32_t* Xv = s_SW + (i + swv) * SP + sv;
              const int32_t wu = *Wu, wv = *Wv, xu = *Xu, xv = *Xv;
              *Wu = xv; *Xu = wv;
              *Wv = xu; *Xv = wu;
            }
          } else {
            // (u0, L): u0 now holds b (walks Ep[b][sigma(u0) + i]), L holds a
            // (walks E[a][u0 + i]); reload from global (rare: 1 pair per class)
            const int32_t sa = __shfl_sync(0xffffffffu, a, sl), sb = __shfl_sync(0xffffffffu, b, sl);
            const int32_t sg = s_sig[su], swu = syu >> 2;
            for (int32_t jj = j + 1 + lane; jj < jmax; jj += 32) {
              const int32_t i = jj - j;
              const int32_t e1 = __ldg(Ep + (int64_t)sb * ldp + sg + i);
              const int32_t e2 = __ldg(E + (int64_t)sa * ld + wrap(su + i));
              s_W[(jj + ofu) * SP + su] = e1;
              s_SW[(i - 1 + swu) * SP + su] = e1;
              s_W[(jj + ofv) * SP + sv] = e2;
            }
          }
        }
      }
#ifdef PM_LS_PROFILE
      tB = clock64();
#endif
      const int any = __syncthreads_or(fired);
#ifdef PM_LS_PROFILE
      ++n_apply;
      const long long tC = clock64();
      t_apply += tC - ts0;
      t_ph[0] += tA - ts0; t_ph[1] += tB - tA; t_ph[2] += tC - tB;
#endif
      if (cend - c <= 1 && !any) B = 2;                 // quiet class: start speculating
      advance(1);
      c = cc + 1;
    }
    // round end: count swaps (line 7 / 11)
    int sw = mysw;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) sw += __shfl_xor_sync(0xffffffffu, sw, o);
    int* red = s_ctl + 8;
    __syncthreads();
    if (lane == 0) red[tid >> 5] = sw;
    __syncthreads();
    int rs = 0;
    for (int w = 0; w < (T >> 5); ++w) rs += red[w];
    if (tid == 0 && rounds < max_log) per_round[rounds] = rs;
#ifdef PM_LS_PROFILE
    if (tid == 0 && max_log >= 1024 && rounds < 128) {
      const long long now = clock64();
      per_round[512 + rounds] = now - t_round;
      per_round[640 + rounds] = n_apply;
      per_round[768 + rounds] = n_spec;
      per_round[896 + rounds] = t_fill;
      per_round[896 + 32 + rounds] = t_spec;
      per_round[896 + 64 + rounds] = t_apply;
      t_round = now;
    }
    if (tid == 32 && max_log >= 1024 && rounds < 16) {
      per_round[256 + rounds] = t_ph[0];
      per_round[256 + 16 + rounds] = t_ph[1];
      per_round[256 + 32 + rounds] = t_ph[2];
    }
    if (tid == 0 && max_log >= 1024 && rounds < 16) {
      per_round[320 + rounds] = t_ph[0];
      per_round[320 + 16 + rounds] = t_ph[1];
      per_round[320 + 32 + rounds] = t_ph[2];
    }
    t_ph[0] = t_ph[1] = t_ph[2] = 0;
    n_apply = n_spec = 0;
    t_fill = t_spec = t_apply = 0;
#endif
    rounds += 1;
    total += rs;
    if (rs == 0) break;
    if (max_rounds > 0 && rounds >= max_rounds) { status = PM_ERR_NOT_CONVERGED; break; }
    if (handoff && rs <= sparse_T) {                   // quiet: sparse rounds take over (k_sparse.cu)
      if (tid == 0) *handoff = 1;
      break;
    }
    B = 1;
    dense = rs > cl.ncls / 2;
  }
  __syncthreads();
  for (int32_t u = tid; u < S; u += T) perm[u] = s_r[u];
  if (tid == 0) { out->status = status; out->rounds = rounds; out->swaps = total; }
}

int32_t ls_window_max_S() { return 2048; }

cudaError_t launch_permute_cols(const int32_t* E, int64_t ldE, int32_t* Ep, int64_t ldp, int32_t S, int32_t m,
                                int32_t ext, cudaStream_t st) {
  const int32_t bx = (m + ext + 4 * 256 - 1) / (4 * 256);
  const int32_t by = S < 65535 ? S : 65535;
  k_permute_cols<<<dim3(bx, by), 256, 0, st>>>(E, ldE, Ep, ldp, S, m, ext);
  note_launch();
  return cudaGetLastError();
}

template <int K, int PPT, int MAXT>
static pm_status_t launch_window_k(const int32_t* E, int64_t ldE, const int32_t* Ep, int64_t ldp, int32_t S,
                                   int32_t* perm, int32_t max_rounds, LsResult* dev_out, int64_t* dev_per_round,
                                   int32_t max_log, cudaStream_t st, int32_t* handoff, int32_t sparse_T) {
  const size_t smem = WinSmem<K>::bytes(S);
  int dev = 0, optin = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  if (smem > (size_t)optin) return PM_ERR_UNSUPPORTED;
  PM_CUDA_TRY(cudaFuncSetAttribute(k_ls_window<K, PPT, MAXT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int32_t npairs = S / 2;
  int threads = (npairs + PPT - 1) / PPT;
  threads = (threads + 31) / 32 * 32;
  if (threads < 32) threads = 32;
  if (threads > MAXT) return PM_ERR_UNSUPPORTED;
  k_ls_window<K, PPT, MAXT><<<1, threads, smem, st>>>(E, ldE, Ep, ldp, S, perm, max_rounds, dev_out, dev_per_round, max_log,
                                                       handoff, sparse_T);
  note_launch();
  PM_CUDA_TRY(cudaGetLastError());
  return PM_OK;
}

pm_status_t run_window(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                       LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st,
                       int32_t* handoff, int32_t sparse_T) {
  if (S > ls_window_max_S()) return PM_ERR_UNSUPPORTED;
  const Classes cl(S);
  const int32_t m = cl.m;
  const int32_t ext = 16 + 8;                                   // >= K + 4 for every K used
  const int64_t ldp = ((int64_t)m + ext + 31) / 32 * 32;
  int32_t* Ep = nullptr;
  PM_CUDA_TRY(pm::scratch_alloc(&Ep, sizeof(int32_t) * (size_t)S * (size_t)ldp, st));
  {
    const int64_t total = (int64_t)S * (m + ext);
    int64_t blocks = (total + 255) / 256;
    if (blocks > 148 * 8) blocks = 148 * 8;
    if (blocks < 1) blocks = 1;
    k_permute_cols<<<(unsigned)blocks, 256, 0, st>>>(E, ldE, Ep, ldp, S, m, ext);
    note_launch();
    PM_CUDA_TRY(cudaGetLastError());
  }
  pm_status_t s;
  if (S <= 1024) s = launch_window_k<16, 1, 512>(E, ldE, Ep, ldp, S, perm, max_rounds, dev_out, dev_per_round, max_log, st,
                                                  handoff, sparse_T);
  else s = launch_window_k<4, 1, 1024>(E, ldE, Ep, ldp, S, perm, max_rounds, dev_out, dev_per_round, max_log, st,
                                                   handoff, sparse_T);
  PM_CUDA_TRY(cudaFreeAsync(Ep, st));
  return s;
}

}  // namespace pm
