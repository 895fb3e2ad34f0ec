// k_sparse.cu -- quiet rounds of Algorithm 2 without touching
// the pairs that cannot fire.
//
// Alg. 2 runs the colour classes of a round in order; a pair (u, v) of class
// c fires iff d[u] + d[v] > E[r[v]][u] + E[r[u]][v] (line 5, reading R6) on
// the state left by classes < c.  A pair's test reads only r and d of its own
// two slots.  So at any class c of a round, a pair whose slots have not been
// swapped yet in this round ("clean") tests exactly as it did on the state at
// the round's start.  The exact sparse round is therefore:
//   1. k_sp_scan (whole GPU): test every pair of every class on the round's
//      start state; stamp the classes that contain a firing pair.
//   2. k_sp_walk (one CTA): walk the classes in order with r and d in shared
//      memory and the set D of slots swapped so far ("dirty").  A class that
//      is not stamped can only fire through pairs with a dirty slot, so only
//      those |D| pairs are tested -- for a window of upcoming classes at once,
//      on the current state (exact as long as nothing fires before: the first
//      firing class is then applied and the walk resumes after it).  A stamped
//      class is tested in full on the current state.
// Every class is thus decided on exactly the state Alg. 2 defines, so r,
// rounds and swaps are bit-identical to every other method (tests/).  Late
// rounds have few swaps, so D stays small and most classes cost nothing.
//
// The dense stage (WINDOW or CLASS) hands over after a round with at most
// sparse_T swaps by setting SpParams::pending; the rounds then loop here in a
// CUDA-graph WHILE node: [k_sp_begin] -> while { k_sp_scan ; k_sp_walk }.
#include <cuda_runtime.h>

#include <cstdlib>
#include <map>
#include <mutex>
#include <tuple>

#include "pm_internal.cuh"

namespace pm {

constexpr int kWalkThreads = 512;
constexpr int kWinMax = 256;             // classes per speculative window
constexpr int kFlSmem = 2048;            // stamped classes kept in shared memory
constexpr int kItemsPerThread = 4;       // pair tests per thread in flight

// Dynamic shared memory of the walk CTA: r, d (int32), dirty list (int32),
// dirty flags (u8).  Beyond the opt-in limit the same arrays live in global
// scratch (one CTA owns them, so plain loads see its own stores).
inline size_t walk_smem_bytes(int32_t S) { return (size_t)S * 13 + 64; }

__global__ void k_sp_set_params(SpParams* dst, SpParams src) { *dst = src; }

// d[x] = E[r[x]][x]; decide whether the sparse loop runs at all.
__global__ void k_sp_begin(SpParams* p, cudaGraphConditionalHandle h) {
  const int32_t S = p->S;
  for (int32_t x = blockIdx.x * blockDim.x + threadIdx.x; x < S; x += gridDim.x * blockDim.x)
    p->d[x] = __ldg(p->E + (int64_t)p->r[x] * p->ldE + x);
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    atomicAdd(p->launches, 1ull);
    const unsigned cont = (p->out->status == PM_OK && p->pending) ? 1u : 0u;
    p->pending = 0;
    p->nd_prev = -1;                             // the dense stage's swaps are not listed: full scan
#ifdef PM_LS_PROFILE
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (p->max_log >= 1024) p->per_round[1023] = (int64_t)t;   // sparse stage start (tools/sp_rounds.py)
#endif
    cudaGraphSetConditional(h, cont);
  }
}

// Full scan from the sigma-permuted copy Ep[t][q] = E[t][2q mod m] (TRAP
// keeps it for the sparse rounds).  For a regular slot y with tile r[y], its
// partner in class c is (2c+1-y) mod m, whose sigma-position is
// (c + (m+1)/2 - sigma(y)) mod m: consecutive classes read consecutive
// entries of row r[y].  So with w_y(c) = E[r[y]][partner_c(y)] - d[y], the
// pair (u, v) of class c fires iff w_u(c) + w_v(c) < 0 (line 5).  Tiles are
// taken in pair-index space: pairs k0 .. k0+kScanP-1 over classes
// c0 .. c0+kScanB-1 hold first slots u0(c0)+t+k and second slots
// u0(c0)+t-k -- two contiguous ranges of kScanP+kScanB-1 slots -- so a tile
// streams each of those slots' 128-byte runs once and tests every pair once
// (a slot-block tiling tests each pair from both of its slots and streams
// every run twice: config 4 first scan 1.07 ms).  Pair 0 (u0, S-1) of even S
// is tested separately.
constexpr int kScanP = 256, kScanB = 32;
constexpr int kScanR = (kScanP + kScanB - 1 + 31) / 32 * 32;   // rows per side (287 -> 288)
constexpr size_t kScanSmem = sizeof(int32_t) * (size_t)(2 * kScanR) * kScanB;

__device__ __forceinline__ void scan_full_ep(const SpParams* __restrict__ p, int32_t stamp, int32_t* sm) {
  const Classes cl(p->S);
  const int32_t m = cl.m, H = cl.half, S = p->S;
  const int32_t KR = (m - 1) / 2;        // regular pairs k = 1 .. KR
  const int32_t* __restrict__ r = p->r;
  const int32_t* __restrict__ d = p->d;
  const int32_t* __restrict__ Ep = p->Ep;
  const int64_t ldp = p->ldp;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
  int32_t* wA = sm;                      // [kScanR][kScanB]: first slots
  int32_t* wB = sm + kScanR * kScanB;    // [kScanR][kScanB]: second slots
  const int32_t nP = (KR + kScanP - 1) / kScanP, nC = (m + kScanB - 1) / kScanB;
  for (int32_t tile = blockIdx.x; tile < nP * nC; tile += gridDim.x) {
    const int32_t k0 = 1 + (tile % nP) * kScanP, c0 = (tile / nP) * kScanB;
    // row j of side A is slot u0(c0) + k0 + j, of side B slot u0(c0) - k0 - (kScanP-1) + j (mod m)
    int32_t baseA = (int32_t)(((int64_t)c0 + H + k0) % m);
    int32_t baseB = (int32_t)(((int64_t)c0 + H - k0 - (kScanP - 1)) % m);
    baseB = baseB < 0 ? baseB + m : baseB;
    const int32_t c = c0 + lane;
    // rows in groups of 32 per warp: lane l fetches row l's tile, d and start
    // position (coalesced), then the warp streams the 32 rows' class runs
    // (one 128-byte load each, all in flight together)
    constexpr int NG = 2 * kScanR / 32;
    for (int32_t grp = warp; grp < NG; grp += nwarp) {
      const bool sideA = grp < kScanR / 32;
      const int32_t row = (sideA ? grp : grp - kScanR / 32) * 32 + lane;
      int32_t y = (sideA ? baseA : baseB) + row;   // < 3m
      y = y >= m ? y - m : y;
      y = y >= m ? y - m : y;
      const int32_t t = __ldg(r + y), dy = __ldg(d + y);
      // sigma-position of class c0's partner: c0 + H - sigma(y) mod m, where
      // sigma(y) = y H mod m is y/2 or (y+m)/2 (m odd) -- no 64-bit remainder
      int32_t q = c0 + H - ((y & 1) ? (y + m) >> 1 : y >> 1);
      q = q < 0 ? q + m : (q >= m ? q - m : q);
      int32_t val[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const int32_t ti = __shfl_sync(0xffffffffu, t, i);
        const int32_t qi = __shfl_sync(0xffffffffu, q, i);
        val[i] = __ldg(Ep + (int64_t)ti * ldp + qi + lane);   // qi + lane < m + 32 <= ldp (cyclic copy)
      }
      int32_t* dst = (sideA ? wA : wB) + (row - lane) * kScanB;
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const int32_t di = __shfl_sync(0xffffffffu, dy, i);
        dst[i * kScanB + lane] = val[i] - di;
      }
    }
    __syncthreads();
    if (c < m) {
      // pair k = k0 + kk at class c0 + lane: first slot = row lane + kk of A,
      // second slot = row lane + kScanP-1 - kk of B (conflict-free: bank = lane)
      for (int32_t kk = warp; kk < kScanP && k0 + kk <= KR; kk += nwarp) {
        if ((int64_t)wA[(lane + kk) * kScanB + lane] + wB[(lane + kScanP - 1 - kk) * kScanB + lane] < 0)
          p->flags[c] = stamp;
      }
    }
    __syncthreads();
  }
  if (S % 2 == 0) {   // the pairs (u0(c), S-1)
    const int32_t* __restrict__ E = p->E;
    const int64_t ld = p->ldE;
    for (int32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < m; c += gridDim.x * blockDim.x) {
      int32_t u0 = c + H;
      u0 = u0 >= m ? u0 - m : u0;
      const int32_t a = __ldg(r + u0), b = __ldg(r + S - 1);
      if ((int64_t)__ldg(d + u0) + __ldg(d + S - 1) >
          (int64_t)__ldg(E + (int64_t)b * ld + u0) + __ldg(E + (int64_t)a * ld + (S - 1)))
        p->flags[c] = stamp;
    }
  }
}

// Stamp every class that has a firing pair on the round's start state.  A
// pair whose slots were not swapped during the previous round did not fire
// then on the same values, so after a sparse round only the pairs of the
// slots it swapped (dprev) are tested; after the dense stage, all pairs
// (streamed from Ep when TRAP left it, else gathered from E).
__global__ void __launch_bounds__(256) k_sp_scan(const SpParams* __restrict__ p) {
  extern __shared__ __align__(16) int32_t sm_scan[];
  if (p->out->status != PM_OK) return;
  if (blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(p->launches, 1ull);
  const Classes cl(p->S);
  const int32_t stamp = (int32_t)p->out->rounds + 1;
  const int32_t ndp = p->nd_prev;
  if (ndp < 0 && p->Ep) {
    scan_full_ep(p, stamp, sm_scan);
    return;
  }
  const int32_t* __restrict__ E = p->E;
  const int32_t* __restrict__ r = p->r;
  const int32_t* __restrict__ d = p->d;
  const int64_t ld = p->ldE;
  const int64_t total = ndp >= 0 ? (int64_t)cl.ncls * ndp : (int64_t)cl.ncls * cl.npairs;
  const int32_t per = ndp >= 0 ? ndp : cl.npairs;
  for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = (int32_t)(idx / per), k = (int32_t)(idx - (int64_t)c * per);
    int32_t u, v;
    if (ndp >= 0) {
      u = __ldg(p->dprev + k);
      v = cl.partner(c, u);
      if (v == u) continue;
    } else {
      cl.pair(c, k, u, v);
    }
    const int32_t a = __ldg(r + u), b = __ldg(r + v);
    const int64_t lhs = (int64_t)__ldg(d + u) + __ldg(d + v);
    if (lhs > (int64_t)__ldg(E + (int64_t)b * ld + u) + __ldg(E + (int64_t)a * ld + v)) p->flags[c] = stamp;
  }
}

// One round of Alg. 2 by one CTA (see the header).  kSmem: r, d and the dirty
// set in shared memory (S <= ~17K), else in global scratch.
template <bool kSmem>
__global__ void __launch_bounds__(kWalkThreads, 1) k_sp_walk(SpParams* p, cudaGraphConditionalHandle h) {
  extern __shared__ __align__(16) int32_t smem[];
  __shared__ int32_t s_nd, s_first[3], s_nf, s_red[32];
  __shared__ int32_t s_fl[kFlSmem];
  const int32_t S = p->S;
  const Classes cl(S);
  const int32_t m = cl.ncls;
  const int tid = threadIdx.x, T = blockDim.x;
  LsResult* o = p->out;
  if (o->status != PM_OK) {                      // uniform
    if (tid == 0) cudaGraphSetConditional(h, 0);
    return;
  }
  int32_t* const base = kSmem ? smem : p->gbuf;
  int32_t* const R = base;
  int32_t* const D = R + S;
  int32_t* const L = D + S;
  uint8_t* const dirty = reinterpret_cast<uint8_t*>(L + S);
  const int32_t* __restrict__ E = p->E;
  const int64_t ld = p->ldE;
  const int32_t stamp = (int32_t)o->rounds + 1;
#ifdef PM_LS_PROFILE
  unsigned long long t_start;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_start));
  int32_t n_win = 0, n_app = 0;
  long long t_ev = 0, t_bar = 0, t_ap = 0, t_pro = 0, t_pa = 0, t_pb = 0, t_pc = 0;
  long long t0 = clock64(), t1 = 0;
#endif
  for (int32_t x = tid; x < S; x += T) {
    R[x] = p->r[x];
    D[x] = p->d[x];
    dirty[x] = 0;
  }
  // stamped classes, in class order (block-wide compaction into p->flist)
  {
    const int32_t chunk = (m + T - 1) / T;
    const int32_t c0 = min(m, tid * chunk), c1 = min(m, c0 + chunk);
    int32_t cnt = 0;
    for (int32_t c = c0; c < c1; ++c) cnt += (p->flags[c] == stamp);
    // exclusive scan over threads
    const int lane = tid & 31, w = tid >> 5;
    int32_t incl = cnt;
#pragma unroll
    for (int o2 = 1; o2 < 32; o2 <<= 1) {
      const int32_t y = __shfl_up_sync(0xffffffffu, incl, o2);
      if (lane >= o2) incl += y;
    }
    if (lane == 31) s_red[w] = incl;
    __syncthreads();
    if (w == 0) {
      int32_t v = (lane < (T >> 5)) ? s_red[lane] : 0;
#pragma unroll
      for (int o2 = 1; o2 < 32; o2 <<= 1) {
        const int32_t y = __shfl_up_sync(0xffffffffu, v, o2);
        if (lane >= o2) v += y;
      }
      s_red[lane] = v;                           // inclusive per warp
      if (lane == 31) s_nf = v;
    }
    __syncthreads();
    int32_t pos = (w > 0 ? s_red[w - 1] : 0) + incl - cnt;
    for (int32_t c = c0; c < c1; ++c)
      if (p->flags[c] == stamp) p->flist[pos++] = c;
  }
  if (tid == 0) { s_nd = 0; s_first[0] = s_first[1] = s_first[2] = INT32_MAX; }
  __syncthreads();
  const int32_t nf = s_nf;
  int32_t fptr = 0;                              // next stamped class: flist[fptr] (uniform)
  int32_t myswaps = 0;

  auto mark = [&](int32_t x) {
    if (!dirty[x]) { dirty[x] = 1; L[atomicAdd(&s_nd, 1)] = x; }
  };
  // test pair (x, y) on the current state; apply the swap if it fires
  auto test_apply = [&](int32_t x, int32_t y) {
    const int32_t a = R[x], b = R[y];
    const int32_t e_bx = __ldg(E + (int64_t)b * ld + x);
    const int32_t e_ay = __ldg(E + (int64_t)a * ld + y);
    if ((int64_t)D[x] + D[y] > (int64_t)e_bx + e_ay) {
      R[x] = b; R[y] = a;
      D[x] = e_bx; D[y] = e_ay;
      mark(x); mark(y);
      ++myswaps;
    }
  };

  // stamped classes in shared memory when they fit
  const int32_t* FL = p->flist;
  if (nf <= kFlSmem) {
    for (int32_t i = tid; i < nf; i += T) s_fl[i] = p->flist[i];
    FL = s_fl;
  }
  __syncthreads();
  const int32_t npairs = cl.npairs;
#ifdef PM_LS_PROFILE
  t_pro = clock64() - t0;
#endif
  int32_t c = 0;
  uint32_t win = 0;                              // window counter: s_first[win % 3]
  int32_t nd_geo = -1, G = 1, g_me = 0, j_me = 0;
  for (;;) {
    const int32_t nd = s_nd;                     // uniform (read after a barrier)
    while (fptr < nf && FL[fptr] < c) ++fptr;
    const int32_t f = (fptr < nf) ? FL[fptr] : m;  // next stamped class >= c
    if (nd == 0) {
      if (f >= m) break;
      c = f;                                     // nothing can fire before f
    }
    if (c >= m) break;
    // Window: the next nw unstamped classes (only pairs with a dirty slot can
    // fire there) and, if it follows them, the stamped class f (all pairs),
    // all tested on the current state; exact up to the first firing class.
    constexpr int U = kItemsPerThread;           // pair tests per thread per batch: all
                                                 // gathers issued before any test
    // thread geometry for nd <= T: G threads per dirty slot (recomputed only
    // when nd changes; nd is uniform)
    if (nd != nd_geo) {
      nd_geo = nd;
      if (nd > 0 && nd <= T) {
        G = T / nd;
        g_me = tid / nd;
        j_me = tid - g_me * nd;
      }
    }
    int32_t K = nd == 0 ? 1 : (nd <= T ? U * G : 1);
    K = K > kWinMax ? kWinMax : K;
    const int32_t nw = min(K, f - c);
    const bool inc_f = f < m && f - c <= K;
    int32_t* first = s_first + (win % 3);
    if (tid == 0) s_first[(win + 1) % 3] = INT32_MAX;   // last read two windows ago
    ++win;
#ifdef PM_LS_PROFILE
    ++n_win;
    t1 = clock64();
#endif
    int32_t my_cc = INT32_MAX, fx = 0, fy = 0, f_bx = 0, f_ay = 0;
    // batch 1: this thread's dirty items (nd <= T: dirty slot L[j_me], classes
    // c + g_me + q*G -- ascending; nw <= U*G so one batch covers them)
    int32_t dcc[U], dy[U], deb[U], dea[U];
    int32_t dx = 0, dDx = 0;
#pragma unroll
    for (int q = 0; q < U; ++q) dcc[q] = INT32_MAX;
    if (nw > 0 && nd <= T && g_me < G) {
      dx = L[j_me];
      const int32_t Rx = R[dx];
      dDx = D[dx];
#pragma unroll
      for (int q = 0; q < U; ++q) {
        const int32_t i = g_me + q * G;
        if (i < nw) {
          const int32_t cq = c + i;
          const int32_t y = cl.partner(cq, dx);
          if (!(y == dx || (dirty[y] && y < dx))) {   // idle slot / tested from y
            dcc[q] = cq; dy[q] = y;
            deb[q] = __ldg(E + (int64_t)R[y] * ld + dx);
            dea[q] = __ldg(E + (int64_t)Rx * ld + y);
          }
        }
      }
    }
#ifdef PM_LS_PROFILE
    const long long tA = clock64();
#endif
    // batch 2: the stamped class f (all pairs), loads in flight with batch 1
    int32_t sx[U], sy[U], seb[U], sea[U];
    bool sok[U];
    const bool f_one_batch = npairs <= U * T;
#pragma unroll
    for (int q = 0; q < U; ++q) {
      const int32_t k = tid + q * T;
      sok[q] = inc_f && f_one_batch && k < npairs;
      if (sok[q]) {
        cl.pair(f, k, sx[q], sy[q]);
        seb[q] = __ldg(E + (int64_t)R[sy[q]] * ld + sx[q]);
        sea[q] = __ldg(E + (int64_t)R[sx[q]] * ld + sy[q]);
      }
    }
#ifdef PM_LS_PROFILE
    const long long tB = clock64();
#endif
#pragma unroll
    for (int q = 0; q < U; ++q)
      if (my_cc == INT32_MAX && dcc[q] != INT32_MAX && (int64_t)dDx + D[dy[q]] > (int64_t)deb[q] + dea[q]) {
        my_cc = dcc[q]; fx = dx; fy = dy[q]; f_bx = deb[q]; f_ay = dea[q];
      }
#ifdef PM_LS_PROFILE
    const long long tC = clock64();
    t_pa += tA - t1; t_pb += tB - tA; t_pc += tC - tB;
#endif
    if (nw > 0 && nd > T) {
      // more dirty slots than threads: class by class
      for (int32_t i = 0; i < nw && my_cc == INT32_MAX; ++i) {
        const int32_t cq = c + i;
        for (int32_t j0 = tid; j0 < nd && my_cc == INT32_MAX; j0 += U * T) {
          int32_t xs[U], ys[U], eb[U], ea[U];
          bool ok[U];
#pragma unroll
          for (int q = 0; q < U; ++q) {
            const int32_t j = j0 + q * T;
            ok[q] = false;
            if (j < nd) {
              const int32_t x = L[j];
              const int32_t y = cl.partner(cq, x);
              if (!(y == x || (dirty[y] && y < x))) {
                ok[q] = true; xs[q] = x; ys[q] = y;
                eb[q] = __ldg(E + (int64_t)R[y] * ld + x);
                ea[q] = __ldg(E + (int64_t)R[x] * ld + y);
              }
            }
          }
#pragma unroll
          for (int q = 0; q < U; ++q)
            if (my_cc == INT32_MAX && ok[q] && (int64_t)D[xs[q]] + D[ys[q]] > (int64_t)eb[q] + ea[q]) {
              my_cc = cq; fx = xs[q]; fy = ys[q]; f_bx = eb[q]; f_ay = ea[q];
            }
        }
      }
    }
#pragma unroll
    for (int q = 0; q < U; ++q)
      if (my_cc == INT32_MAX && sok[q] && (int64_t)D[sx[q]] + D[sy[q]] > (int64_t)seb[q] + sea[q]) {
        my_cc = f; fx = sx[q]; fy = sy[q]; f_bx = seb[q]; f_ay = sea[q];
      }
    if (inc_f && !f_one_batch) {
      // a stamped class with more than U*T pairs
      for (int32_t k0 = tid; k0 < npairs && my_cc == INT32_MAX; k0 += U * T) {
        int32_t xs[U], ys[U], eb[U], ea[U];
        bool ok[U];
#pragma unroll
        for (int q = 0; q < U; ++q) {
          const int32_t k = k0 + q * T;
          ok[q] = k < npairs;
          if (ok[q]) {
            cl.pair(f, k, xs[q], ys[q]);
            eb[q] = __ldg(E + (int64_t)R[ys[q]] * ld + xs[q]);
            ea[q] = __ldg(E + (int64_t)R[xs[q]] * ld + ys[q]);
          }
        }
#pragma unroll
        for (int q = 0; q < U; ++q)
          if (my_cc == INT32_MAX && ok[q] && (int64_t)D[xs[q]] + D[ys[q]] > (int64_t)eb[q] + ea[q]) {
            my_cc = f; fx = xs[q]; fy = ys[q]; f_bx = eb[q]; f_ay = ea[q];
          }
      }
    }
    if (my_cc != INT32_MAX) atomicMin(first, my_cc);
#ifdef PM_LS_PROFILE
    long long t2 = clock64();
    t_ev += t2 - t1;
#endif
    __syncthreads();
#ifdef PM_LS_PROFILE
    { long long t3 = clock64(); t_bar += t3 - t2; t2 = t3; }
#endif
    const int32_t cf = *first;
    if (cf == INT32_MAX) {
      c += nw + (inc_f ? 1 : 0);
      continue;
    }
#ifdef PM_LS_PROFILE
    ++n_app;
#endif
    // classes before cf fire nothing.  Apply class cf: straight from the
    // registers when every thread held at most one of its pairs, else by
    // testing it again (the state has not changed since the window began).
    // (A thread's items of one class are T apart: one per thread iff the
    // class has at most T items.)
    if (nd <= T && (cf != f || npairs <= T)) {
      if (my_cc == cf) {
        const int32_t a = R[fx], b = R[fy];
        R[fx] = b; R[fy] = a;
        D[fx] = f_bx; D[fy] = f_ay;
        mark(fx); mark(fy);
        ++myswaps;
      }
    } else if (cf == f) {
      for (int32_t k = tid; k < npairs; k += T) {
        int32_t u, v;
        cl.pair(cf, k, u, v);
        test_apply(u, v);
      }
    } else {
      for (int32_t j = tid; j < nd; j += T) {
        const int32_t x = L[j];
        const int32_t y = cl.partner(cf, x);
        if (y == x || (dirty[y] && y < x)) continue;   // one test per pair, as in the window
        test_apply(x, y);
      }
    }
    __syncthreads();
#ifdef PM_LS_PROFILE
    t_ap += clock64() - t2;
#endif
    c = cf + 1;
  }
  // ---- round end (line 11)
  __syncthreads();
  for (int32_t x = tid; x < S; x += T) {
    p->r[x] = R[x];
    p->d[x] = D[x];
  }
  const int32_t nd_end = s_nd;
  for (int32_t j = tid; j < nd_end; j += T) p->dprev[j] = L[j];
  if (tid == 0) p->nd_prev = nd_end;
  int32_t sw = myswaps;
#pragma unroll
  for (int o2 = 16; o2 > 0; o2 >>= 1) sw += __shfl_xor_sync(0xffffffffu, sw, o2);
  if ((tid & 31) == 0) s_red[tid >> 5] = sw;
  __syncthreads();
  if (tid == 0) {
    int64_t rs = 0;
    for (int w = 0; w < (T >> 5); ++w) rs += s_red[w];
    if (o->rounds < p->max_log) p->per_round[o->rounds] = rs;
    o->rounds += 1;
    o->swaps += rs;
    unsigned cont = 0;
    if (rs > 0) {
      if (p->max_rounds > 0 && o->rounds >= p->max_rounds) o->status = PM_ERR_NOT_CONVERGED;
      else cont = 1;
    }
    atomicAdd(p->launches, 1ull);
#ifdef PM_LS_PROFILE
    unsigned long long t_end;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
    const int64_t r0 = o->rounds - 1;
    if (p->max_log >= 1024 && r0 < 64) {
      p->per_round[512 + r0] = (int64_t)(t_end - t_start);
      p->per_round[576 + r0] = n_win;
      p->per_round[640 + r0] = n_app;
      p->per_round[704 + r0] = s_nd;
      p->per_round[768 + r0] = nf;
      p->per_round[832 + r0] = (int64_t)t_start;
      p->per_round[896 + r0] = (int64_t)t_end;
      p->per_round[960 + r0] = t_pro;
      p->per_round[448 + r0] = t_ev;
      p->per_round[384 + r0] = t_bar;
      p->per_round[320 + r0] = t_ap;
      p->per_round[256 + r0] = t_pa;
      p->per_round[192 + r0] = t_pb;
      p->per_round[128 + r0] = t_pc;
    }
#endif
    cudaGraphSetConditional(h, cont);
  }
}

// ---------------------------------------------------------------- host ----
struct SpGraph {
  SpParams* dparams = nullptr;
  cudaGraphExec_t exec = nullptr;
};

// Per host thread and bounded, as the CLASS graph cache (k_search.cu).
constexpr size_t kSpCacheMax = 64;
static thread_local std::map<std::tuple<int, int32_t, cudaStream_t, bool, bool, int32_t>, SpGraph> g_sp_graphs;

static int scan_blocks(int32_t S) {
  const int64_t total = (int64_t)Classes(S).ncls * Classes(S).npairs;
  int64_t b = (total + 255) / 256;
  if (b > 148 * 8) b = 148 * 8;
  return b < 1 ? 1 : (int)b;
}

static cudaError_t build_sparse_graph(int32_t S, bool use_smem, bool cluster, SpGraph& out) {
  cudaError_t e = cudaMalloc(&out.dparams, sizeof(SpParams));
  if (e != cudaSuccess) return e;
  cudaGraph_t g = nullptr;
  if ((e = cudaGraphCreate(&g, 0)) != cudaSuccess) return e;
  cudaGraphConditionalHandle h;
  if ((e = cudaGraphConditionalHandleCreate(&h, g, 0, cudaGraphCondAssignDefault)) != cudaSuccess) return e;
  const size_t smem = use_smem ? walk_smem_bytes(S) : 0;
  if (use_smem && !cluster &&
      (e = cudaFuncSetAttribute(k_sp_walk<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) != cudaSuccess)
    return e;
  // [begin] -> while { scan ; walk }
  cudaStream_t cs;
  if ((e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking)) != cudaSuccess) return e;
  if ((e = cudaStreamBeginCaptureToGraph(cs, g, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed)) != cudaSuccess)
    return e;
  const int bb = (S + 255) / 256 > 0 ? ((S + 255) / 256 < 148 ? (S + 255) / 256 : 148) : 1;
  k_sp_begin<<<bb, 256, 0, cs>>>(out.dparams, h);
  cudaStreamCaptureStatus cst;
  const cudaGraphNode_t* deps = nullptr;
  size_t ndeps = 0;
  if ((e = cudaStreamGetCaptureInfo(cs, &cst, nullptr, nullptr, &deps, &ndeps)) != cudaSuccess) return e;
  cudaGraphNodeParams cp = {};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = h;
  cp.conditional.type = cudaGraphCondTypeWhile;
  cp.conditional.size = 1;
  cudaGraphNode_t cnode;
  if ((e = cudaGraphAddNode(&cnode, g, deps, ndeps, &cp)) != cudaSuccess) return e;
  cudaGraph_t body = cp.conditional.phGraph_out[0];
  cudaGraph_t captured = g;
  if ((e = cudaStreamEndCapture(cs, &captured)) != cudaSuccess) return e;
  if ((e = cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed)) != cudaSuccess)
    return e;
  if ((e = cudaFuncSetAttribute(k_sp_scan, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kScanSmem)) !=
      cudaSuccess)
    return e;
  k_sp_scan<<<scan_blocks(S), 256, kScanSmem, cs>>>(out.dparams);
  if (cluster) {
    if ((e = launch_cwalk(out.dparams, h, S, use_smem, cs)) != cudaSuccess) {
      cudaStreamEndCapture(cs, &captured);
      cudaStreamDestroy(cs);
      return e;
    }
  } else if (use_smem) {
    k_sp_walk<true><<<1, kWalkThreads, smem, cs>>>(out.dparams, h);
  } else {
    k_sp_walk<false><<<1, kWalkThreads, 0, cs>>>(out.dparams, h);
  }
  captured = body;
  e = cudaStreamEndCapture(cs, &captured);
  cudaStreamDestroy(cs);
  if (e != cudaSuccess) return e;
  e = cudaGraphInstantiate(&out.exec, g, 0);
  cudaGraphDestroy(g);
  return e;
}

int32_t ls_sparse_threshold(int32_t S, int32_t dense_method) {
  if (S < 2 || !knob("ls_sparse", 1)) return 0;
  const int32_t t = knob("ls_sparse_T", -1);
  if (t >= 0) return t;
  // measured on B200: S <= 2048 (WINDOW + one-CTA walk): a
  // sparse round costs ~2 windows of ~1.3 us per swap plus ~15 us, a WINDOW
  // round ~0.3 us per class; with swaps falling ~3x per round the hand-over
  // sits at ~S^2/1024 swaps (S = 256: 64, 1024: 1024).  S > 2048 (CLASS +
  // cluster walk): the walk's windows are gather-bound once the dirty set
  // holds ~S slots, so hand over below ~3S/4 swaps (S = 4096: after the
  // 2489-swap round, 27 vs 33 ms; S = 16384: after the 4715-swap round,
  // 240 vs 375 ms at S^2/1024).
  // TRAP dense rounds: hand over after the first round with <= 256 swaps up to
  // S = 16384, <= 32 beyond (measured: config 4 whole search 28.3
  // ms at 256 vs 30.1 at 128, 32.7 at 64; configs 2/3 best at 256 too;
  // config 5 584 ms at 32 vs 633-1351 at S/8 = 8192 -- its walk keeps the
  // replicas in global memory and every gather goes to HBM)
  if (dense_method == PM_LS_TRAP) return S <= 16384 ? 256 : 32;
  if (S > 2048) return (int32_t)((int64_t)S * 3 / 4);
  const int64_t t2 = (int64_t)S * S / 1024;
  return (int32_t)(t2 < 1 ? 1 : (t2 > INT32_MAX ? INT32_MAX : t2));
}

pm_status_t sparse_prepare(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                           LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st,
                           SparseRun* run, int32_t pending0, const int32_t* Ep, int64_t ldp) {
  int dev = 0, optin = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  // the walk: one CTA for S <= 2048, a thread-block cluster (k_cwalk.cu)
  // beyond (measured: its cluster barrier per window only pays once the dirty
  // sets outgrow one CTA); PM_LS_CWALK=0/1 forces either
  const int32_t cw_env = knob("ls_cwalk", -1);
  const bool cluster = cw_env < 0 ? S > 2048 : cw_env != 0;
  const bool use_smem = (cluster ? cwalk_smem_ok(S, optin) : walk_smem_bytes(S) + 1024 <= (size_t)optin) &&
                        !knob("ls_sparse_gmem", 0);
  SpGraph sg;
  {
    auto key = std::make_tuple(dev, S, st, use_smem, cluster, cluster ? cwalk_cluster() : 1);
    auto it = g_sp_graphs.find(key);
    if (it == g_sp_graphs.end() && g_sp_graphs.size() >= kSpCacheMax) {
      PM_CUDA_TRY(cudaDeviceSynchronize());
      for (auto& kv : g_sp_graphs) {
        cudaGraphExecDestroy(kv.second.exec);
        cudaFree(kv.second.dparams);
      }
      g_sp_graphs.clear();
    }
    if (it == g_sp_graphs.end()) {
      SpGraph ng;
      PM_CUDA_TRY(build_sparse_graph(S, use_smem, cluster, ng));
      it = g_sp_graphs.emplace(key, ng).first;
    }
    sg = it->second;
  }
  const Classes cl(S);
  const size_t gwords = use_smem ? 0 : (cluster ? cwalk_gbuf_bytes(S) / 4 : (size_t)S * 4);   // R, D, L, dirty
  const size_t words = (size_t)S * 2 /*d, dprev*/ + (size_t)(cl.ncls + 1) * 2 /*flags, flist*/ + gwords;
  int32_t* scratch = nullptr;
  PM_CUDA_TRY(pm::scratch_alloc(&scratch, sizeof(int32_t) * words, st));
  PM_CUDA_TRY(cudaMemsetAsync(scratch + S, 0, sizeof(int32_t) * (size_t)(cl.ncls + 1), st));
  SpParams hp = {};
  hp.E = E; hp.ldE = ldE; hp.r = perm;
  hp.d = scratch;
  hp.flags = scratch + S;
  hp.flist = hp.flags + (cl.ncls + 1);
  hp.dprev = hp.flist + (cl.ncls + 1);
  hp.gbuf = use_smem ? nullptr : hp.dprev + S;
  hp.nd_prev = -1;
  hp.Ep = (Ep && S >= 2 && ldp >= (int64_t)Classes(S).m + 32) ? Ep : nullptr;
  hp.ldp = ldp;
  hp.S = S; hp.max_rounds = max_rounds; hp.max_log = max_log;
  hp.pending = pending0; hp.use_smem = use_smem ? 1 : 0;
  hp.out = dev_out; hp.per_round = dev_per_round;
  hp.launches = device_launch_counter();
  if (!hp.launches) return PM_ERR_CUDA;
  k_sp_set_params<<<1, 1, 0, st>>>(sg.dparams, hp);
  note_launch();
  PM_CUDA_TRY(cudaGetLastError());
  run->pending = &sg.dparams->pending;
  run->exec = sg.exec;
  run->scratch = scratch;
  return PM_OK;
}

__global__ void k_perm_count(const int32_t* __restrict__ perm, int32_t S, int32_t* __restrict__ seen, LsResult* out) {
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < S; u += gridDim.x * blockDim.x) {
    const int32_t t = perm[u];
    if (t < 0 || t >= S) out->status = PM_ERR_NOT_PERMUTATION;
    else atomicAdd(seen + t, 1);
  }
}
__global__ void k_perm_seen(const int32_t* __restrict__ seen, int32_t S, LsResult* out) {
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < S; u += gridDim.x * blockDim.x)
    if (seen[u] != 1) out->status = PM_ERR_NOT_PERMUTATION;
}

cudaError_t launch_perm_check(const int32_t* perm, int32_t S, LsResult* dev_out, cudaStream_t st) {
  int32_t* seen = nullptr;
  cudaError_t e = pm::scratch_alloc(&seen, sizeof(int32_t) * (size_t)S, st);
  if (e != cudaSuccess) return e;
  if ((e = cudaMemsetAsync(seen, 0, sizeof(int32_t) * (size_t)S, st)) != cudaSuccess) return e;
  const int blocks = (S + 255) / 256 < 1184 ? (S + 255) / 256 : 1184;
  k_perm_count<<<blocks, 256, 0, st>>>(perm, S, seen, dev_out);
  k_perm_seen<<<blocks, 256, 0, st>>>(seen, S, dev_out);
  note_launch(2);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  return cudaFreeAsync(seen, st);
}

pm_status_t sparse_launch(SparseRun* run, cudaStream_t st) {
  PM_CUDA_TRY(cudaGraphLaunch(run->exec, st));
  PM_CUDA_TRY(cudaFreeAsync(run->scratch, st));
  return PM_OK;
}

}  // namespace pm
