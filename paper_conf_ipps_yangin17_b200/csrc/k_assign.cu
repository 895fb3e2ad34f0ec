// k_assign.cu -- NEXT-2 of SURVEY §8(f): the paper's *optimization
// algorithm* (Sec. III): the best rearrangement R* (Eq. 3) is
// a minimum-weight perfect matching of the complete bipartite graph with
// w_{u,v} = E(I_u, T_v).  The paper solves it on the CPU with Blossom V
// (1209-1304 s at S = 64^2, Table III).  Here: an epsilon-scaling
// forward auction (Bertsekas) on the GPU, exact for integer weights.
//
// Exactness: costs are scaled by (S + 1); the last phase runs with eps = 1.
// At termination every person i (input tile) holds an object j = sigma(i)
// (target slot) with  C[i][j] + p[j] <= min_k (C[i][k] + p[k]) + eps
// (eps-complementary slackness), so the total scaled cost is within S * eps =
// S < S + 1 of the optimum; scaled costs are multiples of S + 1, hence the
// assignment is optimal.  The certificate (prices) is returned so a caller
// (tests/) can check it independently.
//
// Parallel (Jacobi) bidding in one cooperative grid: every unassigned person
// scans its row with one warp (min, argmin, second min of C[i][k] + p[k]) and
// bids p[j1] + (w2 - w1) + eps on j1 with a packed 64-bit atomicMax; after a
// grid sync each object takes its highest bid and evicts its previous owner.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>

#include "pm_internal.cuh"

namespace cg = cooperative_groups;

namespace pm {

struct AuctionArgs {
  const int32_t* E;
  int64_t ld;
  int32_t S;
  int64_t scale;                 // S + 1
  int32_t eps_shift;             // first epsilon = max(1, max C >> eps_shift)
  int32_t theta;                 // eps divisor per phase
  int64_t* price;                // [S] objects (target slots)
  int32_t* owner;                // [S] object -> person, -1 free
  unsigned long long* bid;       // [S] highest packed bid (price << 16 | person) per object
  unsigned long long* mybid;     // [S] the bid of the k-th listed person this round
  int32_t* myobj;                // [S] the object it went to
  int32_t* list;                 // [2][S] unassigned persons, double-buffered
  int32_t* counters;             // see kC* below
  int32_t max_rounds;            // cap on bidding steps (Jacobi rounds + tail bids) over all phases
  int32_t gs_threshold;          // <= kGsMax: the tail of a phase below this many bidders runs in CTA 0
  int32_t smem_price;            // the tail keeps the prices in shared memory
  int32_t keep_pairs;            // a new phase keeps the pairs that satisfy eps-CS for its eps
};

constexpr int kPersonBits = 16;  // S <= 65536
constexpr int32_t kMaxWeight = 1 << 24;   // E entries must lie in [0, 2^24)
constexpr int kThreads = 512, kWarps = kThreads / 32;
enum { kCLen0 = 0, kCLen1 = 1, kCRounds = 2, kCPhases = 3, kCMaxE = 4, kCBad = 5, kCGsBids = 6, kCGsLast = 7,
       kCHist = 8, kCTotal = 16 };
constexpr int kGsMax = 256;      // Gauss-Seidel tail queue capacity

struct Best {
  int64_t w1, w2;
  int32_t j1;
};

__device__ __forceinline__ Best merge(Best a, Best b) {
  Best r;
  if (b.w1 < a.w1 || (b.w1 == a.w1 && b.j1 < a.j1)) { r.w1 = b.w1; r.j1 = b.j1; r.w2 = min(a.w1, b.w2); }
  else { r.w1 = a.w1; r.j1 = a.j1; r.w2 = min(b.w1, a.w2); }
  return r;
}

__device__ __forceinline__ void consider(Best& b, int64_t w, int32_t j) {
  if (w < b.w1) { b.w2 = b.w1; b.w1 = w; b.j1 = j; }
  else if (w < b.w2) b.w2 = w;
}

// One thread's share of a row scan: min, argmin and second min of
// C[i][j] + p[j] = E[i][j] * scale + p[j] over its columns.  T threads split
// the row; t is this thread's index among them.  kVec: 4 columns per load
// (row 16-byte aligned), scalar tail.
template <bool kVec>
__device__ __forceinline__ Best scan_row(const int32_t* __restrict__ row, const int64_t* price, int32_t S,
                                         int64_t scale, int t, int T) {
  Best b = {INT64_MAX, INT64_MAX, 0};
  if (kVec) {
    const int32_t S4 = S & ~3;
    int32_t j = 4 * t;
    const int32_t step = 4 * T;
    for (; j + step < S4; j += 2 * step) {
      const int4 e0 = __ldg(reinterpret_cast<const int4*>(row + j));
      const int4 e1 = __ldg(reinterpret_cast<const int4*>(row + j + step));
      const longlong2 p00 = *reinterpret_cast<const longlong2*>(price + j);
      const longlong2 p01 = *reinterpret_cast<const longlong2*>(price + j + 2);
      const longlong2 p10 = *reinterpret_cast<const longlong2*>(price + j + step);
      const longlong2 p11 = *reinterpret_cast<const longlong2*>(price + j + step + 2);
      consider(b, e0.x * scale + p00.x, j);
      consider(b, e0.y * scale + p00.y, j + 1);
      consider(b, e0.z * scale + p01.x, j + 2);
      consider(b, e0.w * scale + p01.y, j + 3);
      consider(b, e1.x * scale + p10.x, j + step);
      consider(b, e1.y * scale + p10.y, j + step + 1);
      consider(b, e1.z * scale + p11.x, j + step + 2);
      consider(b, e1.w * scale + p11.y, j + step + 3);
    }
    if (j < S4) {
      const int4 e0 = __ldg(reinterpret_cast<const int4*>(row + j));
      const longlong2 p00 = *reinterpret_cast<const longlong2*>(price + j);
      const longlong2 p01 = *reinterpret_cast<const longlong2*>(price + j + 2);
      consider(b, e0.x * scale + p00.x, j);
      consider(b, e0.y * scale + p00.y, j + 1);
      consider(b, e0.z * scale + p01.x, j + 2);
      consider(b, e0.w * scale + p01.y, j + 3);
    }
    const int32_t jt = S4 + t;
    if (jt < S) consider(b, __ldg(row + jt) * scale + price[jt], jt);
  } else {
    int32_t j = t;
    for (; j + 3 * T < S; j += 4 * T) {
      int32_t e[4];
      int64_t p[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) { e[u] = __ldg(row + j + u * T); p[u] = price[j + u * T]; }
#pragma unroll
      for (int u = 0; u < 4; ++u) consider(b, e[u] * scale + p[u], j + u * T);
    }
    for (; j < S; j += T) consider(b, __ldg(row + j) * scale + price[j], j);
  }
  return b;
}

// min of a non-negative int64 over the warp with two 32-bit redux.sync ops
__device__ __forceinline__ int64_t warp_min_nonneg(int64_t v) {
  const uint32_t hi = (uint32_t)((uint64_t)v >> 32), lo = (uint32_t)v;
  const uint32_t mhi = __reduce_min_sync(0xffffffffu, hi);
  const uint32_t mlo = __reduce_min_sync(0xffffffffu, hi == mhi ? lo : 0xffffffffu);
  return (int64_t)(((uint64_t)mhi << 32) | mlo);
}

// Warp-wide (min, argmin, second min); every lane gets the result.  On ties
// of the minimum the lowest lane's column wins, and the second min equals the
// minimum.  All values are >= 0 (E >= 0, prices >= 0).
__device__ __forceinline__ Best warp_reduce(Best b) {
  Best r;
  r.w1 = warp_min_nonneg(b.w1);
  const int src = __ffs(__ballot_sync(0xffffffffu, b.w1 == r.w1)) - 1;
  r.j1 = __shfl_sync(0xffffffffu, b.j1, src);
  r.w2 = warp_min_nonneg((int)(threadIdx.x & 31) == src ? b.w2 : b.w1);
  return r;
}

__device__ __forceinline__ unsigned long long pack_bid(int64_t price, int32_t person) {
  return ((unsigned long long)price << kPersonBits) | (unsigned long long)person;
}

template <bool kVec>
__global__ void __launch_bounds__(kThreads) k_auction(AuctionArgs a) {
  cg::grid_group grid = cg::this_grid();
  extern __shared__ __align__(16) int64_t s_price[];      // [S] prices + [S] owners in the Gauss-Seidel tail (if a.smem_price)
  __shared__ Best s_best[kWarps];
  __shared__ int32_t s_q[kGsMax];
  __shared__ int32_t s_qn;
  const int32_t S = a.S;
  const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t gsz = (int64_t)gridDim.x * blockDim.x;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int32_t total_warps = gridDim.x * kWarps;
  const int64_t gwarp = gtid >> 5;
  volatile int32_t* ctr = a.counters;
  // ---- validate the weights (range bound keeps packed bids in 64 bits) and find max E
  {
    int32_t mx = 0, bad = 0;
    for (int64_t i = gwarp; i < S; i += total_warps)
      for (int32_t j = lane; j < S; j += 32) {
        const int32_t e = __ldg(a.E + i * a.ld + j);
        mx = max(mx, e);
        bad |= (e < 0 || e >= kMaxWeight);
      }
    if (mx) atomicMax(a.counters + kCMaxE, mx);
    if (bad) atomicOr(a.counters + kCBad, 1);
  }
  for (int64_t j = gtid; j < S; j += gsz) {
    a.price[j] = 0;
    a.bid[j] = 0;
    a.owner[j] = -1;
    a.list[j] = (int32_t)j;                     // phase 1: everyone unassigned
  }
  if (gtid == 0) { ctr[kCLen0] = S; ctr[kCLen1] = 0; }
  grid.sync();
  if (ctr[kCBad]) return;                       // uniform across the grid
  int64_t eps = ((int64_t)ctr[kCMaxE] * a.scale) >> a.eps_shift;
  if (eps < 1) eps = 1;
  int32_t rounds = 0, phase = 0, cur = 0, n_u = S;
  for (;;) {
    // ---- Jacobi rounds: every unassigned person bids at once
    while (n_u > a.gs_threshold && rounds < a.max_rounds) {
      const int32_t* L = a.list + (size_t)cur * S;
      int32_t* Lnext = a.list + (size_t)(cur ^ 1) * S;
      // a group of G warps (same CTA) per unassigned person
      int G = total_warps / n_u;
      G = G >= 16 ? 16 : G >= 8 ? 8 : G >= 4 ? 4 : G >= 2 ? 2 : 1;
      const int32_t ngroups = total_warps / G;
      const int32_t gid = blockIdx.x * (kWarps / G) + warp / G;
      const int wig = warp % G;
      for (int32_t base = 0; base < n_u; base += ngroups) {
        const int32_t k = base + gid;
        Best b = {INT64_MAX, INT64_MAX, 0};
        int32_t i = -1;
        if (k < n_u) {
          i = L[k];
          b = warp_reduce(scan_row<kVec>(a.E + (int64_t)i * a.ld, a.price, S, a.scale, wig * 32 + lane, G * 32));
        }
        if (G > 1) {
          if (lane == 0) s_best[warp] = b;
          __syncthreads();
          if (wig == 0 && lane == 0)
            for (int t = 1; t < G; ++t) b = merge(b, s_best[warp + t]);
          __syncthreads();
        }
        if (k < n_u && wig == 0 && lane == 0) {
          const int64_t gamma = (b.w2 == INT64_MAX ? 0 : b.w2 - b.w1) + eps;   // S == 1: no second object
          const unsigned long long bb = pack_bid(a.price[b.j1] + gamma, i);
          a.mybid[k] = bb;                      // indexed by list position: the resolution
          a.myobj[k] = b.j1;                    // loads them alongside L[k]
          atomicMax(a.bid + b.j1, bb);
        }
      }
      grid.sync();
      // resolution, per bidder: the highest bid on each object wins and evicts
      // the previous owner; losers and evicted persons form the next list
      for (int64_t k = gtid; k < n_u; k += gsz) {
        const int32_t i = L[k];
        const int32_t j = a.myobj[k];
        const unsigned long long bb = a.mybid[k];
        int32_t out = i;
        if (a.bid[j] == bb) {
          a.price[j] = (int64_t)(bb >> kPersonBits);
          out = a.owner[j];
          a.owner[j] = i;
        }
        if (out >= 0) Lnext[atomicAdd(a.counters + (cur ^ 1), 1)] = out;
      }
      ++rounds;
      if (gtid == 0)
        atomicAdd(a.counters + kCHist + (n_u <= 1 ? 0 : n_u <= 4 ? 1 : n_u <= 16 ? 2 : n_u <= 64 ? 3 : 4), 1);
      grid.sync();
      cur ^= 1;
      n_u = ctr[cur];
      if (gtid == 0) ctr[cur ^ 1] = 0;          // the list being refilled next round
    }
    // ---- Gauss-Seidel tail: CTA 0 serves the last few bidders one at a time
    // (the sequential auction of the same phase: each bid is resolved at once)
    if (n_u > 0 && n_u <= a.gs_threshold && rounds < a.max_rounds) {
      if (blockIdx.x == 0) {
        const int64_t* P = a.price;
        int32_t* O = a.owner;
        if (a.smem_price) {
          int32_t* s_owner = reinterpret_cast<int32_t*>(s_price + S);
          for (int32_t j = threadIdx.x; j < S; j += kThreads) { s_price[j] = a.price[j]; s_owner[j] = a.owner[j]; }
          P = s_price;
          O = s_owner;
        }
        const int32_t* L = a.list + (size_t)cur * S;
        if (threadIdx.x < n_u) s_q[threadIdx.x] = L[threadIdx.x];
        if (threadIdx.x == 0) s_qn = n_u;
        __syncthreads();
        int32_t bids = 0;
        while (s_qn > 0 && rounds + bids < a.max_rounds) {
          const int32_t i = s_q[s_qn - 1];
          Best b = warp_reduce(scan_row<kVec>(a.E + (int64_t)i * a.ld, P, S, a.scale, threadIdx.x, kThreads));
          if (lane == 0) s_best[warp] = b;
          __syncthreads();
          if (warp == 0) {
            if (lane < kWarps) b = s_best[lane];
            else b = Best{INT64_MAX, INT64_MAX, 0};     // identity (a duplicate would fake a tie)
            b = warp_reduce(b);
            if (lane == 0) {
              const int64_t np = P[b.j1] + (b.w2 == INT64_MAX ? 0 : b.w2 - b.w1) + eps;
              const_cast<int64_t*>(P)[b.j1] = np;
              a.bid[b.j1] = pack_bid(np, i);    // keeps the Jacobi bid floor monotone
              const int32_t prev = O[b.j1];
              O[b.j1] = i;
              if (prev >= 0) s_q[s_qn - 1] = prev;
              else --s_qn;
            }
          }
          __syncthreads();
          ++bids;
        }
        if (a.smem_price)
          for (int32_t j = threadIdx.x; j < S; j += kThreads) { a.price[j] = P[j]; a.owner[j] = O[j]; }
        if (threadIdx.x == 0) { ctr[kCGsBids] += bids; ctr[kCGsLast] = bids; ctr[cur] = s_qn; }
      }
      grid.sync();
      n_u = ctr[cur];
      rounds += ctr[kCGsLast];                  // uniform: every CTA adds the same count
    }
    ++phase;
    if (gtid == 0) { ctr[kCRounds] = rounds; ctr[kCPhases] = phase; }
    if (eps == 1 || n_u > 0) break;
    eps = eps / a.theta;
    if (eps < 1) eps = 1;
    grid.sync();                                // everyone has read the counters
    if (gtid == 0) { ctr[kCLen0] = 0; ctr[kCLen1] = 0; }
    cur = 0;
    grid.sync();
    // ---- next phase: keep the pairs that satisfy eps-CS for the new eps,
    // free the others (their persons form the first list)
    for (int64_t j = gwarp; j < S; j += total_warps) {
      const int32_t i = a.owner[j];
      if (i < 0) continue;                      // (never: the previous phase assigned everyone)
      const int32_t* row = a.E + (int64_t)i * a.ld;
      bool keep = a.keep_pairs;
      if (keep) {
        const Best b = warp_reduce(scan_row<kVec>(row, a.price, S, a.scale, lane, 32));
        keep = (int64_t)__ldg(row + j) * a.scale + a.price[j] <= b.w1 + eps;
      }
      if (!keep && lane == 0) {
        a.owner[j] = -1;
        a.list[atomicAdd(a.counters + kCLen0, 1)] = i;
      }
    }
    grid.sync();
    n_u = ctr[kCLen0];
  }
  if (gtid == 0) ctr[kCLen0] = n_u;             // unassigned at exit (0 = converged)
}

// Exact optimum of sum_v E[r[v]][v] over bijections r (Eq. 3, P:70 / P:98).
pm_status_t run_assignment(const int32_t* E, int64_t ld, int32_t S, int32_t* perm, int64_t* price_out,
                           int64_t* cost_out_dev, int32_t* h_stats, cudaStream_t st) {
  if (S > (1 << kPersonBits)) return PM_ERR_UNSUPPORTED;
  int dev = 0, sms = 148, coop = 0, per_sm = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev));
  if (!coop) return PM_ERR_UNSUPPORTED;
  const bool vec = (reinterpret_cast<uintptr_t>(E) % 16 == 0) && (ld % 4 == 0);
  void* kfn = vec ? (void*)k_auction<true> : (void*)k_auction<false>;
  int smem_optin = 0;
  PM_CUDA_TRY(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  const size_t static_smem = 8 * 1024;        // s_best, s_q and headroom
  const size_t dyn = (size_t)S * (sizeof(int64_t) + sizeof(int32_t));
  const bool smem_price = knob("auction_smem_price", 1) && dyn + static_smem <= (size_t)smem_optin;
  const size_t dyn_bytes = smem_price ? dyn : 0;
  PM_CUDA_TRY(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn_bytes));
  PM_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfn, kThreads, dyn_bytes));
  if (per_sm < 1) return PM_ERR_UNSUPPORTED;
  const int cap = knob("auction_ctas_per_sm", 1);
  int blocks = sms * (per_sm < cap ? per_sm : cap);

  char* buf = nullptr;
  const size_t bytes = sizeof(int64_t) * 3 * (size_t)S + sizeof(int32_t) * (4 * (size_t)S + kCTotal);
  PM_CUDA_TRY(scratch_alloc(&buf, bytes, st));
  AuctionArgs a = {};
  a.E = E; a.ld = ld; a.S = S; a.scale = (int64_t)S + 1;
  a.price = reinterpret_cast<int64_t*>(buf);
  a.bid = reinterpret_cast<unsigned long long*>(a.price + S);
  a.mybid = a.bid + S;
  a.owner = reinterpret_cast<int32_t*>(a.mybid + S);
  a.myobj = a.owner + S;
  a.list = a.myobj + S;
  a.counters = a.list + 2 * (size_t)S;
  a.theta = knob("auction_theta", 8);
  a.eps_shift = knob("auction_eps_shift", 3);
  a.max_rounds = knob("auction_max_rounds", 1 << 22);
  a.gs_threshold = knob("auction_gs", 8);
  a.smem_price = smem_price;
  a.keep_pairs = knob("auction_keep", 0);
  if (a.theta < 2) a.theta = 2;
  if (a.gs_threshold < 0) a.gs_threshold = 0;
  if (a.gs_threshold > kGsMax) a.gs_threshold = kGsMax;
  PM_CUDA_TRY(cudaMemsetAsync(a.counters, 0, sizeof(int32_t) * kCTotal, st));
  void* params[] = {&a};
  PM_CUDA_TRY(cudaLaunchCooperativeKernel(kfn, blocks, kThreads, params, dyn_bytes, st));
  note_launch();
  // r[v] = owner[v] (input tile at target slot v, Eq. 2's r)
  PM_CUDA_TRY(cudaMemcpyAsync(perm, a.owner, sizeof(int32_t) * S, cudaMemcpyDeviceToDevice, st));
  if (price_out) PM_CUDA_TRY(cudaMemcpyAsync(price_out, a.price, sizeof(int64_t) * S, cudaMemcpyDeviceToDevice, st));
  int32_t hc[kCTotal] = {};
  PM_CUDA_TRY(cudaMemcpyAsync(hc, a.counters, sizeof(hc), cudaMemcpyDeviceToHost, st));
  PM_CUDA_TRY(cudaStreamSynchronize(st));
  PM_CUDA_TRY(cudaFreeAsync(buf, st));
  if (h_stats) { h_stats[0] = hc[kCRounds]; h_stats[1] = hc[kCPhases]; }
  if (hc[kCBad]) return PM_ERR_INVALID;
  if (hc[kCLen0] != 0) return PM_ERR_NOT_CONVERGED;
  if (cost_out_dev) PM_CUDA_TRY(launch_cost(E, ld, S, perm, cost_out_dev, st));
  return PM_OK;
}

}  // namespace pm
