// k_cwalk.cu -- the walk of the sparse rounds (k_sparse.cu) on a thread-block
// cluster: C CTAs on C SMs share the pair tests of every window.
//
// The one-CTA walk is bound by the gathers of one SM (each tested pair reads
// E[r[v]][u] and E[r[u]][v] from L2/HBM, ~1 L1TEX wavefront each): once the
// dirty set D outgrows the CTA it tests one class per window, ~3 us per
// class at S = 4096, slower than a whole-GPU kernel per class.  Here:
//  * every CTA keeps a REPLICA of r, d and D (shared memory up to S ~ 16K,
//    else global scratch), all replicas identical at every window boundary;
//  * a window's tests (dirty pairs of upcoming classes, all pairs of the
//    next stamped class) are split across the C CTAs;
//  * each CTA finds the first firing class among its tests and posts it,
//    with its firing pairs of that class, into a mailbox in EVERY CTA's
//    shared memory (DSMEM stores), then one cluster barrier;
//  * every CTA reads the C mailboxes, takes the smallest class and applies
//    exactly those pairs to its own replica, in mailbox order (so the dirty
//    lists stay identical).  If a CTA found more firing pairs than a mailbox
//    holds, every CTA re-tests that class in full on its replica instead.
// One cluster barrier per window; the decisions are the one-CTA walk's (the
// first firing class, decided on the current state), so r, rounds and swaps
// stay bit-identical to the oracle's replay.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include "pm_internal.cuh"

namespace cg = cooperative_groups;

namespace pm {

namespace cw {
constexpr int kThreads = 512;
constexpr int kU = 4;          // dirty-pair tests per thread per window (loads in flight)
constexpr int kUf = 8;         // stamped-class pair tests per thread (npairs / C / kThreads <= 8)
constexpr int kMail = 16;      // firing pairs one CTA posts per window
constexpr int kWinMax = 256;   // classes per window
constexpr int kFl = 2048;      // stamped classes kept in shared memory
}  // namespace cw

struct CwMail {
  int32_t cls;                 // first firing class among the CTA's tests (INT32_MAX: none)
  int32_t n;                   // its firing pairs of that class, -1 if more than kMail
  int32_t x[cw::kMail], y[cw::kMail], ex[cw::kMail], ey[cw::kMail];   // pair, new d[x], new d[y]
};

// Per-CTA replica: R, D (int32), L (dirty list, int32), dirty flags (u8).
__host__ __device__ inline size_t cwalk_state_bytes(int32_t S) { return ((size_t)S * 13 + 15) / 16 * 16; }

// Block-wide exclusive prefix sum of v (512 threads); returns the total.
__device__ __forceinline__ int32_t cw_block_scan(int32_t v, int32_t& excl, int32_t* s_red) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int32_t incl = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int32_t t = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += t;
  }
  __syncthreads();
  if (lane == 31) s_red[w] = incl;
  __syncthreads();
  if (w == 0) {
    int32_t x = (lane < (int)(blockDim.x >> 5)) ? s_red[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t t = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += t;
    }
    s_red[lane] = x;                   // inclusive per warp
  }
  __syncthreads();
  excl = (w > 0 ? s_red[w - 1] : 0) + incl - v;
  const int32_t total = s_red[(blockDim.x >> 5) - 1];
  __syncthreads();
  return total;
}

template <int C, bool kSmem>
__global__ void __launch_bounds__(cw::kThreads, 1) k_sp_cwalk(SpParams* p, cudaGraphConditionalHandle h) {
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank();
  extern __shared__ __align__(16) int32_t smem[];
  __shared__ CwMail s_mail[2][C];
  constexpr int kFlC = C > 8 ? cw::kFl / 2 : cw::kFl;
  __shared__ int32_t s_fl[kFlC];
  __shared__ int32_t s_nd, s_lmin[2], s_cnt[2], s_red[32];
  const int32_t S = p->S;
  const Classes cl(S);
  const int32_t m = cl.ncls;
  const int tid = threadIdx.x;
  constexpr int T = cw::kThreads;
  LsResult* o = p->out;
  if (o->status != PM_OK) {                      // uniform over the cluster
    if (rank == 0 && tid == 0) cudaGraphSetConditional(h, 0);
    return;
  }
  int32_t* const base = kSmem ? smem : p->gbuf + (size_t)rank * (cwalk_state_bytes(S) / 4);
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
  int32_t n_win = 0, n_split = 0, n_full = 0;
#endif

  for (int32_t x = tid; x < S; x += T) {
    R[x] = p->r[x];
    D[x] = p->d[x];
    dirty[x] = 0;
  }
  // stamped classes, in class order: each CTA compacts them itself when they
  // fit in shared memory, else CTA 0 writes the global list
  int32_t cnt = 0;
  const int32_t chunk = (m + T - 1) / T;
  const int32_t c0 = min(m, tid * chunk), c1 = min(m, c0 + chunk);
  for (int32_t c = c0; c < c1; ++c) cnt += (p->flags[c] == stamp);
  int32_t pos = 0;
  const int32_t nf = cw_block_scan(cnt, pos, s_red);
  const int32_t* FL;
  if (nf <= kFlC) {
    for (int32_t c = c0; c < c1; ++c)
      if (p->flags[c] == stamp) s_fl[pos++] = c;
    FL = s_fl;
  } else {
    if (rank == 0)
      for (int32_t c = c0; c < c1; ++c)
        if (p->flags[c] == stamp) p->flist[pos++] = c;
    FL = p->flist;
  }
  if (tid == 0) s_nd = 0;
  cluster.sync();                                // every CTA running (DSMEM), global flist written

  int32_t myswaps = 0;
  // Every CTA tests all pairs of class cc on its own replica and applies the
  // firing ones (identical in every CTA); new dirty slots are appended in
  // (thread, pair) order through a block scan, so the lists stay identical.
  // Pairs of one class are disjoint, so applying in place is exact.
  auto full_class = [&](int32_t cc) {
    uint64_t bits = 0;
    int32_t cntl = 0;
    int q = 0;
    for (int32_t k = tid; k < cl.npairs; k += T, ++q) {   // <= 64 pairs per thread (S <= 65536)
      int32_t u, v;
      cl.pair(cc, k, u, v);
      const int32_t ebu = __ldg(E + (int64_t)R[v] * ld + u);
      const int32_t eav = __ldg(E + (int64_t)R[u] * ld + v);
      if ((int64_t)D[u] + D[v] > (int64_t)ebu + eav) {
        const int32_t a = R[u], bt = R[v];
        R[u] = bt; R[v] = a;
        D[u] = ebu; D[v] = eav;
        bits |= 1ull << q;
        cntl += (dirty[u] ? 0 : 1) + (dirty[v] ? 0 : 1);
        ++myswaps;
      }
    }
    int32_t excl = 0;
    const int32_t tot = cw_block_scan(cntl, excl, s_red);
    int32_t w = s_nd + excl;
    while (bits) {
      const int qq = __ffsll((long long)bits) - 1;
      bits &= bits - 1;
      int32_t u, v;
      cl.pair(cc, tid + qq * T, u, v);
      if (!dirty[u]) { dirty[u] = 1; L[w++] = u; }
      if (!dirty[v]) { dirty[v] = 1; L[w++] = v; }
    }
    __syncthreads();
    if (tid == 0) s_nd += tot;
    __syncthreads();
  };
  int32_t c = 0, fptr = 0;
  int par = 0;
  for (;;) {
    const int32_t nd = s_nd;                     // uniform, identical in every CTA
    while (fptr < nf && FL[fptr] < c) ++fptr;
    const int32_t f = (fptr < nf) ? FL[fptr] : m;
    if (nd == 0) {
      if (f >= m) break;
      c = f;                                     // nothing can fire before f
    }
    if (c >= m) break;
#ifdef PM_LS_PROFILE
    ++n_win;
#endif
    if (nd > cw::kU * T * C) {                   // more dirty slots than one pass of tests: class c in full
#ifdef PM_LS_PROFILE
      ++n_full;
#endif
      full_class(c);
      c += 1;
      continue;
    }
    // Window: redundant (every CTA tests everything, no cluster traffic) while
    // one CTA's pass covers >= 8 classes and the stamped class fits; else the
    // tests are split across the cluster and exchanged through the mailboxes.
    const int32_t K1 = nd == 0 ? cw::kWinMax : (cw::kU * T) / nd;
    const bool red = K1 >= 8 && cl.npairs <= cw::kUf * T;
    int32_t K = red ? K1 : (nd == 0 ? 1 : (cw::kU * T * C) / nd);
    K = K < 1 ? 1 : (K > cw::kWinMax ? cw::kWinMax : K);
    const int32_t nw = min(K, f - c);
    const bool inc_f = f < m && f - c <= K;

    // ---- this CTA's tests, loads issued before any test ----
    int32_t my_cls = INT32_MAX;
    // dirty items t = i * nd + j (class c + i, dirty slot L[j]), this CTA's chunk [t0, t1)
    const int32_t ni = nw * nd;
    const int32_t ch = red ? ni : (ni + C - 1) / C;
    const int32_t t0 = red ? 0 : rank * ch, t1 = min(ni, t0 + ch);
    int32_t dcls[cw::kU], dx[cw::kU], dy[cw::kU], deb[cw::kU], dea[cw::kU];
#pragma unroll
    for (int q = 0; q < cw::kU; ++q) {
      dcls[q] = INT32_MAX;
      const int32_t t = t0 + tid + q * T;
      if (t < t1) {
        const int32_t i = t / nd, j = t - i * nd;
        const int32_t x = L[j];
        const int32_t cq = c + i;
        const int32_t y = cl.partner(cq, x);
        if (!(y == x || (dirty[y] && y < x))) {  // idle slot / pair tested from y
          dcls[q] = cq; dx[q] = x; dy[q] = y;
          deb[q] = __ldg(E + (int64_t)R[y] * ld + x);
          dea[q] = __ldg(E + (int64_t)R[x] * ld + y);
        }
      }
    }
    // the stamped class f: pairs k of this CTA's range
    const int32_t npc = red ? cl.npairs : (cl.npairs + C - 1) / C;
    const int32_t k0 = red ? 0 : rank * npc, k1 = min(cl.npairs, k0 + npc);
    uint32_t sfire = 0;
    int32_t sx[cw::kUf], sy[cw::kUf], seb[cw::kUf], sea[cw::kUf];
    if (inc_f) {
#pragma unroll
      for (int q = 0; q < cw::kUf; ++q) {
        const int32_t k = k0 + tid + q * T;
        sx[q] = -1;
        if (k < k1) {
          cl.pair(f, k, sx[q], sy[q]);
          seb[q] = __ldg(E + (int64_t)R[sy[q]] * ld + sx[q]);
          sea[q] = __ldg(E + (int64_t)R[sx[q]] * ld + sy[q]);
        }
      }
    }
#pragma unroll
    for (int q = 0; q < cw::kU; ++q)
      if (dcls[q] != INT32_MAX) {
        if ((int64_t)D[dx[q]] + D[dy[q]] > (int64_t)deb[q] + dea[q]) my_cls = min(my_cls, dcls[q]);
        else dcls[q] = INT32_MAX;                // keep only firing items
      }
    if (inc_f) {
#pragma unroll
      for (int q = 0; q < cw::kUf; ++q)
        if (sx[q] >= 0 && (int64_t)D[sx[q]] + D[sy[q]] > (int64_t)seb[q] + sea[q]) sfire |= 1u << q;
      if (sfire) my_cls = min(my_cls, f);
    }
    if (tid == 0) { s_lmin[par] = INT32_MAX; s_cnt[par] = 0; }
    __syncthreads();
    if (my_cls != INT32_MAX) atomicMin(&s_lmin[par], my_cls);
    __syncthreads();
    const int32_t lmin = s_lmin[par];
    if (red) {
      // every CTA decided the same window: apply class lmin from the registers,
      // new dirty slots appended in (thread, item) order
      if (lmin == INT32_MAX) {
        c += nw + (inc_f ? 1 : 0);
        par ^= 1;
        continue;
      }
      int32_t cntl = 0;
#pragma unroll
      for (int q = 0; q < cw::kU; ++q)
        if (dcls[q] == lmin) {
          const int32_t x = dx[q], y = dy[q];
          const int32_t a = R[x], bt = R[y];
          R[x] = bt; R[y] = a;
          D[x] = deb[q]; D[y] = dea[q];
          cntl += (dirty[x] ? 0 : 1) + (dirty[y] ? 0 : 1);
          ++myswaps;
        }
      if (lmin == f) {
#pragma unroll
        for (int q = 0; q < cw::kUf; ++q)
          if ((sfire >> q) & 1u) {
            const int32_t x = sx[q], y = sy[q];
            const int32_t a = R[x], bt = R[y];
            R[x] = bt; R[y] = a;
            D[x] = seb[q]; D[y] = sea[q];
            cntl += (dirty[x] ? 0 : 1) + (dirty[y] ? 0 : 1);
            ++myswaps;
          }
      }
      int32_t excl = 0;
      const int32_t tot = cw_block_scan(cntl, excl, s_red);
      int32_t w = s_nd + excl;
#pragma unroll
      for (int q = 0; q < cw::kU; ++q)
        if (dcls[q] == lmin) {
          if (!dirty[dx[q]]) { dirty[dx[q]] = 1; L[w++] = dx[q]; }
          if (!dirty[dy[q]]) { dirty[dy[q]] = 1; L[w++] = dy[q]; }
        }
      if (lmin == f) {
#pragma unroll
        for (int q = 0; q < cw::kUf; ++q)
          if ((sfire >> q) & 1u) {
            if (!dirty[sx[q]]) { dirty[sx[q]] = 1; L[w++] = sx[q]; }
            if (!dirty[sy[q]]) { dirty[sy[q]] = 1; L[w++] = sy[q]; }
          }
      }
      __syncthreads();
      if (tid == 0) s_nd += tot;
      __syncthreads();
      c = lmin + 1;
      par ^= 1;
      continue;
    }
#ifdef PM_LS_PROFILE
    ++n_split;
#endif
    // ---- post this CTA's firing pairs of class lmin to every CTA's mailbox ----
    auto post = [&](int32_t x, int32_t y, int32_t ex, int32_t ey) {
      const int32_t slot = atomicAdd(&s_cnt[par], 1);
      if (slot < cw::kMail)
        for (int d = 0; d < C; ++d) {
          CwMail* mb = cluster.map_shared_rank(&s_mail[par][rank], d);
          mb->x[slot] = x; mb->y[slot] = y; mb->ex[slot] = ex; mb->ey[slot] = ey;
        }
    };
    if (lmin != INT32_MAX) {
#pragma unroll
      for (int q = 0; q < cw::kU; ++q)
        if (dcls[q] == lmin) post(dx[q], dy[q], deb[q], dea[q]);
      if (lmin == f) {
#pragma unroll
        for (int q = 0; q < cw::kUf; ++q)
          if ((sfire >> q) & 1u) post(sx[q], sy[q], seb[q], sea[q]);
      }
    }
    __syncthreads();
    if (tid < C) {
      CwMail* mb = cluster.map_shared_rank(&s_mail[par][rank], tid);
      mb->cls = lmin;
      mb->n = s_cnt[par] <= cw::kMail ? s_cnt[par] : -1;
    }
    cluster.sync();                              // all mailboxes of this window posted

    int32_t gc = INT32_MAX;
    bool ovf = false;
#pragma unroll
    for (int b2 = 0; b2 < C; ++b2) gc = min(gc, s_mail[par][b2].cls);
    if (gc == INT32_MAX) {
      c += nw + (inc_f ? 1 : 0);
      par ^= 1;
      continue;
    }
#pragma unroll
    for (int b2 = 0; b2 < C; ++b2) ovf |= (s_mail[par][b2].cls == gc && s_mail[par][b2].n < 0);
    if (!ovf) {
      // apply the posted pairs of class gc in mailbox order (one warp; pairs are disjoint)
      if (tid < 32) {
        int32_t ndl = nd;
        for (int b2 = 0; b2 < C; ++b2) {
          const CwMail& mb = s_mail[par][b2];
          if (mb.cls != gc) continue;
          for (int i0 = 0; i0 < mb.n; i0 += 32) {
            const int i = i0 + tid;
            int32_t x = -1, y = -1, nx = 0;
            if (i < mb.n) {
              x = mb.x[i]; y = mb.y[i];
              const int32_t a = R[x], bt = R[y];
              R[x] = bt; R[y] = a;
              D[x] = mb.ex[i]; D[y] = mb.ey[i];  // d[x] = E[r_old[y]][x], d[y] = E[r_old[x]][y]
              nx = (dirty[x] ? 0 : 1) + (dirty[y] ? 0 : 2);
              ++myswaps;
            }
            // dirty-list appends in lane order
            const int32_t cntl = (nx & 1) + (nx >> 1);
            int32_t incl = cntl;
#pragma unroll
            for (int ofs = 1; ofs < 32; ofs <<= 1) {
              const int32_t t = __shfl_up_sync(0xffffffffu, incl, ofs);
              if (tid >= ofs) incl += t;
            }
            int32_t w = ndl + incl - cntl;
            if (nx & 1) { dirty[x] = 1; L[w++] = x; }
            if (nx & 2) { dirty[y] = 1; L[w++] = y; }
            ndl += __shfl_sync(0xffffffffu, incl, 31);
          }
        }
        if (tid == 0) s_nd = ndl;
      }
    } else {
      // a CTA had more firing pairs than its mailbox holds: every CTA tests
      // class gc in full on its replica (unchanged since the window began)
      full_class(gc);
    }
    __syncthreads();
    c = gc + 1;
    par ^= 1;
  }
  // ---- round end (line 11): CTA 0 publishes; the replicas are identical ----
  int32_t e0 = 0;
  const int32_t rs_all = cw_block_scan(myswaps, e0, s_red);
  if (rank == 0) {
    for (int32_t x = tid; x < S; x += T) {
      p->r[x] = R[x];
      p->d[x] = D[x];
    }
    const int32_t nd_end = s_nd;
    for (int32_t j = tid; j < nd_end; j += T) p->dprev[j] = L[j];
    if (tid == 0) {
      p->nd_prev = nd_end;
      const int64_t rs = rs_all;
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
        p->per_round[640 + r0] = n_split;
        p->per_round[704 + r0] = nd_end;
        p->per_round[768 + r0] = nf;
        p->per_round[832 + r0] = (int64_t)t_start;
        p->per_round[896 + r0] = (int64_t)t_end;
        p->per_round[960 + r0] = n_full;
      }
#endif
      cudaGraphSetConditional(h, cont);
    }
  }
}

}  // namespace pm

namespace pm {

namespace {
// cluster sizes: 8 (portable) or 16 (non-portable; tuning ls_cwalk_c)
template <int C>
constexpr size_t cw_static_smem() {
  return sizeof(CwMail) * 2 * C + sizeof(int32_t) * ((C > 8 ? cw::kFl / 2 : cw::kFl) + 40);
}
}  // namespace

// 16 CTAs by default (measured: config 4 whole search 29.4 -> 28.5 ms; the
// windows are bound by the gathers of the cluster's SMs), 8 by tuning
int32_t cwalk_cluster() { return knob("ls_cwalk_c", 16) >= 16 ? 16 : 8; }

bool cwalk_smem_ok(int32_t S, int optin) {
  const size_t st = cwalk_cluster() == 16 ? cw_static_smem<16>() : cw_static_smem<8>();
  return cwalk_state_bytes(S) + st + 1024 <= (size_t)optin;
}
size_t cwalk_gbuf_bytes(int32_t S) { return cwalk_state_bytes(S) * cwalk_cluster(); }

template <int C>
static cudaError_t launch_cwalk_c(SpParams* p, cudaGraphConditionalHandle h, int32_t S, bool smem, cudaStream_t st) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(C, 1, 1);
  cfg.blockDim = dim3(cw::kThreads, 1, 1);
  cfg.dynamicSmemBytes = smem ? cwalk_state_bytes(S) : 0;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = C;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  auto fn = smem ? k_sp_cwalk<C, true> : k_sp_cwalk<C, false>;
  cudaError_t e;
  if (C > 8 && (e = cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1)) != cudaSuccess)
    return e;
  if (smem && (e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        (int)cfg.dynamicSmemBytes)) != cudaSuccess)
    return e;
  return cudaLaunchKernelEx(&cfg, fn, p, h);
}

// One cluster of the walk's CTAs (enqueued on st, e.g. while capturing the
// sparse-round graph).
cudaError_t launch_cwalk(SpParams* p, cudaGraphConditionalHandle h, int32_t S, bool smem, cudaStream_t st) {
  return cwalk_cluster() == 16 ? launch_cwalk_c<16>(p, h, S, smem, st) : launch_cwalk_c<8>(p, h, S, smem, st);
}

}  // namespace pm
