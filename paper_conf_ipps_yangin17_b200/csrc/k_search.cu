// k_search.cu -- Step 3, the parallel approximation (Algorithm 2)
// and the total error (Eq. 2) for sm_100a.
//
// State: r[u] = input tile at target slot u (reading R5) and the maintained
// diagonal d[u] = E[r[u]][u].  A pair (u, v) of class c, a = r[u], b = r[v],
// fires iff d[u] + d[v] > E[b][u] + E[a][v] (line 5, strict: reading R6); on a
// swap r[u] = b, r[v] = a, d[u] = E[b][u], d[v] = E[a][v].  This is line 5's
// four-entry test with two of the entries carried in d (the oracle evaluates
// all four every time), so each pair costs two gathers from E.
//
// Methods (pm_ls_method_t):
//   CLASS  -- the paper's structure: one kernel per colour class, the
//             n-1 class launches of a round captured once into a CUDA graph
//             whose while-node repeats rounds on the device until a round
//             has no swap (no host round trip per round).
#include <cuda_runtime.h>

#include <map>
#include <mutex>
#include <tuple>

#include "pm_internal.cuh"

namespace pm {

// Device-resident parameters of one search (fixed address per cached graph).
struct LsParams {
  const int32_t* E;
  int64_t ldE;
  int32_t* r;
  int32_t* d;          // maintained diagonal, int32 [S] (CLASS method scratch)
  int32_t* seen;       // permutation check, int32 [S]
  int32_t S;
  int32_t max_rounds;
  int32_t max_log;
  int32_t sparse_T;    // hand over to sparse rounds after a round with <= sparse_T swaps
  unsigned long long round_swaps;
  LsResult* out;
  int64_t* per_round;
  int32_t* handoff;    // SpParams::pending, or NULL
  unsigned long long* launches;   // device-side launch counter (graph kernels)
};

// ------------------------------------------------------------- CLASS -----
// Parameters travel as a kernel argument (no pageable H2D copy, no host sync).
__global__ void k_ls_set_params(LsParams* dst, LsParams src) { *dst = src; }

__global__ void k_ls_check_init(LsParams* p) {
  const int32_t S = p->S;
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < S; u += gridDim.x * blockDim.x) {
    const int32_t t = p->r[u];
    if (t < 0 || t >= S) {
      p->out->status = PM_ERR_NOT_PERMUTATION;
      continue;
    }
    atomicAdd(p->seen + t, 1);
    p->d[u] = p->E[(int64_t)t * p->ldE + u];
  }
}

__global__ void k_ls_check_seen(LsParams* p) {
  const int32_t S = p->S;
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < S; u += gridDim.x * blockDim.x)
    if (p->seen[u] != 1) p->out->status = PM_ERR_NOT_PERMUTATION;
}

// One colour class P_{c+1}: every pair concurrently (Alg. 2 line 4).
__global__ void __launch_bounds__(256) k_ls_class(const LsParams* __restrict__ p, int32_t c) {
  if (blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(p->launches, 1ull);
  if (p->out->status != PM_OK) return;
  const Classes cl(p->S);
  const int32_t k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= cl.npairs) return;
  int32_t u, v;
  cl.pair(c, k, u, v);
  int32_t* r = p->r;
  int32_t* d = p->d;
  const int32_t* E = p->E;
  const int64_t ld = p->ldE;
  const int32_t a = r[u], b = r[v];
  const int32_t e_bu = __ldg(E + (int64_t)b * ld + u);
  const int32_t e_av = __ldg(E + (int64_t)a * ld + v);
  const int32_t du = d[u], dv = d[v];
  if ((int64_t)du + dv > (int64_t)e_bu + e_av) {
    r[u] = b; r[v] = a;
    d[u] = e_bu; d[v] = e_av;
    atomicAdd(const_cast<unsigned long long*>(&p->round_swaps), 1ull);
  }
}

// Alg. 2 line 11 (+ the max_rounds cap): decide whether the while-node loops.
__global__ void k_ls_round_end(LsParams* p, cudaGraphConditionalHandle h) {
  LsResult* o = p->out;
  unsigned cont = 0;
  atomicAdd(p->launches, 1ull);
  if (o->status == PM_OK) {
    const int64_t sw = (int64_t)p->round_swaps;
    p->round_swaps = 0;
    if (o->rounds < p->max_log) p->per_round[o->rounds] = sw;
    o->rounds += 1;
    o->swaps += sw;
    if (sw > 0) {
      if (p->max_rounds > 0 && o->rounds >= p->max_rounds) o->status = PM_ERR_NOT_CONVERGED;
      else if (p->handoff && sw <= p->sparse_T) *p->handoff = 1;   // quiet: sparse rounds take over
      else cont = 1;
    }
  }
  cudaGraphSetConditional(h, cont);
}

struct ClassGraph {
  LsParams* dparams = nullptr;
  cudaGraphExec_t exec = nullptr;
};

// One cache per host thread (a cached graph reads one device params struct,
// so two threads sharing a stream handle -- the legacy default stream,
// cudaStreamPerThread -- must not share an entry); bounded: beyond
// kGraphCacheMax entries the thread's cache is dropped after a device sync.
constexpr size_t kGraphCacheMax = 64;
static thread_local std::map<std::tuple<int, int32_t, cudaStream_t>, ClassGraph> g_graphs;

static cudaError_t build_class_graph(int32_t S, cudaStream_t st, ClassGraph& out) {
  const Classes cl(S);
  cudaError_t e = cudaMalloc(&out.dparams, sizeof(LsParams));
  if (e != cudaSuccess) return e;
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
  // Populate the loop body by capturing one round onto a private stream.
  cudaStream_t cs;
  if ((e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking)) != cudaSuccess) return e;
  if ((e = cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed)) != cudaSuccess)
    return e;
  const int threads = 256;
  const int blocks = (cl.npairs + threads - 1) / threads;
  for (int32_t c = 0; c < cl.ncls; ++c) k_ls_class<<<blocks > 0 ? blocks : 1, threads, 0, cs>>>(out.dparams, c);
  k_ls_round_end<<<1, 1, 0, cs>>>(out.dparams, h);
  cudaGraph_t captured = body;
  e = cudaStreamEndCapture(cs, &captured);
  cudaStreamDestroy(cs);
  if (e != cudaSuccess) return e;
  e = cudaGraphInstantiate(&out.exec, g, 0);
  cudaGraphDestroy(g);
  (void)st;
  return e;
}

static pm_status_t run_class(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                             LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st,
                             int32_t* handoff, int32_t sparse_T) {
  int dev = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  ClassGraph cg;
  {
    auto key = std::make_tuple(dev, S, st);
    auto it = g_graphs.find(key);
    if (it == g_graphs.end() && g_graphs.size() >= kGraphCacheMax) {
      PM_CUDA_TRY(cudaDeviceSynchronize());
      for (auto& kv : g_graphs) {
        cudaGraphExecDestroy(kv.second.exec);
        cudaFree(kv.second.dparams);
      }
      g_graphs.clear();
    }
    if (it == g_graphs.end()) {
      ClassGraph ng;
      PM_CUDA_TRY(build_class_graph(S, st, ng));
      it = g_graphs.emplace(key, ng).first;
    }
    cg = it->second;
  }
  int32_t* scratch = nullptr;   // d [S] + seen [S]
  PM_CUDA_TRY(pm::scratch_alloc(&scratch, sizeof(int32_t) * 2 * (size_t)(S > 0 ? S : 1), st));
  PM_CUDA_TRY(cudaMemsetAsync(scratch + S, 0, sizeof(int32_t) * (size_t)S, st));
  LsParams hp = {};
  hp.E = E; hp.ldE = ldE; hp.r = perm; hp.d = scratch; hp.seen = scratch + S;
  hp.S = S; hp.max_rounds = max_rounds; hp.max_log = max_log;
  hp.round_swaps = 0; hp.out = dev_out; hp.per_round = dev_per_round;
  hp.handoff = handoff; hp.sparse_T = sparse_T;
  hp.launches = device_launch_counter();
  if (!hp.launches) return PM_ERR_CUDA;
  k_ls_set_params<<<1, 1, 0, st>>>(cg.dparams, hp);
  const int blocks = (S + 255) / 256 > 0 ? (S + 255) / 256 : 1;
  k_ls_check_init<<<blocks, 256, 0, st>>>(cg.dparams);
  k_ls_check_seen<<<blocks, 256, 0, st>>>(cg.dparams);
  note_launch(3);
  PM_CUDA_TRY(cudaGetLastError());
  PM_CUDA_TRY(cudaGraphLaunch(cg.exec, st));   // its kernels count themselves on the device
  PM_CUDA_TRY(cudaFreeAsync(scratch, st));
  return PM_OK;
}

pm_status_t ls_method_supported(int32_t S, int32_t method) {
  if (method == PM_LS_AUTO) method = pm_ls_auto_method(S);
  if (method == PM_LS_TRAP && (S < ls_trap_min_S() || (S & 1))) return PM_ERR_UNSUPPORTED;
  if (method == PM_LS_WINDOW && S > ls_window_max_S()) return PM_ERR_UNSUPPORTED;
  return PM_OK;
}

pm_status_t run_local_search(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                             int32_t method, LsResult* dev_out, int64_t* dev_per_round, int32_t max_log,
                             cudaStream_t st, int32_t* used_method, int32_t* ep_buf, size_t ep_bytes,
                             bool ep_ready) {
  if (method == PM_LS_AUTO) method = pm_ls_auto_method(S);
  if (used_method) *used_method = method;
  {
    const pm_status_t v = ls_method_supported(S, method);
    if (v != PM_OK) return v;
  }
  const int32_t sparse_T = (method == PM_LS_CLASS || method == PM_LS_WINDOW || method == PM_LS_TRAP)
                               ? ls_sparse_threshold(S, method) : 0;
  // TRAP's sigma-permuted copy of E lives through the sparse rounds too: their
  // first (full) scan streams its rows instead of gathering from E
  ScopedScratch ep(st);
  int64_t ldp = 0;
  const int32_t* Ep_use = nullptr;
  if (method == PM_LS_TRAP) {
    PM_CUDA_TRY(launch_perm_check(perm, S, dev_out, st));
    if (ep_buf && ep_bytes >= trap_ep_bytes(S)) {   // the caller's buffer (pm_local_search_ep/_sigma_async)
      if (ep_ready) {
        ldp = trap_ep_ld(S);                         // built with E (pm_error_matrix_sigma)
      } else {
        const pm_status_t se = trap_build_ep_into(E, ldE, S, st, ep_buf, &ldp);
        if (se != PM_OK) return se;
      }
      Ep_use = ep_buf;
    } else {
      int32_t* Ep = nullptr;
      const pm_status_t se = trap_build_ep(E, ldE, S, st, &Ep, &ldp);
      ep.p = Ep;
      if (se != PM_OK) return se;
      Ep_use = Ep;
    }
  }
  SparseRun sr;
  ScopedScratch sps(st);
  if (sparse_T > 0) {
    const pm_status_t s = sparse_prepare(E, ldE, S, perm, max_rounds, dev_out, dev_per_round, max_log, st, &sr, 0,
                                         Ep_use, ldp);
    if (s != PM_OK) return s;
    sps.p = sr.scratch;   // freed here on an error path; sparse_launch frees it otherwise
  }
  pm_status_t s;
  switch (method) {
    case PM_LS_CLASS:
      s = run_class(E, ldE, S, perm, max_rounds, dev_out, dev_per_round, max_log, st, sr.pending, sparse_T);
      break;
    case PM_LS_TRAP:
      s = run_trap(E, ldE, S, perm, max_rounds, dev_out, dev_per_round, max_log, st, sr.pending, sparse_T,
                   Ep_use, ldp);
      break;
    case PM_LS_WINDOW:
      s = run_window(E, ldE, S, perm, max_rounds, dev_out, dev_per_round, max_log, st, sr.pending, sparse_T);
      break;
    case PM_LS_WALK: {
      // every round a sparse round: start-state scan + cluster walk (S >= 2;
      // S = 1 has no colour class: one empty round, as the class graph runs it)
      if (S < 2) return run_class(E, ldE, S, perm, max_rounds, dev_out, dev_per_round, max_log, st, nullptr, 0);
      PM_CUDA_TRY(launch_perm_check(perm, S, dev_out, st));
      SparseRun wr;
      const pm_status_t s0 = sparse_prepare(E, ldE, S, perm, max_rounds, dev_out, dev_per_round, max_log, st, &wr, 1);
      if (s0 != PM_OK) return s0;
      return sparse_launch(&wr, st);
    }
    default:
      return PM_ERR_UNSUPPORTED;
  }
  if (sparse_T > 0) {
    if (s != PM_OK) return s;
    sps.p = nullptr;
    return sparse_launch(&sr, st);
  }
  return s;
}

// ------------------------------------------------------------ Eq. (2) ----
template <class Rows>
__global__ void __launch_bounds__(256) k_cost(const Rows E, int32_t S, const int32_t* __restrict__ perm,
                                              unsigned long long* __restrict__ cost) {
  // up to 8 gathers per thread, all r loads then all E loads in flight (two
  // memory round trips instead of one per gather)
  constexpr int U = 8;
  long long s = 0;
  const int32_t stride = gridDim.x * blockDim.x;
  for (int32_t u0 = blockIdx.x * blockDim.x + threadIdx.x; u0 < S; u0 += U * stride) {
    int32_t rq[U];
#pragma unroll
    for (int q = 0; q < U; ++q) rq[q] = (u0 + q * stride < S) ? __ldg(perm + u0 + q * stride) : -1;
#pragma unroll
    for (int q = 0; q < U; ++q)
      if (rq[q] >= 0) s += __ldg(E(rq[q]) + (u0 + q * stride));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  __shared__ long long red[8];
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    long long t = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += red[w];
    if (gridDim.x == 1) *cost = (unsigned long long)t;   // one block: no zeroing, no atomic
    else atomicAdd(cost, (unsigned long long)t);
  }
}

template <class Rows>
static cudaError_t launch_cost_rows(const Rows& E, int32_t S, const int32_t* perm, int64_t* d_cost,
                                    cudaStream_t st) {
  int blocks = (S + 2047) / 2048;   // <= 8 gathers per thread
  if (blocks < 1) blocks = 1;
  if (blocks > 148) blocks = 148;
  if (blocks > 1) {
    cudaError_t e = cudaMemsetAsync(d_cost, 0, sizeof(int64_t), st);
    if (e != cudaSuccess) return e;
  }
  k_cost<Rows><<<blocks, 256, 0, st>>>(E, S, perm, reinterpret_cast<unsigned long long*>(d_cost));
  note_launch();
  return cudaGetLastError();
}

cudaError_t launch_cost(const int32_t* E, int64_t ldE, int32_t S, const int32_t* perm, int64_t* d_cost,
                        cudaStream_t st) {
  return launch_cost_rows(PlainRows{E, ldE}, S, perm, d_cost, st);
}

cudaError_t launch_cost_sharded(const ShardRows& rows, int32_t S, const int32_t* perm, int64_t* d_cost,
                                cudaStream_t st) {
  return launch_cost_rows(rows, S, perm, d_cost, st);
}

}  // namespace pm

namespace pm {
int32_t ls_class_launches_per_round(int32_t S) { return Classes(S).ncls + 1; }

// r := identity (Alg. 1/2 start from the input image as given, reading R7).
__global__ void k_iota(int32_t* perm, int32_t S) {
  for (int32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < S; u += gridDim.x * blockDim.x) perm[u] = u;
}
cudaError_t launch_iota(int32_t* perm, int32_t S, cudaStream_t st) {
  int blocks = (S + 255) / 256;
  if (blocks < 1) blocks = 1;
  if (blocks > 1184) blocks = 1184;
  k_iota<<<blocks, 256, 0, st>>>(perm, S);
  note_launch();
  return cudaGetLastError();
}
}  // namespace pm
