// pm_internal.cuh -- shared internals of libpm.so (CUDA path only; the CPU
// oracle under oracle/ shares nothing with this file).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <atomic>

#include "../../include/pm.h"

namespace pm {

// ----------------------------------------------------------------------------
// Launch accounting (pm_launch_count): every kernel launch in this library
// goes through note_launch().
extern std::atomic<int64_t> g_launches;
inline void note_launch(int64_t n = 1) { g_launches.fetch_add(n, std::memory_order_relaxed); }

// Stream-ordered scratch from a library-owned memory pool per device that keeps
// up to kPoolKeepBytes mapped between calls: the scratch of repeated calls is
// served without re-mapping (the default pool returns memory to the driver at
// every synchronisation, ~1 ms per call); pm_scratch_trim() releases it all.
cudaError_t scratch_alloc(void** p, size_t bytes, cudaStream_t st);
constexpr uint64_t kPoolKeepBytes = 4ull << 30;   // pool release threshold
template <typename T>
inline cudaError_t scratch_alloc(T** p, size_t bytes, cudaStream_t st) {
  return scratch_alloc(reinterpret_cast<void**>(p), bytes, st);
}

// Tuning overrides (pm_tuning_set): the measured defaults unless a test or a
// development tool overrode them through the ABI.  Never read from the
// environment; every override keeps results bit-exact.
int32_t knob(const char* name, int32_t dflt);
bool tuning_name_ok(const char* name);

// Scratch owned by a scope: freed (stream-ordered) on every return path.
struct ScopedScratch {
  void* p = nullptr;
  cudaStream_t st = nullptr;
  explicit ScopedScratch(cudaStream_t s) : st(s) {}
  ScopedScratch(const ScopedScratch&) = delete;
  ScopedScratch& operator=(const ScopedScratch&) = delete;
  ~ScopedScratch() { if (p) cudaFreeAsync(p, st); }
  template <typename T> T* as() const { return static_cast<T*>(p); }
};

#define PM_CUDA_TRY(expr)                         \
  do {                                            \
    cudaError_t _e = (expr);                      \
    if (_e != cudaSuccess) return PM_ERR_CUDA;    \
  } while (0)

// ----------------------------------------------------------------------------
// Colour classes of K_S (Theorem 1; groups P:152-203), generated on the
// fly.  0-indexed slots, class c in [0, ncls).  Reading R8: with m = S-1 (S
// even) or m = S (S odd), class c pairs slots whose sum is 2c+1 (mod m); its
// fixed point u0 = (c + (m+1)/2) mod m (the solution of 2u0 == 2c+1) is joined
// to slot S-1 when S is even and idles when S is odd.  Enumerated here as
// pair k:  k == 0 -> (u0, S-1) [even S];  k >= 1 -> (u0+k, u0-k) mod m.
struct Classes {
  int32_t S, m, half, ncls, npairs;  // half = (m+1)/2
  __host__ __device__ explicit Classes(int32_t S_) : S(S_) {
    m = (S % 2 == 0) ? S - 1 : S;
    half = (m + 1) / 2;
    ncls = (S < 2) ? 0 : m;
    npairs = S / 2;
  }
  __host__ __device__ __forceinline__ int32_t fixed_point(int32_t c) const {
    int32_t u0 = c + half;
    return u0 >= m ? u0 - m : u0;
  }
  // Pair k in [0, npairs) of class c as (u, v).  (Odd S: the fixed point idles
  // and is not enumerated.)
  __host__ __device__ __forceinline__ void pair(int32_t c, int32_t k, int32_t& u, int32_t& v) const {
    int32_t u0 = fixed_point(c);
    if (S % 2 == 0) {
      if (k == 0) { u = u0; v = S - 1; return; }
    } else {
      k += 1;  // odd S: pairs k = 1 .. (S-1)/2
    }
    int32_t a = u0 + k; if (a >= m) a -= m;
    int32_t b = u0 - k; if (b < 0) b += m;
    u = a; v = b;
  }
  // Partner of slot x in class c (x itself if it idles: odd S fixed point).
  __host__ __device__ __forceinline__ int32_t partner(int32_t c, int32_t x) const {
    int32_t u0 = fixed_point(c);
    if (S % 2 == 0) {
      if (x == S - 1) return u0;
      if (x == u0) return S - 1;
    } else if (x == u0) {
      return x;
    }
    int32_t p = 2 * c + 1 - x;  // in (-m, 2m)
    if (p < 0) p += m;
    else if (p >= m) p -= m;
    return p;
  }
};

// ----------------------------------------------------------------------------
// Internal launchers (defined in k_sad.cu / k_search.cu).
cudaError_t launch_pack(const uint8_t* img, int32_t N, int32_t M, int32_t C, uint8_t* tiles,
                        int64_t ld_tiles, int32_t tile_begin, int32_t tile_end, cudaStream_t st);
// Ep (optional): also write TRAP's sigma-permuted copy Ep[row0 + r][sigma(v)]
// (+ its cyclic extension) in the epilogue -- only when the plan has no
// split-K (sad_split_plan false); the caller permutes E afterwards otherwise.
cudaError_t launch_sad(const uint8_t* A, const uint8_t* B, int64_t ldt, int32_t nrows, int32_t S,
                       int32_t P, int32_t* E, int64_t ldE, cudaStream_t st, int32_t* Ep = nullptr,
                       int64_t ldp = 0, int32_t row0 = 0);
bool sad_split_plan(int32_t nrows, int32_t S, int32_t P);
cudaError_t launch_render(const uint8_t* img, int32_t N, int32_t M, int32_t C, const int32_t* perm,
                          uint8_t* out, cudaStream_t st);
// Step 1 fused into the E kernel's loader (no packed tiles): requires
// sad_image_ok (a tile row is a whole number of 16-byte pieces, P % 64 == 0).
bool sad_image_ok(const uint8_t* I, const uint8_t* T, int32_t N, int32_t M, int32_t C);
cudaError_t launch_sad_image(const uint8_t* I, const uint8_t* T, int32_t N, int32_t M, int32_t C,
                             int32_t row_begin, int32_t row_end, int32_t* E, int64_t ldE, cudaStream_t st,
                             int32_t* Ep = nullptr, int64_t ldp = 0);

// Device-side result of one search; layout = the int64 [3] of
// pm_local_search_async's d_result: {status, rounds, swaps}.
struct LsResult {
  int64_t status;  // pm_status_t
  int64_t rounds;
  int64_t swaps;
};
cudaError_t launch_iota(int32_t* perm, int32_t S, cudaStream_t st);
// Runs the whole search; writes device results (LsResult + per-round swaps)
// into dev_out (LsResult) and dev_per_round (int64 [max_log]).
pm_status_t run_local_search(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm,
                             int32_t max_rounds, int32_t method, LsResult* dev_out,
                             int64_t* dev_per_round, int32_t max_log, cudaStream_t st,
                             int32_t* used_method, int32_t* ep_buf = nullptr, size_t ep_bytes = 0,
                             bool ep_ready = false);
int32_t ls_class_launches_per_round(int32_t S);
int32_t ls_window_max_S();
// Ep[t][pos] = E[t][2 pos mod m], pos in [0, m + ext) (sigma-permuted rows, k_window.cu)
cudaError_t launch_permute_cols(const int32_t* E, int64_t ldE, int32_t* Ep, int64_t ldp, int32_t S, int32_t m,
                                int32_t ext, cudaStream_t st);
pm_status_t run_window(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                       LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st,
                       int32_t* handoff = nullptr, int32_t sparse_T = 0);
constexpr int kMaxRanks = 8;

// Where row g of E (or of its sigma-permuted copy) lives: one matrix, or
// row shards across the ranks of a multi-GPU world (rank o holds rows
// [rb[o], rb[o+1]) at base[o], a peer pointer).
struct PlainRows {
  const int32_t* base;
  int64_t ld;
  __device__ __forceinline__ const int32_t* operator()(int32_t g) const { return base + (int64_t)g * ld; }
};
struct ShardRows {
  const int32_t* base[kMaxRanks];
  int32_t rb[kMaxRanks + 1];
  int32_t world;
  int64_t ld;
  __device__ __forceinline__ const int32_t* operator()(int32_t g) const {
    int o = 0;
    while (o + 1 < world && g >= rb[o + 1]) ++o;
    return base[o] + (int64_t)(g - rb[o]) * ld;
  }
};

cudaError_t launch_cost(const int32_t* E, int64_t ldE, int32_t S, const int32_t* perm, int64_t* d_cost,
                        cudaStream_t st);
// Eq. (2) over row-sharded E (peer-mapped shards)
cudaError_t launch_cost_sharded(const ShardRows& rows, int32_t S, const int32_t* perm, int64_t* d_cost,
                                cudaStream_t st);

// ---- sparse rounds (k_sparse.cu): quiet rounds of Alg. 2 ----
struct SpParams {
  const int32_t* E;
  int64_t ldE;
  int32_t* r;                  // = the caller's perm
  int32_t* d;                  // [S] diagonal E[r[x]][x]
  int32_t* flags;              // [ncls + 1] round stamp of classes with a pair firing at round start
  int32_t* flist;              // [ncls + 1] stamped classes of the current round, in order
  int32_t* gbuf;               // walk arrays when shared memory is too small (else NULL)
  int32_t S, max_rounds, max_log;
  int32_t pending;             // set by the dense stage when it hands over
  int32_t use_smem;
  int32_t nd_prev;             // slots swapped in the previous sparse round (-1: unknown)
  int32_t* dprev;              // [S] their list
  const int32_t* Ep;           // sigma-permuted copy of E (or NULL): the full scan streams its rows
  int64_t ldp;
  LsResult* out;
  int64_t* per_round;
  unsigned long long* launches;   // device-side launch counter (graph kernels)
};
struct SparseRun {
  int32_t* pending = nullptr;  // device flag the dense stage sets
  cudaGraphExec_t exec = nullptr;
  int32_t* scratch = nullptr;
};
// The walk on a thread-block cluster (k_cwalk.cu).
bool cwalk_smem_ok(int32_t S, int optin);
int32_t cwalk_cluster();   // CTAs of the walk's cluster (8, or 16 by tuning)
size_t cwalk_gbuf_bytes(int32_t S);
cudaError_t launch_cwalk(SpParams* p, cudaGraphConditionalHandle h, int32_t S, bool smem, cudaStream_t st);
// Swap-count threshold at which the dense stage (WINDOW / CLASS) hands over
// to sparse rounds; 0 = never.
int32_t ls_sparse_threshold(int32_t S, int32_t dense_method);
// Enqueue the parameter upload (before the dense stage) ...
// pending0 = 1 runs every round as a sparse round (PM_LS_WALK); the caller
// has checked that perm is a bijection.
pm_status_t sparse_prepare(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                           LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st,
                           SparseRun* run, int32_t pending0 = 0, const int32_t* Ep = nullptr, int64_t ldp = 0);
// dev_out->status = PM_ERR_NOT_PERMUTATION unless perm is a bijection of [0, S).
cudaError_t launch_perm_check(const int32_t* perm, int32_t S, LsResult* dev_out, cudaStream_t st);
// ... and the sparse-round graph (after it).
pm_status_t sparse_launch(SparseRun* run, cudaStream_t st);
// Per-device counter of kernels launched from inside CUDA graphs (device
// loops), added to pm_launch_count().
unsigned long long* device_launch_counter();
int64_t device_launch_total();

// Temporal-blocked whole-GPU search (k_trap.cu).
int32_t ls_trap_min_S();
pm_status_t run_trap(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                     LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st,
                     int32_t* handoff, int32_t sparse_T, const int32_t* Ep = nullptr, int64_t ldp = 0);
// The sigma-permuted copy Ep[t][q] = E[t][2q mod m] (q < m + 48, cyclic) that
// TRAP stages from while E <= 2 GiB (trap_ep), or NULL: allocated from the
// scratch pool on st; the caller frees it.
pm_status_t trap_build_ep(const int32_t* E, int64_t ldE, int32_t S, cudaStream_t st, int32_t** Ep, int64_t* ldp);
// Its leading dimension and size (S rows); built into a caller-owned buffer by
// trap_build_ep_into (pm_local_search_ep_async).
int64_t trap_ep_ld(int32_t S);
size_t trap_ep_bytes(int32_t S);
bool trap_ep_wanted(int32_t S);   // would trap_build_ep build the copy for S (trap_ep rule)?
pm_status_t trap_build_ep_into(const int32_t* E, int64_t ldE, int32_t S, cudaStream_t st, int32_t* Ep, int64_t* ldp);

// Multi-rank TRAP (k_trap.cu).
struct TrapRank;
size_t trap_ws_bytes(int32_t S);
pm_status_t trap_multi_supported(int32_t S, int64_t ldE, int32_t world);
// PM_OK if `method` (resolved: not AUTO) runs at this S, else PM_ERR_UNSUPPORTED
pm_status_t ls_method_supported(int32_t S, int32_t method);
size_t trap_ws_zero_bytes(int32_t S);
pm_status_t trap_multi_emulated(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t world,
                                int32_t max_rounds, LsResult* dev_out, int64_t* dev_per_round, int32_t max_log,
                                cudaStream_t st);
pm_status_t trap_multi_rank(const int32_t* E, int64_t ldE, int32_t S, int32_t* const* perm_peers,
                            void* const* ws_peers, int32_t rank, int32_t world, int32_t max_rounds,
                            LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st);
size_t trap_ws_bytes_sharded(int32_t S, int32_t rows);
pm_status_t trap_multi_rank_sharded(const int32_t* const* E_peers, const int32_t* rb, int64_t ldE, int32_t S,
                                    int32_t* const* perm_peers, void* const* ws_peers, int32_t rank, int32_t world,
                                    int32_t max_rounds, LsResult* dev_out, cudaStream_t st);
pm_status_t trap_multi_emulated_sharded(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t world,
                                        int32_t max_rounds, LsResult* dev_out, cudaStream_t st);

// Histogram matching of I to T (k_hist.cu, reading R12).
int32_t hist_max_channels();
pm_status_t run_histogram_match(const uint8_t* I, const uint8_t* T, int32_t N, int32_t C, uint8_t* out,
                                cudaStream_t st);

// Exact min-weight perfect matching by eps-scaling auction (k_assign.cu).
// h_stats (nullable): {bidding rounds, phases}.  Synchronises st.
pm_status_t run_assignment(const int32_t* E, int64_t ld, int32_t S, int32_t* perm, int64_t* price_out,
                           int64_t* cost_out_dev, int32_t* h_stats, cudaStream_t st);

}  // namespace pm
