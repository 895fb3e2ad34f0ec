// pm_abi.cu -- the extern "C" entry points of libpm.so (include/pm.h):
// argument validation, scratch management and the calls into the kernels of
// k_sad.cu / k_search.cu.  No compute happens here; there is no CPU fallback.
#include <cuda_runtime.h>

#include <algorithm>
#include <vector>

#include "pm_internal.cuh"

#include <cstring>
#include <map>
#include <mutex>
#include <string>

namespace pm {
std::atomic<int64_t> g_launches{0};

// ---- scratch pool ----------------------------------------------------------
static std::mutex g_pool_mu;
static cudaMemPool_t g_pools[64] = {};

cudaError_t scratch_alloc(void** p, size_t bytes, cudaStream_t st) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  cudaMemPool_t pool;
  {
    std::lock_guard<std::mutex> lk(g_pool_mu);
    if (!g_pools[dev]) {
      cudaMemPoolProps props = {};
      props.allocType = cudaMemAllocationTypePinned;
      props.location.type = cudaMemLocationTypeDevice;
      props.location.id = dev;
      if ((e = cudaMemPoolCreate(&g_pools[dev], &props)) != cudaSuccess) return e;
      // keep up to kPoolKeepBytes mapped between calls (the per-call scratch of
      // configs 1-4 is served without re-mapping); anything beyond goes back to
      // the driver at the next synchronisation (pm.h "Ownership")
      uint64_t thr = kPoolKeepBytes;
      if ((e = cudaMemPoolSetAttribute(g_pools[dev], cudaMemPoolAttrReleaseThreshold, &thr)) != cudaSuccess)
        return e;
    }
    pool = g_pools[dev];
  }
  return cudaMallocFromPoolAsync(p, bytes, pool, st);
}

// ---- tuning overrides (tests / development; never read from the environment)
static std::mutex g_tune_mu;
static std::map<std::string, int32_t> g_tune;

static const char* const kTuningNames[] = {
    "trap_variant", "trap_W", "trap_cluster", "trap_nbsync", "trap_cpc", "trap_prof", "trap_ep", "trap_vec",
    "trap_spec",    "trap_wait_ms", "trap_coal", "sad_plan",
    "ls_sparse",    "ls_sparse_T", "ls_cwalk", "ls_sparse_gmem", "ls_cwalk_c",
    "auction_gs",   "auction_keep", "auction_smem_price", "auction_theta", "auction_eps_shift",
    "auction_max_rounds", "auction_ctas_per_sm"};

bool tuning_name_ok(const char* name) {
  if (!name) return false;
  for (const char* n : kTuningNames)
    if (std::strcmp(n, name) == 0) return true;
  return false;
}

int32_t knob(const char* name, int32_t dflt) {
  std::lock_guard<std::mutex> lk(g_tune_mu);
  if (g_tune.empty()) return dflt;
  auto it = g_tune.find(name);
  return it == g_tune.end() ? dflt : it->second;
}

static std::mutex g_ctr_mu;
static unsigned long long* g_dev_ctr[64] = {};

unsigned long long* device_launch_counter() {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
  std::lock_guard<std::mutex> lk(g_ctr_mu);
  if (!g_dev_ctr[dev]) {
    unsigned long long* p = nullptr;
    if (cudaMalloc(&p, sizeof(unsigned long long)) != cudaSuccess) return nullptr;
    if (cudaMemset(p, 0, sizeof(unsigned long long)) != cudaSuccess) return nullptr;
    g_dev_ctr[dev] = p;
  }
  return g_dev_ctr[dev];
}

int64_t device_launch_total() {
  int cur = 0;
  if (cudaGetDevice(&cur) != cudaSuccess) return 0;
  int64_t total = 0;
  std::lock_guard<std::mutex> lk(g_ctr_mu);
  for (int dev = 0; dev < 64; ++dev) {
    if (!g_dev_ctr[dev]) continue;
    unsigned long long v = 0;
    if (cudaSetDevice(dev) == cudaSuccess &&
        cudaMemcpy(&v, g_dev_ctr[dev], sizeof(v), cudaMemcpyDeviceToHost) == cudaSuccess)
      total += (int64_t)v;
  }
  cudaSetDevice(cur);
  return total;
}
}  // namespace pm

using namespace pm;

namespace {

constexpr int32_t kMaxLog = 1024;   // per-round swap log kept on the device

bool valid_image_args(int32_t N, int32_t M, int32_t C) {
  if (N <= 0 || M <= 0 || C <= 0) return false;
  if (N % M != 0) return false;                        // P:57, S = (N/M)^2
  const int64_t P = (int64_t)M * M * C;
  if (P * 255 > INT32_MAX) return false;               // reading R11: int32 E
  const int64_t g = N / M;
  if (g * g > INT32_MAX / 2) return false;
  return true;
}

struct DevBuf {
  void* p = nullptr;
  cudaStream_t st = nullptr;
  ~DevBuf() { if (p) cudaFreeAsync(p, st); }
};

// PM_LS_* values 2 and 4 were retired in round 2 (dominated methods)
bool valid_method(int32_t method) {
  return method == PM_LS_AUTO || method == PM_LS_CLASS || method == PM_LS_WINDOW || method == PM_LS_WALK ||
         method == PM_LS_TRAP;
}

bool valid_ls_args(const int32_t* d_E, int64_t ld_E, int32_t S, const int32_t* d_perm, int32_t max_rounds,
                   int32_t method) {
  if (!d_E || !d_perm || S < 1 || ld_E < S || max_rounds < 0) return false;
  return valid_method(method);
}

// Synchronous local search: scratch, launch, read back.
pm_status_t local_search_impl(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                              int32_t max_rounds, int32_t method, int32_t* h_rounds, int64_t* h_swaps,
                              int64_t* h_per_round, int32_t len, cudaStream_t st) {
  if (!valid_ls_args(d_E, ld_E, S, d_perm, max_rounds, method)) return PM_ERR_INVALID;
  DevBuf buf;
  buf.st = st;
  const size_t bytes = sizeof(LsResult) + sizeof(int64_t) * kMaxLog;
  PM_CUDA_TRY(pm::scratch_alloc(&buf.p, bytes, st));
  LsResult* dres = reinterpret_cast<LsResult*>(buf.p);
  int64_t* dlog = reinterpret_cast<int64_t*>(reinterpret_cast<char*>(buf.p) + sizeof(LsResult));
  PM_CUDA_TRY(cudaMemsetAsync(buf.p, 0, bytes, st));
  int32_t used = method;
  pm_status_t s = run_local_search(d_E, ld_E, S, d_perm, max_rounds, method, dres, dlog, kMaxLog, st, &used);
  if (s != PM_OK) return s;
  LsResult hres;
  std::vector<int64_t> hlog;
  PM_CUDA_TRY(cudaMemcpyAsync(&hres, dres, sizeof(hres), cudaMemcpyDeviceToHost, st));
  if (h_per_round && len > 0) {
    hlog.resize(std::min(len, kMaxLog));
    PM_CUDA_TRY(cudaMemcpyAsync(hlog.data(), dlog, sizeof(int64_t) * hlog.size(), cudaMemcpyDeviceToHost, st));
  }
  PM_CUDA_TRY(cudaStreamSynchronize(st));
  if (h_rounds) *h_rounds = (int32_t)hres.rounds;
  if (h_swaps) *h_swaps = hres.swaps;
  if (h_per_round && len > 0)   // entries at and beyond `rounds` are zero
    for (size_t i = 0; i < hlog.size(); ++i) h_per_round[i] = hlog[i];
  return (pm_status_t)hres.status;
}

}  // namespace

extern "C" {

const char* pm_status_string(pm_status_t s) {
  switch (s) {
    case PM_OK: return "PM_OK";
    case PM_ERR_INVALID: return "PM_ERR_INVALID: invalid argument";
    case PM_ERR_CUDA: return "PM_ERR_CUDA: CUDA runtime error";
    case PM_ERR_NOT_CONVERGED: return "PM_ERR_NOT_CONVERGED: max_rounds reached before a zero-swap round";
    case PM_ERR_UNSUPPORTED: return "PM_ERR_UNSUPPORTED: not supported by this build/device";
    case PM_ERR_NOT_PERMUTATION: return "PM_ERR_NOT_PERMUTATION: perm is not a bijection of [0, S)";
    case PM_ERR_TIMEOUT: return "PM_ERR_TIMEOUT: a peer rank did not arrive in time";
  }
  return "PM_ERR_?: unknown status";
}

int64_t pm_tile_stride(int32_t M, int32_t C) {
  if (M <= 0 || C <= 0) return 0;
  const int64_t P = (int64_t)M * M * C;
  return (P + 63) / 64 * 64;
}

pm_status_t pm_pack_tiles(const uint8_t* d_img, int32_t N, int32_t M, int32_t C, uint8_t* d_tiles,
                          int64_t ld_tiles, pm_stream_t stream) {
  if (!d_img || !d_tiles || !valid_image_args(N, M, C)) return PM_ERR_INVALID;
  if (ld_tiles < (int64_t)M * M * C || ld_tiles % 16 != 0) return PM_ERR_INVALID;
  const int32_t g = N / M;
  PM_CUDA_TRY(launch_pack(d_img, N, M, C, d_tiles, ld_tiles, 0, g * g, (cudaStream_t)stream));
  return PM_OK;
}

pm_status_t pm_error_matrix_tiles(const uint8_t* d_input_tiles, const uint8_t* d_target_tiles,
                                  int64_t ld_tiles, int32_t S, int32_t P, int32_t row_begin, int32_t row_end,
                                  int32_t* d_E, int64_t ld_E, pm_stream_t stream) {
  if (S < 1 || P < 1 || (int64_t)P * 255 > INT32_MAX) return PM_ERR_INVALID;
  if (ld_tiles < P || ld_tiles % 64 != 0) return PM_ERR_INVALID;
  if (row_begin < 0 || row_end > S || row_begin > row_end || ld_E < S) return PM_ERR_INVALID;
  if (row_begin == row_end) return PM_OK;
  if (!d_input_tiles || !d_target_tiles || !d_E) return PM_ERR_INVALID;
  PM_CUDA_TRY(launch_sad(d_input_tiles + (int64_t)row_begin * ld_tiles, d_target_tiles, ld_tiles,
                         row_end - row_begin, S, P, d_E, ld_E, (cudaStream_t)stream));
  return PM_OK;
}

// Steps 1-2 for rows [row_begin, row_end), and (Ep != NULL) TRAP's
// sigma-permuted copy of those rows in the same pass (arguments validated by
// the callers).
static pm_status_t error_matrix_impl(const uint8_t* d_input, const uint8_t* d_target, int32_t N, int32_t M,
                                     int32_t C, int32_t row_begin, int32_t row_end, int32_t* d_E, int64_t ld_E,
                                     cudaStream_t st, int32_t* Ep) {
  const int32_t g = N / M;
  const int32_t S = g * g;
  const int64_t ldp = Ep ? trap_ep_ld(S) : 0;
  const int32_t nrows = row_end - row_begin;
  // split-K plans accumulate E with atomics: the copy is permuted afterwards
  const bool split = Ep && sad_split_plan(nrows, S, M * M * C);
  int32_t* Ep_k = split ? nullptr : Ep;
  // Step 1 fused into the E loader where the two pack launches would cost more
  // than the loader's per-stage address arithmetic (measured: fused ~8 % slower
  // per pair at S >= 16384, pack overhead dominant at S <= 4096).
  if (S <= 4096 && sad_image_ok(d_input, d_target, N, M, C)) {
    PM_CUDA_TRY(launch_sad_image(d_input, d_target, N, M, C, row_begin, row_end, d_E, ld_E, st, Ep_k, ldp));
  } else {
    const int64_t ldt = pm_tile_stride(M, C);
    DevBuf buf;
    buf.st = st;
    PM_CUDA_TRY(pm::scratch_alloc(&buf.p, (size_t)ldt * ((size_t)nrows + S), st));
    uint8_t* tI = reinterpret_cast<uint8_t*>(buf.p);
    uint8_t* tT = tI + (size_t)ldt * nrows;
    PM_CUDA_TRY(launch_pack(d_input, N, M, C, tI, ldt, row_begin, row_end, st));
    PM_CUDA_TRY(launch_pack(d_target, N, M, C, tT, ldt, 0, S, st));
    PM_CUDA_TRY(launch_sad(tI, tT, ldt, nrows, S, M * M * C, d_E, ld_E, st, Ep_k, ldp, row_begin));
  }
  if (split) PM_CUDA_TRY(launch_permute_cols(d_E, ld_E, Ep + (int64_t)row_begin * ldp, ldp, nrows, S - 1, 48, st));
  return PM_OK;
}

pm_status_t pm_error_matrix(const uint8_t* d_input, const uint8_t* d_target, int32_t N, int32_t M, int32_t C,
                            int32_t row_begin, int32_t row_end, int32_t* d_E, int64_t ld_E,
                            pm_stream_t stream) {
  if (!valid_image_args(N, M, C)) return PM_ERR_INVALID;
  const int32_t g = N / M;
  const int32_t S = g * g;
  if (row_begin < 0 || row_end > S || row_begin > row_end || ld_E < S) return PM_ERR_INVALID;
  if (row_begin == row_end) return PM_OK;   // empty shard: nothing to do, pointers unused
  if (!d_input || !d_target || !d_E) return PM_ERR_INVALID;
  return error_matrix_impl(d_input, d_target, N, M, C, row_begin, row_end, d_E, ld_E, (cudaStream_t)stream,
                           nullptr);
}

pm_status_t pm_error_matrix_sigma(const uint8_t* d_input, const uint8_t* d_target, int32_t N, int32_t M,
                                  int32_t C, int32_t* d_E, int64_t ld_E, int32_t* d_Ep, size_t ep_bytes,
                                  pm_stream_t stream) {
  if (!valid_image_args(N, M, C)) return PM_ERR_INVALID;
  const int32_t g = N / M;
  const int32_t S = g * g;
  if (!d_input || !d_target || !d_E || !d_Ep || ld_E < S || ep_bytes < trap_ep_bytes(S) ||
      (reinterpret_cast<uintptr_t>(d_Ep) & 15))
    return PM_ERR_INVALID;
  if (S < 2 || (S & 1)) return PM_ERR_UNSUPPORTED;   // the copy is defined for m = S-1 odd
  return error_matrix_impl(d_input, d_target, N, M, C, 0, S, d_E, ld_E, (cudaStream_t)stream, d_Ep);
}

int32_t pm_num_colors(int32_t S) { return Classes(S).ncls; }

pm_status_t pm_edge_coloring(int32_t S, int32_t class_begin, int32_t class_end, int32_t* h_pairs) {
  const Classes cl(S);
  if (S < 2 || !h_pairs || class_begin < 0 || class_end > cl.ncls || class_begin > class_end)
    return PM_ERR_INVALID;
  const int32_t per = S / 2;
  std::vector<std::pair<int32_t, int32_t>> grp;
  for (int32_t c = class_begin; c < class_end; ++c) {
    grp.clear();
    for (int32_t k = 0; k < cl.npairs; ++k) {
      int32_t u, v;
      cl.pair(c, k, u, v);
      grp.emplace_back(std::min(u, v), std::max(u, v));
    }
    std::sort(grp.begin(), grp.end());   // the paper lists pairs by smaller index
    int32_t* out = h_pairs + (int64_t)(c - class_begin) * per * 2;
    int32_t k = 0;
    for (; k < (int32_t)grp.size(); ++k) { out[2 * k] = grp[k].first; out[2 * k + 1] = grp[k].second; }
    for (; k < per; ++k) { out[2 * k] = -1; out[2 * k + 1] = -1; }
  }
  return PM_OK;
}

pm_status_t pm_local_search(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm, int32_t max_rounds,
                            int32_t* h_rounds, int64_t* h_swaps, pm_stream_t stream) {
  return local_search_impl(d_E, ld_E, S, d_perm, max_rounds, PM_LS_AUTO, h_rounds, h_swaps, nullptr, 0,
                           (cudaStream_t)stream);
}

pm_status_t pm_local_search_ex(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm, int32_t max_rounds,
                               int32_t method, int32_t* h_rounds, int64_t* h_swaps, int64_t* h_swaps_per_round,
                               int32_t len, pm_stream_t stream) {
  return local_search_impl(d_E, ld_E, S, d_perm, max_rounds, method, h_rounds, h_swaps, h_swaps_per_round, len,
                           (cudaStream_t)stream);
}

pm_status_t pm_local_search_async(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                  int32_t max_rounds, int32_t method, int64_t* d_result, pm_stream_t stream) {
  if (!d_result || !valid_ls_args(d_E, ld_E, S, d_perm, max_rounds, method)) return PM_ERR_INVALID;
  {
    const pm_status_t v = ls_method_supported(S, method);
    if (v != PM_OK) return v;
  }
  cudaStream_t st = (cudaStream_t)stream;
  PM_CUDA_TRY(cudaMemsetAsync(d_result, 0, sizeof(LsResult), st));
  int32_t used = method;
  return run_local_search(d_E, ld_E, S, d_perm, max_rounds, method, reinterpret_cast<LsResult*>(d_result),
                          nullptr, 0, st, &used);
}

size_t pm_sigma_copy_bytes(int32_t S) { return trap_ep_bytes(S); }

pm_status_t pm_local_search_ep_async(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                     int32_t max_rounds, int32_t method, int32_t* d_Ep, size_t ep_bytes,
                                     int64_t* d_result, pm_stream_t stream) {
  if (!d_result || !d_Ep || ep_bytes < trap_ep_bytes(S) || (reinterpret_cast<uintptr_t>(d_Ep) & 15) ||
      !valid_ls_args(d_E, ld_E, S, d_perm, max_rounds, method))
    return PM_ERR_INVALID;
  {
    const pm_status_t v = ls_method_supported(S, method);
    if (v != PM_OK) return v;
  }
  cudaStream_t st = (cudaStream_t)stream;
  PM_CUDA_TRY(cudaMemsetAsync(d_result, 0, sizeof(LsResult), st));
  int32_t used = method;
  return run_local_search(d_E, ld_E, S, d_perm, max_rounds, method, reinterpret_cast<LsResult*>(d_result),
                          nullptr, 0, st, &used, d_Ep, ep_bytes);
}

pm_status_t pm_local_search_sigma_async(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                        int32_t max_rounds, int32_t method, const int32_t* d_Ep, size_t ep_bytes,
                                        int64_t* d_result, pm_stream_t stream) {
  if (!d_result || !d_Ep || ep_bytes < trap_ep_bytes(S) || (reinterpret_cast<uintptr_t>(d_Ep) & 15) ||
      !valid_ls_args(d_E, ld_E, S, d_perm, max_rounds, method))
    return PM_ERR_INVALID;
  {
    const pm_status_t v = ls_method_supported(S, method);
    if (v != PM_OK) return v;
  }
  cudaStream_t st = (cudaStream_t)stream;
  PM_CUDA_TRY(cudaMemsetAsync(d_result, 0, sizeof(LsResult), st));
  int32_t used = method;
  // (the copy is only read: ep_ready)
  return run_local_search(d_E, ld_E, S, d_perm, max_rounds, method, reinterpret_cast<LsResult*>(d_result),
                          nullptr, 0, st, &used, const_cast<int32_t*>(d_Ep), ep_bytes, true);
}

size_t pm_trap_workspace_bytes(int32_t S) { return (S < 2) ? 0 : trap_ws_bytes(S); }

pm_status_t pm_trap_workspace_reset(void* d_ws, int32_t S, pm_stream_t stream) {
  if (!d_ws || S < 2) return PM_ERR_INVALID;
  PM_CUDA_TRY(cudaMemsetAsync(d_ws, 0, trap_ws_zero_bytes(S), (cudaStream_t)stream));
  return PM_OK;
}

pm_status_t pm_local_search_multi_async(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* const* d_perm_peers,
                                        void* const* d_ws_peers, int32_t rank, int32_t world, int32_t max_rounds,
                                        int64_t* d_result, pm_stream_t stream) {
  if (!d_E || !d_perm_peers || !d_ws_peers || !d_result || ld_E < S || max_rounds < 0) return PM_ERR_INVALID;
  if (world < 1 || rank < 0 || rank >= world) return PM_ERR_INVALID;
  for (int r = 0; r < world; ++r)
    if (!d_perm_peers[r] || !d_ws_peers[r]) return PM_ERR_INVALID;
  {
    const pm_status_t v = trap_multi_supported(S, ld_E, world);
    if (v != PM_OK) return v;
  }
  cudaStream_t st = (cudaStream_t)stream;
  PM_CUDA_TRY(cudaMemsetAsync(d_result, 0, sizeof(LsResult), st));
  return trap_multi_rank(d_E, ld_E, S, d_perm_peers, d_ws_peers, rank, world, max_rounds,
                         reinterpret_cast<LsResult*>(d_result), nullptr, 0, st);
}

pm_status_t pm_local_search_multi_emulated(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                           int32_t world, int32_t max_rounds, int32_t* h_rounds, int64_t* h_swaps,
                                           pm_stream_t stream) {
  if (!d_E || !d_perm || ld_E < S || max_rounds < 0 || world < 1) return PM_ERR_INVALID;
  {
    const pm_status_t v = trap_multi_supported(S, ld_E, world);
    if (v != PM_OK) return v;
  }
  cudaStream_t st = (cudaStream_t)stream;
  DevBuf buf;
  buf.st = st;
  PM_CUDA_TRY(pm::scratch_alloc(&buf.p, sizeof(LsResult), st));
  LsResult* dres = reinterpret_cast<LsResult*>(buf.p);
  PM_CUDA_TRY(cudaMemsetAsync(dres, 0, sizeof(LsResult), st));
  pm_status_t s = trap_multi_emulated(d_E, ld_E, S, d_perm, world, max_rounds, dres, nullptr, 0, st);
  if (s != PM_OK) return s;
  LsResult h;
  PM_CUDA_TRY(cudaMemcpyAsync(&h, dres, sizeof(h), cudaMemcpyDeviceToHost, st));
  PM_CUDA_TRY(cudaStreamSynchronize(st));
  if (h_rounds) *h_rounds = (int32_t)h.rounds;
  if (h_swaps) *h_swaps = h.swaps;
  return (pm_status_t)h.status;
}

size_t pm_trap_workspace_bytes_sharded(int32_t S, int32_t rows) {
  return (S < 2 || rows < 0 || rows > S) ? 0 : trap_ws_bytes_sharded(S, rows);
}

pm_status_t pm_local_search_sharded_async(const int32_t* const* d_E_peers, const int32_t* h_row_begin, int64_t ld_E,
                                          int32_t S, int32_t* const* d_perm_peers, void* const* d_ws_peers,
                                          int32_t rank, int32_t world, int32_t max_rounds, int64_t* d_result,
                                          pm_stream_t stream) {
  if (!d_E_peers || !h_row_begin || !d_perm_peers || !d_ws_peers || !d_result || ld_E < S || max_rounds < 0)
    return PM_ERR_INVALID;
  if (world < 1 || world > 8 || rank < 0 || rank >= world) return PM_ERR_INVALID;
  if (h_row_begin[0] != 0 || h_row_begin[world] != S) return PM_ERR_INVALID;
  for (int r = 0; r < world; ++r) {
    if (!d_perm_peers[r] || !d_ws_peers[r] || h_row_begin[r + 1] < h_row_begin[r]) return PM_ERR_INVALID;
    if (!d_E_peers[r] && h_row_begin[r + 1] > h_row_begin[r]) return PM_ERR_INVALID;
  }
  {
    const pm_status_t v = trap_multi_supported(S, ld_E, world);
    if (v != PM_OK) return v;
  }
  cudaStream_t st = (cudaStream_t)stream;
  PM_CUDA_TRY(cudaMemsetAsync(d_result, 0, sizeof(LsResult), st));
  return trap_multi_rank_sharded(d_E_peers, h_row_begin, ld_E, S, d_perm_peers, d_ws_peers, rank, world, max_rounds,
                                 reinterpret_cast<LsResult*>(d_result), st);
}

pm_status_t pm_local_search_sharded_emulated(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                             int32_t world, int32_t max_rounds, int32_t* h_rounds, int64_t* h_swaps,
                                             pm_stream_t stream) {
  if (!d_E || !d_perm || ld_E < S || max_rounds < 0 || world < 1 || world > 8) return PM_ERR_INVALID;
  {
    const pm_status_t v = trap_multi_supported(S, ld_E, world);
    if (v != PM_OK) return v;
  }
  cudaStream_t st = (cudaStream_t)stream;
  DevBuf buf;
  buf.st = st;
  PM_CUDA_TRY(pm::scratch_alloc(&buf.p, sizeof(LsResult), st));
  LsResult* dres = reinterpret_cast<LsResult*>(buf.p);
  PM_CUDA_TRY(cudaMemsetAsync(dres, 0, sizeof(LsResult), st));
  pm_status_t s = trap_multi_emulated_sharded(d_E, ld_E, S, d_perm, world, max_rounds, dres, st);
  if (s != PM_OK) return s;
  LsResult h;
  PM_CUDA_TRY(cudaMemcpyAsync(&h, dres, sizeof(h), cudaMemcpyDeviceToHost, st));
  PM_CUDA_TRY(cudaStreamSynchronize(st));
  if (h_rounds) *h_rounds = (int32_t)h.rounds;
  if (h_swaps) *h_swaps = h.swaps;
  return (pm_status_t)h.status;
}

int32_t pm_ls_auto_method(int32_t S) {
  // measured on B200 (whole search incl. sparse rounds): TRAP for
  // even S >= 256 (config 1/2/3/4: 0.42/1.50/10.7/111 ms against WINDOW
  // 0.46/1.98 and CLASS 28.6/240); below, WINDOW up to its shared-memory
  // limit, then the graph of per-class kernels
  if (S >= ls_trap_min_S() && (S % 2) == 0) return PM_LS_TRAP;
  return (S <= ls_window_max_S()) ? PM_LS_WINDOW : PM_LS_CLASS;
}

pm_status_t pm_cost_async(const int32_t* d_E, int64_t ld_E, int32_t S, const int32_t* d_perm, int64_t* d_cost,
                          pm_stream_t stream) {
  if (!d_E || !d_perm || !d_cost || S < 1 || ld_E < S) return PM_ERR_INVALID;
  PM_CUDA_TRY(launch_cost(d_E, ld_E, S, d_perm, d_cost, (cudaStream_t)stream));
  return PM_OK;
}

pm_status_t pm_cost_sharded_async(const int32_t* const* d_E_peers, const int32_t* h_row_begin, int32_t world,
                                  int64_t ld_E, int32_t S, const int32_t* d_perm, int64_t* d_cost,
                                  pm_stream_t stream) {
  if (!d_E_peers || !h_row_begin || !d_perm || !d_cost || S < 1 || ld_E < S) return PM_ERR_INVALID;
  if (world < 1 || world > kMaxRanks || h_row_begin[0] != 0 || h_row_begin[world] != S) return PM_ERR_INVALID;
  ShardRows rows = {};
  rows.world = world;
  rows.ld = ld_E;
  for (int o = 0; o < world; ++o) {
    if (h_row_begin[o + 1] < h_row_begin[o]) return PM_ERR_INVALID;
    if (!d_E_peers[o] && h_row_begin[o + 1] > h_row_begin[o]) return PM_ERR_INVALID;
    rows.base[o] = d_E_peers[o];
  }
  for (int o = 0; o <= world; ++o) rows.rb[o] = h_row_begin[o];
  PM_CUDA_TRY(launch_cost_sharded(rows, S, d_perm, d_cost, (cudaStream_t)stream));
  return PM_OK;
}

pm_status_t pm_cost(const int32_t* d_E, int64_t ld_E, int32_t S, const int32_t* d_perm, int64_t* h_cost,
                    pm_stream_t stream) {
  if (!h_cost) return PM_ERR_INVALID;
  cudaStream_t st = (cudaStream_t)stream;
  DevBuf buf;
  buf.st = st;
  PM_CUDA_TRY(pm::scratch_alloc(&buf.p, sizeof(int64_t), st));
  pm_status_t s = pm_cost_async(d_E, ld_E, S, d_perm, reinterpret_cast<int64_t*>(buf.p), stream);
  if (s != PM_OK) return s;
  PM_CUDA_TRY(cudaMemcpyAsync(h_cost, buf.p, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  PM_CUDA_TRY(cudaStreamSynchronize(st));
  return PM_OK;
}

pm_status_t pm_init_identity(int32_t* d_perm, int32_t S, pm_stream_t stream) {
  if (!d_perm || S < 1) return PM_ERR_INVALID;
  PM_CUDA_TRY(launch_iota(d_perm, S, (cudaStream_t)stream));
  return PM_OK;
}

pm_status_t pm_photomosaic_async(const uint8_t* d_input, const uint8_t* d_target, int32_t N, int32_t M, int32_t C,
                                 int32_t* d_E, int64_t ld_E, int32_t* d_perm, int32_t method, int64_t* d_result,
                                 pm_stream_t stream) {
  if (!d_input || !d_target || !d_E || !d_perm || !d_result || !valid_image_args(N, M, C)) return PM_ERR_INVALID;
  if (!valid_method(method)) return PM_ERR_INVALID;
  const int32_t g = N / M;
  const int32_t S = g * g;
  if (ld_E < S) return PM_ERR_INVALID;
  {
    const pm_status_t v = ls_method_supported(S, method);   // before Steps 1-2 are enqueued
    if (v != PM_OK) return v;
  }
  cudaStream_t st = (cudaStream_t)stream;
  // TRAP stages from the sigma-permuted copy of E: write it in the E pass
  // (pm_error_matrix_sigma) when the search would build it anyway
  const int32_t used = method == PM_LS_AUTO ? pm_ls_auto_method(S) : method;
  ScopedScratch ep(st);
  if (used == PM_LS_TRAP && trap_ep_wanted(S)) {
    PM_CUDA_TRY(pm::scratch_alloc(&ep.p, trap_ep_bytes(S), st));
    pm_status_t s = pm_error_matrix_sigma(d_input, d_target, N, M, C, d_E, ld_E, ep.as<int32_t>(),
                                          trap_ep_bytes(S), stream);                        // Steps 1-2 (+ copy)
    if (s != PM_OK) return s;
    PM_CUDA_TRY(launch_iota(d_perm, S, st));                                                // r = identity
    s = pm_local_search_sigma_async(d_E, ld_E, S, d_perm, 0, method, ep.as<int32_t>(), trap_ep_bytes(S),
                                    d_result, stream);                                      // Alg. 2
    if (s != PM_OK) return s;
  } else {
    pm_status_t s = pm_error_matrix(d_input, d_target, N, M, C, 0, S, d_E, ld_E, stream);   // Steps 1-2
    if (s != PM_OK) return s;
    PM_CUDA_TRY(launch_iota(d_perm, S, st));                                                // r = identity
    s = pm_local_search_async(d_E, ld_E, S, d_perm, 0, method, d_result, stream);           // Alg. 2
    if (s != PM_OK) return s;
  }
  PM_CUDA_TRY(launch_cost(d_E, ld_E, S, d_perm, d_result + 3, st));                       // Eq. (2)
  return PM_OK;
}

pm_status_t pm_photomosaic(const uint8_t* d_input, const uint8_t* d_target, int32_t N, int32_t M, int32_t C,
                           int32_t* d_E, int64_t ld_E, int32_t* d_perm, int32_t method, int32_t* h_rounds,
                           int64_t* h_swaps, int64_t* h_cost, pm_stream_t stream) {
  cudaStream_t st = (cudaStream_t)stream;
  DevBuf buf;   // {status, rounds, swaps, cost}
  buf.st = st;
  if (!d_input || !d_target || !d_E || !d_perm || !valid_image_args(N, M, C)) return PM_ERR_INVALID;
  PM_CUDA_TRY(pm::scratch_alloc(&buf.p, 4 * sizeof(int64_t), st));
  pm_status_t s = pm_photomosaic_async(d_input, d_target, N, M, C, d_E, ld_E, d_perm, method,
                                       reinterpret_cast<int64_t*>(buf.p), stream);
  if (s != PM_OK) return s;
  int64_t h[4];
  PM_CUDA_TRY(cudaMemcpyAsync(h, buf.p, sizeof(h), cudaMemcpyDeviceToHost, st));
  PM_CUDA_TRY(cudaStreamSynchronize(st));
  if (h_rounds) *h_rounds = (int32_t)h[1];
  if (h_swaps) *h_swaps = h[2];
  if (h_cost) *h_cost = h[3];
  return (pm_status_t)h[0];
}

pm_status_t pm_photomosaic_host(const uint8_t* h_input, const uint8_t* h_target, int32_t N, int32_t M, int32_t C,
                                int32_t method, int32_t* h_perm, int32_t* h_rounds, int64_t* h_swaps,
                                int64_t* h_cost, pm_stream_t stream) {
  if (!h_input || !h_target || !h_perm || !valid_image_args(N, M, C) || !valid_method(method))
    return PM_ERR_INVALID;
  cudaStream_t st = (cudaStream_t)stream;
  const int32_t g = N / M;
  const int64_t S = (int64_t)g * g;
  {
    const pm_status_t v = ls_method_supported((int32_t)S, method);
    if (v != PM_OK) return v;
  }
  const size_t img = (size_t)N * N * C;
  const size_t bytes = 64 + 2 * img + sizeof(int32_t) * (size_t)S * (size_t)S + sizeof(int32_t) * (size_t)S + 64;
  DevBuf buf;
  buf.st = st;
  PM_CUDA_TRY(pm::scratch_alloc(&buf.p, bytes, st));
  char* base = reinterpret_cast<char*>(buf.p);
  int64_t* dres = reinterpret_cast<int64_t*>(base);          // {status, rounds, swaps, cost}
  int32_t* dE = reinterpret_cast<int32_t*>(base + 64);
  int32_t* dperm = dE + S * S;
  uint8_t* dI = reinterpret_cast<uint8_t*>(dperm + S);
  uint8_t* dT = dI + img;
  PM_CUDA_TRY(cudaMemcpyAsync(dI, h_input, img, cudaMemcpyHostToDevice, st));
  PM_CUDA_TRY(cudaMemcpyAsync(dT, h_target, img, cudaMemcpyHostToDevice, st));
  pm_status_t s = pm_photomosaic_async(dI, dT, N, M, C, dE, S, dperm, method, dres, stream);
  if (s != PM_OK) return s;
  // the result and r back in stream order, one host synchronisation
  int64_t h[4];
  PM_CUDA_TRY(cudaMemcpyAsync(h_perm, dperm, sizeof(int32_t) * (size_t)S, cudaMemcpyDeviceToHost, st));
  PM_CUDA_TRY(cudaMemcpyAsync(h, dres, sizeof(h), cudaMemcpyDeviceToHost, st));
  PM_CUDA_TRY(cudaStreamSynchronize(st));
  if (h_rounds) *h_rounds = (int32_t)h[1];
  if (h_swaps) *h_swaps = h[2];
  if (h_cost) *h_cost = h[3];
  return (pm_status_t)h[0];
}

pm_status_t pm_render(const uint8_t* d_input, int32_t N, int32_t M, int32_t C, const int32_t* d_perm,
                      uint8_t* d_out, pm_stream_t stream) {
  if (!valid_image_args(N, M, C)) return PM_ERR_INVALID;
  if (!d_input || !d_perm || !d_out || d_out == d_input) return PM_ERR_INVALID;
  PM_CUDA_TRY(launch_render(d_input, N, M, C, d_perm, d_out, (cudaStream_t)stream));
  return PM_OK;
}

pm_status_t pm_histogram_match(const uint8_t* d_input, const uint8_t* d_target, int32_t N, int32_t C,
                               uint8_t* d_out, pm_stream_t stream) {
  if (!d_input || !d_target || !d_out || N < 1 || C < 1) return PM_ERR_INVALID;
  if (C > hist_max_channels()) return PM_ERR_UNSUPPORTED;
  if (d_out == d_target && d_target != d_input) return PM_ERR_INVALID;   // the target is read after the input's map
  return run_histogram_match(d_input, d_target, N, C, d_out, (cudaStream_t)stream);
}

pm_status_t pm_optimal_assignment(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm, int64_t* d_price,
                                  int32_t* h_rounds, int64_t* h_cost, pm_stream_t stream) {
  if (!d_E || !d_perm || S < 1 || ld_E < S) return PM_ERR_INVALID;
  cudaStream_t st = (cudaStream_t)stream;
  DevBuf buf;
  buf.st = st;
  if (h_cost) PM_CUDA_TRY(pm::scratch_alloc(&buf.p, sizeof(int64_t), st));
  int32_t stats[2] = {0, 0};
  const pm_status_t s = run_assignment(d_E, ld_E, S, d_perm, d_price, reinterpret_cast<int64_t*>(buf.p), stats, st);
  if (h_rounds) *h_rounds = stats[0];
  if (s != PM_OK) return s;
  if (h_cost) {
    PM_CUDA_TRY(cudaMemcpyAsync(h_cost, buf.p, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    PM_CUDA_TRY(cudaStreamSynchronize(st));
  }
  return PM_OK;
}

int64_t pm_launch_count(void) { return g_launches.load() + device_launch_total(); }

pm_status_t pm_tuning_set(const char* name, int32_t value) {
  if (!tuning_name_ok(name)) return PM_ERR_INVALID;
  std::lock_guard<std::mutex> lk(g_tune_mu);
  g_tune[name] = value;
  return PM_OK;
}

void pm_tuning_reset(void) {
  std::lock_guard<std::mutex> lk(g_tune_mu);
  g_tune.clear();
}

pm_status_t pm_scratch_trim(void) {
  int dev = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  if (dev < 0 || dev >= 64) return PM_ERR_CUDA;
  std::lock_guard<std::mutex> lk(g_pool_mu);
  if (g_pools[dev]) PM_CUDA_TRY(cudaMemPoolTrimTo(g_pools[dev], 0));
  return PM_OK;
}

size_t pm_scratch_reserved_bytes(void) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 0;
  std::lock_guard<std::mutex> lk(g_pool_mu);
  if (!g_pools[dev]) return 0;
  uint64_t v = 0;
  if (cudaMemPoolGetAttribute(g_pools[dev], cudaMemPoolAttrReservedMemCurrent, &v) != cudaSuccess) return 0;
  return (size_t)v;
}

}  // extern "C"
