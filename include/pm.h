/*
 * pm.h -- C-ABI of the B200 (sm_100a) photomosaic hot path
 * (Yang, Ito & Nakano, "Photomosaic Generation by Rearranging Subimages,
 * with GPU Acceleration", IPDPS workshops 2017).  Library: libpm.so.
 *
 * "P:<n>" cites line n of the paper text; "reading Rk" cites DESIGN.md's list
 * of readings where the paper is silent or garbled.
 *
 * Conventions for every entry point
 *   - d_* : device pointer on the CURRENT CUDA device; h_* : host pointer.
 *   - stream : a cudaStream_t (NULL = legacy default stream).  Device work is
 *     enqueued on it; functions that return host scalars synchronise it.
 *   - Ownership: the caller allocates and frees every buffer it passes.  The
 *     library keeps no state between calls except cached launch plans and
 *     its scratch pool; scratch comes from a stream-ordered pool on
 *     `stream` and is freed (to the pool) before return -- see
 *     pm_scratch_trim for what the pool keeps.
 *   - Errors: every argument is validated before any launch
 *     (PM_ERR_INVALID, nothing enqueued).  CUDA failures map to PM_ERR_CUDA.
 *     No C++ exception crosses this boundary.  Outputs are undefined on error.
 *   - There is no CPU fallback: every step runs in this library's kernels.
 *   - Thread-safe across distinct streams.
 *   - All arithmetic is integer: results are bit-exact by construction.
 */
#ifndef PM_H_
#define PM_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

struct CUstream_st;                       /* = cudaStream_t */
typedef struct CUstream_st* pm_stream_t;

typedef enum {
  PM_OK = 0,
  PM_ERR_INVALID = 1,        /* bad argument; nothing was launched            */
  PM_ERR_CUDA = 2,           /* a CUDA runtime call or launch failed          */
  PM_ERR_NOT_CONVERGED = 3,  /* max_rounds reached before a zero-swap round   */
  PM_ERR_UNSUPPORTED = 4,    /* valid, but outside what this build supports   */
  PM_ERR_NOT_PERMUTATION = 5, /* d_perm is not a bijection of [0, S)   */
  PM_ERR_TIMEOUT = 6         /* multi-GPU: a peer rank did not arrive within
                                the wait limit (pm_local_search_multi_async) */
} pm_status_t;

/* Local-search implementation selector for pm_local_search_ex.  Every method
 * returns the same r, rounds and per-round swaps (Alg. 2 is deterministic
 * under readings R5-R10); they differ only in speed and in the S they take.
 * Values 2 and 4 (the single-CTA and pair-window methods of round 1,
 * dominated on every S) are retired: PM_ERR_INVALID. */
typedef enum {
  PM_LS_AUTO = 0,      /* pick the fastest method supported for S            */
  PM_LS_CLASS = 1,     /* one kernel per colour class P_i, the paper's own
                          launch structure, replayed as a CUDA graph  */
  PM_LS_WINDOW = 3,    /* one CTA, plus a shared-memory window of each slot's
                          upcoming E entries streamed ahead of the classes
                          (S <= 2048)                                         */
  PM_LS_WALK = 5,      /* every round as a sparse round: a whole-GPU test of
                          every pair on the round's start state marks the
                          classes that can fire, then a thread-block cluster
                          walks the classes in order, testing only those
                          classes and the pairs of already-swapped slots;
                          rounds looped on the device (CUDA-graph WHILE node) */
  PM_LS_TRAP = 6       /* many SMs, temporal blocking of the class sequence:
                          pair k of class c+1 depends only on pairs k-1..k+1
                          of class c, so a chunk's warps replay T classes on
                          the slots of pairs [k0-T, k1+T) in shared memory
                          (E entries staged as per-tile stride-2 runs) and
                          publish pairs [k0, k1) to the neighbour chunks
                          only: one thread-block cluster (DSMEM st.async +
                          mbarrier, S <= 1024) or a persistent cooperative
                          grid (per-chunk phase flags); quiet rounds then
                          run as sparse rounds; even S >= 256 (AUTO)         */
} pm_ls_method_t;

const char* pm_status_string(pm_status_t s);

/* Packed tile stride in bytes: P = M*M*C rounded up to a multiple of 64
 * (the zero padding adds |0-0| = 0 to every E entry). */
int64_t pm_tile_stride(int32_t M, int32_t C);

/* Step 1: cut an N x N image into S = (N/M)^2 tiles of M x M.
 *   d_img   : u8 [N][N][C], row-major HWC, no padding (reading R2).
 *   d_tiles : u8 [S][ld_tiles], ld_tiles >= pm_tile_stride(M, C), multiple of
 *             16.  Tile u = grid cell (u / (N/M), u % (N/M)) (raster, reading
 *             R4); bytes in (y, x, c) order; bytes [M*M*C, ld_tiles) zeroed.
 * Async on stream.  PM_ERR_INVALID unless N % M == 0, M >= 1, C >= 1. */
pm_status_t pm_pack_tiles(const uint8_t* d_img, int32_t N, int32_t M, int32_t C,
                          uint8_t* d_tiles, int64_t ld_tiles, pm_stream_t stream);

/* Step 2, Eq. (1):
 *   E[(u - row_begin) * ld_E + v] = sum_{y,x < M, c < C} |I_u(y,x,c) - T_v(y,x,c)|
 * for input tiles u in [row_begin, row_end) and every target tile v in
 * [0, S), S = (N/M)^2 -- the weight w_{u,v} of P:94 (rows = input tiles).
 *   d_input, d_target : u8 [N][N][C] HWC images (as pm_pack_tiles).
 *   d_E : int32, (row_end - row_begin) rows of ld_E >= S entries.
 * Requires 255*M*M*C <= INT32_MAX (reading R11).  Async on stream (packs both
 * images into scratch tiles, then runs the VABSDIFF4 SAD kernel). */
pm_status_t pm_error_matrix(const uint8_t* d_input, const uint8_t* d_target,
                            int32_t N, int32_t M, int32_t C,
                            int32_t row_begin, int32_t row_end,
                            int32_t* d_E, int64_t ld_E, pm_stream_t stream);

/* Step 2 on already-packed tiles (pm_pack_tiles layout, same ld_tiles for
 * both), for callers that keep the tiles resident:
 *   E[(u - row_begin) * ld_E + v] = sum_{k < P} |Itiles[u][k] - Ttiles[v][k]|,
 * u in [row_begin, row_end), v in [0, S).  P = M*M*C; bytes P..ld_tiles-1
 * must be zero in both (pm_pack_tiles guarantees it).  Async on stream. */
pm_status_t pm_error_matrix_tiles(const uint8_t* d_input_tiles, const uint8_t* d_target_tiles,
                                  int64_t ld_tiles, int32_t S, int32_t P,
                                  int32_t row_begin, int32_t row_end,
                                  int32_t* d_E, int64_t ld_E, pm_stream_t stream);

/* Theorem 1: number of non-empty edge groups of K_S:
 * S - 1 for even S, S for odd S, 0 for S < 2. */
int32_t pm_num_colors(int32_t S);

/* Edge groups P_{class_begin+1} .. P_{class_end}, 0-indexed slots,
 * in the paper's group order and, inside a group, by increasing smaller index
 * (exactly the printed K_16 table for S = 16).  Host-side, for tests and
 * inspection; the kernels generate the same groups on the fly (reading R8:
 * pairs u + v == 2i + 1 (mod m), m = S-1 for even S, m = S for odd S; the
 * fixed point joins vertex S when S is even and idles when S is odd).
 *   h_pairs : int32 [class_end - class_begin][S/2][2], each (u, v) with u < v;
 *             for odd S the last entry of every group is (-1, -1). */
pm_status_t pm_edge_coloring(int32_t S, int32_t class_begin, int32_t class_end, int32_t* h_pairs);

/* Step 3, Algorithm 2: parallel 2-swap local search over the
 * edge groups, groups in order i = 1..S, all pairs of a group concurrently,
 * rounds repeated until a round performs no swap.  Slot-indexed (reading R5):
 * for each pair (u, v) of the group, with a = r[u], b = r[v],
 *   if E[a][u] + E[b][v] > E[b][u] + E[a][v]   (strict, reading R6)
 *   then r[u] = b, r[v] = a.
 *   d_E    : int32 [S][ld_E] from pm_error_matrix (rows = input tiles).
 *   d_perm : int32 [S]; in: the initial rearrangement (identity per the
 *            paper, reading R7; any bijection resumes exactly), out: final r.
 *            r[u] = input tile placed at target slot u (Eq. 2's r).
 *   max_rounds : 0 = until convergence; else stop after that many rounds and
 *            return PM_ERR_NOT_CONVERGED (d_perm then holds the state after
 *            the last full round, so calling again resumes bit-identically).
 *   h_rounds : rounds executed, counting the final zero-swap round (R10).
 *   h_swaps  : total swaps.
 * Synchronises `stream`.  PM_ERR_NOT_PERMUTATION if d_perm is not a
 * bijection (checked on the device before any swap). */
pm_status_t pm_local_search(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                            int32_t max_rounds, int32_t* h_rounds, int64_t* h_swaps,
                            pm_stream_t stream);

/* pm_local_search with an explicit method (pm_ls_method_t) and an optional
 * per-round swap log h_swaps_per_round[0 .. min(rounds, len)-1] (may be NULL;
 * entries from index `rounds` on are written as zero, up to len). */
pm_status_t pm_local_search_ex(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                               int32_t max_rounds, int32_t method,
                               int32_t* h_rounds, int64_t* h_swaps,
                               int64_t* h_swaps_per_round, int32_t len,
                               pm_stream_t stream);

/* Algorithm 2 without any host synchronisation (for pipelines and graphs):
 * as pm_local_search, but the outcome is written to DEVICE memory
 *   d_result : int64 [3] = {status (pm_status_t), rounds, swaps}
 * when the enqueued work completes.  The return value only reports argument
 * and launch errors. */
pm_status_t pm_local_search_async(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                  int32_t max_rounds, int32_t method, int64_t* d_result,
                                  pm_stream_t stream);

/* pm_local_search_async with the sigma-permuted copy of E in a CALLER-OWNED
 * buffer.  Method TRAP stages its per-tile E runs from
 * Ep[t][q] = E[t][2q mod m] (q < m + 48 cyclic, m = S-1),
 * which pm_local_search_async builds in library scratch for every call: at
 * S = 65536 that is 16 GiB mapped and released per call (~100 ms).  Here the
 * copy is built into d_Ep instead, so a caller that searches repeatedly
 * allocates it once.
 *   pm_sigma_copy_bytes : bytes d_Ep must hold for S (0 for S < 2).
 *   d_Ep      : device buffer of at least pm_sigma_copy_bytes(S) bytes,
 *               16-byte aligned, owned by the caller; overwritten (any other
 *               method leaves it untouched).
 * Results are identical to pm_local_search_async (Alg. 2).
 * PM_ERR_INVALID for a NULL, misaligned or too small d_Ep, else as
 * pm_local_search_async. */
size_t pm_sigma_copy_bytes(int32_t S);
/* Steps 1-2 (Eq. 1; all S rows) AND the sigma-permuted copy in one
 * pass: the E kernel writes each entry E[u][v] also to d_Ep[u][sigma(v)]
 * (and to d_Ep[u][sigma(v) + m] when sigma(v) < 48), saving the separate
 * read + write of E that pm_local_search_ep_async / pm_local_search_async
 * spend on it.  d_E, ld_E as pm_error_matrix (row_begin = 0, row_end = S);
 * d_Ep as pm_local_search_ep_async (16-byte aligned, PM_ERR_INVALID
 * otherwise).  S must be even (m = S-1 odd), else PM_ERR_UNSUPPORTED.
 * Asynchronous on `stream`. */
pm_status_t pm_error_matrix_sigma(const uint8_t* d_input, const uint8_t* d_target, int32_t N, int32_t M,
                                  int32_t C, int32_t* d_E, int64_t ld_E, int32_t* d_Ep, size_t ep_bytes,
                                  pm_stream_t stream);
/* pm_local_search_async on a copy d_Ep that already holds E's
 * sigma-permuted rows (from pm_error_matrix_sigma or pm_local_search_ep_async
 * on this E; read only; 16-byte aligned).  A stale copy gives wrong results:
 * the caller keeps it in step with E.  PM_ERR_INVALID for a NULL, misaligned
 * or too small d_Ep. */
pm_status_t pm_local_search_sigma_async(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                        int32_t max_rounds, int32_t method, const int32_t* d_Ep, size_t ep_bytes,
                                        int64_t* d_result, pm_stream_t stream);
pm_status_t pm_local_search_ep_async(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                     int32_t max_rounds, int32_t method, int32_t* d_Ep, size_t ep_bytes,
                                     int64_t* d_result, pm_stream_t stream);

/* Multi-GPU Algorithm 2 (method PM_LS_TRAP split across ranks,
 * one rank per GPU of one NVLink box).  The colour classes are global
 * perfect matchings, so the search does not shard into independent parts;
 * instead rank r runs the TRAP phases on its contiguous share of the pair
 * chunks and exchanges, per phase, only the slots of the chunks at its range
 * ends with its neighbour ranks -- peer stores of (r, d) plus a phase flag
 * (release/acquire at system scope) into their workspaces -- and, once per
 * round, the round's swap count (peer atomics + a cross-rank barrier).
 * Every rank holds the whole of E (replicated; e.g. gathered from the
 * row shards of pm_error_matrix).  Results are bit-identical to
 * pm_local_search.
 *   pm_trap_workspace_bytes : per-rank workspace size for S.
 *   pm_trap_workspace_reset : zero a workspace's counters and flags (every
 *            rank's, followed by a cross-process barrier, before a search).
 *   pm_local_search_multi_async : this rank's part; d_perm_peers[o] and
 *            d_ws_peers[o] (host arrays of `world` device pointers) are rank
 *            o's perm (int32 [S], the same bijection on every rank on entry,
 *            the final r on every rank on exit) and workspace, mapped into
 *            this process (peer access / IPC); d_result as
 *            pm_local_search_async (this rank's copy).  All ranks must run
 *            concurrently (the kernels wait on each other).
 *   pm_local_search_multi_emulated : test hook -- all `world` ranks in one
 *            launch on the current device (own workspaces and perms), the
 *            exchange protocol unchanged; d_perm in/out as pm_local_search.
 * world <= 8; S even, >= 256, and at least `world` pair chunks (S/64 chunks
 * while E is L2-resident or S > 16384, else S/128): else PM_ERR_UNSUPPORTED,
 * before anything is enqueued.  Every cross-GPU wait is bounded (20 s): a
 * rank whose peer never arrives stops and reports PM_ERR_TIMEOUT in
 * d_result (d_perm is then unspecified on that rank). */
size_t pm_trap_workspace_bytes(int32_t S);
pm_status_t pm_trap_workspace_reset(void* d_ws, int32_t S, pm_stream_t stream);
pm_status_t pm_local_search_multi_async(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* const* d_perm_peers,
                                        void* const* d_ws_peers, int32_t rank, int32_t world, int32_t max_rounds,
                                        int64_t* d_result, pm_stream_t stream);
pm_status_t pm_local_search_multi_emulated(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                           int32_t world, int32_t max_rounds, int32_t* h_rounds, int64_t* h_swaps,
                                           pm_stream_t stream);

/* Multi-GPU Algorithm 2 over ROW-SHARDED E (the north_star
 * layout): rank o holds only rows [h_row_begin[o], h_row_begin[o+1]) of E
 * (e.g. its own pm_error_matrix row block), in a buffer mapped into every
 * peer (d_E_peers[o] points at that shard's first row; leading dimension
 * ld_E >= S elements, the same on every rank).  The protocol is that of
 * pm_local_search_multi_async; the only difference is where E is read:
 * each rank first writes the sigma-permuted copy of its own rows (reading
 * R10's contiguous-run layout, DESIGN 6.1) into its workspace, and each
 * TRAP tile then reads E[t][.] from the rank that owns row t, through
 * NVLink peer loads -- no rank holds, gathers or replicates all of E.  Every
 * round runs TRAP (no sparse rounds, which would need the whole matrix).
 * Results are bit-identical to pm_local_search.
 *   pm_trap_workspace_bytes_sharded : per-rank workspace size for S and
 *            that rank's row count (the replicated-mode workspace followed
 *            by its permuted rows); reset with pm_trap_workspace_reset.
 *   pm_local_search_sharded_async : this rank's part.  h_row_begin : host
 *            int32 [world+1], 0 = h_row_begin[0] <= ... <= h_row_begin[world]
 *            = S, identical on every rank; d_E_peers, d_perm_peers,
 *            d_ws_peers : host arrays of `world` device pointers (a rank
 *            with no rows may pass NULL for its shard).  All ranks must run
 *            concurrently; every wait is bounded as above.
 *   pm_local_search_sharded_emulated : test hook -- E is split evenly into
 *            `world` separate shard buffers on the current device and all
 *            ranks run in one launch; d_perm in/out as pm_local_search.
 * Unsupported shapes: as pm_local_search_multi_async (PM_ERR_UNSUPPORTED
 * before anything is enqueued); bad pointers / row bounds: PM_ERR_INVALID. */
size_t pm_trap_workspace_bytes_sharded(int32_t S, int32_t rows);
pm_status_t pm_local_search_sharded_async(const int32_t* const* d_E_peers, const int32_t* h_row_begin, int64_t ld_E,
                                          int32_t S, int32_t* const* d_perm_peers, void* const* d_ws_peers,
                                          int32_t rank, int32_t world, int32_t max_rounds, int64_t* d_result,
                                          pm_stream_t stream);
pm_status_t pm_local_search_sharded_emulated(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                             int32_t world, int32_t max_rounds, int32_t* h_rounds, int64_t* h_swaps,
                                             pm_stream_t stream);

/* The method PM_LS_AUTO selects for S on the current device (host-only). */
int32_t pm_ls_auto_method(int32_t S);

/* r := identity (Alg. 1/2 start from the input image as given, P:116-120,
 * reading R7).  d_perm : int32 [S].  Async on stream. */
pm_status_t pm_init_identity(int32_t* d_perm, int32_t S, pm_stream_t stream);

/* Eq. (2): *h_cost = sum_u E[r[u]][u] (int64, reading R11).
 * Synchronises `stream`. */
pm_status_t pm_cost(const int32_t* d_E, int64_t ld_E, int32_t S, const int32_t* d_perm,
                    int64_t* h_cost, pm_stream_t stream);

/* Eq. (2) without the host sync: d_cost (int64 [1], device) is overwritten. */
pm_status_t pm_cost_async(const int32_t* d_E, int64_t ld_E, int32_t S, const int32_t* d_perm,
                          int64_t* d_cost, pm_stream_t stream);

/* Eq. (2) over ROW-SHARDED E (the layout of pm_local_search_sharded_async):
 * d_E_peers / h_row_begin / world / ld_E as there (peer-mapped shards, host
 * arrays); d_perm int32 [S] on this device; d_cost (int64 [1], device) is
 * overwritten with sum_u E[r[u]][u], each term read from the shard owning row
 * r[u].  Async on stream; PM_ERR_INVALID on bad pointers or bounds. */
pm_status_t pm_cost_sharded_async(const int32_t* const* d_E_peers, const int32_t* h_row_begin, int32_t world,
                                  int64_t ld_E, int32_t S, const int32_t* d_perm, int64_t* d_cost,
                                  pm_stream_t stream);

/* The whole approximation pipeline of Sec. V in one call, on
 * device buffers: Step 1 + Step 2 into d_E (caller-owned, [S][ld_E]), r :=
 * identity, Algorithm 2 (method as pm_local_search_ex), Eq. (2).
 * Outputs d_perm (int32 [S]) and the host scalars.  Synchronises `stream`. */
pm_status_t pm_photomosaic(const uint8_t* d_input, const uint8_t* d_target,
                           int32_t N, int32_t M, int32_t C,
                           int32_t* d_E, int64_t ld_E, int32_t* d_perm, int32_t method,
                           int32_t* h_rounds, int64_t* h_swaps, int64_t* h_cost,
                           pm_stream_t stream);

/* pm_photomosaic without any host synchronisation: d_result (int64 [4],
 * device) receives {status, rounds, swaps, cost} when the work completes. */
pm_status_t pm_photomosaic_async(const uint8_t* d_input, const uint8_t* d_target,
                                 int32_t N, int32_t M, int32_t C,
                                 int32_t* d_E, int64_t ld_E, int32_t* d_perm, int32_t method,
                                 int64_t* d_result, pm_stream_t stream);

/* Same pipeline from HOST images to HOST results (the end-to-end call):
 * copies h_input / h_target (u8 [N][N][C]) to the device, runs
 * pm_photomosaic with library-owned scratch, copies r back to h_perm
 * (int32 [S]).  Pinned host memory gives full PCIe/C2C bandwidth; pageable
 * memory works but is slower.  Synchronises `stream`. */
pm_status_t pm_photomosaic_host(const uint8_t* h_input, const uint8_t* h_target,
                                int32_t N, int32_t M, int32_t C, int32_t method,
                                int32_t* h_perm, int32_t* h_rounds, int64_t* h_swaps,
                                int64_t* h_cost, pm_stream_t stream);

/* The resulting photomosaic R (Sec. V P:247 "writes the resulting
 * photomosaic image to the global memory"): target slot u of d_out shows
 * input tile r[u] = d_perm[u] of d_input, pixel for pixel (raster tiles,
 * (y, x, c) order, reading R4).  d_input / d_out: u8 [N][N][C] HWC, distinct
 * buffers; d_perm: int32 [S] (not validated as a bijection here).  Async. */
pm_status_t pm_render(const uint8_t* d_input, int32_t N, int32_t M, int32_t C, const int32_t* d_perm,
                      uint8_t* d_out, pm_stream_t stream);

/* Adjusting the input image's intensity distribution to the target's before
 * Step 1 (Sec. II: "the distribution of an input image is changed to
 * that of a target image using the histogram equalization [10]"; reading
 * R12): for every channel c separately, with C_I(k) and C_T(k) the numbers
 * of pixels of level <= k in channel c of d_input and d_target,
 *   d_out(y, x, c) = min{ z : C_T(z) >= C_I(d_input(y, x, c)) }
 * (histogram specification on cumulative counts -- integers, no rounding).
 *   d_input, d_target : u8 [N][N][C] HWC (the same N and C); C <= 4.
 *   d_out : u8 [N][N][C]; may be d_input (in place), not d_target.
 * Not part of pm_photomosaic*: the hot path takes its images as given
 * (reading R12); call this first to reproduce the paper's preprocessing.
 * Async on stream. */
pm_status_t pm_histogram_match(const uint8_t* d_input, const uint8_t* d_target, int32_t N, int32_t C,
                               uint8_t* d_out, pm_stream_t stream);

/* The paper's optimization algorithm (Sec. III): the best
 * rearrangement R* (Eq. 3), i.e. a minimum-weight perfect matching of
 * the complete bipartite graph input tiles x target slots with
 * w_{u,v} = E[u][v], which the paper computes on the CPU with Blossom V
 * (P:102).  Here an exact GPU eps-scaling auction on the integer weights
 * scaled by S + 1, finishing at eps = 1 (reading R16).
 *   d_E     : int32 [S][ld_E] (rows = input tiles), entries in [0, 2^24)
 *             (checked on the device: PM_ERR_INVALID after the launch if not).
 *   d_perm  : int32 [S], out: r[v] = input tile at target slot v, with
 *             sum_v E[r[v]][v] minimal over all bijections.  When several
 *             bijections are optimal, which one is returned is unspecified
 *             and may differ between calls (the bidder lists are built with
 *             atomics); the cost never does.
 *   d_price : int64 [S] or NULL, out: the final object prices p[v], a
 *             certificate: with C = (S + 1) * E, every u = r[v] satisfies
 *             C[u][v] + p[v] <= min_w (C[u][w] + p[w]) + 1.
 *   h_rounds: bidding rounds executed (nullable).
 *   h_cost  : sum_v E[r[v]][v] (int64, nullable).
 * S <= 65536; needs cooperative launch (PM_ERR_UNSUPPORTED otherwise).
 * PM_ERR_NOT_CONVERGED if the internal round cap (2^22) is hit.
 * Synchronises `stream`. */
pm_status_t pm_optimal_assignment(const int32_t* d_E, int64_t ld_E, int32_t S, int32_t* d_perm,
                                  int64_t* d_price, int32_t* h_rounds, int64_t* h_cost,
                                  pm_stream_t stream);

/* Number of this library's kernel launches by the calling process so far
 * (for launch accounting in benchmarks): host-side launches plus the kernels
 * that device-side graph loops (CLASS rounds, sparse rounds)
 * launched, which count themselves on the device -- so this call reads a
 * device counter back and synchronises with the devices it has used. */
int64_t pm_launch_count(void);

/* Tuning overrides, for tests and development tools only.  Every method
 * reads its geometry and hand-over choices from measured defaults; these
 * calls override one of them process-wide (never read from the
 * environment).  Results stay bit-exact under every override -- only speed
 * and the set of supported S change (an override that a launch cannot honour
 * returns PM_ERR_UNSUPPORTED from the search).
 *   name  : one of "trap_variant" (chunk geometry 0..7), "trap_W" (owned
 *           pairs per chunk), "trap_cluster" (0 grid, 1 cluster), "trap_nbsync",
 *           "trap_cpc", "trap_ep" (sigma-permuted staging: 0 off, 1 auto,
 *           2 always), "trap_vec", "trap_spec" (speculative class steps: 0 off, 1 quiet rounds,
 *           2 always), "trap_coal" (warp-cooperative staging), "trap_prof",
 *           "trap_wait_ms" (bound of the multi-GPU waits, default 20000),
 *           "ls_sparse" (0: no sparse rounds), "ls_sparse_T" (hand-over swap
 *           count), "ls_cwalk" (0 one-CTA walk, 1 cluster walk),
 *           "ls_sparse_gmem", "auction_gs", "auction_keep",
 *           "auction_smem_price", "auction_theta", "auction_eps_shift",
 *           "auction_max_rounds", "auction_ctas_per_sm".
 * PM_ERR_INVALID for an unknown name.  pm_tuning_reset restores every
 * default.  Not synchronised with searches running on other threads. */
pm_status_t pm_tuning_set(const char* name, int32_t value);
void pm_tuning_reset(void);

/* Scratch.  Every call takes its scratch from a library-owned stream-ordered
 * pool on the current device and frees it before returning (in stream
 * order).  The pool keeps up to 4 GiB mapped between calls so repeated calls
 * do not re-map memory; memory beyond that returns to the driver at the next
 * synchronisation.  pm_scratch_trim releases everything the pool holds that
 * no pending work uses (call after synchronising the streams used);
 * pm_scratch_reserved_bytes reports what the pool holds now. */
pm_status_t pm_scratch_trim(void);
size_t pm_scratch_reserved_bytes(void);

#ifdef __cplusplus
}
#endif
#endif /* PM_H_ */
