// k_trap.cu -- Algorithm 2 on many SMs by temporal blocking of
// the colour-class sequence (method PM_LS_TRAP).
//
// Structure used.  Class c pairs slot u0+k with u0-k (mod m), k = 1..K, and
// u0 with S-1 (k = 0), where u0 = c + (m+1)/2 and K = S/2 - 1 (Theorem 1,
// P:139; R8).  From class c to c+1, u0 advances by one, so the two slots of
// pair k at class c+1 are the first slot of pair k+1 and the second slot of
// pair k-1 at class c (the ends reflect: pair 0 keeps S-1, pair K takes its
// own second slot).  The state of pair k after class c+1 therefore depends on
// pairs k-1..k+1 after class c only: a 1-D three-point stencil in k over the
// class index.  Alg. 2's exact result for the pairs [k0, k1) after T more
// classes is a function of the state of pairs [k0-T, k1+T) alone.
//
// Kernel.  A phase covers T consecutive classes of a round.  The pairs are cut
// into chunks of W owned pairs; a group of warps takes a chunk, copies the
// state (r, d) of the slots of its extended range [k0-T, k1+T) into shared
// memory, replays the T classes on it (the valid range shrinks by one pair per
// side and class: overlapped tiling) and publishes the slots of its owned
// pairs.  Two modes:
//   grid    -- persistent cooperative grid, any S; r and d in global memory.
//              With W >= 2T a chunk writes its owned slots into buffer
//              (q+1) mod 3 and releases a per-chunk phase flag, and waits
//              only for its two neighbours' flags (every earlier reader of
//              that buffer generation lies within two chunks); one grid
//              barrier per round for the swap count.  Else one grid barrier
//              per phase with two buffers.
//   cluster -- one thread-block cluster (<= 16 CTAs, one chunk each) holds
//              every chunk; each CTA keeps replicas of r and d, published
//              slots go to the replicas of the neighbouring chunks' CTAs by
//              st.async, completing on the receiver's mbarrier (expect_tx),
//              one cluster barrier per round (small S).
// The multi-rank kernel at the end of the file runs the grid mode across
// the GPUs of one box (pm_local_search_multi_async).
// Each pair test is line 5 with two entries carried in d (as every method
// here): d[u] + d[v] > E[r[v]][u] + E[r[u]][v], strict (R6).
//
// E entries a chunk needs.  The partner of slot y in class c is 2c+1-y
// (mod m), so a tile that stays at y meets partners advancing by 2 per class,
// and after a swap its new partner is its old slot + 2.  A tile starting at
// slot s0 with class-c0 partner p0 is thus only ever tested against slots
// p0 + 2j and s0 + 2j (j <= T) -- two stride-2 runs of its E row -- unless it
// passes through pair 0 (slot S-1 meets u0, u0+1, ...), which only tiles
// within T pairs of pair 0 can reach: for them the contiguous run
// E[t][u0 .. u0+2T+1] is staged too, and E[t][S-1] for every tile.  Each slot
// state carries indices of the staged entries of its tile's current partner
// (pp) and of slot + 2 (po): no swap -> pp += inc; swap -> (pp, po) <- (po,
// pp + inc) -- inc = 1 in a compact stride-2 run, 2 in the contiguous run.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <atomic>
#include <cstdio>
#include <type_traits>
#include <cstdlib>

#include "pm_internal.cuh"

namespace cg = cooperative_groups;

namespace pm {

struct TrapParams {
  const int32_t* E;
  int64_t ldE;
  int32_t* rbuf[3];            // rbuf[0] = the caller's perm
  int32_t* dbuf[3];
  int4* sbuf[3];               // grid mode: per-slot state {tile g, d = E[g][x], E[g][S-1], 0}; phase q reads q % 3
  unsigned int* flags;         // grid mode, neighbour sync: phases completed per chunk
  int32_t nbsync;              // grid mode: wait for the neighbour chunks only (W >= 2T)
  int32_t S, max_rounds, max_log, sparse_T;
  int32_t W, nchunks;
  int32_t gsz;                 // warps per chunk group (= PPL)
  int32_t vec;                 // 16-byte staging allowed (PM_TRAP_VEC, default 1)
  const int32_t* Ep;           // sigma-permuted copy of E (or NULL), leading dimension ldp
  int64_t ldp;
  int32_t prof;                // trap_prof: CTA 0 thread 0 phase timers -> per_round[192..196]
  int32_t spec;                // speculative class steps (trap_spec, default 1)
  int32_t coal;                // warp-cooperative (coalesced) staging of the Ep runs
  unsigned int* bar;           // grid barrier counter (zeroed before launch)
  unsigned long long* rsw;     // [3] swaps per round, rotating (grid mode)
  LsResult* out;
  int64_t* per_round;
  int32_t* handoff;
};

template <int PPL, int T, bool EP>
struct TrapSmem {
  static constexpr int X = 32 * PPL;        // pairs of an extended range
  static constexpr int L = 2 * X;           // slots (= tiles) of an extended range
  // staged row of local tile i: span0 [0, SP) holds the tile's partner run,
  // span1 [SP, 2SP) its own-slot run, E[g][S-1] at CL.  From E's rows (EP
  // false): E[g][(p0 & ~3) + q] (16-byte copies; the runs p0 + 2j, s0 + 2j,
  // j <= T, are entries (p0 & 3) + 2j); from the sigma-permuted rows (EP):
  // the same runs are contiguous, SPP entries each
  static constexpr int SPP = (T + 1 + 3 + 3) / 4 * 4;
  static constexpr int SP = EP ? SPP : (2 * T + 4 + 3) / 4 * 4;
  static constexpr int CL = 2 * SP;
  static constexpr int RS = 2 * SP + 4;
  static constexpr int NC = 2 * T + 2;      // pair-0 light-cone tiles (at most)
  static constexpr int NU = (2 * T + 2 + 3 + 3) / 4 * 4;   // their span of E[g][u0 + z], z <= 2T+1
  static constexpr int UOFF = L * RS;       // cone rows follow the rows (one index space)
  static constexpr int MOFF = (UOFF + NC * NU + 1) / 2 * 2;   // 3 rotating 64-bit class masks (speculative steps)
  static constexpr int ints = (L * (4 + 1) + MOFF + 6 + 3) / 4 * 4;   // state + g + rows + cone rows + masks
  static constexpr size_t bytes = sizeof(int32_t) * (size_t)ints;
};


// Speculative class steps pay only once most chunk-phases are quiet: a pass
// (every remaining class tested, the first firing class applied) costs a few
// chain steps, and a phase needs 1 + (firing classes) passes, so busy chunks
// get slower while quiet ones get faster -- and in the chain of
// neighbour-synchronised chunks the slow ones pace everybody.  The firing
// classes per chunk and phase of this round are predicted from the previous
// round's swaps, which fall ~3x per round from round 1 on: f = (prev / 3) *
// X * T / (classes * pairs).  Crossovers measured per mode (round 2,
// DESIGN.md): grid 192 x 48 (E in HBM; also 224 x 44) dense wins at f = 0.32
// and loses at 0.12 -> threshold 0.2; grid 128 x 32 spec wins at f = 0.39 -> 0.5; cluster
// mode (DSMEM hand-off, configs 1-2) spec wins up to f ~ 1 -> 1.2.  mode:
// trap_spec (0 never, 1 this rule, 2 always).  Results are identical either
// way.
__device__ __forceinline__ bool spec_round(int32_t mode, int64_t prev_rs, int32_t X, int32_t T, int32_t ncls,
                                           int32_t npairs, bool clu) {
  if (mode == 2) return true;
  if (mode != 1 || prev_rs < 0) return false;
  const int64_t thr10 = clu ? 12 : (X >= 192 ? 2 : 5);   // threshold x 10
  return prev_rs * (int64_t)X * T * 10 < thr10 * 3 * (int64_t)ncls * npairs;
}

__device__ __forceinline__ int32_t wrap_m(int32_t x, int32_t m) {
  x = x < 0 ? x + m : x;
  return x >= m ? x - m : x;
}

// sigma(y) = y (m+1)/2 mod m for 0 <= y < m, m odd
__device__ __forceinline__ int32_t sigma_m(int32_t y, int32_t m) { return (y & 1) ? (y + m) >> 1 : y >> 1; }

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ void cp_async4(int32_t* dst, const int32_t* src) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(s), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16(int32_t* dst, const int32_t* src) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s), "l"(src) : "memory");
}
// E[row][first .. first + n) (n = 4 * pieces) into dst (16-byte aligned): one
// 16-byte copy per piece when the span is in the regular columns and rows are
// 16-byte aligned, else entry by entry with the column taken mod m.
__device__ __forceinline__ void stage_span(int32_t* dst, const int32_t* row, int32_t first, int32_t n, int32_t m,
                                           bool vec) {
  if (vec && first + n <= m) {
    for (int32_t q = 0; q < n; q += 4) cp_async16(dst + q, row + first + q);
  } else {
    for (int32_t q = 0; q < n; ++q) {
      int32_t y = first + q;
      y = y >= m ? y - m : y;
      cp_async4(dst + q, row + y);
    }
  }
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// Barrier of the nthr threads of one chunk group (named barrier id >= 1).
__device__ __forceinline__ void group_sync(int id, int nthr) {
  if (nthr == 32) __syncwarp();
  else asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthr) : "memory");
}

__device__ __forceinline__ void grid_barrier(unsigned int* bar, unsigned int target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(bar) : "memory");
    unsigned int v;
    do {
      asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
    } while (v < target);
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
  }
  __syncthreads();
}

// ---- cluster mode: DSMEM stores that complete on the receiver's mbarrier ----
__device__ __forceinline__ uint32_t smem_u32(const void* ptr) { return (uint32_t)__cvta_generic_to_shared(ptr); }
__device__ __forceinline__ uint32_t cluster_addr(uint32_t a, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
  return r;
}
__device__ __forceinline__ void st_async_v2(uint32_t raddr, int32_t x, int32_t y, uint32_t rmbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v2.s32 [%0], {%1, %2}, [%3];" ::"r"(raddr),
               "r"(x), "r"(y), "r"(rmbar)
               : "memory");
}
__device__ __forceinline__ void mbar_init(uint64_t* mbar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(mbar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* mbar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(mbar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait_parity(uint64_t* mbar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred P1;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n"
      " @!P1 bra WAIT_%=;\n}\n" ::"r"(smem_u32(mbar)),
      "r"(parity)
      : "memory");
}

// Local slot j of a chunk's extended range [a, b): j < nA -> slot u0 + a + j
// (first slots), j < nA + nB -> slot u0 - (a2 + j - nA) (second slots),
// j = nA + nB -> S - 1 (only when a == 0).  Pair k at step t (class c0 + t)
// has slots u0 + t + k and u0 + t - k (or S - 1 for k = 0).

struct TrapChunk {
  int32_t a, b, a2, nA, nB, Lc, K, m, Tp;
  __device__ __forceinline__ void local_slots(int32_t t, int32_t k, int32_t& j1, int32_t& j2) const {
    const int32_t o1 = t + k;
    j1 = (o1 <= K) ? o1 - a : nA + (m - o1 - a2);
    const int32_t o2 = t - k;
    j2 = (k == 0) ? Lc - 1 : ((o2 >= 0) ? o2 - a : nA + (k - t - a2));
  }
  __device__ __forceinline__ int32_t slot_of(int32_t j, int32_t u0, int32_t S) const {
    if (j < nA) return wrap_m(u0 + a + j, m);
    if (j < nA + nB) return wrap_m(u0 - (a2 + j - nA), m);
    return S - 1;
  }
  // index of local tile i in the pair-0 light cone (low chunks), -1 if outside:
  // local slots 0..Tp (first), nA..nA+Tp-1 (second), Lc-1 (S-1)
  __device__ __forceinline__ int32_t cone(int32_t i) const {
    if (a != 0) return -1;
    if (i <= Tp) return i;
    if (i >= nA && i < nA + Tp) return Tp + 1 + (i - nA);
    if (i == Lc - 1) return 2 * Tp + 1;
    return -1;
  }
};

// One chunk of one phase: stage (state via `src`, E rows from global), replay
// Tp classes.  Returns the swaps of the owned pairs.
template <int PPL, int T, bool EP, typename Rows, typename Src>
__device__ __forceinline__ int trap_chunk(const TrapChunk& C, int32_t k0, int32_t k1, int32_t c0, int32_t u0,
                                          const Rows& erows, bool aligned, int32_t S, Src src,
                                          int4* s_st, int32_t* s_g, int32_t* s_E, int gt, int bar_id,
                                          bool vec, unsigned long long* tprof,
                                          const Rows& eprows, bool spec, bool coal) {
  using SM = TrapSmem<PPL, T, EP>;
  static_assert(T <= 64, "one mask bit per class of a phase");
  const unsigned long long t_in = tprof ? gtimer() : 0;   // trap_prof: tprof[1] issue, tprof[2] copy wait
  constexpr int RS = SM::RS, X = SM::X, GT = X;   // one pair position per thread
  const int32_t m = C.m, K = C.K, Tp = C.Tp, Lc = C.Lc;
  const bool low = (C.a == 0);
  int32_t* s_U = s_E + SM::UOFF;
  // ---- one thread per local slot j (= local tile j): its state, then its
  // tile's E row pieces, every copy independent of the others.  Both slots'
  // states are loaded before any copy is issued (two L2 round trips in
  // flight together) ----
  constexpr int NJ = (SM::L + GT - 1) / GT;   // slots per thread (2)
  int32_t xs[NJ], gs[NJ], ds[NJ], els[NJ];   // els: E[g][S-1] when the state carries it, else -1
  int32_t colA[NJ], colB[NJ];                 // coalesced staging: start columns of the two runs in Ep
#pragma unroll
  for (int i = 0; i < NJ; ++i) {
    const int32_t j = gt + i * GT;
    xs[i] = 0; gs[i] = 0; ds[i] = 0; els[i] = -1;
    if (j < Lc) {
      xs[i] = C.slot_of(j, u0, S);
      src(xs[i], gs[i], ds[i], els[i]);
    }
  }
#pragma unroll
  for (int i = 0; i < NJ; ++i) {
    const int32_t j = gt + i * GT;
    if (j >= Lc) continue;
    const int32_t x = xs[i], g = gs[i], d = ds[i];
    s_g[j] = g;
    const bool fx = (x == S - 1);
    const int32_t ci = C.cone(j);
    // p0 = partner in class c0 (the fixed tile's runs are unused)
    const int32_t p0 = fx ? u0 : wrap_m(2 * c0 + 1 - x, m);
    const int32_t s0 = fx ? u0 : x;
    const int32_t* row = erows(g);
    int32_t* dst = s_E + j * RS;
    if (EP) {
      // sigma-permuted rows: Ep[g][q] = E[g][2q mod m], so the stride-2 run
      // from column y is the contiguous run from q = sigma(y) = y (m+1)/2
      // (m = S-1 is odd, so (m+1)/2 is the inverse of 2 mod m: sigma(y) = y/2
      // for even y, (y+m)/2 for odd y -- no 64-bit remainder, which was four
      // calls of the division routine per thread and phase)
      const int32_t sp = sigma_m(p0, m);
      const int32_t ss = sigma_m(s0, m);
      s_st[j] = fx ? make_int4(j | (1 << 16), d, SM::UOFF + ci * SM::NU + (u0 & 3), 0)
                   : make_int4(j | (1 << 16), d, j * RS + (sp & 3), j * RS + SM::SP + (ss & 3) + 1);
      const int32_t* prow = eprows(g);
      colA[i] = sp & ~3;
      colB[i] = ss & ~3;
      if (!coal) {
        for (int32_t q = 0; q < SM::SPP; q += 4) cp_async16(dst + q, prow + (sp & ~3) + q);
        for (int32_t q = 0; q < SM::SPP; q += 4) cp_async16(dst + SM::SP + q, prow + (ss & ~3) + q);
      }
    } else {
      s_st[j] = fx ? make_int4(j | (1 << 16), d, SM::UOFF + ci * SM::NU + (u0 & 3), 0)
                   : make_int4(j | (2 << 16), d, j * RS + (p0 & 3), j * RS + SM::SP + (s0 & 3) + 2);
      stage_span(dst, row, p0 & ~3, SM::SP, m, vec);
      stage_span(dst + SM::SP, row, s0 & ~3, SM::SP, m, vec);
    }
    if (els[i] >= 0) dst[SM::CL] = els[i];          // carried by the published state (grid mode)
    else cp_async4(dst + SM::CL, row + (S - 1));
    // the pair-0 light cone's run E[g][u0 .. u0+2T+1] is contiguous (every
    // entry used): 16-byte pieces whenever the rows are aligned.  (With
    // 4-byte copies chunk 0 -- the only one with a cone -- was the straggler
    // that paced the whole chunk chain: config 4 TRAP round 5.5 -> 5.0 ms.)
    if (ci >= 0) stage_span(s_U + ci * SM::NU, row, u0 & ~3, SM::NU, m, aligned || vec);
  }
  if (EP && coal) {
    // warp-cooperative copies of the runs of the warp's 32 slots: one warp
    // instruction moves one run type (partner runs, then own-slot runs) of
    // SPI = 32 / NP consecutive slots, lane l taking 16-byte piece l % NP of
    // slot l / NP's run -- a few whole runs per instruction (contiguous
    // pieces, ~2 lines each) instead of 32 pieces of 32 different runs.
    // Lane l's (slot offset, piece) is fixed, so an instruction costs one
    // 64-bit pointer shuffle and compile-time shared-memory offsets (the
    // former piece-by-piece mapping spent ~25 instructions per copy on its
    // divisions and three shuffles: 31 % of the kernel's instructions).
    constexpr int NP = SM::SPP / 4;           // 16-byte pieces per run
    constexpr int SPI = 32 / NP;              // slots per warp instruction
    static_assert(SPI >= 1, "a run must fit one warp instruction");
    constexpr int NINS = (32 + SPI - 1) / SPI;
    const int lane = gt & 31;
    const int wbase = gt - lane;
    const int so = lane / NP, qo = 4 * (lane - so * NP);
    const bool act = so < SPI;
    int32_t* const dst0 = s_E + (wbase + so) * RS + qo;
#pragma unroll
    for (int i = 0; i < NJ; ++i) {
      const int32_t* pa = eprows(gs[i]) + colA[i];
      const int32_t* pb = eprows(gs[i]) + colB[i];
#pragma unroll
      for (int run = 0; run < 2; ++run) {
#pragma unroll
        for (int ins = 0; ins < NINS; ++ins) {
          const int sl = ins * SPI + so;      // the slot (of the warp's 32) this lane copies for
          const int32_t* src = (const int32_t*)__shfl_sync(0xffffffffu, (unsigned long long)(run ? pb : pa), sl & 31);
          if (act && sl < 32 && wbase + sl + i * GT < Lc)
            cp_async16(dst0 + (ins * SPI + i * GT) * RS + (run ? SM::SP : 0), src + qo);
        }
      }
    }
  }
  if (spec && gt < 6) s_E[SM::MOFF + gt] = 0;
  const unsigned long long t_iss = tprof ? gtimer() : 0;
  cp_async_wait_all();
  group_sync(bar_id, GT);
  unsigned long long t0 = tprof ? gtimer() : 0;
  if (tprof) { tprof[1] += t_iss - t_in; tprof[2] += t0 - t_iss; }
  // ---- Tp classes on the extended range: thread gt takes pair k = a + gt,
  // valid while t <= tmax (the trapezoid); its local slots are linear in t ----
  int mysw = 0;
  const int32_t k = C.a + gt;
  const bool own = (k >= k0 && k < k1);
  int32_t tmax = -1;
  if (k < C.b) {
    tmax = Tp - 1;
    if (!low) tmax = min(tmax, k - C.a);
    if (C.b != K + 1) tmax = min(tmax, C.b - 1 - k);
  }
  const int32_t tk = K - k, b1 = k - C.a, c1 = C.nA + m - C.a2 - k;   // j1 = t <= tk ? b1 + t : c1 - t
  const int32_t b2 = -k - C.a, c2 = C.nA + k - C.a2;                   // j2 = t >= k ? b2 + t : c2 - t
  if (spec) {
    // Speculative steps (exact).  The state of every slot is stored as of the
    // last class that changed it, with its partner-entry index in the form
    // z' = z - t * inc (z advances by inc per class while the slot does not
    // swap), so class t >= tc can be tested on the state left by class tc-1
    // directly: as long as no valid pair of classes [tc, t) fires, every slot
    // a valid pair of class t reads is unchanged since tc (the trapezoid:
    // valid pairs read only slots written by valid pairs).  One pass tests
    // every remaining class of the phase at once (a bit per class), the OR
    // over the chunk gives the first class t* in which a valid pair fires;
    // exactly the firing pairs of t* are applied (the pairs of a class are
    // disjoint) and the next pass resumes at t* + 1.  A quiet phase thus
    // costs one parallel pass instead of Tp dependent steps.
    unsigned long long* s_or = reinterpret_cast<unsigned long long*>(s_E + SM::MOFF);   // reset before the staging barrier
    int32_t tc = 0;
    uint32_t it = 0;
    while (tc < Tp) {
      const int32_t tl = min(Tp, tmax + 1);
      unsigned long long mask = 0;
#pragma unroll 8
      for (int32_t t = tc; t < tl; ++t) {
        const int32_t j1 = (t <= tk) ? b1 + t : c1 - t;
        const int32_t j2 = (k == 0) ? Lc - 1 : ((t >= k) ? b2 + t : c2 - t);
        const int4 A = s_st[j1], B = s_st[j2];
        const int32_t e_bu = s_E[B.z + t * (B.x >> 16)];
        const int32_t e_av = s_E[(k == 0) ? (A.x & 0xffff) * RS + SM::CL : A.z + t * (A.x >> 16)];
        mask |= (A.y + B.y > e_bu + e_av) ? (1ull << t) : 0ull;
      }
      unsigned long long* slot = s_or + (it % 3u);
      if (gt == 0) s_or[(it + 1) % 3u] = 0ull;   // last read two passes ago
      const uint32_t wlo = __reduce_or_sync(0xffffffffu, (uint32_t)mask);
      const uint32_t whi = (T > 32) ? __reduce_or_sync(0xffffffffu, (uint32_t)(mask >> 32)) : 0u;
      const unsigned long long wor = ((unsigned long long)whi << 32) | wlo;
      if ((gt & 31) == 0 && wor) atomicOr(slot, wor);
      group_sync(bar_id, GT);
      const unsigned long long all = *slot;
      ++it;
      if (all == 0ull) break;                  // nothing fires in [tc, Tp): the phase is decided
      const int32_t ts = __ffsll((long long)all) - 1;   // first firing class
      if ((mask >> ts) & 1ull) {               // apply my pair of class ts (state unchanged since tc)
        const int32_t j1 = (ts <= tk) ? b1 + ts : c1 - ts;
        const int32_t j2 = (k == 0) ? Lc - 1 : ((ts >= k) ? b2 + ts : c2 - ts);
        const int4 fA = s_st[j1], fB = s_st[j2];
        const int32_t ia = fA.x >> 16, ib = fB.x >> 16;
        const int32_t f_bu = s_E[fB.z + ts * ib];
        const int32_t f_av = s_E[(k == 0) ? (fA.x & 0xffff) * RS + SM::CL : fA.z + ts * ia];
        int4 nA, nB;
        if (k == 0) {                 // B leaves S-1 for slot u0+ts (next partner u0+ts+2), A enters S-1
          const int32_t rb = SM::UOFF + C.cone(fB.x & 0xffff) * SM::NU + (u0 & 3) + ts + 2;
          nA = make_int4((fB.x & 0xffff) | (2 << 16), f_bu, rb - 2 * (ts + 1), rb);
          nB = make_int4((fA.x & 0xffff) | (1 << 16), f_av, SM::UOFF + C.cone(fA.x & 0xffff) * SM::NU + (u0 & 3), 0);
        } else {
          nA = make_int4(fB.x, f_bu, fB.w - (ts + 1) * ib, fB.z + (ts + 1) * ib);
          nB = make_int4(fA.x, f_av, fA.w - (ts + 1) * ia, fA.z + (ts + 1) * ia);
        }
        s_st[j1] = nA;
        s_st[j2] = nB;
        mysw += own ? 1 : 0;
      }
      group_sync(bar_id, GT);
      tc = ts + 1;
    }
  } else {
    for (int32_t t = 0; t < Tp; ++t) {
      if (t <= tmax) {
        const int32_t j1 = (t <= tk) ? b1 + t : c1 - t;
        const int32_t j2 = (k == 0) ? Lc - 1 : ((t >= k) ? b2 + t : c2 - t);
        const int4 A = s_st[j1], B = s_st[j2];
        const int32_t e_bu = s_E[B.z];
        const int32_t e_av = s_E[(k == 0) ? (A.x & 0xffff) * RS + SM::CL : A.z];
        const int32_t ia = A.x >> 16, ib = B.x >> 16;
        const bool sw = A.y + B.y > e_bu + e_av;
        int4 nA = sw ? make_int4(B.x, e_bu, B.w, B.z + ib) : make_int4(A.x, A.y, A.z + ia, A.w);
        int4 nB = sw ? make_int4(A.x, e_av, A.w, A.z + ia) : make_int4(B.x, B.y, B.z + ib, B.w);
        if (k == 0 && sw) {   // B leaves S-1 for slot u0+t (next partner u0+t+2), A enters S-1
          const int32_t rb = SM::UOFF + C.cone(B.x & 0xffff) * SM::NU + (u0 & 3) + t + 2;
          nA = make_int4((B.x & 0xffff) | (2 << 16), e_bu, rb, rb);
          nB = make_int4((A.x & 0xffff) | (1 << 16), e_av, SM::UOFF + C.cone(A.x & 0xffff) * SM::NU + (u0 & 3) + t + 1, 0);
        }
        s_st[j1] = nA;
        s_st[j2] = nB;
        mysw += (sw && own) ? 1 : 0;
      }
      group_sync(bar_id, GT);
    }
  }
  if (tprof) *tprof += gtimer() - t0;
  return mysw;
}

template <int PPL, int T, bool CLU, bool EP>
__global__ void __launch_bounds__(256, 1)
k_ls_trap(const TrapParams p) {
  using SM = TrapSmem<PPL, T, EP>;
  constexpr int L = SM::L, X = SM::X;
  extern __shared__ __align__(16) int32_t sm[];
  constexpr int GT = X;                        // threads per chunk group (PPL warps)
  const int cpc = blockDim.x / GT;             // chunk groups per CTA
  const int grp = threadIdx.x / GT;
  const int gt = threadIdx.x - grp * GT;
  int32_t* ws = sm + (size_t)grp * SM::ints;
  int4* s_st = reinterpret_cast<int4*>(ws);
  int32_t* s_g = ws + 4 * L;
  int32_t* s_E = s_g + L;
  const int32_t S = p.S;
  // cluster mode (one chunk per CTA): replica {r, d} of every slot, ping-pong
  // [2][S]; mbar[b] completes when the neighbours' slots for buffer b landed
  int2* rep = reinterpret_cast<int2*>(sm + (size_t)cpc * SM::ints);
  __shared__ int32_t s_cta_sw;
  __shared__ unsigned long long s_rs, s_rsw[3];
  __shared__ __align__(8) uint64_t s_mbar[2];

  const int32_t* __restrict__ E = p.E;
  const int64_t ld = p.ldE;
  const bool aligned = ((ld & 3) == 0) && ((reinterpret_cast<uintptr_t>(E) & 15) == 0);
  const bool vec = p.vec && aligned;   // 16-byte row pieces
  const PlainRows er{E, ld}, epr{p.Ep, p.ldp};
  const Classes cl(S);
  const int32_t m = cl.m, H = cl.half, K = cl.npairs - 1, ncls = cl.ncls;
  const int32_t W = p.W;
  const unsigned nblk = gridDim.x;
  unsigned int bar_target = 0;
  const int ngrp_tot = nblk * cpc;
  const int gid = blockIdx.x * cpc + grp;

  if (p.out->status != PM_OK) return;   // grid-uniform (written before launch)

  if (threadIdx.x == 0) { s_cta_sw = 0; s_rsw[0] = s_rsw[1] = s_rsw[2] = 0ull; }
  // d[x] = E[r[x]][x] (the maintained diagonal)
  // bytes of published slots this CTA receives per phase: chunks ch-1..ch+1
  // each send 2 slots x 8 bytes per owned pair
  uint32_t rx_bytes = 0;
  if (CLU) {
    for (int dch = -1; dch <= 1; ++dch) {
      const int32_t c2 = (int32_t)blockIdx.x + dch;
      if (c2 >= 0 && c2 < p.nchunks) rx_bytes += 16u * (uint32_t)(min((c2 + 1) * W, K + 1) - c2 * W);
    }
    for (int32_t x = threadIdx.x; x < S; x += blockDim.x) {
      const int32_t g = __ldcg(p.rbuf[0] + x);
      rep[x] = make_int2(g, __ldg(E + (int64_t)g * ld + x));
    }
    if (threadIdx.x == 0) {
      mbar_init(&s_mbar[0], 1);
      mbar_init(&s_mbar[1], 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    cg::this_cluster().sync();
  } else {
    for (int32_t x = blockIdx.x * blockDim.x + threadIdx.x; x < S; x += nblk * blockDim.x) {
      const int32_t g = __ldcg(p.rbuf[0] + x);
      const int32_t* row = E + (int64_t)g * ld;
      __stcg(p.sbuf[0] + x, make_int4(g, __ldg(row + x), __ldg(row + (S - 1)), 0));
    }
    bar_target += nblk;
    grid_barrier(p.bar, bar_target);
  }

  int cur = 0;
  int32_t rounds = 0;
  int64_t total = 0;
  int status = PM_OK;
  // PM_TRAP_PROF = 1: CTA 0, 2: the last CTA, 3: the middle one
  const unsigned pblk = p.prof == 2 ? nblk - 1 : (p.prof == 3 ? nblk / 2 : 0);
  const bool prof = p.prof && blockIdx.x == pblk && threadIdx.x == 0 && p.max_log >= 200;
  unsigned long long t_ld = 0, t_bar = 0, t_pub = 0, n_ph = 0, tq = prof ? gtimer() : 0;
  unsigned long long t_stv[3] = {0, 0, 0}, t_fw = 0;   // steps, issue, copy wait; neighbour-flag wait
  unsigned long long& t_st = t_stv[0];
  const unsigned long long t_start0 = tq;
  const int npass = (p.nchunks + ngrp_tot - 1) / ngrp_tot;
  uint32_t nph_cl = 0;   // cluster mode: phases completed (mbarrier parity)
  uint32_t qph = 0;      // grid mode: phases completed
  int64_t prev_rs = -1;   // swaps of the previous round (-1: none yet)
  for (;;) {
    const bool spec = spec_round(p.spec, prev_rs, X, T, ncls, K + 1, CLU);
    if (!CLU && blockIdx.x == 0 && threadIdx.x == 0) p.rsw[(rounds + 1) % 3] = 0ull;
    for (int32_t c0 = 0; c0 < ncls; c0 += T) {
      const int32_t Tp = min(T, ncls - c0);
      const int32_t u0 = wrap_m(c0 + H, m);
      int mysw = 0;
      for (int pass = 0; pass < npass; ++pass) {
        const int32_t ch = gid + pass * ngrp_tot;
        const bool have = ch < p.nchunks;
        TrapChunk C;
        const int32_t k0 = ch * W, k1 = min(k0 + W, K + 1);
        C.a = max(k0 - Tp, 0); C.b = min(k1 + Tp, K + 1);
        C.a2 = max(C.a, 1);
        C.nA = C.b - C.a; C.nB = C.b - C.a2;
        C.Lc = C.nA + C.nB + (C.a == 0 ? 1 : 0);
        C.K = K; C.m = m; C.Tp = Tp;
        if (have) {
          if (CLU) {
            const int2* rr = rep + cur * S;
            mysw += trap_chunk<PPL, T, EP>(C, k0, k1, c0, u0, er, aligned, S,
                                       [&](int32_t x, int32_t& g, int32_t& d, int32_t& el) { const int2 v = rr[x]; g = v.x; d = v.y; el = -1; },
                                       s_st, s_g, s_E, gt, 1 + grp, vec, prof ? t_stv : nullptr, epr, spec, p.coal);
          } else {
            const int bi = p.nbsync ? (int)(qph % 3u) : cur;
            const int4* __restrict__ sc = bi == 0 ? p.sbuf[0] : (bi == 1 ? p.sbuf[1] : p.sbuf[2]);
            if (p.nbsync && qph > 0) {
              // the neighbour chunks' slots of phase qph - 1 (W >= 2T: every
              // reader of this buffer's previous generation is within two
              // chunks, and those finished it before our neighbours did theirs)
              const unsigned long long tw0 = prof ? gtimer() : 0;
              if (gt == 0) {
#pragma unroll
                for (int dch = -1; dch <= 1; dch += 2) {
                  const int32_t c2 = ch + dch;
                  if (c2 < 0 || c2 >= p.nchunks) continue;
                  unsigned int v;
                  do {
                    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p.flags + c2) : "memory");
                  } while (v < qph);
                }
              }
              group_sync(1 + grp, GT);
              if (prof) t_fw += gtimer() - tw0;
            }
            mysw += trap_chunk<PPL, T, EP>(C, k0, k1, c0, u0, er, aligned, S,
                                       [&](int32_t x, int32_t& g, int32_t& d, int32_t& el) {
                                         const int4 v = __ldcg(sc + x); g = v.x; d = v.y; el = v.z;
                                       },
                                       s_st, s_g, s_E, gt, 1 + grp, vec, prof ? t_stv : nullptr, epr, spec, p.coal);
          }
          if (prof) { const unsigned long long t = gtimer(); t_ld += t - tq; tq = t; }
          // ---- publish the slots of the owned pairs (class c0 + Tp - 1) ----
          for (int32_t kq = gt; kq < X; kq += GT) {
            const int32_t k = C.a + kq;
            if (k >= k0 && k < k1) {
              int32_t j1, j2;
              C.local_slots(Tp - 1, k, j1, j2);
              const int32_t x1 = C.slot_of(j1, u0, S), x2 = C.slot_of(j2, u0, S);
              const int4 A = s_st[j1], B = s_st[j2];
              const int32_t g1 = s_g[A.x & 0xffff], g2 = s_g[B.x & 0xffff];
              if (CLU) {
                // to the replicas of the CTAs of chunks ch-1, ch, ch+1 (every slot of
                // a chunk's next extended range is published by one of them: W > T),
                // each store completing on the receiver's mbarrier for that buffer
                const int nx = cur ^ 1;
                const uint32_t a1 = smem_u32(rep + nx * S + x1), a2 = smem_u32(rep + nx * S + x2);
                const uint32_t am = smem_u32(&s_mbar[nx]);
                for (int dch = -1; dch <= 1; ++dch) {
                  const int32_t c2 = ch + dch;
                  if (c2 < 0 || c2 >= p.nchunks) continue;
                  const uint32_t rm = cluster_addr(am, c2);
                  st_async_v2(cluster_addr(a1, c2), g1, A.y, rm);
                  st_async_v2(cluster_addr(a2, c2), g2, B.y, rm);
                }
              } else {
                // {tile, d, E[tile][S-1]}: the reader needs no second round trip
                const int bn = p.nbsync ? (int)((qph + 1u) % 3u) : (cur ^ 1);
                int4* sn = bn == 0 ? p.sbuf[0] : (bn == 1 ? p.sbuf[1] : p.sbuf[2]);
                __stcg(sn + x1, make_int4(g1, A.y, s_E[(A.x & 0xffff) * SM::RS + SM::CL], 0));
                __stcg(sn + x2, make_int4(g2, B.y, s_E[(B.x & 0xffff) * SM::RS + SM::CL], 0));
              }
            }
          }
        }
        if (prof) { const unsigned long long t = gtimer(); t_pub += t - tq; }
        group_sync(1 + grp, GT);
        if (!CLU && p.nbsync && have && gt == 0) {   // this chunk's slots of phase qph are out
          // (the release is cumulative: the group's publish stores happen
          // before it through the barrier above)
          asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p.flags + ch), "r"(qph + 1u) : "memory");
        }
      }
      // swaps of this phase -> the round counter
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) mysw += __shfl_xor_sync(0xffffffffu, mysw, o);
      if ((threadIdx.x & 31) == 0 && mysw) atomicAdd(&s_cta_sw, mysw);
      cur ^= 1;
      __syncthreads();
      // the CTA's swaps of the round leave the CTA once, before the round's
      // last barrier: cluster -> its own slot s_rsw[round % 3] (read by every
      // CTA over DSMEM after the barrier), grid -> one global atomic
      if (c0 + T >= ncls && threadIdx.x == 0) {
        if (CLU) s_rsw[rounds % 3] = (unsigned long long)s_cta_sw;
        else if (s_cta_sw) atomicAdd(p.rsw + rounds % 3, (unsigned long long)s_cta_sw);
        s_cta_sw = 0;
      }
      if (CLU) {
        // wait for the neighbours' slots of the next phase (buffer cur, now);
        // mbar[b] is used every other phase: parity = its use count & 1
        if (threadIdx.x == 0) mbar_arrive_expect_tx(&s_mbar[cur], rx_bytes);
        mbar_wait_parity(&s_mbar[cur], (uint32_t)(nph_cl >> 1) & 1u);
        ++nph_cl;
        if (c0 + T >= ncls) cg::this_cluster().sync();   // round end: every CTA's s_rsw slot is set
      } else if (!p.nbsync || c0 + T >= ncls) {   // neighbour sync: one grid barrier per round
        bar_target += nblk;
        grid_barrier(p.bar, bar_target);
      }
      ++qph;
      if (prof) { const unsigned long long t = gtimer(); t_bar += t - tq; tq = t; ++n_ph; }
    }
    // round end (Alg. 2 lines 10-11)
    if (CLU) {
      if (threadIdx.x < 32) {
        unsigned long long v = 0;
        for (int b = threadIdx.x; b < (int)nblk; b += 32) v += *cg::this_cluster().map_shared_rank(&s_rsw[rounds % 3], b);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (threadIdx.x == 0) s_rs = v;
      }
    } else if (threadIdx.x == 0) {
      s_rs = *((volatile unsigned long long*)(p.rsw + rounds % 3));
    }
    __syncthreads();
    const int64_t rs = (int64_t)s_rs;
    prev_rs = rs;
    if (blockIdx.x == 0 && threadIdx.x == 0 && rounds < p.max_log) p.per_round[rounds] = rs;
    if (prof && rounds < 32) p.per_round[224 + rounds] = (int64_t)gtimer();   // round end times (trap_prof)
    rounds += 1;
    total += rs;
    __syncthreads();   // (a CTA's s_rsw slot is rewritten three rounds later)
    if (rs == 0) break;
    if (p.max_rounds > 0 && rounds >= p.max_rounds) { status = PM_ERR_NOT_CONVERGED; break; }
    if (p.handoff && rs <= p.sparse_T) {
      if (blockIdx.x == 0 && threadIdx.x == 0) *p.handoff = 1;
      break;
    }
  }
  if (prof) {
    p.per_round[197] = (int64_t)t_start0;
    p.per_round[192] = (int64_t)(t_ld - t_st); p.per_round[193] = (int64_t)t_st;
    p.per_round[194] = (int64_t)t_bar; p.per_round[195] = (int64_t)n_ph;
    p.per_round[196] = (int64_t)t_pub;
    p.per_round[198] = (int64_t)t_fw; p.per_round[199] = (int64_t)t_stv[1]; p.per_round[200] = (int64_t)t_stv[2];
  }
  if (CLU) {
    // every CTA writes the slots of its owned pairs in the last class
    // (ncls - 1) from its own replica (it published them to itself)
    for (int pass = 0; pass < npass; ++pass) {
      const int32_t ch = gid + pass * ngrp_tot;
      if (ch >= p.nchunks) continue;
      const int32_t k0 = ch * W, k1 = min(k0 + W, K + 1);
      for (int32_t k = k0 + gt; k < k1; k += GT) {
        int32_t u, v;
        cl.pair(ncls - 1, k, u, v);
        p.rbuf[0][u] = rep[cur * S + u].x;
        p.rbuf[0][v] = rep[cur * S + v].x;
      }
    }
    cg::this_cluster().sync();   // no CTA exits while others may still touch its smem
  } else {   // the final state is in buffer qph % 3 (nbsync) or cur: copy to perm
    const int bf = p.nbsync ? (int)(qph % 3u) : cur;
    const int4* src = bf == 0 ? p.sbuf[0] : (bf == 1 ? p.sbuf[1] : p.sbuf[2]);
    for (int32_t x = blockIdx.x * blockDim.x + threadIdx.x; x < S; x += nblk * blockDim.x)
      p.rbuf[0][x] = __ldcg(src + x).x;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    p.out->status = status;
    p.out->rounds = rounds;
    p.out->swaps = total;
  }
}

int32_t ls_trap_min_S() { return 256; }

template <int PPL, int T, bool EP>
static pm_status_t launch_trap_ep(TrapParams& hp, cudaStream_t st) {
  using SM = TrapSmem<PPL, T, EP>;
  constexpr int X = SM::X;
  static_assert(X > 2 * T + 1, "chunk must own more than T pairs");
  int dev = 0, nsm = 0, optin = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  const Classes cl(hp.S);
  const int32_t npairs = cl.npairs;
  int32_t W = knob("trap_W", X - 2 * T);
  if (W < T + 1 || W > X - 2 * T) W = X - 2 * T;   // W > T: neighbours publish every halo slot
  hp.W = W;
  hp.nchunks = (npairs + W - 1) / W;
  const int gsz = PPL;   // warps per chunk group: one pair position per thread
  hp.gsz = gsz;
  // cluster mode when every chunk fits one cluster of <= 16 CTAs
  const size_t rep_bytes = sizeof(int32_t) * 4 * (size_t)hp.S;
  int mode = knob("trap_cluster", -1);   // -1 auto, 0 grid, 1 cluster
  int max_cpc_cl = ((size_t)optin > rep_bytes) ? (int)(((size_t)optin - rep_bytes) / SM::bytes) : 0;
  if (max_cpc_cl > 8 / gsz) max_cpc_cl = 8 / gsz;
  // (cluster mode: one chunk per CTA, its neighbours' CTAs = chunks ch +- 1)
  const bool cl_ok = max_cpc_cl >= 1 && hp.nchunks <= 16 && W > T;
  // measured: the cluster pays while every CTA holds one chunk
  // (config 2: 1.50 vs 1.66 ms); with several chunks per CTA the staging of
  // 16 SMs loses to the grid's (config 3: 11.8 vs 10.7 ms)
  if (mode < 0) mode = cl_ok ? 1 : 0;
  if (mode == 1 && !cl_ok) return PM_ERR_UNSUPPORTED;
  if (mode == 1) {
    const int cpc_cl = 1;
    const int nblk = hp.nchunks;
    if (nblk > 16) return PM_ERR_UNSUPPORTED;
    const size_t smem = SM::bytes * cpc_cl + rep_bytes;
    const int threads = 32 * gsz * cpc_cl;
    auto fn = k_ls_trap<PPL, T, true, EP>;
    PM_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    if (nblk > 8) PM_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(nblk);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = nblk;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    int ncl = 0;
    PM_CUDA_TRY(cudaOccupancyMaxActiveClusters(&ncl, fn, &cfg));
    if (ncl < 1) return PM_ERR_UNSUPPORTED;
    PM_CUDA_TRY(cudaLaunchKernelEx(&cfg, fn, hp));
    note_launch();
    return PM_OK;
  }
  // grid mode: cpc chunk groups per CTA, enough CTAs for one pass if possible;
  // neighbour synchronisation (chunk flags, three state buffers) when W >= 2T
  hp.nbsync = (W >= 2 * T) ? knob("trap_nbsync", 1) : 0;
  int max_cpc = (int)((size_t)optin / SM::bytes);
  if (max_cpc > 8 / gsz) max_cpc = 8 / gsz;
  if (max_cpc < 1) return PM_ERR_UNSUPPORTED;
  int cpc = knob("trap_cpc", (hp.nchunks + nsm - 1) / nsm);
  if (cpc < 1) cpc = 1;
  if (cpc > max_cpc) cpc = max_cpc;
  const size_t smem = SM::bytes * cpc;
  const int threads = 32 * gsz * cpc;
  auto fn = k_ls_trap<PPL, T, false, EP>;
  PM_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  PM_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, smem));
  if (occ < 1) return PM_ERR_UNSUPPORTED;
  int grid = (hp.nchunks + cpc - 1) / cpc;
  if (grid > nsm * occ) grid = nsm * occ;
  void* args[] = {(void*)&hp};
  PM_CUDA_TRY(cudaLaunchCooperativeKernel((const void*)fn, dim3(grid), dim3(threads), args, smem, st));
  note_launch();
  return PM_OK;
}

// sigma-permuted copy of E (trap_ep: 1 auto, 2 always, 0 never).  Auto
// builds it whenever it takes at most 1/8 of the device's memory (22 GiB on
// a B200, E itself being as large; the total is queried once per device --
// cudaMemGetInfo per call costs ~0.6 ms and synchronises): since the staging
// became warp-cooperative and the 192 x 48 geometry needs its compact rows,
// it pays at every size (config 5, measured: whole search 970 ms from E's
// rows with 64 x 16 chunks vs 584 ms with the 16 GiB copy and 192 x 48; in
// round 1, before both, it lost there: 1.09 vs 1.25 s).
static size_t device_total_mem() {
  static std::atomic<size_t> totals[64];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 0;
  size_t t = totals[dev].load();
  if (t == 0) {
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, dev) != cudaSuccess) return 0;
    t = prop.totalGlobalMem;
    totals[dev].store(t);
  }
  return t;
}

int64_t trap_ep_ld(int32_t S) { return ((int64_t)S - 1 + 48 + 31) / 32 * 32; }
size_t trap_ep_bytes(int32_t S) { return S < 2 ? 0 : sizeof(int32_t) * (size_t)S * (size_t)trap_ep_ld(S); }

pm_status_t trap_build_ep_into(const int32_t* E, int64_t ldE, int32_t S, cudaStream_t st, int32_t* Ep,
                               int64_t* ldp) {
  *ldp = trap_ep_ld(S);
  PM_CUDA_TRY(launch_permute_cols(E, ldE, Ep, *ldp, S, S - 1, 48, st));
  return PM_OK;
}

bool trap_ep_wanted(int32_t S) {
  const int32_t ep_mode = knob("trap_ep", 1);
  if (ep_mode == 0 || S < 2) return false;
  return ep_mode == 2 || trap_ep_bytes(S) <= device_total_mem() / 8;
}

pm_status_t trap_build_ep(const int32_t* E, int64_t ldE, int32_t S, cudaStream_t st, int32_t** Ep,
                          int64_t* ldp) {
  *Ep = nullptr;
  *ldp = 0;
  const int32_t ep_mode = knob("trap_ep", 1);
  if (ep_mode == 0) return PM_OK;
  const int32_t m = S - 1, ext = 48;
  const int64_t l = trap_ep_ld(S);
  const size_t bytes = sizeof(int32_t) * (size_t)S * (size_t)l;
  if (ep_mode == 1 && bytes > device_total_mem() / 8) return PM_OK;
  *ldp = l;
  PM_CUDA_TRY(pm::scratch_alloc(Ep, bytes, st));
  PM_CUDA_TRY(launch_permute_cols(E, ldE, *Ep, *ldp, S, m, ext, st));
  return PM_OK;
}

// The staging layout depends on whether the runs come from the sigma-permuted
// copy (EP: contiguous runs, half the shared memory per tile) or from E.
template <int PPL, int T>
static pm_status_t launch_trap(TrapParams& hp, cudaStream_t st) {
  if (hp.Ep) return launch_trap_ep<PPL, T, true>(hp, st);
  return launch_trap_ep<PPL, T, false>(hp, st);   // PM_ERR_UNSUPPORTED if its layout exceeds shared memory
}

pm_status_t run_trap(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t max_rounds,
                     LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st,
                     int32_t* handoff, int32_t sparse_T, const int32_t* Ep_in, int64_t ldp_in) {
  if (S < ls_trap_min_S() || (S & 1)) return PM_ERR_UNSUPPORTED;
  // (run_local_search checks the permutation before building Ep)
  // scratch: 3 round counters, barrier counter, chunk flags [S/2], then the
  // three generations of packed slot states (int4 [S] each)
  const size_t n = (size_t)S;
  ScopedScratch scr(st), ep(st);
  const size_t head = (64 + sizeof(unsigned int) * (n / 2 + 16) + 15) / 16 * 16;
  const size_t bytes = head + sizeof(int4) * 3 * n;
  PM_CUDA_TRY(pm::scratch_alloc(&scr.p, bytes, st));
  char* scratch = scr.as<char>();
  unsigned long long* rsw = reinterpret_cast<unsigned long long*>(scratch);
  unsigned int* bar = reinterpret_cast<unsigned int*>(scratch + 32);
  unsigned int* flags = reinterpret_cast<unsigned int*>(scratch + 64);
  int4* base = reinterpret_cast<int4*>(scratch + head);
  PM_CUDA_TRY(cudaMemsetAsync(scratch, 0, head, st));
  TrapParams hp = {};
  hp.E = E; hp.ldE = ldE;
  hp.rbuf[0] = perm;
  hp.sbuf[0] = base; hp.sbuf[1] = base + n; hp.sbuf[2] = base + 2 * n;
  hp.flags = flags;
  hp.S = S; hp.max_rounds = max_rounds; hp.max_log = max_log;
  hp.sparse_T = sparse_T; hp.handoff = handoff;
  hp.bar = bar; hp.rsw = rsw;
  hp.out = dev_out; hp.per_round = dev_per_round;
  hp.prof = knob("trap_prof", 0);
  hp.coal = knob("trap_coal", 1);
  hp.spec = knob("trap_spec", 1);
  // sigma-permuted rows (the runs become contiguous: 5 instead of 9 16-byte
  // pieces per run at T = 16 from L2, dense sectors instead of stride-2 ones
  // from HBM)
  // (measured: config 2 1.25 -> 1.18 ms, config 4 67.4 -> 62.3 ms; config 5
  // 1.09 -> 1.25 s -- building the 16 GiB copy costs more than it saves)
  if (Ep_in) {
    hp.Ep = Ep_in; hp.ldp = ldp_in;
  } else {
    int32_t* Ep = nullptr;
    int64_t ldp = 0;
    const pm_status_t se = trap_build_ep(E, ldE, S, st, &Ep, &ldp);
    ep.p = Ep;
    if (se != PM_OK) return se;
    hp.Ep = Ep; hp.ldp = ldp;
  }
  // 16-byte span copies pay while E is L2-resident (config 2/3 staging 2.55 ->
  // 1.80 / 3.2 -> 2.1 us per phase); from HBM the 4-byte entry copies of the
  // used runs win (config 4: 5.0 vs 10.8 us)
  hp.vec = knob("trap_vec", (int64_t)S * ldE * 4 <= (96ll << 20) ? 1 : 0);
  const int32_t variant = knob("trap_variant", -1);
  switch (variant) {
    case 0: return launch_trap<2, 16>(hp, st);
    case 1: return launch_trap<1, 8>(hp, st);
    case 2: return launch_trap<2, 8>(hp, st);
    case 3: return launch_trap<4, 16>(hp, st);
    case 4: return launch_trap<4, 8>(hp, st);
    case 5: return launch_trap<4, 32>(hp, st);
    case 6: return launch_trap<6, 48>(hp, st);
    case 7: return launch_trap<7, 44>(hp, st);
    default:
      // measured (whole search, configs 1/2/3/4): 128-pair ranges
      // x 32 classes 0.338/1.049/6.14/36.6 ms, 64 x 16 0.353/1.172/7.73/54.9,
      // 192 x 48 0.353/1.107/6.20/34.5 -- so 192 x 48 once E is beyond L2
      // (it needs the sigma-permuted copy's compact staging), 128 x 32 below;
      // from E's own rows (E > 2 GiB, config 5) 64 x 16 (round 1: 1.21 vs
      // 1.32 s for 128 x 32)
      if (!hp.Ep) return launch_trap<2, 16>(hp, st);
      if ((int64_t)S * ldE * 4 > (96ll << 20)) {
        // 192 x 48 (96 owned pairs) unless its chunks need more passes per
        // phase over the SMs than 224 x 44 (136 owned pairs, 222 KB of
        // staging): config 5 has 342 chunks = 3 passes on 148 SMs, 241 = 2
        // passes (measured: TRAP round 34 -> ~24 ms); config 4
        // (86 chunks) keeps 192 x 48
        int dev = 0, nsm = 148;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        const int64_t np = Classes(S).npairs;
        const int64_t pass48 = ((np + 95) / 96 + nsm - 1) / nsm, pass44 = ((np + 135) / 136 + nsm - 1) / nsm;
        if (pass44 < pass48) return launch_trap<7, 44>(hp, st);
        return launch_trap<6, 48>(hp, st);
      }
      return launch_trap<4, 32>(hp, st);
  }
}


// =====================================================================
// Multi-rank TRAP (one rank per GPU; NVLink peer memory).  The chunks are
// split into `world` contiguous ranges; rank r runs the grid-mode phases on
// its range with the neighbour synchronisation above, except that a chunk
// publishes its owned slots (and its phase flag) to the rank(s) owning
// chunks ch-1, ch, ch+1 -- by peer stores when another rank owns them.  E
// is replicated (every rank holds all of it).  Once per round every rank
// adds its swap count to every rank's round total and passes a cross-rank
// barrier; at the end every chunk writes its owned slots' final tiles into
// every rank's perm, so every rank returns the whole result.  The same
// kernel runs all ranks inside one launch on one device for the test hook
// pm_local_search_multi_emulated (peer pointers are then plain pointers).
struct TrapRank {                 // one rank's workspace (see trap_ws_layout)
  int32_t* rbuf[3];
  int32_t* dbuf[3];
  unsigned int* flags;            // [nchunks] phases completed, per chunk
  unsigned int* bar;              // this rank's grid barrier counter
  unsigned int* xbar;             // cross-rank barrier counter
  unsigned long long* rtot;       // [3] round swap totals (all ranks add, system-scope atomics)
  unsigned int* abort;            // set when a wait timed out (every wait of the launch watches it)
  int32_t* perm;
  const int32_t* E;
  const int32_t* Ep;              // this rank's sigma-permuted copy of E (or NULL)
};
struct TrapMultiParams {
  TrapRank rk[kMaxRanks];
  int64_t ldE, ldp;
  int32_t S, max_rounds, max_log, W, nchunks, world, rank0, ctas_per_rank, vec;
  LsResult* out;                  // written by the launch's first rank
  int64_t* per_round;
  int32_t* handoff;               // the first rank's sparse-round flag (or NULL)
  int32_t sparse_T;
  int32_t spec;                   // speculative class steps
  int32_t coal;                   // coalesced staging of the Ep runs
  unsigned long long wait_ns;     // bound of every cross-rank wait
  // E row-sharded across the ranks (SH kernels): row g of E and of Ep is read
  // from its owner's shard (peer memory); no rank holds all of E
  ShardRows esh, epsh;
  int32_t sh_aligned;             // SH: every shard's rows are 16-byte aligned
};

__device__ __forceinline__ int32_t chunk_begin(int32_t r, int32_t nchunks, int32_t world) {
  return (int32_t)(((int64_t)r * nchunks) / world);
}
__device__ __forceinline__ int32_t chunk_owner(int32_t ch, int32_t nchunks, int32_t world) {
  int32_t r = 0;
  while (r + 1 < world && chunk_begin(r + 1, nchunks, world) <= ch) ++r;
  return r;
}
// Every cross-GPU wait is bounded: a rank that waits longer than the limit
// (TrapMultiParams::wait_ns, 20 s unless tuned) for a peer sets its
// workspace's abort flag (and, best effort, every peer's), reports
// PM_ERR_TIMEOUT and leaves; every other wait of the launch also watches the
// flag, so no CTA spins forever behind a dead rank.

__device__ __forceinline__ unsigned int ld_acquire_sys(const unsigned int* a) {
  unsigned int v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_acquire_sys64(const unsigned long long* a) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(a) : "memory");
  return v;
}
__device__ __forceinline__ void raise_abort(const TrapMultiParams& p, int32_t r) {
  for (int o = 0; o < p.world; ++o)
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;" ::"l"(p.rk[o].abort), "r"(1u) : "memory");
  __threadfence_system();
  (void)r;
}
// wait until *a >= target; false if the launch aborted or the wait timed out
// (then the abort is raised)
__device__ __forceinline__ bool wait_ge_sys(const TrapMultiParams& p, int32_t r, const unsigned int* a,
                                            unsigned int target) {
  const unsigned long long t0 = gtimer();
  unsigned int n = 0;
  while (ld_acquire_sys(a) < target) {
    if ((++n & 63u) == 0) {
      if (ld_acquire_sys(p.rk[r].abort)) return false;
      if (gtimer() - t0 > p.wait_ns) { raise_abort(p, r); return false; }
    }
  }
  return true;
}
// the rank's own grid barrier, abortable
__device__ __forceinline__ bool grid_barrier_mr(const TrapMultiParams& p, int32_t r, unsigned int* bar,
                                                unsigned int target) {
  __syncthreads();
  __shared__ int s_ok;
  if (threadIdx.x == 0) {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(bar) : "memory");
    s_ok = wait_ge_sys(p, r, bar, target) ? 1 : 0;
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
  }
  __syncthreads();
  return s_ok != 0;
}
__device__ __forceinline__ bool sys_barrier_arrive_wait(const TrapMultiParams& p, int32_t r, unsigned int target) {
  // every rank's leader: arrive at every rank's counter, wait for its own
  __threadfence_system();
  for (int o = 0; o < p.world; ++o)
    asm volatile("red.release.sys.global.add.u32 [%0], 1;" ::"l"(p.rk[o].xbar) : "memory");
  return wait_ge_sys(p, r, p.rk[r].xbar, target);
}

template <int PPL, int T, bool EP, bool SH>
__global__ void __launch_bounds__(256, 1)
k_ls_trap_mr(const TrapMultiParams p) {
  using SM = TrapSmem<PPL, T, EP>;
  constexpr int L = SM::L, X = SM::X, GT = X;
  extern __shared__ __align__(16) int32_t sm[];
  const int cpc = blockDim.x / GT;
  const int grp = threadIdx.x / GT;
  const int gt = threadIdx.x - grp * GT;
  int32_t* ws = sm + (size_t)grp * SM::ints;
  int4* s_st = reinterpret_cast<int4*>(ws);
  int32_t* s_g = ws + 4 * L;
  int32_t* s_E = s_g + L;
  __shared__ int32_t s_cta_sw;
  __shared__ unsigned long long s_rs;

  const int32_t r = p.rank0 + (int32_t)(blockIdx.x / p.ctas_per_rank);
  const int32_t lb = (int32_t)(blockIdx.x % p.ctas_per_rank);
  const bool leader = (lb == 0 && threadIdx.x == 0);
  const TrapRank& me = p.rk[r];
  const int32_t* __restrict__ E = me.E;
  const int64_t ld = p.ldE;
  const int32_t S = p.S;
  // p.vec: 16-byte row pieces allowed (the host checked the alignment of every shard)
  const bool aligned = SH ? p.sh_aligned != 0 : (((ld & 3) == 0) && ((reinterpret_cast<uintptr_t>(E) & 15) == 0));
  const bool vec = p.vec && aligned;
  using Rows = typename std::conditional<SH, ShardRows, PlainRows>::type;
  Rows er, epr;
  if constexpr (SH) {
    er = p.esh;
    epr = p.epsh;
  } else {
    er = PlainRows{E, ld};
    epr = PlainRows{me.Ep, p.ldp};
  }
  const Classes cl(S);
  const int32_t m = cl.m, H = cl.half, K = cl.npairs - 1, ncls = cl.ncls;
  const int32_t W = p.W, world = p.world, nch = p.nchunks;
  const int32_t cb = chunk_begin(r, nch, world), ce = chunk_begin(r + 1, nch, world);
  const unsigned nloc = p.ctas_per_rank;
  unsigned int bar_target = 0;
  if (p.out->status != PM_OK) return;   // uniform (written before launch)

  __shared__ int32_t s_abort, s_gab[8];   // s_gab[grp]: written by that group's thread 0 only
  unsigned int xtarget = 0;
  if (threadIdx.x == 0) { s_cta_sw = 0; s_abort = 0; }
  if (gt == 0) s_gab[grp] = 0;
  bool ok = true;
  if (SH) {
    // every rank's E shard and its permuted rows were written before that
    // rank's launch (stream order): after one cross-rank barrier every
    // peer's shard is complete and may be read
    __syncthreads();
    if (leader) {
      xtarget += (unsigned)world;
      if (!sys_barrier_arrive_wait(p, r, xtarget)) s_abort = 1;
    }
    bar_target += nloc;
    ok = grid_barrier_mr(p, r, me.bar, bar_target) && !s_abort;
  }
  if (ok)
    for (int32_t x = lb * blockDim.x + threadIdx.x; x < S; x += nloc * blockDim.x)
      __stcg(me.dbuf[0] + x, __ldg(er(__ldcg(me.rbuf[0] + x)) + x));
  bar_target += nloc;
  ok = grid_barrier_mr(p, r, me.bar, bar_target) && ok;

  uint32_t q = 0;
  int32_t rounds = 0;
  int64_t total = 0;
  int status = PM_OK;
  int64_t prev_rs = -1;
  while (ok) {
    const bool spec = spec_round(p.spec, prev_rs, X, T, ncls, K + 1, false);
    if (leader) me.rtot[(rounds + 1) % 3] = 0ull;
    for (int32_t c0 = 0; c0 < ncls && ok; c0 += T) {
      const int32_t Tp = min(T, ncls - c0);
      const int32_t u0 = wrap_m(c0 + H, m);
      const int bi = (int)(q % 3u), bn = (int)((q + 1u) % 3u);
      int mysw = 0;
      for (int32_t ch = cb + lb * cpc + grp; ch < ce + (int32_t)(nloc * cpc); ch += (int32_t)(nloc * cpc)) {
        const bool have = ch < ce;
        if (have && q > 0 && gt == 0) {
          for (int dch = -1; dch <= 1; dch += 2) {
            const int32_t c2 = ch + dch;
            if (c2 < 0 || c2 >= nch) continue;
            if (!wait_ge_sys(p, r, me.flags + c2, q)) { s_gab[grp] = 1; s_abort = 1; break; }
          }
        }
        group_sync(1 + grp, GT);
        if (s_gab[grp]) break;   // group-uniform: written by this group's thread 0 before the sync
        if (have) {
          TrapChunk C;
          const int32_t k0 = ch * W, k1 = min(k0 + W, K + 1);
          C.a = max(k0 - Tp, 0); C.b = min(k1 + Tp, K + 1);
          C.a2 = max(C.a, 1);
          C.nA = C.b - C.a; C.nB = C.b - C.a2;
          C.Lc = C.nA + C.nB + (C.a == 0 ? 1 : 0);
          C.K = K; C.m = m; C.Tp = Tp;
          const int32_t* __restrict__ rc = me.rbuf[bi];
          const int32_t* __restrict__ dc = me.dbuf[bi];
          mysw += trap_chunk<PPL, T, EP>(C, k0, k1, c0, u0, er, aligned, S,
                                     [&](int32_t x, int32_t& g, int32_t& d, int32_t& el) { g = __ldcg(rc + x); d = __ldcg(dc + x); el = -1; },
                                     s_st, s_g, s_E, gt, 1 + grp, vec, nullptr, epr, spec, p.coal);
          // publish the owned slots to the ranks owning chunks ch-1, ch, ch+1
          int32_t own[3];
          int nown = 0;
          for (int dch = -1; dch <= 1; ++dch) {
            const int32_t c2 = ch + dch;
            if (c2 < 0 || c2 >= nch) continue;
            const int32_t o = chunk_owner(c2, nch, world);
            bool dup = false;
            for (int i = 0; i < nown; ++i) dup |= (own[i] == o);
            if (!dup) own[nown++] = o;
          }
          const int32_t k = C.a + gt;
          if (k >= k0 && k < k1) {
            int32_t j1, j2;
            C.local_slots(Tp - 1, k, j1, j2);
            const int32_t x1 = C.slot_of(j1, u0, S), x2 = C.slot_of(j2, u0, S);
            const int4 A = s_st[j1], B = s_st[j2];
            const int32_t g1 = s_g[A.x & 0xffff], g2 = s_g[B.x & 0xffff];
            for (int i = 0; i < nown; ++i) {
              const TrapRank& ro = p.rk[own[i]];
              __stcg(ro.rbuf[bn] + x1, g1); __stcg(ro.dbuf[bn] + x1, A.y);
              __stcg(ro.rbuf[bn] + x2, g2); __stcg(ro.dbuf[bn] + x2, B.y);
            }
          }
          group_sync(1 + grp, GT);
          if (gt == 0) {
            bool remote = false;
            for (int i = 0; i < nown; ++i) remote |= (own[i] != r);
            if (remote) __threadfence_system();   // peer ranks: system scope
            else __threadfence();
            for (int i = 0; i < nown; ++i) {
              if (own[i] != r)
                asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p.rk[own[i]].flags + ch), "r"(q + 1u)
                             : "memory");
              else
                asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p.rk[own[i]].flags + ch), "r"(q + 1u)
                             : "memory");
            }
          }
        }
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) mysw += __shfl_xor_sync(0xffffffffu, mysw, o);
      if ((threadIdx.x & 31) == 0 && mysw) atomicAdd(&s_cta_sw, mysw);
      ++q;
      __syncthreads();
      if (s_abort) { ok = false; break; }
      if (c0 + T >= ncls) {
        // round end: every CTA's count to every rank's total (system-scope
        // atomics: the adds of several GPUs meet in one counter), then the
        // rank barrier and the cross-rank barrier, then the rank barrier again
        if (threadIdx.x == 0) {   // (thread 0 alone reads and resets the CTA's count)
          const int cta_sw = s_cta_sw;
          if (cta_sw)
            for (int o = 0; o < world; ++o) atomicAdd_system(p.rk[o].rtot + rounds % 3, (unsigned long long)cta_sw);
          s_cta_sw = 0;
        }
        bar_target += nloc;
        if (!grid_barrier_mr(p, r, me.bar, bar_target)) { ok = false; break; }
        if (leader) {
          xtarget += (unsigned)world;
          if (!sys_barrier_arrive_wait(p, r, xtarget)) s_abort = 1;
        }
        bar_target += nloc;
        if (!grid_barrier_mr(p, r, me.bar, bar_target) || s_abort) { ok = false; break; }
      }
    }
    if (!ok) break;
    if (threadIdx.x == 0) s_rs = ld_acquire_sys64(me.rtot + rounds % 3);
    __syncthreads();
    const int64_t rs = (int64_t)s_rs;
    prev_rs = rs;
    if (leader && r == p.rank0 && rounds < p.max_log) p.per_round[rounds] = rs;
    rounds += 1;
    total += rs;
    __syncthreads();
    if (rs == 0) break;
    if (p.max_rounds > 0 && rounds >= p.max_rounds) { status = PM_ERR_NOT_CONVERGED; break; }
    if (p.handoff && rs <= p.sparse_T) {   // quiet: every rank continues alone (sparse rounds, same result)
      if (leader && r == p.rank0) *p.handoff = 1;
      break;
    }
  }
  if (!ok) {   // a peer did not arrive in time: report and leave (nothing is written to perm)
    if (leader && r == p.rank0) {
      p.out->status = PM_ERR_TIMEOUT;
      p.out->rounds = rounds;
      p.out->swaps = total;
      if (p.handoff) *p.handoff = 0;
    }
    return;
  }
  // every chunk's owned slots (class ncls - 1) into every rank's perm
  const int32_t* fin = me.rbuf[q % 3u];
  for (int32_t ch = cb + lb * cpc + grp; ch < ce; ch += (int32_t)(nloc * cpc)) {
    const int32_t k0 = ch * W, k1 = min(k0 + W, K + 1);
    for (int32_t k = k0 + gt; k < k1; k += GT) {
      int32_t u, v;
      cl.pair(ncls - 1, k, u, v);
      const int32_t gu = __ldcg(fin + u), gv = __ldcg(fin + v);
      for (int o = 0; o < world; ++o) {
        __stcg(p.rk[o].perm + u, gu);
        __stcg(p.rk[o].perm + v, gv);
      }
    }
  }
  bar_target += nloc;
  ok = grid_barrier_mr(p, r, me.bar, bar_target);
  if (leader) {
    xtarget += (unsigned)world;
    if (ok) ok = sys_barrier_arrive_wait(p, r, xtarget);
    if (r == p.rank0) {
      p.out->status = ok ? status : PM_ERR_TIMEOUT;
      p.out->rounds = rounds;
      p.out->swaps = total;
    }
  }
}

// Per-rank workspace: 3 round totals, barrier counters, chunk flags, r1, r2,
// d0, d1, d2 (the rank's perm is r0).
size_t trap_ws_bytes(int32_t S) {
  const size_t n = (size_t)S;
  return 128 + sizeof(unsigned int) * (n / 2 + 16) + sizeof(int32_t) * 5 * n;
}
static void trap_ws_layout(void* ws, int32_t S, int32_t* perm, const int32_t* E, TrapRank& rk) {
  const size_t n = (size_t)S;
  char* b = static_cast<char*>(ws);
  rk.rtot = reinterpret_cast<unsigned long long*>(b);
  rk.bar = reinterpret_cast<unsigned int*>(b + 32);
  rk.xbar = reinterpret_cast<unsigned int*>(b + 64);
  rk.abort = reinterpret_cast<unsigned int*>(b + 96);
  rk.flags = reinterpret_cast<unsigned int*>(b + 128);
  int32_t* base = reinterpret_cast<int32_t*>(b + 128 + sizeof(unsigned int) * (n / 2 + 16));
  rk.rbuf[0] = perm; rk.rbuf[1] = base; rk.rbuf[2] = base + n;
  rk.dbuf[0] = base + 2 * n; rk.dbuf[1] = base + 3 * n; rk.dbuf[2] = base + 4 * n;
  rk.perm = perm;
  rk.E = E;
  rk.Ep = nullptr;
}
size_t trap_ws_zero_bytes(int32_t S) { return 128 + sizeof(unsigned int) * ((size_t)S / 2 + 16); }

// Launch `nloc` ranks [rank0, rank0 + nloc) of a world on the current device.
template <int PPL, int T, bool EP, bool SH = false>
static pm_status_t launch_trap_multi(TrapRank* ranks, int32_t world, int32_t rank0, int32_t nloc, int64_t ldE,
                                     int32_t S, int32_t max_rounds, LsResult* dev_out, int64_t* dev_per_round,
                                     int32_t max_log, cudaStream_t st, int32_t* handoff, int32_t sparse_T,
                                     int64_t ldp, const ShardRows* esh = nullptr, const ShardRows* epsh = nullptr) {
  using SM = TrapSmem<PPL, T, EP>;
  if (S < ls_trap_min_S() || (S & 1) || world < 1 || world > kMaxRanks || nloc < 1) return PM_ERR_UNSUPPORTED;
  int dev = 0, nsm = 0, optin = 0;
  PM_CUDA_TRY(cudaGetDevice(&dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  PM_CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  TrapMultiParams hp = {};
  for (int i = 0; i < world; ++i) hp.rk[i] = ranks[i];
  hp.ldE = ldE; hp.S = S; hp.max_rounds = max_rounds; hp.max_log = max_log;
  hp.W = SM::X - 2 * T;    // W = 2T: the neighbour synchronisation holds
  hp.nchunks = (Classes(S).npairs + hp.W - 1) / hp.W;
  if (hp.nchunks < world) return PM_ERR_UNSUPPORTED;
  hp.world = world; hp.rank0 = rank0;
  hp.vec = ((int64_t)S * ldE * 4 <= (96ll << 20)) ? 1 : 0;
  hp.out = dev_out; hp.per_round = dev_per_round;
  hp.handoff = handoff; hp.sparse_T = sparse_T;
  hp.ldp = ldp;
  hp.wait_ns = (unsigned long long)knob("trap_wait_ms", 20000) * 1000000ull;
  hp.spec = knob("trap_spec", 1);
  hp.coal = knob("trap_coal", 1);
  if (SH) {
    hp.esh = *esh;
    hp.epsh = *epsh;
    bool al = (ldE & 3) == 0;
    for (int o = 0; o < world; ++o) al = al && (reinterpret_cast<uintptr_t>(esh->base[o]) & 15) == 0;
    hp.sh_aligned = al ? 1 : 0;
    hp.vec = hp.vec && al;
  }
  const int per_rank_chunks = (hp.nchunks + world - 1) / world;
  int cpc = (per_rank_chunks * nloc + nsm - 1) / nsm;
  int max_cpc = (int)((size_t)optin / SM::bytes);
  if (max_cpc > 8 / PPL) max_cpc = 8 / PPL;
  if (cpc < 1) cpc = 1;
  if (cpc > max_cpc) cpc = max_cpc;
  const size_t smem = SM::bytes * cpc;
  const int threads = SM::X * cpc;
  auto fn = k_ls_trap_mr<PPL, T, EP, SH>;
  PM_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  PM_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, smem));
  if (occ < 1) return PM_ERR_UNSUPPORTED;
  int cpr = (per_rank_chunks + cpc - 1) / cpc;        // CTAs per rank
  if (cpr * nloc > nsm * occ) cpr = (nsm * occ) / nloc;
  if (cpr < 1) return PM_ERR_UNSUPPORTED;
  hp.ctas_per_rank = cpr;
  void* args[] = {(void*)&hp};
  PM_CUDA_TRY(cudaLaunchCooperativeKernel((const void*)fn, dim3(cpr * nloc), dim3(threads), args, smem, st));
  note_launch();
  return PM_OK;
}

static bool ep_expected(int32_t S) {   // trap_build_ep's rule, before anything is allocated
  const int32_t mode = knob("trap_ep", 1);
  if (mode == 0) return false;
  const int64_t l = ((int64_t)S - 1 + 48 + 31) / 32 * 32;
  return mode == 2 || sizeof(int32_t) * (size_t)S * (size_t)l <= device_total_mem() / 8;
}
static int32_t trap_multi_variant(int32_t S, int64_t ldE) {
  int32_t v = knob("trap_variant", -1);
  if (v != 0 && v != 5 && v != 6)
    v = ((int64_t)S * ldE * 4 > (96ll << 20)) ? (ep_expected(S) ? 6 : 5) : 0;
  return v;
}
// Chunk geometry as the single-GPU path: 64 x 16 while E is L2-resident
// (small S: enough chunks for every rank), else 192 x 48 with the
// sigma-permuted copy, 128 x 32 without (trap_variant 0 / 5 / 6 force one).
pm_status_t run_trap_multi(TrapRank* ranks, int32_t world, int32_t rank0, int32_t nloc, int64_t ldE, int32_t S,
                           int32_t max_rounds, LsResult* dev_out, int64_t* dev_per_round, int32_t max_log,
                           cudaStream_t st, int32_t* handoff = nullptr, int32_t sparse_T = 0, int64_t ldp = 0) {
  const bool ep = ranks[rank0].Ep != nullptr;
  const int32_t v = trap_multi_variant(S, ldE);
  if (v == 6 && ep)
    return launch_trap_multi<6, 48, true>(ranks, world, rank0, nloc, ldE, S, max_rounds, dev_out, dev_per_round,
                                          max_log, st, handoff, sparse_T, ldp);
  if (v == 5 || v == 6)
    return ep ? launch_trap_multi<4, 32, true>(ranks, world, rank0, nloc, ldE, S, max_rounds, dev_out, dev_per_round,
                                               max_log, st, handoff, sparse_T, ldp)
              : launch_trap_multi<4, 32, false>(ranks, world, rank0, nloc, ldE, S, max_rounds, dev_out, dev_per_round,
                                                max_log, st, handoff, sparse_T, ldp);
  return ep ? launch_trap_multi<2, 16, true>(ranks, world, rank0, nloc, ldE, S, max_rounds, dev_out, dev_per_round,
                                             max_log, st, handoff, sparse_T, ldp)
            : launch_trap_multi<2, 16, false>(ranks, world, rank0, nloc, ldE, S, max_rounds, dev_out, dev_per_round,
                                              max_log, st, handoff, sparse_T, ldp);
}


// Can the multi-rank kernel take (S, world)?  Checked before anything is
// enqueued (pm.h: arguments are validated before any launch).
pm_status_t trap_multi_supported(int32_t S, int64_t ldE, int32_t world) {
  if (world < 1 || world > kMaxRanks) return PM_ERR_INVALID;
  if (S < ls_trap_min_S() || (S & 1)) return PM_ERR_UNSUPPORTED;
  const int32_t v = trap_multi_variant(S, ldE);
  const int32_t W = v == 6 ? 96 : (v == 5 ? 64 : 32);   // X - 2T of the geometry
  if ((Classes(S).npairs + W - 1) / W < world) return PM_ERR_UNSUPPORTED;
  return PM_OK;
}

// All ranks of a world on the current device, one launch (test hook).
pm_status_t trap_multi_emulated(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t world,
                                int32_t max_rounds, LsResult* dev_out, int64_t* dev_per_round, int32_t max_log,
                                cudaStream_t st) {
  {
    const pm_status_t v = trap_multi_supported(S, ldE, world);
    if (v != PM_OK) return v;
  }
  PM_CUDA_TRY(launch_perm_check(perm, S, dev_out, st));
  const size_t wsb = (trap_ws_bytes(S) + 255) / 256 * 256;
  const size_t pb = ((size_t)S * sizeof(int32_t) + 255) / 256 * 256;
  ScopedScratch bufs(st), sps(st), ep(st);
  PM_CUDA_TRY(pm::scratch_alloc(&bufs.p, (wsb + pb) * world, st));
  char* buf = bufs.as<char>();
  TrapRank ranks[kMaxRanks];
  for (int r = 0; r < world; ++r) {
    char* ws = buf + (wsb + pb) * r;
    int32_t* pr = reinterpret_cast<int32_t*>(ws + wsb);
    PM_CUDA_TRY(cudaMemsetAsync(ws, 0, trap_ws_zero_bytes(S), st));
    PM_CUDA_TRY(cudaMemcpyAsync(pr, perm, sizeof(int32_t) * S, cudaMemcpyDeviceToDevice, st));
    trap_ws_layout(ws, S, pr, E, ranks[r]);
  }
  int64_t ldp = 0;
  {
    int32_t* Ep = nullptr;
    const pm_status_t se = trap_build_ep(E, ldE, S, st, &Ep, &ldp);
    ep.p = Ep;
    if (se != PM_OK) return se;
  }
  // quiet rounds: every rank would continue alone with the same sparse
  // rounds; here rank world-1 (the farthest from the launch's first) does
  const int32_t sparse_T = ls_sparse_threshold(S, PM_LS_TRAP);
  SparseRun sr;
  if (sparse_T > 0) {
    const pm_status_t s0 = sparse_prepare(E, ldE, S, ranks[world - 1].perm, max_rounds, dev_out, dev_per_round,
                                          max_log, st, &sr, 0, ep.as<int32_t>(), ldp);
    if (s0 != PM_OK) return s0;
    sps.p = sr.scratch;   // freed here on an error path; sparse_launch frees it otherwise
  }
  for (int r = 0; r < world; ++r) ranks[r].Ep = ep.as<int32_t>();
  pm_status_t s = run_trap_multi(ranks, world, 0, world, ldE, S, max_rounds, dev_out, dev_per_round, max_log, st,
                                 sr.pending, sparse_T, ldp);
  if (s != PM_OK) return s;
  if (sparse_T > 0) {
    sps.p = nullptr;
    const pm_status_t s1 = sparse_launch(&sr, st);
    if (s1 != PM_OK) return s1;
  }
  PM_CUDA_TRY(cudaMemcpyAsync(perm, ranks[world - 1].perm, sizeof(int32_t) * S, cudaMemcpyDeviceToDevice, st));
  return PM_OK;
}

// One rank of a multi-GPU world: ws_peers[o] / perm_peers[o] are rank o's
// workspace and perm mapped into this process (peer memory); every
// workspace zeroed and every perm holding the same bijection before any
// rank launches.
pm_status_t trap_multi_rank(const int32_t* E, int64_t ldE, int32_t S, int32_t* const* perm_peers,
                            void* const* ws_peers, int32_t rank, int32_t world, int32_t max_rounds,
                            LsResult* dev_out, int64_t* dev_per_round, int32_t max_log, cudaStream_t st) {
  if (rank < 0 || rank >= world) return PM_ERR_INVALID;
  {
    const pm_status_t v = trap_multi_supported(S, ldE, world);
    if (v != PM_OK) return v;
  }
  // a non-bijection would send out-of-range tile indices into E; every rank
  // holds the same perm, so every rank's kernel returns at once (status set)
  PM_CUDA_TRY(launch_perm_check(perm_peers[rank], S, dev_out, st));
  TrapRank ranks[kMaxRanks];
  for (int r = 0; r < world; ++r) trap_ws_layout(ws_peers[r], S, perm_peers[r], E, ranks[r]);
  // quiet rounds: this rank continues alone (sparse rounds on its own copy
  // of r and E -- every rank reaches the same result, no exchange)
  const int32_t sparse_T = ls_sparse_threshold(S, PM_LS_TRAP);
  ScopedScratch sps(st), ep(st);
  int64_t ldp = 0;
  {
    int32_t* Ep = nullptr;
    const pm_status_t se = trap_build_ep(E, ldE, S, st, &Ep, &ldp);
    ep.p = Ep;
    if (se != PM_OK) return se;
  }
  SparseRun sr;
  if (sparse_T > 0) {
    const pm_status_t s0 = sparse_prepare(E, ldE, S, perm_peers[rank], max_rounds, dev_out, dev_per_round, max_log,
                                          st, &sr, 0, ep.as<int32_t>(), ldp);
    if (s0 != PM_OK) return s0;
    sps.p = sr.scratch;
  }
  ranks[rank].Ep = ep.as<int32_t>();   // only this rank's entry is read by this launch
  const pm_status_t s = run_trap_multi(ranks, world, rank, 1, ldE, S, max_rounds, dev_out, dev_per_round, max_log,
                                       st, sr.pending, sparse_T, ldp);
  if (s != PM_OK) return s;
  if (sparse_T > 0) {
    sps.p = nullptr;
    return sparse_launch(&sr, st);
  }
  return PM_OK;
}

// ---------------------------------------------------------------------
// Row-sharded E (north_star's multi-GPU layout): rank o holds rows
// [rb[o], rb[o+1]) of E, and builds the sigma-permuted copy of the same rows
// into its workspace; every rank reads any tile's runs from the owner's
// shard through peer memory, so no rank holds (or all-gathers) all of E.  No
// sparse rounds (they would gather all of E): TRAP runs every round.
static int64_t ep_ld(int32_t S) { return ((int64_t)S - 1 + 48 + 31) / 32 * 32; }
static size_t ws_head_sharded(int32_t S) { return (trap_ws_bytes(S) + 255) / 256 * 256; }
size_t trap_ws_bytes_sharded(int32_t S, int32_t rows) {
  return ws_head_sharded(S) + sizeof(int32_t) * (size_t)rows * (size_t)ep_ld(S);
}

static pm_status_t check_shards(const int32_t* rb, int32_t S, int32_t world) {
  if (world < 1 || world > kMaxRanks || !rb || rb[0] != 0 || rb[world] != S) return PM_ERR_INVALID;
  for (int o = 0; o < world; ++o)
    if (rb[o + 1] < rb[o]) return PM_ERR_INVALID;
  return PM_OK;
}

static pm_status_t launch_sharded(TrapRank* ranks, int32_t world, int32_t rank0, int32_t nloc, int64_t ldE,
                                  int32_t S, int32_t max_rounds, LsResult* dev_out, int64_t* dev_per_round,
                                  int32_t max_log, cudaStream_t st, const ShardRows& esh, const ShardRows& epsh) {
  const int64_t ldp = epsh.ld;
  const int32_t v = trap_multi_variant(S, ldE);
  if (v == 6)
    return launch_trap_multi<6, 48, true, true>(ranks, world, rank0, nloc, ldE, S, max_rounds, dev_out, dev_per_round,
                                                max_log, st, nullptr, 0, ldp, &esh, &epsh);
  if (v == 5)
    return launch_trap_multi<4, 32, true, true>(ranks, world, rank0, nloc, ldE, S, max_rounds, dev_out, dev_per_round,
                                                max_log, st, nullptr, 0, ldp, &esh, &epsh);
  return launch_trap_multi<2, 16, true, true>(ranks, world, rank0, nloc, ldE, S, max_rounds, dev_out, dev_per_round,
                                              max_log, st, nullptr, 0, ldp, &esh, &epsh);
}

pm_status_t trap_multi_rank_sharded(const int32_t* const* E_peers, const int32_t* rb, int64_t ldE, int32_t S,
                                    int32_t* const* perm_peers, void* const* ws_peers, int32_t rank, int32_t world,
                                    int32_t max_rounds, LsResult* dev_out, cudaStream_t st) {
  {
    const pm_status_t v = check_shards(rb, S, world);
    if (v != PM_OK) return v;
    if (rank < 0 || rank >= world) return PM_ERR_INVALID;
    const pm_status_t w = trap_multi_supported(S, ldE, world);
    if (w != PM_OK) return w;
  }
  PM_CUDA_TRY(launch_perm_check(perm_peers[rank], S, dev_out, st));
  const size_t head = ws_head_sharded(S);
  const int64_t ldp = ep_ld(S);
  ShardRows esh = {}, epsh = {};
  esh.world = epsh.world = world;
  esh.ld = ldE;
  epsh.ld = ldp;
  TrapRank ranks[kMaxRanks];
  for (int o = 0; o < world; ++o) {
    trap_ws_layout(ws_peers[o], S, perm_peers[o], nullptr, ranks[o]);
    esh.base[o] = E_peers[o];
    epsh.base[o] = reinterpret_cast<const int32_t*>(static_cast<const char*>(ws_peers[o]) + head);
  }
  for (int o = 0; o <= world; ++o) esh.rb[o] = epsh.rb[o] = rb[o];
  // this rank's rows of Ep, into its own workspace (peers read them after
  // the kernel's opening cross-rank barrier)
  const int32_t rows = rb[rank + 1] - rb[rank];
  if (rows > 0)
    PM_CUDA_TRY(launch_permute_cols(E_peers[rank], ldE, const_cast<int32_t*>(epsh.base[rank]), ldp, rows, S - 1, 48,
                                    st));
  return launch_sharded(ranks, world, rank, 1, ldE, S, max_rounds, dev_out, nullptr, 0, st, esh, epsh);
}

// Every rank of a world in one launch on the current device (test hook): E's
// rows copied into `world` separate shard buffers, each with its own Ep rows.
pm_status_t trap_multi_emulated_sharded(const int32_t* E, int64_t ldE, int32_t S, int32_t* perm, int32_t world,
                                        int32_t max_rounds, LsResult* dev_out, cudaStream_t st) {
  {
    const pm_status_t w = trap_multi_supported(S, ldE, world);
    if (w != PM_OK) return w;
  }
  PM_CUDA_TRY(launch_perm_check(perm, S, dev_out, st));
  int32_t rb[kMaxRanks + 1];
  for (int o = 0; o <= world; ++o) rb[o] = (int32_t)(((int64_t)S * o) / world);
  const size_t head = ws_head_sharded(S);
  const int64_t ldp = ep_ld(S);
  const size_t pb = ((size_t)S * sizeof(int32_t) + 255) / 256 * 256;
  size_t total = 0;
  size_t off_ws[kMaxRanks], off_perm[kMaxRanks], off_e[kMaxRanks];
  for (int o = 0; o < world; ++o) {
    const int32_t rows = rb[o + 1] - rb[o];
    off_ws[o] = total;
    total += (trap_ws_bytes_sharded(S, rows) + 255) / 256 * 256;
    off_perm[o] = total;
    total += pb;
    off_e[o] = total;
    total += ((size_t)rows * (size_t)ldE * sizeof(int32_t) + 255) / 256 * 256;
  }
  ScopedScratch buf(st);
  PM_CUDA_TRY(pm::scratch_alloc(&buf.p, total, st));
  char* b = buf.as<char>();
  ShardRows esh = {}, epsh = {};
  esh.world = epsh.world = world;
  esh.ld = ldE;
  epsh.ld = ldp;
  TrapRank ranks[kMaxRanks];
  for (int o = 0; o < world; ++o) {
    const int32_t rows = rb[o + 1] - rb[o];
    void* ws = b + off_ws[o];
    int32_t* pr = reinterpret_cast<int32_t*>(b + off_perm[o]);
    int32_t* es = reinterpret_cast<int32_t*>(b + off_e[o]);
    PM_CUDA_TRY(cudaMemsetAsync(ws, 0, trap_ws_zero_bytes(S), st));
    PM_CUDA_TRY(cudaMemcpyAsync(pr, perm, sizeof(int32_t) * S, cudaMemcpyDeviceToDevice, st));
    if (rows > 0)
      PM_CUDA_TRY(cudaMemcpy2DAsync(es, sizeof(int32_t) * ldE, E + (int64_t)rb[o] * ldE, sizeof(int32_t) * ldE,
                                    sizeof(int32_t) * S, rows, cudaMemcpyDeviceToDevice, st));
    trap_ws_layout(ws, S, pr, nullptr, ranks[o]);
    esh.base[o] = es;
    epsh.base[o] = reinterpret_cast<const int32_t*>(static_cast<char*>(ws) + head);
    if (rows > 0)
      PM_CUDA_TRY(launch_permute_cols(es, ldE, const_cast<int32_t*>(epsh.base[o]), ldp, rows, S - 1, 48, st));
  }
  for (int o = 0; o <= world; ++o) esh.rb[o] = epsh.rb[o] = rb[o];
  const pm_status_t s = launch_sharded(ranks, world, 0, world, ldE, S, max_rounds, dev_out, nullptr, 0, st, esh, epsh);
  if (s != PM_OK) return s;
  PM_CUDA_TRY(cudaMemcpyAsync(perm, ranks[world - 1].perm, sizeof(int32_t) * S, cudaMemcpyDeviceToDevice, st));
  return PM_OK;
}
}  // namespace pm
