// k_sad.cu -- Step 1 (tile packing) and Step 2 (the all-pairs tile
// error matrix, Eq. 1) for sm_100a.
//
// Eq. (1) is an L1 / sum-of-absolute-differences metric (reading R1), which is
// not bilinear, so it does not map onto tcgen05 tensor cores (the exact
// threshold-decomposition form would need 255x the MACs; DESIGN.md "E
// kernel").  It runs on the integer ALU pipe instead: one
// `vabsdiff4.u32.u32.u32.add` (SASS VABSDIFF4.U8.ACC) consumes 4 byte pairs
// and accumulates into an int32; it issues at 64 /clk/SM, half the IADD3
// rate (~124 /clk/SM in the same microbenchmark, tools/ubench_alu.cu,
// profiles/r01_ubench_alu.txt).  The kernel is a register-blocked "SAD-GEMM":
//   * CTA tile 128 (input tiles u) x 64 (target tiles v), 256 threads, each
//     thread 8 x 4 outputs, two CTAs per SM (the 128 x 128 / 8 x 8 variant
//     measured ~3 % slower at every size); rows ty + 16 i, cols tx + 16 j ->
//     conflict-free LDS.128 on a 80-byte padded smem row stride;
//   * K (the P bytes of a tile) streamed in 128-byte chunks (64 when K is not
//     a multiple of 32 words) through a 4-stage cp.async.cg ring (16-byte
//     copies, L2-only): 6 main-loop iterations per tile at P = 768;
//   * per 4 K-words a thread issues 12 LDS.128 and 128 VABSDIFF4 (8 x 8 tile: 16 and 256);
//   * split-K over gridDim.z available (integer red.add is exact and
//     order-independent), chosen on the host only when it pays (measured:
//     never at configs 1-5);
//   * optionally the epilogue also writes TRAP's sigma-permuted copy of E
//     (pm_error_matrix_sigma).
#include "pm_internal.cuh"

namespace pm {

// ---------------------------------------------------------------- Step 1 ---
// One thread per 4 output bytes of the packed layout; tile t in
// [tile_begin, tile_end) goes to row t - tile_begin of `tiles`.
__global__ void k_pack(const uint8_t* __restrict__ img, int32_t N, int32_t M, int32_t C,
                       uint8_t* __restrict__ tiles, int64_t ld_tiles, int32_t tile_begin,
                       int32_t tile_end) {
  const int32_t g = N / M;
  const int32_t P = M * M * C;
  const int64_t words_per_tile = ld_tiles / 4;
  const int64_t total = (int64_t)(tile_end - tile_begin) * words_per_tile;
  for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < total;
       w += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t = tile_begin + w / words_per_tile;
    const int32_t k0 = (int32_t)(w % words_per_tile) * 4;
    const int64_t ty = t / g, tx = t % g;
    uint32_t out = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int32_t k = k0 + q;
      uint32_t byte = 0;
      if (k < P) {
        const int32_t pix = k / C, c = k - pix * C;
        const int32_t y = pix / M, x = pix - y * M;
        byte = img[((ty * M + y) * (int64_t)N + tx * M + x) * C + c];
      }
      out |= byte << (8 * q);
    }
    reinterpret_cast<uint32_t*>(tiles + (t - tile_begin) * ld_tiles)[k0 / 4] = out;
  }
}

cudaError_t launch_pack(const uint8_t* img, int32_t N, int32_t M, int32_t C, uint8_t* tiles,
                        int64_t ld_tiles, int32_t tile_begin, int32_t tile_end, cudaStream_t st) {
  const int64_t total = (int64_t)(tile_end - tile_begin) * (ld_tiles / 4);
  if (total <= 0) return cudaSuccess;
  int64_t blocks = (total + 255) / 256;
  if (blocks > 148 * 16) blocks = 148 * 16;
  k_pack<<<(unsigned)blocks, 256, 0, st>>>(img, N, M, C, tiles, ld_tiles, tile_begin, tile_end);
  note_launch();
  return cudaGetLastError();
}

// ------------------------------------------------------------- render R ---
// The photomosaic: target slot u of R shows input tile r[u].
// One thread per output byte (coalesced writes; the reads are row segments of
// the source tile).
__global__ void k_render(const uint8_t* __restrict__ img, int32_t N, int32_t M, int32_t C,
                         const int32_t* __restrict__ perm, uint8_t* __restrict__ out) {
  const int32_t g = N / M;
  const int64_t total = (int64_t)N * N * C;
  const int64_t rowb = (int64_t)N * C;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t py = i / rowb;
    const int32_t rem = (int32_t)(i - py * rowb);
    const int32_t px = rem / C, c = rem - px * C;
    const int32_t uy = (int32_t)(py / M), y = (int32_t)(py - (int64_t)uy * M);
    const int32_t ux = px / M, x = px - ux * M;
    const int32_t t = __ldg(perm + (int64_t)uy * g + ux);
    const int32_t ty = t / g, tx = t - ty * g;
    out[i] = __ldg(img + ((int64_t)(ty * M + y) * N + tx * M + x) * C + c);
  }
}

cudaError_t launch_render(const uint8_t* img, int32_t N, int32_t M, int32_t C, const int32_t* perm,
                          uint8_t* out, cudaStream_t st) {
  const int64_t total = (int64_t)N * N * C;
  int64_t blocks = (total + 255) / 256;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks < 1) blocks = 1;
  k_render<<<(unsigned)blocks, 256, 0, st>>>(img, N, M, C, perm, out);
  note_launch();
  return cudaGetLastError();
}

// ---------------------------------------------------------------- Step 2 ---
namespace sad {
constexpr int kThreads = 256;
constexpr int BM = 128;          // tile rows (input tiles u); BN (target tiles v) is 128 or 64
constexpr int kStages = 4;
// K words (4 bytes each) per pipeline stage: 32 when K is a multiple of 32
// words (P = 768: 6 instead of 12 main-loop iterations per tile, each with
// its barrier and copy issue -- config 4 E 3.47 -> 3.26 ms, 80 -> 85 % of the
// ALU peak), else 16.  Padded smem row stride KW + 4 words (conflict-free
// LDS.128 for both).
template <int BN, int KW>
constexpr int smem_bytes() { return kStages * (BM + BN) * (KW + 4) * 4; }   // 60 / 110 KiB at BN = 64
inline int stage_words(int64_t kw) { return (kw % 32 == 0) ? 32 : 16; }
}  // namespace sad

__device__ __forceinline__ uint32_t sad4(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("vabsdiff4.u32.u32.u32.add %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}

__device__ __forceinline__ void cp_async16(uint32_t* smem, const void* gmem) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

// Where the K bytes of a tile live.  Packed: tile t at A + t*ldt (bytes
// contiguous).  Image (Step 1 fused into the loader, used when a tile row is a
// whole number of 16-byte pieces): tile t = grid cell (t / g, t % g) of a u8
// HWC image; its 16-byte piece p is row y = p / R (R = M*C/16 pieces per tile
// row) at byte offset (p % R)*16 of that row, i.e. the same (y, x, c) byte
// order as k_pack produces.
struct SadGeom {
  const uint8_t* A;        // input tiles (packed, already offset by row_begin) or input image
  const uint8_t* B;        // target tiles or target image
  int64_t ldt;             // packed: tile stride in bytes
  int64_t rowbytes;        // image: N*C
  int32_t a_tile0;         // image: tile index of local row 0 (row_begin)
  int32_t g, M, R, MC;     // image: tiles per grid row, tile side, pieces per tile row, M*C
  int32_t e_row0;          // row of Ep that local row 0 goes to (the sigma copy, when written)
  int32_t vec_out;         // 0: scalar epilogue; >= 1: E rows 16-byte aligned (staged epilogue); 2: also S/2 % 4 == 0
};

template <bool kImage>
__device__ __forceinline__ const uint8_t* sad_tile_base(const SadGeom& geo, const uint8_t* img, int32_t t) {
  if (kImage) {
    const int32_t ty = t / geo.g, tx = t - ty * geo.g;
    return img + (int64_t)ty * geo.M * geo.rowbytes + (int64_t)tx * geo.MC;
  }
  return img + (int64_t)t * geo.ldt;
}

// nrows rows of A (input tiles), S columns (target tiles).  kw_split: K words
// handled by one blockIdx.z slice.  BN = 128: 8 x 8 outputs per thread, one
// CTA per SM; BN = 64: 8 x 4, two CTAs per SM (for grids too small to fill
// 148 SMs with 128 x 128 tiles without split-K).
template <bool kAtomic, bool kImage, int BN, int KW>
__global__ void __launch_bounds__(sad::kThreads, BN == 128 ? 1 : 2)
k_sad(SadGeom geo, int32_t nrows, int32_t S, int32_t kw_split, int32_t* __restrict__ E, int64_t ldE,
      int32_t* __restrict__ Ep, int64_t ldp) {
  using namespace sad;
  constexpr int BKW = KW;                              // K words per pipeline stage
  constexpr int ROWW = KW + 4;                         // padded smem row stride in words
  constexpr int NJ = BN / 16;                          // output columns per thread
  extern __shared__ __align__(16) uint32_t smem[];
  uint32_t* sA = smem;                                 // [kStages][BM][ROWW]
  uint32_t* sB = smem + kStages * BM * ROWW;           // [kStages][BN][ROWW]

  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
  const int32_t row0 = blockIdx.y * BM, col0 = blockIdx.x * BN;
  const int32_t piece0 = blockIdx.z * kw_split / 4;    // first 16-byte piece of this K slice
  const int nkb = kw_split / BKW;

  // Loader: per stage, BM (BN) rows x 4 BKW B = PPR BM (PPR BN) 16-byte
  // pieces per operand (PPR = BKW / 4); thread tid copies pieces
  // q = tid + h * 256 (row q / PPR, part q % PPR).
  constexpr int PPR = BKW / 4;
  constexpr int HA = BM * PPR / kThreads, HB = BN * PPR / kThreads;
  const uint8_t* baseA[HA];
  const uint8_t* baseB[HB];
  const int part = tid % PPR;
#pragma unroll
  for (int h = 0; h < HA; ++h) {
    int32_t ra = row0 + (tid + h * kThreads) / PPR; if (ra >= nrows) ra = nrows - 1;   // clamp: loaded, never stored
    baseA[h] = sad_tile_base<kImage>(geo, geo.A, kImage ? geo.a_tile0 + ra : ra);
  }
#pragma unroll
  for (int h = 0; h < HB; ++h) {
    int32_t rb = col0 + (tid + h * kThreads) / PPR; if (rb >= S) rb = S - 1;
    baseB[h] = sad_tile_base<kImage>(geo, geo.B, rb);
  }
  auto load_stage = [&](int kb, int stage) {
    const int32_t p = piece0 + kb * (BKW / 4) + part;
    int64_t off;
    if (kImage) {
      const int32_t y = p / geo.R;
      off = (int64_t)y * geo.rowbytes + (p - y * geo.R) * 16;
    } else {
      off = (int64_t)p * 16;
    }
#pragma unroll
    for (int h = 0; h < HA; ++h) cp_async16(sA + stage * BM * ROWW + ((tid + h * kThreads) / PPR) * ROWW + part * 4, baseA[h] + off);
#pragma unroll
    for (int h = 0; h < HB; ++h) cp_async16(sB + stage * BN * ROWW + ((tid + h * kThreads) / PPR) * ROWW + part * 4, baseB[h] + off);
  };

  uint32_t acc[8][NJ];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[i][j] = 0u;

#pragma unroll
  for (int s = 0; s < kStages - 1; ++s) {
    if (s < nkb) load_stage(s, s);
    cp_async_commit();
  }

  for (int kb = 0; kb < nkb; ++kb) {
    cp_async_wait<kStages - 2>();
    __syncthreads();   // stage kb landed for all; stage kb-1 fully consumed
    {
      const int nk = kb + kStages - 1;
      if (nk < nkb) load_stage(nk, nk % kStages);
      cp_async_commit();
    }
    const int stage = kb % kStages;
    const uint32_t* a_base = sA + stage * BM * ROWW + ty * ROWW;
    const uint32_t* b_base = sB + stage * BN * ROWW + tx * ROWW;
#pragma unroll
    for (int kk = 0; kk < BKW; kk += 4) {
      uint4 a[8], b[NJ];
#pragma unroll
      for (int i = 0; i < 8; ++i) a[i] = *reinterpret_cast<const uint4*>(a_base + i * 16 * ROWW + kk);
#pragma unroll
      for (int j = 0; j < NJ; ++j) b[j] = *reinterpret_cast<const uint4*>(b_base + j * 16 * ROWW + kk);
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
          uint32_t t = acc[i][j];
          t = sad4(a[i].x, b[j].x, t);
          t = sad4(a[i].y, b[j].y, t);
          t = sad4(a[i].z, b[j].z, t);
          t = sad4(a[i].w, b[j].w, t);
          acc[i][j] = t;
        }
    }
  }
  cp_async_wait<0>();

  // Full tiles with 16-byte-aligned rows (geo.vec_out): the outputs go
  // through shared memory and leave as coalesced 16-byte stores -- E's rows,
  // and the sigma copy's two contiguous runs per row (even columns -> q =
  // col/2, odd -> (col + m)/2 = col/2 + S/2) -- instead of one 4-byte store
  // per entry (and two per entry of the copy).
  const int32_t mq = S - 1;
  if (!kAtomic && geo.vec_out && row0 + BM <= nrows && col0 + BN < S) {   // (col0 + BN <= m: every column in the copy)
    constexpr int OS = BN + 16;                         // padded row stride: conflict-free fills
    static_assert(BM * OS * 4 <= kStages * (BM + BN) * ROWW * 4, "staged tile fits the pipeline smem");
    __syncthreads();                                    // every warp done with the pipeline buffers
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < NJ; ++j) smem[(ty + 16 * i) * OS + tx + 16 * j] = acc[i][j];
    __syncthreads();
    constexpr int NV = BM * BN / 4 / kThreads;          // 16-byte pieces per thread
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      const int idx = tid + v * kThreads;
      const int r = idx / (BN / 4), c4 = idx - r * (BN / 4);
      const uint4 val = *reinterpret_cast<const uint4*>(smem + r * OS + 4 * c4);
      *reinterpret_cast<uint4*>(E + (int64_t)(row0 + r) * ldE + col0 + 4 * c4) = val;
    }
    if (Ep) {
      const bool odd_vec = geo.vec_out > 1;             // S/2 % 4 == 0: the odd run is 16-byte aligned too
#pragma unroll
      for (int v = 0; v < NV; ++v) {
        const int idx = tid + v * kThreads;
        const int r = idx / (BN / 4), w = idx - r * (BN / 4);
        const int par = w >= BN / 8 ? 1 : 0, k4 = w - par * (BN / 8);
        const uint32_t* srow = smem + r * OS + 8 * k4 + par;
        const uint4 val = make_uint4(srow[0], srow[2], srow[4], srow[6]);
        const int32_t q0 = (col0 >> 1) + (par ? (S >> 1) : 0) + 4 * k4;
        int32_t* prow = Ep + (int64_t)(geo.e_row0 + row0 + r) * ldp;
        if (!par || odd_vec) {
          *reinterpret_cast<uint4*>(prow + q0) = val;
        } else {
          prow[q0] = (int32_t)val.x; prow[q0 + 1] = (int32_t)val.y;
          prow[q0 + 2] = (int32_t)val.z; prow[q0 + 3] = (int32_t)val.w;
        }
        if (q0 < 48) {                                  // the cyclic extension, q + m for q < 48
          const uint32_t vv[4] = {val.x, val.y, val.z, val.w};
#pragma unroll
          for (int e = 0; e < 4; ++e)
            for (int32_t qq = q0 + e + mq; qq < mq + 48; qq += mq) prow[qq] = (int32_t)vv[e];
        }
      }
    }
    return;
  }

#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int32_t row = row0 + ty + 16 * i;
    if (row >= nrows) continue;
    int32_t* erow = E + (int64_t)row * ldE;
#pragma unroll
    for (int j = 0; j < NJ; ++j) {
      const int32_t col = col0 + tx + 16 * j;
      if (col >= S) continue;
      if (kAtomic) atomicAdd(erow + col, (int32_t)acc[i][j]);
      else erow[col] = (int32_t)acc[i][j];
      // the sigma-permuted copy TRAP stages from (k_trap.cu), written in the
      // same pass (no separate read + write of E): Ep[row][q] = E[row][2q mod m]
      // for q < m + 48 cyclic, m = S - 1 odd -> column col lands at
      // q = sigma(col) = col/2 (even) or (col+m)/2 (odd), and again at q + m,
      // q + 2m, ... below m + 48
      if (!kAtomic && Ep) {
        const int32_t m = S - 1;
        if (col < m) {
          const int32_t q = (col & 1) ? (col + m) >> 1 : col >> 1;
          int32_t* prow = Ep + (int64_t)(geo.e_row0 + row) * ldp;
          prow[q] = (int32_t)acc[i][j];
          for (int32_t qq = q + m; qq < m + 48; qq += m) prow[qq] = (int32_t)acc[i][j];   // (m < 48: wraps again)
        }
      }
    }
  }
}

// Host-side tiling choice: 128 x 128 or 128 x 64 tiles (two CTAs per SM,
// half the work per tile), each with split-K over the divisors of nkb.
// Cost = waves * per-CTA work, biased by measured factors.
struct SadPlan { int bn, split; };
static SadPlan choose_plan(int64_t nrows, int64_t S, int nkb, int sms) {
  SadPlan best{128, 1};
  double best_cost = 1e300;
  const int64_t gy = (nrows + sad::BM - 1) / sad::BM;
  for (int s = 1; s <= nkb; ++s) {
    if (nkb % s) continue;
    if (s > 1 && nkb / s < 2) break;
    const int64_t ctas = gy * ((S + 127) / 128) * s;
    const double cost = (double)((ctas + sms - 1) / sms) * (nkb / s) * (s > 1 ? 1.35 : 1.0);
    if (cost < best_cost - 1e-9) { best_cost = cost; best = {128, s}; }
  }
  // half-size tiles, two CTAs per SM.  Factors measured (round 2, configs
  // 2-4, tools/e_bench.py): 128 x 64 tiles are ~3 % faster than 128 x 128 at
  // any size (0.48 per half-size tile), and split-K never paid (its memset
  // and atomics: x1.35)
  for (int s = 1; s <= nkb; ++s) {
    if (nkb % s) continue;
    if (s > 1 && nkb / s < 2) break;
    const int64_t ctas = gy * ((S + 63) / 64) * s;
    const double cost = (double)((ctas + sms - 1) / sms) * (nkb / s) * 0.48 * (s > 1 ? 1.35 : 1.0);
    if (cost < best_cost - 1e-9) { best_cost = cost; best = {64, s}; }
  }
  // tuning: sad_plan = 1000 * bn + split forces a plan (tests / tools)
  const int32_t forced = knob("sad_plan", 0);
  if (forced > 0) {
    const int bn = forced / 1000 == 64 ? 64 : 128, sp = forced % 1000;
    if (sp >= 1 && nkb % sp == 0) best = {bn, sp};
  }
  return best;
}

template <bool kAtomic, bool kImage, int BN, int KW>
static cudaError_t sad_set_attr() {
  return cudaFuncSetAttribute(k_sad<kAtomic, kImage, BN, KW>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              sad::smem_bytes<BN, KW>());
}
template <int KW>
static cudaError_t sad_set_attr_all() {
  cudaError_t e;
  if ((e = sad_set_attr<false, false, 128, KW>()) != cudaSuccess) return e;
  if ((e = sad_set_attr<true, false, 128, KW>()) != cudaSuccess) return e;
  if ((e = sad_set_attr<false, true, 128, KW>()) != cudaSuccess) return e;
  if ((e = sad_set_attr<true, true, 128, KW>()) != cudaSuccess) return e;
  if ((e = sad_set_attr<false, false, 64, KW>()) != cudaSuccess) return e;
  if ((e = sad_set_attr<false, true, 64, KW>()) != cudaSuccess) return e;
  if ((e = sad_set_attr<true, false, 64, KW>()) != cudaSuccess) return e;
  return sad_set_attr<true, true, 64, KW>();
}

// One launch of the chosen plan for a stage width KW.
template <int KW>
static void sad_launch_kw(const SadGeom& g2, bool image, int bn, int split, int32_t nrows, int32_t S, int kw,
                          int64_t gy, int32_t* E, int64_t ldE, int32_t* Ep, int64_t ldp, cudaStream_t st) {
  using namespace sad;
  if (bn == 64) {
    dim3 grid((unsigned)((S + 63) / 64), (unsigned)gy, (unsigned)split);
    constexpr int sm = smem_bytes<64, KW>();
    if (split > 1) {
      if (image) k_sad<true, true, 64, KW><<<grid, kThreads, sm, st>>>(g2, nrows, S, kw / split, E, ldE, nullptr, 0);
      else k_sad<true, false, 64, KW><<<grid, kThreads, sm, st>>>(g2, nrows, S, kw / split, E, ldE, nullptr, 0);
    } else {
      if (image) k_sad<false, true, 64, KW><<<grid, kThreads, sm, st>>>(g2, nrows, S, kw, E, ldE, Ep, ldp);
      else k_sad<false, false, 64, KW><<<grid, kThreads, sm, st>>>(g2, nrows, S, kw, E, ldE, Ep, ldp);
    }
  } else {
    dim3 grid((unsigned)((S + 127) / 128), (unsigned)gy, (unsigned)split);
    constexpr int sm = smem_bytes<128, KW>();
    if (split > 1) {   // (split-K accumulates: the sigma copy follows E, launch_sad_sigma)
      if (image) k_sad<true, true, 128, KW><<<grid, kThreads, sm, st>>>(g2, nrows, S, kw / split, E, ldE, nullptr, 0);
      else k_sad<true, false, 128, KW><<<grid, kThreads, sm, st>>>(g2, nrows, S, kw / split, E, ldE, nullptr, 0);
    } else {
      if (image) k_sad<false, true, 128, KW><<<grid, kThreads, sm, st>>>(g2, nrows, S, kw, E, ldE, Ep, ldp);
      else k_sad<false, false, 128, KW><<<grid, kThreads, sm, st>>>(g2, nrows, S, kw, E, ldE, Ep, ldp);
    }
  }
}

static cudaError_t launch_sad_geom(const SadGeom& geo, bool image, int32_t nrows, int32_t S, int32_t P,
                                   int32_t* E, int64_t ldE, cudaStream_t st, int32_t* Ep = nullptr,
                                   int64_t ldp = 0) {
  using namespace sad;
  if (nrows <= 0 || S <= 0) return cudaSuccess;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  static std::atomic<uint64_t> attr_done{0};   // one bit per device ordinal
  if (dev < 64 && !(attr_done.load() & (1ull << dev))) {
    cudaError_t e;
    if ((e = sad_set_attr_all<16>()) != cudaSuccess) return e;
    if ((e = sad_set_attr_all<32>()) != cudaSuccess) return e;
    attr_done.fetch_or(1ull << dev);
  }
  const int kw = image ? P / 4 : (int)(geo.ldt / 4);
  const int KWs = stage_words(kw);
  const int nkb = kw / KWs;
  const int64_t gy = (nrows + BM - 1) / BM;
  if (gy > 65535) return cudaErrorInvalidValue;
  const SadPlan plan = choose_plan(nrows, S, nkb, sms);
  const int split = plan.split;
  SadGeom g2 = geo;
  g2.vec_out = ((ldE & 3) == 0 && (reinterpret_cast<uintptr_t>(E) & 15) == 0 &&
                (!Ep || (reinterpret_cast<uintptr_t>(Ep) & 15) == 0))
                   ? (((S / 2) % 4 == 0) ? 2 : 1) : 0;
  if (split > 1) {
    // split-K accumulates with red.add: zero the [nrows][S] window of E first
    cudaError_t e = (ldE == S)
        ? cudaMemsetAsync(E, 0, sizeof(int32_t) * (size_t)nrows * S, st)
        : cudaMemset2DAsync(E, sizeof(int32_t) * ldE, 0, sizeof(int32_t) * S, nrows, st);
    if (e != cudaSuccess) return e;
  }
  if (KWs == 32) sad_launch_kw<32>(g2, image, plan.bn, split, nrows, S, kw, gy, E, ldE, Ep, ldp, st);
  else sad_launch_kw<16>(g2, image, plan.bn, split, nrows, S, kw, gy, E, ldE, Ep, ldp, st);
  note_launch();
  return cudaGetLastError();
}

cudaError_t launch_sad(const uint8_t* A, const uint8_t* B, int64_t ldt, int32_t nrows, int32_t S,
                       int32_t P, int32_t* E, int64_t ldE, cudaStream_t st, int32_t* Ep, int64_t ldp,
                       int32_t row0) {
  SadGeom geo = {};
  geo.A = A; geo.B = B; geo.ldt = ldt;
  geo.e_row0 = row0;
  return launch_sad_geom(geo, false, nrows, S, P, E, ldE, st, Ep, ldp);
}

bool sad_split_plan(int32_t nrows, int32_t S, int32_t P) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return choose_plan(nrows, S, (P / 4) / sad::stage_words(P / 4), sms).split > 1;
}

bool sad_image_ok(const uint8_t* I, const uint8_t* T, int32_t N, int32_t M, int32_t C) {
  const int64_t MC = (int64_t)M * C, P = MC * M;
  return MC % 16 == 0 && P % 64 == 0 && ((int64_t)N * C) % 16 == 0 &&
         (reinterpret_cast<uintptr_t>(I) % 16) == 0 && (reinterpret_cast<uintptr_t>(T) % 16) == 0;
}

cudaError_t launch_sad_image(const uint8_t* I, const uint8_t* T, int32_t N, int32_t M, int32_t C,
                             int32_t row_begin, int32_t row_end, int32_t* E, int64_t ldE, cudaStream_t st,
                             int32_t* Ep, int64_t ldp) {
  SadGeom geo = {};
  geo.A = I; geo.B = T;
  geo.e_row0 = row_begin;
  geo.rowbytes = (int64_t)N * C;
  geo.a_tile0 = row_begin;
  geo.g = N / M; geo.M = M; geo.MC = M * C; geo.R = M * C / 16;
  const int32_t S = geo.g * geo.g;
  return launch_sad_geom(geo, true, row_end - row_begin, S, M * M * C, E, ldE, st, Ep, ldp);
}

}  // namespace pm
