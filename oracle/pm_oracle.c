/*
 * pm_oracle.c -- plain, slow, obviously-correct CPU oracle for the hot path of
 * Yang, Ito & Nakano, "Photomosaic Generation by Rearranging Subimages, with
 * GPU Acceleration" (IPDPS workshops 2017).  "P:<n>" = line n of the paper
 * text (/root/reference/PAPER.md, not present at run time).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code, header, table or helper with the CUDA path
 * (paper_conf_ipps_yangin17_b200/csrc) and must never be called by it.
 *
 * Everything here is integer arithmetic; there is no floating point.  Loops
 * follow the paper's definitions in the paper's order, with no blocking,
 * fusion or reordering.  Indices are 0-based (the paper's I_1 is slot 0;
 * DESIGN.md reading R4).  OpenMP (if compiled with -fopenmp) only splits
 * independent iterations (rows of E; pairs inside one colour class, which
 * are disjoint by Theorem 1) -- it never changes a result.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#ifdef _OPENMP
#include <omp.h>
#endif

/* ------------------------------------------------------------------------ */
/* Step 1: divide an N x N image into S = (N/M)^2 tiles of M x M.
 * Tile u is grid cell (ty, tx) = (u / g, u % g), g = N / M (raster order,
 * reading R4).  Pixels are HWC u8 (C channels, reading R2).  Tile bytes are
 * written in (y, x, c) order; E does not depend on this order (Eq. 1 is a
 * sum).                                                                      */
void or_tiles(const uint8_t* img, int32_t N, int32_t M, int32_t C, uint8_t* tiles) {
  int32_t g = N / M;
  int64_t S = (int64_t)g * g;
  int64_t P = (int64_t)M * M * C;
  for (int64_t u = 0; u < S; ++u) {
    int64_t ty = u / g, tx = u % g;
    for (int64_t y = 0; y < M; ++y)
      for (int64_t x = 0; x < M; ++x)
        for (int64_t c = 0; c < C; ++c)
          tiles[u * P + (y * M + x) * C + c] =
              img[((ty * M + y) * (int64_t)N + tx * M + x) * C + c];
  }
}

/* ------------------------------------------------------------------------ */
/* Eq. (1): E(I_u, T_v) = sum_{1<=i,j<=M} |e_{i,j}|, e = I_u - T_v at
 * each pixel (reading R1: signed difference of 8-bit values, so E is the L1
 * distance; colour: summed over channels, reading R2).  Computed
 * straight from the two images, one pixel at a time.                         */
int32_t or_error_entry(const uint8_t* I, const uint8_t* T, int32_t N, int32_t M, int32_t C,
                       int64_t u, int64_t v) {
  int64_t g = N / M;
  int64_t uy = u / g, ux = u % g, vy = v / g, vx = v % g;
  int32_t s = 0;
  for (int64_t i = 0; i < M; ++i)
    for (int64_t j = 0; j < M; ++j)
      for (int64_t c = 0; c < C; ++c) {
        int32_t a = I[((uy * M + i) * (int64_t)N + ux * M + j) * C + c];
        int32_t b = T[((vy * M + i) * (int64_t)N + vx * M + j) * C + c];
        int32_t e = a - b;
        s += e < 0 ? -e : e;
      }
  return s;
}

/* Step 2: E(I_u, T_v) for input tiles u in [row_begin, row_end) and
 * all target tiles v; E[(u - row_begin) * S + v] (w_{u,v} orientation). */
void or_error_matrix(const uint8_t* I, const uint8_t* T, int32_t N, int32_t M, int32_t C,
                     int64_t row_begin, int64_t row_end, int32_t* E) {
  int64_t g = N / M, S = g * g;
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t u = row_begin; u < row_end; ++u)
    for (int64_t v = 0; v < S; ++v)
      E[(u - row_begin) * S + v] = or_error_entry(I, T, N, M, C, u, v);
}

/* ------------------------------------------------------------------------ */
/* Theorem 1: K_n is n-edge-colourable for odd n, (n-1)-edge-
 * colourable for even n.  Number of non-empty edge groups P_i.             */
int32_t or_num_colors(int32_t S) {
  if (S < 2) return 0;
  return (S % 2 == 0) ? S - 1 : S;
}

/* Edge groups P_1..P_m, 0-indexed slots.  Reading R8 (the round-
 * robin 1-factorisation that reproduces the printed K_16 groups exactly):
 * with m = S-1 (S even) or m = S (S odd) and 1-indexed vertices,
 *   P_i = {(u, v) : 1 <= u < v <= m, u + v == 2i + 1 (mod m)}
 *         + {(w, S)} for the w in 1..m with 2w == 2i + 1 (mod m)  (S even only).
 * Pairs of a group are listed by increasing smaller index, as printed.
 * Output: pairs[(i - class_begin) * (S/2) + k][0..1] = (u, v), u < v,
 * 0-indexed; for odd S the last pair slot of each class is (-1, -1).       */
int32_t or_edge_coloring(int32_t S, int32_t class_begin, int32_t class_end, int32_t* pairs) {
  int32_t ncls = or_num_colors(S);
  if (S < 2 || class_begin < 0 || class_end > ncls || class_begin > class_end) return 1;
  int32_t m = (S % 2 == 0) ? S - 1 : S;
  int32_t per = S / 2;
  for (int32_t cls = class_begin; cls < class_end; ++cls) {
    int32_t i = cls + 1;                 /* paper's group index, 1-based */
    int32_t target = (2 * i + 1) % m;
    int32_t k = 0;
    int32_t* out = pairs + (int64_t)(cls - class_begin) * per * 2;
    /* For each u in 1..m the congruence u + v == 2i+1 (mod m) has exactly one
     * solution v in 1..m; if that v is u itself, u is the group's fixed point
     * and (S even) is joined to vertex S.  Emit each pair once, at its
     * smaller index, so pairs come out by increasing smaller index.        */
    for (int32_t u = 1; u <= m; ++u) {
      int32_t v = ((target - u) % m + m) % m;
      if (v == 0) v = m;
      if (v == u) {
        if (S % 2 == 0) v = S; else continue;   /* odd S: fixed point idles */
      }
      if (u < v) {
        out[2 * k + 0] = u - 1;
        out[2 * k + 1] = v - 1;
        ++k;
      }
    }
    for (; k < per; ++k) { out[2 * k] = -1; out[2 * k + 1] = -1; }
  }
  return 0;
}

/* ------------------------------------------------------------------------ */
/* Eq. (2): Error(R, T) = sum_u E(r(I_u), T_u), with r[u] = the input
 * tile placed at target slot u (reading R5).  int64 (reading R11).          */
int64_t or_cost(const int32_t* E, int64_t ldE, int32_t S, const int32_t* r) {
  int64_t s = 0;
  for (int64_t u = 0; u < S; ++u) s += E[(int64_t)r[u] * ldE + u];
  return s;
}

/* ------------------------------------------------------------------------ */
/* Algorithm 2, parallel approximation, replayed serially.
 * Reading R5: I_u is the tile currently at slot u, i.e. r[u]; so
 *   E(I_u,T_u) = E[r[u]][u],  E(I_v,T_u) = E[r[v]][u].
 * Line 5 is used literally (four E entries, strict '>', reading R6).
 * Start: identity unless the caller passes another r (reading R7 / resume).
 * Groups in order i = 1..S (P_S empty for even S), reading R8.  Pairs inside
 * a group are disjoint, so their order is irrelevant; OpenMP may split them.
 * A round = one pass of lines 3-10; rounds counts the final zero-swap round
 * (reading R10).  max_rounds = 0: no cap.  Returns 0 if converged, 3 if the
 * cap stopped it first.  swaps_per_round may be NULL (else >= max_rounds or
 * enough entries for the run).                                              */
int32_t or_local_search(const int32_t* E, int64_t ldE, int32_t S, int32_t* r, int32_t max_rounds,
                        int32_t* rounds_out, int64_t* swaps_out, int64_t* swaps_per_round,
                        int32_t swaps_per_round_len) {
  int32_t ncls = or_num_colors(S);
  int32_t per = S / 2;
  int32_t* groups = NULL;
  if (ncls > 0) {
    groups = (int32_t*)malloc(sizeof(int32_t) * 2 * (size_t)per * (size_t)ncls);
    if (!groups) return 2;
    or_edge_coloring(S, 0, ncls, groups);
  }
  int32_t rounds = 0;
  int64_t total = 0;
  int32_t status = 0;
  int flag;
  do {                                                     /* line 1: repeat   */
    if (max_rounds > 0 && rounds >= max_rounds) { status = 3; break; }
    flag = 0;                                              /* line 2           */
    int64_t sw = 0;
    for (int32_t cls = 0; cls < ncls; ++cls) {             /* line 3: i = 1..S */
      const int32_t* g = groups + (int64_t)cls * per * 2;
#pragma omp parallel for reduction(+ : sw) schedule(static)
      for (int32_t k = 0; k < per; ++k) {                  /* line 4           */
        int32_t u = g[2 * k], v = g[2 * k + 1];
        if (u < 0) continue;
        int64_t Iu = r[u], Iv = r[v];
        int64_t lhs = (int64_t)E[Iu * ldE + u] + E[Iv * ldE + v];   /* E(I_u,T_u)+E(I_v,T_v) */
        int64_t rhs = (int64_t)E[Iv * ldE + u] + E[Iu * ldE + v];   /* E(I_v,T_u)+E(I_u,T_v) */
        if (lhs > rhs) {                                   /* line 5           */
          r[u] = (int32_t)Iv;                              /* line 6: swap     */
          r[v] = (int32_t)Iu;
          sw += 1;                                         /* line 7: flag     */
        }
      }
    }
    if (sw > 0) flag = 1;
    if (swaps_per_round && rounds < swaps_per_round_len) swaps_per_round[rounds] = sw;
    total += sw;
    rounds += 1;
  } while (flag != 0);                                     /* line 11          */
  free(groups);
  if (rounds_out) *rounds_out = rounds;
  if (swaps_out) *swaps_out = total;
  return status;
}

/* Algorithm 1, serial approximation: all u < v in lexicographic
 * order, swap on strict '>' (same slot-indexed reading).  NEXT-4 in SURVEY;
 * kept here because it is short and gives Table I's "approx CPU" column. */
int32_t or_serial_local_search(const int32_t* E, int64_t ldE, int32_t S, int32_t* r,
                               int32_t max_rounds, int32_t* rounds_out, int64_t* swaps_out) {
  int32_t rounds = 0;
  int64_t total = 0;
  int flag;
  int32_t status = 0;
  do {
    if (max_rounds > 0 && rounds >= max_rounds) { status = 3; break; }
    flag = 0;
    for (int32_t u = 0; u < S; ++u)
      for (int32_t v = u + 1; v < S; ++v) {
        int64_t Iu = r[u], Iv = r[v];
        if ((int64_t)E[Iu * ldE + u] + E[Iv * ldE + v] > (int64_t)E[Iv * ldE + u] + E[Iu * ldE + v]) {
          r[u] = (int32_t)Iv;
          r[v] = (int32_t)Iu;
          flag = 1;
          total += 1;
        }
      }
    rounds += 1;
  } while (flag != 0);
  if (rounds_out) *rounds_out = rounds;
  if (swaps_out) *swaps_out = total;
  return status;
}

/* ------------------------------------------------------------------------ */
/* Section III: the optimum is a minimum-weight perfect matching of
 * the complete bipartite graph with w_{u,v} = E(I_u, T_v).  Kuhn-Munkres
 * (Hungarian method, refs [11],[12]) in its O(S^3) shortest-
 * augmenting-path form with row/column potentials, int64 arithmetic.
 * Rows = input tiles u, columns = target slots v.
 * Outputs: r[v] = input tile matched to slot v (same meaning as Eq. 2's r),
 * *cost, and the dual (p[u], q[v]) with p[u] + q[v] <= E[u][v] for all
 * (u, v), equality on the matching, sum p + sum q = cost (LP duality: a
 * certificate of optimality that can be checked without trusting this code). */
int32_t or_hungarian(const int32_t* E, int64_t ldE, int32_t S, int32_t* r, int64_t* cost,
                     int64_t* p_out, int64_t* q_out) {
  int64_t n = S;
  const int64_t INF = (int64_t)1 << 62;
  int64_t* pu = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));   /* row potentials    */
  int64_t* pv = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));   /* column potentials */
  int64_t* match = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t)); /* column -> row, 1-based */
  int64_t* way = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
  int64_t* minv = (int64_t*)malloc(sizeof(int64_t) * ((size_t)n + 1));
  char* used = (char*)malloc((size_t)n + 1);
  if (!pu || !pv || !match || !way || !minv || !used) return 2;
  for (int64_t i = 1; i <= n; ++i) {
    match[0] = i;
    int64_t j0 = 0;
    for (int64_t j = 0; j <= n; ++j) { minv[j] = INF; used[j] = 0; }
    do {
      used[j0] = 1;
      int64_t i0 = match[j0], delta = INF, j1 = 0;
      for (int64_t j = 1; j <= n; ++j) {
        if (used[j]) continue;
        int64_t cur = (int64_t)E[(i0 - 1) * ldE + (j - 1)] - pu[i0] - pv[j];
        if (cur < minv[j]) { minv[j] = cur; way[j] = j0; }
        if (minv[j] < delta) { delta = minv[j]; j1 = j; }
      }
      for (int64_t j = 0; j <= n; ++j) {
        if (used[j]) { pu[match[j]] += delta; pv[j] -= delta; }
        else minv[j] -= delta;
      }
      j0 = j1;
    } while (match[j0] != 0);
    do {
      int64_t j1 = way[j0];
      match[j0] = match[j1];
      j0 = j1;
    } while (j0);
  }
  int64_t c = 0;
  for (int64_t j = 1; j <= n; ++j) {
    r[j - 1] = (int32_t)(match[j] - 1);
    c += E[(match[j] - 1) * ldE + (j - 1)];
  }
  *cost = c;
  /* Dual of  min sum w x  s.t. rows/cols sum to 1:  max sum p + sum q,
   * p_u + q_v <= w_{u,v}.  Here p = pu, q = pv.                         */
  if (p_out) for (int64_t i = 0; i < n; ++i) p_out[i] = pu[i + 1];
  if (q_out) for (int64_t j = 0; j < n; ++j) q_out[j] = pv[j + 1];
  free(pu); free(pv); free(match); free(way); free(minv); free(used);
  return 0;
}

/* ------------------------------------------------------------------------ */
/* The resulting photomosaic R ("writes the resulting photomosaic
 * image"): target slot u of R shows input tile r[u], pixel by pixel, in the
 * same raster tile geometry as Step 1 (reading R4).                         */
void or_render(const uint8_t* I, int32_t N, int32_t M, int32_t C, const int32_t* r, uint8_t* R) {
  int64_t g = N / M, S = g * g;
  for (int64_t u = 0; u < S; ++u) {
    int64_t t = r[u];
    int64_t uy = u / g, ux = u % g, ty = t / g, tx = t % g;
    for (int64_t y = 0; y < M; ++y)
      for (int64_t x = 0; x < M; ++x)
        for (int64_t c = 0; c < C; ++c)
          R[((uy * M + y) * (int64_t)N + ux * M + x) * C + c] =
              I[((ty * M + y) * (int64_t)N + tx * M + x) * C + c];
  }
}

int32_t or_num_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

void or_set_num_threads(int32_t t) {
#ifdef _OPENMP
  if (t > 0) omp_set_num_threads(t);
#else
  (void)t;
#endif
}

/* ------------------------------------------------------------------------ */
/* Histogram matching of the input image to the target (Sec. II: "the
 * distribution of an input image is changed to that of a target image using
 * the histogram equalization [10]").  Reading R12: histogram
 * specification in its exact integer form, per channel c, L = 256 levels:
 *   h_I[k], h_T[k]  = pixel counts of level k in channel c of I and T;
 *   C_I[k], C_T[k]  = cumulative counts sum_{j <= k} h[j];
 *   map[k]          = the smallest level z with C_T[z] >= C_I[k]
 *                     (z = G^{-1}(T(k)) of [10] with the cumulative
 *                     distributions compared as counts: both images have
 *                     N*N pixels, so no division and no rounding);
 *   out(y, x, c)    = map[I(y, x, c)].
 * I, T, out: u8 [N][N][C] HWC; out may alias I.                            */
void or_histogram_match(const uint8_t* I, const uint8_t* T, int32_t N, int32_t C, uint8_t* out) {
  int64_t n = (int64_t)N * N;
  for (int32_t c = 0; c < C; ++c) {
    int64_t hI[256], hT[256], cI[256], cT[256];
    uint8_t map[256];
    for (int k = 0; k < 256; ++k) { hI[k] = 0; hT[k] = 0; }
    for (int64_t p = 0; p < n; ++p) {
      hI[I[p * C + c]] += 1;
      hT[T[p * C + c]] += 1;
    }
    int64_t sI = 0, sT = 0;
    for (int k = 0; k < 256; ++k) {
      sI += hI[k]; cI[k] = sI;
      sT += hT[k]; cT[k] = sT;
    }
    for (int k = 0; k < 256; ++k) {
      int z = 0;
      while (z < 255 && cT[z] < cI[k]) ++z;
      map[k] = (uint8_t)z;
    }
    for (int64_t p = 0; p < n; ++p) out[p * C + c] = map[I[p * C + c]];
  }
}
