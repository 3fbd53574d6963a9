/*
 * apsp_oracle.c — TEST INFRASTRUCTURE ONLY. The plain, slow, obviously correct
 * CPU oracle for the all-pairs shortest paths (APSP) hot path of
 *   Xia, Agrawal, Jiang, Ramnath, "Scaling and Selecting GPU Methods for All
 *   Pairs Shortest Paths (APSP) Computations", IPDPS 2022.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library. It shares no code, header,
 * constant or helper with the CUDA path under paper_conf_ipps_xia0ar22_b200/.
 *
 * Arithmetic: the paper stores distances as C `int`. The oracle
 * computes integer distances in int64 (so no intermediate can overflow) and
 * real-valued distances in double (fp64), and marks "no path" with its own
 * sentinel: ORACLE_INF_I64 = INT64_MAX for integers, +infinity for doubles.
 * Relaxations that involve a missing edge are skipped (the paper's "infinity",
 * PAPER.md:60), so the sentinel never takes part in an addition.
 *
 * Functions and the passage each follows:
 *   oracle_init_*     PAPER.md:60  (§II-A) "initializes the matrix dist with the
 *                     input weights for the edges (which will be infinity when
 *                     there are no edges)"; diagonal = 0 (a vertex reaches
 *                     itself by the empty path, PAPER.md:56 definition of dist);
 *                     duplicate arcs keep the smallest weight (DESIGN.md
 *                     reading R3); a self-loop of weight w gives min(0, w) (R2).
 *   oracle_fw_*       PAPER.md:60  (§II-A) the plain Floyd–Warshall: an outer
 *                     loop over k; in iteration k every pair (i, j) is checked
 *                     for a shorter path via v_k. `k_iters` < n stops after the
 *                     first k_iters outer iterations, which leaves
 *                     dist[i][j] = shortest i->j path whose intermediate
 *                     vertices all lie in {0..k_iters-1} (the FW invariant).
 *                     Negative cycles (reading R6): if dist[k][k] < 0 when
 *                     iteration k starts, the input holds a negative cycle;
 *                     the function returns 1 and the matrix is unspecified.
 *   oracle_dijkstra_row_*  PAPER.md:66 (§II-B) Dijkstra's algorithm, one
 *                     source, binary heap; non-negative weights only. Used to
 *                     check sampled rows of the full-size results and as an
 *                     independent pin of oracle_fw_* on small graphs.
 *   oracle_bellman_ford_row_i64  PAPER.md:68 (§II-B) Bellman–Ford, one source,
 *                     any weights; returns 1 on a reachable negative cycle.
 *   oracle_certify_rows_i32  the shortest-path optimality conditions (Bellman
 *                     equations of the single-source problem)
 *                     as an O(m)-per-row exactness certificate for claimed
 *                     int32 rows with strictly positive weights; checks every
 *                     row of the full-size (n=262144) results.
 *
 * Parity pins (tests/test_oracle.py, -m "not gpu"): closed forms (grid =
 * Manhattan distance, directed ring, weighted path, complete graph, disjoint
 * union), brute-force simple-path enumeration for n <= 7, Dijkstra vs FW vs
 * Bellman–Ford cross-checks, potential reweighting, invariants.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define ORACLE_INF_I64 INT64_MAX

/* ---------------------------------------------------------------- init -- */

/* dist (n*n, row-major): dist[i][j] = weight of arc i->j, +inf if none,
 * dist[i][i] = min(0, self loops). Integer weights. */
void oracle_init_i64(int64_t n, const int64_t* row_ptr, const int32_t* col,
                     const int64_t* w, int64_t* dist) {
  for (int64_t i = 0; i < n; ++i)
    for (int64_t j = 0; j < n; ++j) dist[i * n + j] = (i == j) ? 0 : ORACLE_INF_I64;
  for (int64_t u = 0; u < n; ++u)
    for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
      int64_t v = col[e];
      if (w[e] < dist[u * n + v]) dist[u * n + v] = w[e];
    }
}

void oracle_init_f64(int64_t n, const int64_t* row_ptr, const int32_t* col,
                     const double* w, double* dist) {
  for (int64_t i = 0; i < n; ++i)
    for (int64_t j = 0; j < n; ++j) dist[i * n + j] = (i == j) ? 0.0 : INFINITY;
  for (int64_t u = 0; u < n; ++u)
    for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
      int64_t v = col[e];
      if (w[e] < dist[u * n + v]) dist[u * n + v] = w[e];
    }
}

/* ------------------------------------------------------ Floyd–Warshall -- */

/* Plain FW. Runs outer iterations k = k_begin .. k_end-1
 * (k_begin > 0 continues an earlier call on the same matrix).
 * Returns 1 if a negative cycle was detected (dist unspecified), else 0.
 * The i-loop of one outer iteration is split over OpenMP threads: row k and
 * column k do not change during iteration k when dist[k][k] == 0, so the rows
 * are independent within an iteration. */
int oracle_fw_i64(int64_t n, int64_t* dist, int64_t k_begin, int64_t k_end) {
  for (int64_t k = k_begin; k < k_end; ++k) {
    if (dist[k * n + k] < 0) return 1;
    const int64_t* rowk = dist + k * n;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
      int64_t dik = dist[i * n + k];
      if (dik == ORACLE_INF_I64) continue;
      int64_t* rowi = dist + i * n;
      for (int64_t j = 0; j < n; ++j) {
        int64_t dkj = rowk[j];
        if (dkj == ORACLE_INF_I64) continue;
        if (dik + dkj < rowi[j]) rowi[j] = dik + dkj;
      }
    }
  }
  return 0;
}

int oracle_fw_f64(int64_t n, double* dist, int64_t k_begin, int64_t k_end) {
  for (int64_t k = k_begin; k < k_end; ++k) {
    if (dist[k * n + k] < 0) return 1;
    const double* rowk = dist + k * n;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
      double dik = dist[i * n + k];
      if (isinf(dik)) continue;
      double* rowi = dist + i * n;
      for (int64_t j = 0; j < n; ++j) {
        double dkj = rowk[j];
        if (isinf(dkj)) continue;
        if (dik + dkj < rowi[j]) rowi[j] = dik + dkj;
      }
    }
  }
  return 0;
}

/* ------------------------------------------------------------ Dijkstra -- */

typedef struct { int64_t key; int64_t v; } hent_i;
typedef struct { double key; int64_t v; } hent_d;

static void heap_push_i(hent_i* h, int64_t* sz, int64_t key, int64_t v) {
  int64_t i = (*sz)++;
  h[i].key = key; h[i].v = v;
  while (i > 0) {
    int64_t p = (i - 1) / 2;
    if (h[p].key <= h[i].key) break;
    hent_i t = h[p]; h[p] = h[i]; h[i] = t; i = p;
  }
}
static hent_i heap_pop_i(hent_i* h, int64_t* sz) {
  hent_i top = h[0];
  h[0] = h[--(*sz)];
  int64_t i = 0;
  for (;;) {
    int64_t l = 2 * i + 1, r = l + 1, m = i;
    if (l < *sz && h[l].key < h[m].key) m = l;
    if (r < *sz && h[r].key < h[m].key) m = r;
    if (m == i) break;
    hent_i t = h[m]; h[m] = h[i]; h[i] = t; i = m;
  }
  return top;
}
static void heap_push_d(hent_d* h, int64_t* sz, double key, int64_t v) {
  int64_t i = (*sz)++;
  h[i].key = key; h[i].v = v;
  while (i > 0) {
    int64_t p = (i - 1) / 2;
    if (h[p].key <= h[i].key) break;
    hent_d t = h[p]; h[p] = h[i]; h[i] = t; i = p;
  }
}
static hent_d heap_pop_d(hent_d* h, int64_t* sz) {
  hent_d top = h[0];
  h[0] = h[--(*sz)];
  int64_t i = 0;
  for (;;) {
    int64_t l = 2 * i + 1, r = l + 1, m = i;
    if (l < *sz && h[l].key < h[m].key) m = l;
    if (r < *sz && h[r].key < h[m].key) m = r;
    if (m == i) break;
    hent_d t = h[m]; h[m] = h[i]; h[i] = t; i = m;
  }
  return top;
}

/* Single-source Dijkstra with lazy deletion; weights >= 0.
 * out[v] = shortest src->v distance, ORACLE_INF_I64 if unreachable.
 * Returns 0, or -1 on allocation failure / negative weight. */
int oracle_dijkstra_row_i64(int64_t n, const int64_t* row_ptr, const int32_t* col,
                            const int64_t* w, int64_t src, int64_t* out) {
  int64_t m = row_ptr[n];
  for (int64_t e = 0; e < m; ++e) if (w[e] < 0) return -1;
  hent_i* h = (hent_i*)malloc(sizeof(hent_i) * (size_t)(m + 1));
  char* done = (char*)calloc((size_t)n, 1);
  if (!h || !done) { free(h); free(done); return -1; }
  for (int64_t v = 0; v < n; ++v) out[v] = ORACLE_INF_I64;
  int64_t sz = 0;
  out[src] = 0;
  heap_push_i(h, &sz, 0, src);
  while (sz > 0) {
    hent_i t = heap_pop_i(h, &sz);
    if (done[t.v]) continue;
    done[t.v] = 1;
    for (int64_t e = row_ptr[t.v]; e < row_ptr[t.v + 1]; ++e) {
      int64_t v = col[e];
      int64_t nd = t.key + w[e];
      if (nd < out[v]) { out[v] = nd; heap_push_i(h, &sz, nd, v); }
    }
  }
  free(h); free(done);
  return 0;
}

int oracle_dijkstra_row_f64(int64_t n, const int64_t* row_ptr, const int32_t* col,
                            const double* w, int64_t src, double* out) {
  int64_t m = row_ptr[n];
  for (int64_t e = 0; e < m; ++e) if (w[e] < 0) return -1;
  hent_d* h = (hent_d*)malloc(sizeof(hent_d) * (size_t)(m + 1));
  char* done = (char*)calloc((size_t)n, 1);
  if (!h || !done) { free(h); free(done); return -1; }
  for (int64_t v = 0; v < n; ++v) out[v] = INFINITY;
  int64_t sz = 0;
  out[src] = 0.0;
  heap_push_d(h, &sz, 0.0, src);
  while (sz > 0) {
    hent_d t = heap_pop_d(h, &sz);
    if (done[t.v]) continue;
    done[t.v] = 1;
    for (int64_t e = row_ptr[t.v]; e < row_ptr[t.v + 1]; ++e) {
      int64_t v = col[e];
      double nd = t.key + w[e];
      if (nd < out[v]) { out[v] = nd; heap_push_d(h, &sz, nd, v); }
    }
  }
  free(h); free(done);
  return 0;
}

/* Many Dijkstra rows at once (one source per OpenMP iteration): out is
 * n_src x n. Used for sampled-row parity at full size. Returns 0 or -1. */
int oracle_dijkstra_rows_i64(int64_t n, const int64_t* row_ptr, const int32_t* col,
                             const int64_t* w, int64_t n_src, const int64_t* srcs,
                             int64_t* out) {
  int bad = 0;
#pragma omp parallel for schedule(dynamic, 1) reduction(| : bad)
  for (int64_t s = 0; s < n_src; ++s)
    if (oracle_dijkstra_row_i64(n, row_ptr, col, w, srcs[s], out + s * n) != 0) bad |= 1;
  return bad ? -1 : 0;
}

int oracle_dijkstra_rows_f64(int64_t n, const int64_t* row_ptr, const int32_t* col,
                             const double* w, int64_t n_src, const int64_t* srcs,
                             double* out) {
  int bad = 0;
#pragma omp parallel for schedule(dynamic, 1) reduction(| : bad)
  for (int64_t s = 0; s < n_src; ++s)
    if (oracle_dijkstra_row_f64(n, row_ptr, col, w, srcs[s], out + s * n) != 0) bad |= 1;
  return bad ? -1 : 0;
}

/* -------------------------------------------------------- Bellman–Ford -- */

/* Single-source Bellman–Ford: relax every arc, n-1 rounds; a
 * further improving relaxation means a negative cycle reachable from src
 * (returns 1). out[v] = ORACLE_INF_I64 when unreachable. */
int oracle_bellman_ford_row_i64(int64_t n, const int64_t* row_ptr, const int32_t* col,
                                const int64_t* w, int64_t src, int64_t* out) {
  for (int64_t v = 0; v < n; ++v) out[v] = ORACLE_INF_I64;
  out[src] = 0;
  for (int64_t round = 0; round < n; ++round) {
    int changed = 0;
    for (int64_t u = 0; u < n; ++u) {
      if (out[u] == ORACLE_INF_I64) continue;
      for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
        int64_t v = col[e];
        if (out[u] + w[e] < out[v]) { out[v] = out[u] + w[e]; changed = 1; }
      }
    }
    if (!changed) return 0;
    if (round == n - 1) return 1;
  }
  return 0;
}

/* --------------------------------------------- optimality certificate -- */

/* Shortest-path optimality certificate for claimed distance rows (SURVEY.md
 * §8(c) "full-scale exactness"; the Bellman equations of PAPER.md:66-68's
 * single-source problem). For a graph whose arc weights are all STRICTLY
 * positive, a row d = D[s][.] equals the true shortest distances from s iff
 *   (i)   d[s] = 0;
 *   (ii)  every arc (u,v,w) with d[u] finite has d[v] <= d[u] + w
 *         (an "unreachable" d[v] violates it);
 *   (iii) every v != s with d[v] finite has an arc (u,v,w) with d[u] finite
 *         and d[v] = d[u] + w.
 * Proof: (ii) along a shortest s->v path gives d[v] <= dist(s,v) (and finite
 * whenever v is reachable); following (iii) backwards from v gives a walk
 * into v of length d[v] whose d-values strictly decrease (w > 0), so it
 * cannot repeat a vertex and must end at the only vertex with no tight arc
 * required, s: d[v] >= dist(s,v). Cost O(m) per row, no triple loop, so it
 * checks every row of the n=262144 result.
 *
 * rows: cnt rows of an int32 matrix (row i is source s = r0 + i), ld elements
 * apart, `inf` the value that marks "no path". Integers are compared in int64.
 * Returns the number of rows that fail; -1 if some weight is <= 0. If fail_row
 * is non-NULL it receives the first failing source (or -1). */
int64_t oracle_certify_rows_i32(int64_t n, const int64_t* row_ptr, const int32_t* col,
                                const int64_t* w, int64_t r0, int64_t cnt,
                                const int32_t* rows, int64_t ld, int32_t inf,
                                int64_t* fail_row) {
  for (int64_t e = 0; e < row_ptr[n]; ++e)
    if (w[e] <= 0) return -1;
  int64_t bad = 0, first = -1;
#pragma omp parallel
  {
    unsigned char* tight = (unsigned char*)malloc((size_t)(n > 0 ? n : 1));
#pragma omp for schedule(dynamic, 16) reduction(+ : bad)
    for (int64_t i = 0; i < cnt; ++i) {
      const int32_t* d = rows + i * ld;
      const int64_t s = r0 + i;
      int ok = (d[s] == 0);
      memset(tight, 0, (size_t)n);
      for (int64_t u = 0; u < n && ok; ++u) {
        if (d[u] == inf) continue;
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
          const int64_t v = col[e];
          const int64_t via = (int64_t)d[u] + w[e];
          if (d[v] == inf || (int64_t)d[v] > via) { ok = 0; break; }   /* (ii) */
          if ((int64_t)d[v] == via) tight[v] = 1;
        }
      }
      for (int64_t v = 0; v < n && ok; ++v)
        if (v != s && d[v] != inf && !tight[v]) ok = 0;                /* (iii) */
      if (!ok) {
        bad += 1;
#pragma omp critical
        if (first < 0 || s < first) first = s;
      }
    }
    free(tight);
  }
  if (fail_row) *fail_row = first;
  return bad;
}

int oracle_omp_max_threads(void) {
#ifdef _OPENMP
  extern int omp_get_max_threads(void);
  return omp_get_max_threads();
#else
  return 1;
#endif
}
