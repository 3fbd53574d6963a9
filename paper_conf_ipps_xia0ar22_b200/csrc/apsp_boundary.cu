// apsp_boundary.cu — the boundary algorithm (Djidjev et al.; PAPER.md:139-150,
// eq. (1); out-of-core form Algorithm 3) on one B200, built
// from the same sm_100a kernels as the blocked Floyd–Warshall path.
//
//   step 1  partition (given by the caller: comp[v] in [0, k)); a vertex with an
//           arc to another component is a boundary node
//   step 2  dist2 = APSP inside every component: blocked FW on the diagonal
//           blocks A(i,i) (Alg. 3 l.1-3); all components advance one round per
//           launch (batched phase 1, phase 2 and phase 3). The diagonal blocks
//           live in a strip of n_pad rows x s_max columns (component i's rows
//           hold its block in columns [0, s_pad[i])): "S_dia" of P:186
//   step 3  boundary graph: inter-component arcs + virtual edges dist2(u,v)
//           between boundary nodes of one component (Alg. 3 l.4);
//           dist3 = blocked FW on `bound` (Alg. 3 l.5): "S_bound" of P:186
//   step 4  dist4, one block row A(i, :) at a time (Alg. 3 l.12-17): with
//           C2B[i] = A(i,i)(C_i, B_i) and B2C[j] = A(j,j)(B_j, C_j) (l.6-11),
//           tmp_i = C2B[i] (x) bound(B_i, :), then A(i,j) = tmp_i(:, B_j) (x) B2C[j]
//           for j != i and A(i,i) = min(dist2(i,i), tmp_i(:, B_i) (x) B2C[i]).
//           Block rows are batched into groups; every group is one batched
//           launch of each product.
//
// Placement of the n_pad x n_pad result (l.20 "Transfer A(i,j) back to CPU"):
//   in core      the whole result stays in HBM (one group, no transfer);
//   out of core  (the result does not fit the device budget, or forced) the
//                paper's scheme: S_rem = L - S_dia - S_bound is split
//                into two buffers on two streams; each buffer accumulates the
//                block rows of N_row = S_rem / (N_max n W) component iterations
//                (here: as many whole block rows as fit half of the share of
//                S_rem given to the buffers) and is then copied to pinned host
//                memory while the other stream computes the next group into
//                the other buffer. Reading R21: device memory left beyond the
//                two buffers keeps the LAST block rows resident in HBM (no
//                transfer, computed on a third stream); with a small budget
//                nothing is resident and every block row streams, as in the paper.
// Exactness: a path from C_i to C_j (j != i) leaves C_i at its first boundary
// node and enters C_j at its last one; its middle part is a path of the
// boundary graph whose intra-component detours are virtual edges. Paths inside
// one component either avoid boundary nodes (dist2) or are covered the same way.
//
// Layout (Fig. 1a): vertices are relabelled so that every component is
// a contiguous block with its boundary nodes first; blocks are padded to 128
// (the tile) and boundary sets to 32 (the depth chunk) with further vertices of
// the component treated as boundary (any superset of the boundary keeps eq. (1)
// exact) or isolated dummies. The result is kept in this order; apsp_get_dist
// gathers rows and columns back into the caller's order.
#include "apsp_internal.h"
#include "apsp_sched.cuh"

#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

namespace apsp {

namespace {

struct Launch {
  int first = 0, count = 0;  // descriptors [first, first+count)
  int pfirst = 0;            // prefix array segment (count + 1 entries)
  long long tiles = 0;
  int cls = 2;
  double relax = 0;
};

// A run of consecutive components [c0, c1) whose block rows are produced together.
struct Group {
  int c0 = 0, c1 = 0;
  int slot = -1;                 // streamed: output buffer / stream 0 or 1; resident: -1
  long long row0 = 0, rows = 0;  // new-order rows [row0, row0 + rows)
  Launch prod1, prod2, prodd;
  std::vector<int> no_bnd;       // components of this group without boundary nodes (fix-ups)
};

struct Bnd {
  int k = 0;
  long long n_pad = 0, NB_pad = 0, s_max = 0, nb_real = 0;
  std::vector<long long> off, s_pad, nb_pad, boff;
  std::vector<int> new_id;    // original vertex -> new index
  void* strip = nullptr;      // n_pad x s_max: dist2 diagonal blocks (S_dia)
  void* bound = nullptr;      // NB_pad x NB_pad (S_bound)
  void* D_res = nullptr;      // rows [res_row0, n_pad) x n_pad resident in HBM
  long long res_row0 = 0;     // rows [0, res_row0) stream to the pinned host matrix
  void* host = nullptr;       // pinned res_row0 x n_pad
  void* buf[2] = {nullptr, nullptr};     // out-of-core output buffers (buf_rows x n_pad each)
  void* tmpb[3] = {nullptr, nullptr, nullptr};  // tmp rows per slot (0, 1, resident = 2)
  long long buf_rows = 0, tmp_rows = 0;
  cudaStream_t xs[2] = {nullptr, nullptr};
  cudaEvent_t ev_ready = nullptr, ev_done[2] = {nullptr, nullptr};
  bool ooc = false, need_fill = false;
  std::vector<Group> groups;
  void* inf_row = nullptr;    // max(NB_pad, s_max) elements of infinity
  std::vector<void*> dev;     // every other device allocation (freed together)
  int* d_new_id = nullptr;
  long long* d_irp = nullptr;  // intra-component CSR over the n_pad new rows (block-local columns)
  int* d_icol = nullptr;
  void* d_iw = nullptr;
  long long* d_brp = nullptr;  // boundary-graph CSR over NB_pad rows (bound columns)
  int* d_bcol = nullptr;
  void* d_bw = nullptr;
  int* d_rowcomp_b = nullptr;  // bound row -> component (-1: padding)
  long long *d_off = nullptr, *d_boff = nullptr, *d_nbpad = nullptr;
  void* d_desc = nullptr;
  long long* d_pref = nullptr;
  std::vector<Launch> p2, p3;  // dist2 rounds
  std::vector<void*> p1_tiles;  // per dist2 round: device array of pivot-tile pointers
  std::vector<int> p1_count;
  int* d_rowmap = nullptr;      // get_dist staging
  void* d_stage = nullptr;
  void* d_src = nullptr;        // out of core: rows gathered from host / HBM before the column gather
  int* d_ident = nullptr;
  long long stage_rows = 0;
};

Bnd* B_(Handle* h) { return static_cast<Bnd*>(h->bnd); }

template <typename T> T inf_value();
template <> int inf_value<int>() { return APSP_INF_I32; }
template <> float inf_value<float>() { return INFINITY; }

// bound(B_c, B_c) = min(arcs, dist2 restricted to the boundary nodes): the virtual edges
template <typename T>
__global__ void bound_merge_kernel(T* bound, long long ldb, const T* strip, long long lds, const int* rowcomp_b,
                                   const long long* off, const long long* boff, const long long* nbp) {
  const long long r = blockIdx.x;
  const int c = rowcomp_b[r];
  if (c < 0) return;
  const T* src = strip + (off[c] + (r - boff[c])) * lds;
  T* dst = bound + r * ldb + boff[c];
  for (long long x = threadIdx.x; x < nbp[c]; x += blockDim.x) dst[x] = src[x] < dst[x] ? src[x] : dst[x];
}

template <typename T>
struct Builder {
  std::vector<MinPlusDesc<T>> descs;
  std::vector<long long> pref;
  long long cur = 0;
  Launch begin(int cls) {
    Launch L;
    L.first = (int)descs.size();
    L.pfirst = (int)pref.size();
    L.cls = cls;
    pref.push_back(0);
    cur = 0;
    return L;
  }
  void add(Launch& L, const MinPlusDesc<T>& d) {
    const long long t = (long long)d.tiles_i * d.tiles_j;
    if (t <= 0 || d.K <= 0) return;
    descs.push_back(d);
    cur += t;
    pref.push_back(cur);
    L.relax += (double)t * kTile * kTile * d.K;
  }
  void end(Launch& L) {
    L.count = (int)descs.size() - L.first;
    L.tiles = cur;
  }
};

template <typename T>
apsp_status dupload(Handle* h, std::vector<void*>& keep, T** dst, const T* src, size_t count) {
  apsp_status st;
  *dst = nullptr;
  if (count == 0) return APSP_OK;
  void* p = nullptr;
  if ((st = h->cuda(cudaMalloc(&p, count * sizeof(T)), "cudaMalloc boundary"))) return st;
  keep.push_back(p);
  h->device_bytes += count * sizeof(T);
  *dst = static_cast<T*>(p);
  return h->cuda(cudaMemcpy(p, src, count * sizeof(T), cudaMemcpyHostToDevice), "H2D boundary");
}

// Where block rows go: in core (one resident group) or the out-of-core split of
// P:184-197 (two streamed buffers, plus resident block rows from leftover memory, R21).
apsp_status plan_placement(Handle* h, const apsp_config& cfg, long long fixed) {
  Bnd* b = B_(h);
  const long long W = h->elem, n_pad = b->n_pad, NB = b->NB_pad;
  const long long incore = n_pad * n_pad * W + n_pad * NB * W;  // result + tmp for all block rows
  const long long avail = device_free_bytes(h->device, fixed + incore);
  if (avail < 0) return h->fail(APSP_ECUDA, "cudaMemGetInfo failed");
  const long long L = cfg.device_budget_bytes > 0 ? cfg.device_budget_bytes : avail - (1ll << 30);
  if (!cfg.force_out_of_core && fixed + incore <= L) {
    b->ooc = false;
    b->res_row0 = 0;
    b->tmp_rows = n_pad;
    Group g;
    g.c0 = 0;
    g.c1 = b->k;
    g.row0 = 0;
    g.rows = n_pad;
    b->groups.push_back(g);
    return APSP_OK;
  }
  // out of core: S_rem = L - S_dia - S_bound (- the other fixed buffers)
  b->ooc = true;
  const long long S_rem = L - fixed;
  const long long per_row = (n_pad + NB) * W;  // one output row of a buffer + its tmp row
  // each buffer: at most ~1 GiB of output rows and a quarter of S_rem (so at least half of it
  // can keep whole block rows resident, R21), at least one block row (N_max); when S_rem is
  // too small for that, the paper's split: the two buffers share S_rem
  const long long cap_rows = std::max<long long>(1, (1ll << 30) / (n_pad * W));
  long long buf_rows = std::min<long long>(cap_rows, S_rem / 4 / per_row);
  if (buf_rows < b->s_max) buf_rows = std::min<long long>(std::max(cap_rows, b->s_max), S_rem / 2 / per_row);
  // forced (force_out_of_core / ooc_stream_all): the paper's setting, every block row streams,
  // in at least ~4 groups so the two buffers alternate even on small graphs
  const bool stream_all = cfg.force_out_of_core || cfg.ooc_stream_all;
  if (stream_all) buf_rows = std::max(b->s_max, std::min(buf_rows, n_pad / 4));
  if (buf_rows < b->s_max)
    return h->fail(APSP_ENOMEM, "boundary out of core: S_rem = %lld B leaves %lld rows per buffer < N_max = %lld",
                   S_rem, buf_rows, b->s_max);
  // resident block rows from the end while memory allows (each also needs no tmp: the resident
  // groups share one tmp of buf_rows rows)
  long long left = S_rem - 2 * buf_rows * per_row - buf_rows * NB * W;
  int c_res = b->k;
  while (!stream_all && c_res > 0 && left >= b->s_pad[c_res - 1] * n_pad * W) {
    left -= b->s_pad[c_res - 1] * n_pad * W;
    --c_res;
  }
  if (left < 0) c_res = b->k;  // no room for the resident tmp: stream everything
  b->res_row0 = c_res < b->k ? b->off[c_res] : n_pad;
  b->buf_rows = buf_rows;
  b->tmp_rows = buf_rows;
  // streamed groups of whole block rows (N_row components each), alternating slots
  int slot = 0;
  for (int c = 0; c < c_res;) {
    Group g;
    g.c0 = c;
    g.row0 = b->off[c];
    while (c < c_res && b->off[c] + b->s_pad[c] - g.row0 <= buf_rows) ++c;
    g.c1 = c;
    g.rows = b->off[c - 1] + b->s_pad[c - 1] - g.row0;
    g.slot = slot;
    slot ^= 1;
    b->groups.push_back(g);
  }
  for (int c = c_res; c < b->k;) {  // resident groups (tmp of buf_rows rows)
    Group g;
    g.c0 = c;
    g.row0 = b->off[c];
    while (c < b->k && b->off[c] + b->s_pad[c] - g.row0 <= buf_rows) ++c;
    g.c1 = c;
    g.rows = b->off[c - 1] + b->s_pad[c - 1] - g.row0;
    b->groups.push_back(g);
  }
  return APSP_OK;
}

template <typename T>
apsp_status setup_t(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col, const T* w,
                    const int32_t* comp, int k) {
  Bnd* b = B_(h);
  apsp_status st;
  const long long n = h->n;
  b->k = k;
  // ---- step 1: boundary nodes, component-blocked order ------------------------
  std::vector<char> isb(n, 0);
  for (long long u = 0; u < n; ++u)
    for (long long e = row_ptr[u]; e < row_ptr[u + 1]; ++e)
      if (comp[col[e]] != comp[u]) isb[u] = isb[col[e]] = 1;
  std::vector<std::vector<int>> members(k);
  for (long long v = 0; v < n; ++v)
    if (isb[v]) members[comp[v]].push_back((int)v);
  std::vector<long long> nbr(k);
  for (int c = 0; c < k; ++c) nbr[c] = (long long)members[c].size();
  for (long long v = 0; v < n; ++v)
    if (!isb[v]) members[comp[v]].push_back((int)v);
  b->off.resize(k);
  b->s_pad.resize(k);
  b->nb_pad.resize(k);
  b->boff.resize(k);
  long long o = 0, bo = 0;
  for (int c = 0; c < k; ++c) {
    const long long s = (long long)members[c].size();
    b->nb_pad[c] = (nbr[c] + 31) / 32 * 32;
    b->s_pad[c] = std::max<long long>(kTile, (std::max(s, b->nb_pad[c]) + kTile - 1) / kTile * kTile);
    b->off[c] = o;
    b->boff[c] = bo;
    o += b->s_pad[c];
    bo += b->nb_pad[c];
    b->s_max = std::max(b->s_max, b->s_pad[c]);
    b->nb_real += nbr[c];
    if (b->nb_pad[c] == 0) b->need_fill = true;
  }
  b->n_pad = o;
  b->NB_pad = std::max<long long>(kTile, (bo + kTile - 1) / kTile * kTile);
  h->n_pad = b->n_pad;
  h->ld = b->n_pad;
  b->new_id.assign(n, -1);
  std::vector<int> old_of(b->n_pad, -1), rowcomp_b(b->NB_pad, -1);
  for (int c = 0; c < k; ++c) {
    for (size_t p = 0; p < members[c].size(); ++p) {
      b->new_id[members[c][p]] = (int)(b->off[c] + (long long)p);
      old_of[b->off[c] + p] = members[c][p];
    }
    for (long long r = 0; r < b->nb_pad[c]; ++r) rowcomp_b[b->boff[c] + r] = c;
  }
  // ---- CSRs in the new order (host bookkeeping, no distance arithmetic) -------
  std::vector<long long> irp(b->n_pad + 1, 0), brp(b->NB_pad + 1, 0);
  std::vector<int> icol, bcol;
  std::vector<T> iw, bw;
  for (long long r = 0; r < b->n_pad; ++r) {
    const int u = old_of[r];
    if (u >= 0)
      for (long long e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
        const int v = col[e];
        if (comp[v] == comp[u]) {
          icol.push_back((int)(b->new_id[v] - b->off[comp[u]]));
          iw.push_back(w[e]);
        }
      }
    irp[r + 1] = (long long)icol.size();
  }
  for (long long rb = 0; rb < b->NB_pad; ++rb) {
    const int c = rowcomp_b[rb];
    const int u = c >= 0 ? old_of[b->off[c] + (rb - b->boff[c])] : -1;
    if (u >= 0)
      for (long long e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
        const int v = col[e];
        const int cv = comp[v];
        if (cv != c) {  // both ends are boundary nodes (slot < boundary count of their component)
          bcol.push_back((int)(b->boff[cv] + (b->new_id[v] - b->off[cv])));
          bw.push_back(w[e]);
        }
      }
    brp[rb + 1] = (long long)bcol.size();
  }
  // ---- placement ---------------------------------------------------------------
  const size_t es = h->elem;
  const long long NB = b->NB_pad, ldg = b->s_max;
  const long long inf_len = std::max(NB, b->s_max);
  const long long fixed = b->n_pad * ldg * es + NB * NB * es + inf_len * es +
                          (long long)(irp.size() + brp.size()) * 8 + (long long)(icol.size() + bcol.size()) * 8 +
                          (8ll << 20);  // descriptors, staging
  if ((st = plan_placement(h, cfg, fixed))) return st;
  // ---- device state --------------------------------------------------------------
  auto dmalloc = [&](void** p, size_t bytes, const char* what) -> apsp_status {
    apsp_status s2 = h->cuda(cudaMallocAsync(p, bytes, h->stream), what);
    if (!s2) h->device_bytes += bytes;
    return s2;
  };
  if ((st = dmalloc(&b->strip, (size_t)b->n_pad * ldg * es, "cudaMalloc dist2 strip"))) return st;
  if ((st = dmalloc(&b->bound, (size_t)NB * NB * es, "cudaMalloc bound"))) return st;
  if (b->res_row0 < b->n_pad &&
      (st = dmalloc(&b->D_res, (size_t)(b->n_pad - b->res_row0) * b->n_pad * es, "cudaMalloc dist")))
    return st;
  const bool any_res = b->res_row0 < b->n_pad;
  if (any_res && (st = dmalloc(&b->tmpb[2], (size_t)b->tmp_rows * NB * es, "cudaMalloc tmp")))
    return st;
  if (b->ooc) {
    for (int s = 0; s < 2; ++s) {
      if ((st = dmalloc(&b->buf[s], (size_t)b->buf_rows * b->n_pad * es, "cudaMalloc boundary buffer"))) return st;
      if ((st = dmalloc(&b->tmpb[s], (size_t)b->tmp_rows * NB * es, "cudaMalloc tmp"))) return st;
      if ((st = h->cuda(cudaStreamCreateWithFlags(&b->xs[s], cudaStreamNonBlocking), "stream"))) return st;
      if ((st = h->cuda(cudaEventCreateWithFlags(&b->ev_done[s], cudaEventDisableTiming), "event"))) return st;
    }
    if ((st = h->cuda(cudaEventCreateWithFlags(&b->ev_ready, cudaEventDisableTiming), "event"))) return st;
    if (b->res_row0 > 0) {
      const size_t hb = (size_t)b->res_row0 * b->n_pad * es;
      if ((st = h->cuda(cudaHostAlloc(&b->host, hb, cudaHostAllocDefault), "cudaHostAlloc boundary result")))
        return st;
      h->host_bytes += hb;
    }
  }
  if ((st = dmalloc(&b->inf_row, (size_t)inf_len * es, "cudaMalloc inf"))) return st;
  auto& K = b->dev;
  if ((st = dupload<int>(h, K, &b->d_new_id, b->new_id.data(), n))) return st;
  if ((st = dupload<long long>(h, K, &b->d_irp, irp.data(), irp.size()))) return st;
  if ((st = dupload<int>(h, K, &b->d_icol, icol.data(), icol.size()))) return st;
  {
    T* p = nullptr;
    if ((st = dupload<T>(h, K, &p, iw.data(), iw.size()))) return st;
    b->d_iw = p;
  }
  if ((st = dupload<long long>(h, K, &b->d_brp, brp.data(), brp.size()))) return st;
  if ((st = dupload<int>(h, K, &b->d_bcol, bcol.data(), bcol.size()))) return st;
  {
    T* p = nullptr;
    if ((st = dupload<T>(h, K, &p, bw.data(), bw.size()))) return st;
    b->d_bw = p;
  }
  if ((st = dupload<int>(h, K, &b->d_rowcomp_b, rowcomp_b.data(), rowcomp_b.size()))) return st;
  if ((st = dupload<long long>(h, K, &b->d_off, b->off.data(), k))) return st;
  if ((st = dupload<long long>(h, K, &b->d_boff, b->boff.data(), k))) return st;
  if ((st = dupload<long long>(h, K, &b->d_nbpad, b->nb_pad.data(), k))) return st;
  if ((st = h->cuda(cudaStreamSynchronize(h->stream), "boundary alloc sync"))) return st;

  // ---- batched min-plus descriptors -------------------------------------------------
  T* S = static_cast<T*>(b->strip);
  T* bound = static_cast<T*>(b->bound);
  const T* infr = static_cast<const T*>(b->inf_row);
  const long long ld = b->n_pad;
  Builder<T> bl;
  // step 2 (dist2): round r of every component's blocked FW, on the strip (ld = s_max)
  const long long R = b->s_max / kTile;
  for (long long r = 0; r < R; ++r) {
    std::vector<T*> piv;
    Launch L2 = bl.begin(1);
    for (int c = 0; c < k; ++c) {
      const long long nbc = b->s_pad[c] / kTile;
      if (r >= nbc) continue;
      T* base = S + b->off[c] * ldg;
      T* band = base + r * kTile * ldg;
      piv.push_back(band + r * kTile);
      MinPlusDesc<T> d0 = mkdesc<T>(band, band, band + r * kTile, band, ldg, ldg, ldg, 1, (int)(nbc - 1), -1, (int)r);
      MinPlusDesc<T> d1 = mkdesc<T>(base + r * kTile, base + r * kTile, base + r * kTile, band + r * kTile, ldg, ldg,
                                    ldg, (int)(nbc - 1), 1, (int)r, -1);
      d0.K = d1.K = kTile;
      bl.add(L2, d0);
      bl.add(L2, d1);
    }
    bl.end(L2);
    b->p2.push_back(L2);
    Launch L3 = bl.begin(2);
    for (int c = 0; c < k; ++c) {
      const long long nbc = b->s_pad[c] / kTile;
      if (r >= nbc) continue;
      T* base = S + b->off[c] * ldg;
      MinPlusDesc<T> d = mkdesc<T>(base, base, base + r * kTile, base + r * kTile * ldg, ldg, ldg, ldg,
                                   (int)(nbc - 1), (int)(nbc - 1), (int)r, (int)r);
      d.K = kTile;
      bl.add(L3, d);
    }
    bl.end(L3);
    b->p3.push_back(L3);
    T** dp = nullptr;
    if ((st = dupload<T*>(h, K, &dp, piv.data(), piv.size()))) return st;
    b->p1_tiles.push_back(dp);
    b->p1_count.push_back((int)piv.size());
  }
  // step 4 per group: out(c) = first element of block row c in its destination (ld = n_pad)
  for (auto& g : b->groups) {
    T* dst = g.slot >= 0 ? static_cast<T*>(b->buf[g.slot])
                         : static_cast<T*>(b->D_res) + (g.row0 - b->res_row0) * ld;
    T* tmp = static_cast<T*>(b->tmpb[g.slot >= 0 ? g.slot : 2]);
    if (!b->ooc) tmp = static_cast<T*>(b->tmpb[2]);
    // product 1: tmp_c = C2B[c] (x) bound(B_c, :)  (non-accumulating: Cin = +inf row, ldc_in 0)
    g.prod1 = bl.begin(2);
    for (int c = g.c0; c < g.c1; ++c) {
      if (b->nb_pad[c] == 0) {
        g.no_bnd.push_back(c);
        continue;
      }
      MinPlusDesc<T> d = mkdesc<T>(tmp + (b->off[c] - g.row0) * NB, infr, S + b->off[c] * ldg, bound + b->boff[c] * NB,
                                   NB, ldg, NB, (int)(b->s_pad[c] / kTile), (int)(NB / kTile), -1, -1);
      d.ldc_in = 0;
      d.K = (int)b->nb_pad[c];
      bl.add(g.prod1, d);
    }
    bl.end(g.prod1);
    // product 2, off-diagonal blocks: A(c,j) = tmp_c(:, B_j) (x) B2C[j]
    g.prod2 = bl.begin(2);
    for (int c = g.c0; c < g.c1; ++c) {
      if (b->nb_pad[c] == 0) continue;
      for (int j = 0; j < k; ++j) {
        if (j == c) continue;
        MinPlusDesc<T> d = mkdesc<T>(dst + (b->off[c] - g.row0) * ld + b->off[j], infr,
                                     tmp + (b->off[c] - g.row0) * NB + b->boff[j], S + b->off[j] * ldg, ld, NB, ldg,
                                     (int)(b->s_pad[c] / kTile), (int)(b->s_pad[j] / kTile), -1, -1);
        d.ldc_in = 0;
        d.K = (int)b->nb_pad[j];
        bl.add(g.prod2, d);
      }
    }
    bl.end(g.prod2);
    // product 2, diagonal blocks: A(c,c) = min(dist2(c,c), tmp_c(:, B_c) (x) B2C[c])
    g.prodd = bl.begin(2);
    for (int c = g.c0; c < g.c1; ++c) {
      if (b->nb_pad[c] == 0) continue;
      T* blk = S + b->off[c] * ldg;
      MinPlusDesc<T> d = mkdesc<T>(dst + (b->off[c] - g.row0) * ld + b->off[c], blk,
                                   tmp + (b->off[c] - g.row0) * NB + b->boff[c], blk, ld, NB, ldg,
                                   (int)(b->s_pad[c] / kTile), (int)(b->s_pad[c] / kTile), -1, -1);
      d.ldc_in = ldg;
      d.K = (int)b->nb_pad[c];
      bl.add(g.prodd, d);
    }
    bl.end(g.prodd);
  }
  {
    MinPlusDesc<T>* dd = nullptr;
    if ((st = dupload<MinPlusDesc<T>>(h, K, &dd, bl.descs.data(), bl.descs.size()))) return st;
    b->d_desc = dd;
  }
  if ((st = dupload<long long>(h, K, &b->d_pref, bl.pref.data(), bl.pref.size()))) return st;
  return h->cuda(launch_fill<T>(static_cast<T*>(b->inf_row), inf_len, inf_value<T>(), h->stream), "fill inf");
}

template <typename T>
apsp_status batched(Handle* h, const Launch& L, cudaStream_t s) {
  Bnd* b = B_(h);
  if (L.count <= 0) return APSP_OK;
  h->ev_begin(L.cls, s);
  apsp_status st = h->cuda(launch_minplus_batched<T>(static_cast<const MinPlusDesc<T>*>(b->d_desc) + L.first,
                                                     b->d_pref + L.pfirst, L.count, L.tiles, s),
                           "batched min-plus");
  h->ev_end(L.relax, s);
  return st;
}

template <typename T>
apsp_status init_t(Handle* h) {
  Bnd* b = B_(h);
  apsp_status st;
  const long long ldg = b->s_max;
  T* S = static_cast<T*>(b->strip);
  if ((st = h->cuda(launch_fill<T>(S, b->n_pad * ldg, inf_value<T>(), h->stream), "fill strip"))) return st;
  // dist2 init: each diagonal block from the intra-component arcs
  for (int c = 0; c < b->k; ++c) {
    const long long o = b->off[c];
    if ((st = h->cuda(launch_init_rows<T>(S + o * ldg, ldg, b->s_pad[c], 0, b->s_pad[c], b->s_pad[c], b->d_irp + o,
                                          0, b->d_icol, static_cast<const T*>(b->d_iw), h->stream),
                      "init dist2")))
      return st;
  }
  return h->cuda(cudaMemsetAsync(h->d_flag, 0, sizeof(int), h->stream), "memset flag");
}

// Step 4 for one group on stream s: products into the group's destination, fix-ups for
// components without boundary nodes (their block rows / columns are +inf but for the
// dist2 block), then (streamed groups) the copy of the group's rows to pinned host memory.
template <typename T>
apsp_status run_group(Handle* h, const Group& g, cudaStream_t s) {
  Bnd* b = B_(h);
  apsp_status st;
  const long long ld = b->n_pad;
  T* dst = g.slot >= 0 ? static_cast<T*>(b->buf[g.slot]) : static_cast<T*>(b->D_res) + (g.row0 - b->res_row0) * ld;
  if (b->need_fill) {
    h->ev_begin(3, s);
    st = h->cuda(launch_fill<T>(dst, g.rows * ld, inf_value<T>(), s), "fill block rows");
    h->ev_end(0, s);
    if (st) return st;
  }
  if ((st = batched<T>(h, g.prod1, s))) return st;
  if ((st = batched<T>(h, g.prod2, s))) return st;
  if ((st = batched<T>(h, g.prodd, s))) return st;
  for (int c : g.no_bnd) {  // no boundary node: A(c,c) = dist2(c,c), the rest of the row stays +inf
    const long long o = b->off[c];
    if ((st = h->cuda(launch_min_into<T>(dst + (o - g.row0) * ld + o, ld, static_cast<const T*>(b->strip) + o * b->s_max,
                                         b->s_max, b->s_pad[c], b->s_pad[c], s),
                      "dist2 block")))
      return st;
  }
  if (g.slot >= 0) {  // Alg. 3 l.20: the accumulated N_row block rows go back to the CPU
    h->ev_begin(3, s);
    st = h->cuda(cudaMemcpyAsync(static_cast<char*>(b->host) + (size_t)g.row0 * ld * h->elem, dst,
                                 (size_t)g.rows * ld * h->elem, cudaMemcpyDeviceToHost, s),
                 "D2H block rows");
    h->ev_end(0, s);
    if (st) return st;
  }
  return APSP_OK;
}

template <typename T>
apsp_status run_t(Handle* h) {
  Bnd* b = B_(h);
  apsp_status st;
  cudaStream_t s = h->stream;
  const long long NB = b->NB_pad, ldg = b->s_max;
  T* S = static_cast<T*>(b->strip);
  T* bound = static_cast<T*>(b->bound);
  // ---- step 2: dist2, all components one round per launch -----------------
  for (size_t r = 0; r < b->p2.size(); ++r) {
    h->ev_begin(0, s);
    if ((st = h->cuda(launch_phase1_batched<T>(static_cast<T* const*>(b->p1_tiles[r]), b->p1_count[r], ldg, h->d_flag,
                                               s),
                      "phase1 batched")))
      return st;
    h->ev_end((double)b->p1_count[r] * kTile * kTile * kTile, s);
    if ((st = batched<T>(h, b->p2[r], s))) return st;
    if ((st = batched<T>(h, b->p3[r], s))) return st;
  }
  // ---- step 3: boundary graph (arcs + virtual edges), dist3 ---------------------
  h->ev_begin(3, s);
  if ((st = h->cuda(launch_init_rows<T>(bound, NB, NB, 0, NB, NB, b->d_brp, 0, b->d_bcol,
                                        static_cast<const T*>(b->d_bw), s),
                    "init bound")))
    return st;
  bound_merge_kernel<T><<<(unsigned)NB, 128, 0, s>>>(bound, NB, S, ldg, b->d_rowcomp_b, b->d_off, b->d_boff,
                                                     b->d_nbpad);
  if ((st = h->cuda(cudaGetLastError(), "bound merge"))) return st;
  h->ev_end(0, s);
  if ((st = fw_closure<T>(h, bound, NB, NB, 0, NB / kTile, s))) return st;
  // ---- step 4: dist4, group by group ---------------------------------------------------
  if (b->ooc) {
    if ((st = h->cuda(cudaEventRecord(b->ev_ready, s), "event"))) return st;
    for (int x = 0; x < 2; ++x)
      if ((st = h->cuda(cudaStreamWaitEvent(b->xs[x], b->ev_ready, 0), "wait"))) return st;
  }
  // streamed groups alternate between the two buffers / streams (a buffer's next
  // group waits in stream order for its previous D2H); resident groups run on the main stream
  for (const auto& g : b->groups)
    if (g.slot >= 0 && (st = run_group<T>(h, g, b->xs[g.slot]))) return st;
  for (const auto& g : b->groups)
    if (g.slot < 0 && (st = run_group<T>(h, g, s))) return st;
  if (b->ooc)
    for (int x = 0; x < 2; ++x) {
      if ((st = h->cuda(cudaEventRecord(b->ev_done[x], b->xs[x]), "event"))) return st;
      if ((st = h->cuda(cudaStreamWaitEvent(s, b->ev_done[x], 0), "wait"))) return st;
    }
  return APSP_OK;
}

}  // namespace

apsp_status bnd_setup(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col, const void* w,
                      const int32_t* comp, int k) {
  h->bnd = new Bnd();
  apsp_status st = h->dtype == APSP_I32
                       ? setup_t<int>(h, cfg, row_ptr, col, static_cast<const int*>(w), comp, k)
                       : setup_t<float>(h, cfg, row_ptr, col, static_cast<const float*>(w), comp, k);
  if (st) return st;
  if ((st = bnd_reinit(h))) return st;
  return h->cuda(cudaStreamSynchronize(h->stream), "boundary init sync");
}

apsp_status bnd_reinit(Handle* h) {
  h->fw_done = false;
  h->canonical = false;
  return h->dtype == APSP_I32 ? init_t<int>(h) : init_t<float>(h);
}

apsp_status bnd_run(Handle* h) { return h->dtype == APSP_I32 ? run_t<int>(h) : run_t<float>(h); }

long long bnd_boundary_nodes(const Handle* h) { return h->bnd ? static_cast<const Bnd*>(h->bnd)->nb_real : 0; }

long long bnd_ooc_rows(const Handle* h) {
  const Bnd* b = static_cast<const Bnd*>(h->bnd);
  return b && b->ooc ? b->buf_rows : 0;
}

// Rows [r0, r0+cnt) in the caller's order: in core one gather of rows and columns from the
// resident matrix; out of core the needed rows (component order) are first brought into a
// device staging block (H2D from the pinned host matrix or D2D from the resident rows).
apsp_status bnd_get_rows(Handle* h, long long r0, long long cnt, void* out, long long ld_out) {
  Bnd* b = B_(h);
  apsp_status st;
  const long long n = h->n, n_pad = b->n_pad;
  const size_t es = h->elem;
  const long long blk = std::max<long long>(1, std::min<long long>(cnt, (64ll << 20) / (n_pad * (long long)es)));
  const bool staged = b->res_row0 > 0;
  if (b->stage_rows < blk) {
    cudaFree(b->d_stage);
    cudaFree(b->d_rowmap);
    cudaFree(b->d_src);
    cudaFree(b->d_ident);
    b->d_stage = b->d_src = nullptr;
    b->d_rowmap = b->d_ident = nullptr;
    if ((st = h->cuda(cudaMalloc(&b->d_stage, blk * n * es), "cudaMalloc stage"))) return st;
    if ((st = h->cuda(cudaMalloc(&b->d_rowmap, blk * sizeof(int)), "cudaMalloc rowmap"))) return st;
    if (staged) {
      if ((st = h->cuda(cudaMalloc(&b->d_src, blk * n_pad * es), "cudaMalloc stage src"))) return st;
      std::vector<int> id(blk);
      for (long long t = 0; t < blk; ++t) id[t] = (int)t;
      if ((st = h->cuda(cudaMalloc(&b->d_ident, blk * sizeof(int)), "cudaMalloc ident"))) return st;
      if ((st = h->cuda(cudaMemcpy(b->d_ident, id.data(), blk * sizeof(int), cudaMemcpyHostToDevice), "H2D ident")))
        return st;
    }
    b->stage_rows = blk;
  }
  for (long long r = r0; r < r0 + cnt; r += blk) {
    const long long rr = std::min(blk, r0 + cnt - r);
    const void* src = b->D_res;
    const int* rowmap = b->d_rowmap;
    long long src_ld = n_pad;
    if (staged) {  // component-order rows -> d_src rows 0..rr-1
      for (long long t = 0; t < rr; ++t) {
        const long long nr = b->new_id[r + t];
        char* d = static_cast<char*>(b->d_src) + (size_t)t * n_pad * es;
        if (nr < b->res_row0)
          st = h->cuda(cudaMemcpyAsync(d, static_cast<const char*>(b->host) + (size_t)nr * n_pad * es, n_pad * es,
                                       cudaMemcpyHostToDevice, h->stream),
                       "H2D row");
        else
          st = h->cuda(cudaMemcpyAsync(d, static_cast<const char*>(b->D_res) + (size_t)(nr - b->res_row0) * n_pad * es,
                                       n_pad * es, cudaMemcpyDeviceToDevice, h->stream),
                       "D2D row");
        if (st) return st;
      }
      src = b->d_src;
      rowmap = b->d_ident;
    } else if ((st = h->cuda(cudaMemcpyAsync(b->d_rowmap, b->new_id.data() + r, rr * sizeof(int),
                                             cudaMemcpyHostToDevice, h->stream),
                             "H2D rowmap"))) {
      return st;
    }
    cudaError_t e = h->dtype == APSP_I32
                        ? launch_gather<int>(static_cast<const int*>(src), src_ld, rowmap, b->d_new_id,
                                             static_cast<int*>(b->d_stage), n, rr, n, h->stream)
                        : launch_gather<float>(static_cast<const float*>(src), src_ld, rowmap, b->d_new_id,
                                               static_cast<float*>(b->d_stage), n, rr, n, h->stream);
    if ((st = h->cuda(e, "gather"))) return st;
    if ((st = h->cuda(cudaMemcpy2DAsync(static_cast<char*>(out) + (r - r0) * ld_out * es, ld_out * es, b->d_stage,
                                        n * es, n * es, rr, cudaMemcpyDeviceToHost, h->stream),
                      "D2H dist")))
      return st;
    if ((st = h->cuda(cudaStreamSynchronize(h->stream), "get_dist sync"))) return st;  // rowmap / stage reuse
  }
  return APSP_OK;
}

void bnd_free(Handle* h) {
  Bnd* b = B_(h);
  if (!b) return;
  for (int x = 0; x < 2; ++x)
    if (b->xs[x]) cudaStreamSynchronize(b->xs[x]);
  if (h->stream) {
    for (void* p : {b->strip, b->bound, b->D_res, b->buf[0], b->buf[1], b->tmpb[0], b->tmpb[1], b->tmpb[2],
                    b->inf_row})
      if (p) cudaFreeAsync(p, h->stream);
    cudaStreamSynchronize(h->stream);
  }
  for (int x = 0; x < 2; ++x) {
    if (b->xs[x]) cudaStreamDestroy(b->xs[x]);
    if (b->ev_done[x]) cudaEventDestroy(b->ev_done[x]);
  }
  if (b->ev_ready) cudaEventDestroy(b->ev_ready);
  if (b->host) cudaFreeHost(b->host);
  for (void* p : b->dev) cudaFree(p);
  cudaFree(b->d_stage);
  cudaFree(b->d_rowmap);
  cudaFree(b->d_src);
  cudaFree(b->d_ident);
  delete b;
  h->bnd = nullptr;
}

}  // namespace apsp
