// apsp_boundary.cu — the boundary algorithm (Djidjev et al.; PAPER.md:139-150,
// eq. (1); out-of-core form Algorithm 3) on one B200, built
// from the same sm_100a kernels as the blocked Floyd–Warshall path.
//
//   step 1  partition (given by the caller: comp[v] in [0, k)); a vertex with an
//           arc to another component is a boundary node
//   step 2  dist2 = APSP inside every component: blocked FW on the diagonal
//           blocks A(i,i) (Alg. 3 l.1-3); all components advance one round per
//           launch (batched phase 1, phase 2 and phase 3)
//   step 3  boundary graph: inter-component arcs + virtual edges dist2(u,v)
//           between boundary nodes of one component (Alg. 3 l.4);
//           dist3 = blocked FW on `bound` (Alg. 3 l.5)
//   step 4  dist4 = C2B[i] (x) bound(i,j) (x) B2C[j] (eq. (1); Alg. 3 l.12-17):
//           tmp(C_i, :) = C2B[i] (x) bound(B_i, :) for all i in one batched
//           launch; A(i,j) = tmp(C_i, B_j) (x) B2C[j] for all j != i in one
//           batched launch; A(i,i) = min(dist2(i,i), tmp(C_i, B_i) (x) B2C[i])
//           out of place, then copied back.
// Exactness: a path from C_i to C_j (j != i) leaves C_i at its first boundary
// node and enters C_j at its last one; its middle part is a path of the
// boundary graph whose intra-component detours are virtual edges. Paths inside
// one component either avoid boundary nodes (dist2) or are covered the same way.
//
// Layout (Fig. 1a): vertices are relabelled so that every component is
// a contiguous block with its boundary nodes first; blocks are padded to 128
// (the tile) and boundary sets to 32 (the depth chunk) with further vertices of
// the component treated as boundary (any superset of the boundary keeps eq. (1)
// exact) or isolated dummies. The n x n result stays on the device in this
// order; apsp_get_dist gathers rows and columns back into the caller's order.
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

struct Bnd {
  int k = 0;
  long long n_pad = 0, NB_pad = 0, s_max = 0, nb_real = 0;
  std::vector<long long> off, s_pad, nb_pad, boff;
  std::vector<int> new_id;  // original vertex -> new index
  void* D = nullptr;        // n_pad x n_pad, component-blocked order
  void* bound = nullptr;    // NB_pad x NB_pad
  void* tmp = nullptr;      // n_pad x NB_pad (rows of C_i hold tmp_i)
  void* scratch = nullptr;  // n_pad x s_max (new diagonal blocks, row-aligned with D)
  void* inf_row = nullptr;  // max(NB_pad, s_max) elements of infinity
  std::vector<void*> dev;   // every other device allocation (freed together)
  int* d_new_id = nullptr;
  long long* d_irp = nullptr;  // intra-component CSR over the n_pad new rows (block-local columns)
  int* d_icol = nullptr;
  void* d_iw = nullptr;
  long long* d_brp = nullptr;  // boundary-graph CSR over NB_pad rows (bound columns)
  int* d_bcol = nullptr;
  void* d_bw = nullptr;
  int* d_rowcomp = nullptr;    // new row -> component
  int* d_rowcomp_b = nullptr;  // bound row -> component (-1: padding)
  long long *d_off = nullptr, *d_boff = nullptr, *d_spad = nullptr, *d_nbpad = nullptr;
  void* d_desc = nullptr;
  long long* d_pref = nullptr;
  std::vector<Launch> p2, p3;  // dist2 rounds
  Launch prod1, prod2, prodd;
  std::vector<void*> p1_tiles;  // per dist2 round: device array of pivot-tile pointers
  std::vector<int> p1_count;
  int* d_rowmap = nullptr;      // get_dist staging
  void* d_stage = nullptr;
  long long stage_rows = 0;
};

Bnd* B_(Handle* h) { return static_cast<Bnd*>(h->bnd); }

template <typename T> T inf_value();
template <> int inf_value<int>() { return APSP_INF_I32; }
template <> float inf_value<float>() { return INFINITY; }

template <typename T>
__global__ void bound_merge_kernel(T* bound, long long ldb, const T* D, long long ld, const int* rowcomp_b,
                                   const long long* off, const long long* boff, const long long* nbp) {
  const long long r = blockIdx.x;
  const int c = rowcomp_b[r];
  if (c < 0) return;
  const T* src = D + (off[c] + (r - boff[c])) * ld + off[c];
  T* dst = bound + r * ldb + boff[c];
  for (long long x = threadIdx.x; x < nbp[c]; x += blockDim.x) dst[x] = src[x] < dst[x] ? src[x] : dst[x];
}

template <typename T>
__global__ void diag_copy_kernel(T* D, long long ld, const T* S, long long lds, const int* rowcomp,
                                 const long long* off, const long long* spad, const long long* nbp) {
  const long long r = blockIdx.x;
  const int c = rowcomp[r];
  if (nbp[c] == 0) return;  // no boundary node: the block is dist2 already
  const T* src = S + r * lds;
  T* dst = D + r * ld + off[c];
  for (long long x = threadIdx.x; x < spad[c]; x += blockDim.x) dst[x] = src[x];
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

template <typename T>
apsp_status setup_t(Handle* h, const int64_t* row_ptr, const int32_t* col, const T* w, const int32_t* comp, int k) {
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
  }
  b->n_pad = o;
  b->NB_pad = std::max<long long>(kTile, (bo + kTile - 1) / kTile * kTile);
  h->n_pad = b->n_pad;
  h->ld = b->n_pad;
  b->new_id.assign(n, -1);
  std::vector<int> old_of(b->n_pad, -1), rowcomp(b->n_pad, 0), rowcomp_b(b->NB_pad, -1);
  for (int c = 0; c < k; ++c) {
    for (size_t p = 0; p < members[c].size(); ++p) {
      b->new_id[members[c][p]] = (int)(b->off[c] + (long long)p);
      old_of[b->off[c] + p] = members[c][p];
    }
    for (long long r = 0; r < b->s_pad[c]; ++r) rowcomp[b->off[c] + r] = c;
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
  // ---- device state --------------------------------------------------------------
  const size_t es = h->elem;
  auto dmalloc = [&](void** p, size_t bytes, const char* what) -> apsp_status {
    apsp_status s2 = h->cuda(cudaMallocAsync(p, bytes, h->stream), what);
    if (!s2) h->device_bytes += bytes;
    return s2;
  };
  if ((st = dmalloc(&b->D, (size_t)b->n_pad * b->n_pad * es, "cudaMalloc dist"))) return st;
  if ((st = dmalloc(&b->bound, (size_t)b->NB_pad * b->NB_pad * es, "cudaMalloc bound"))) return st;
  if ((st = dmalloc(&b->tmp, (size_t)b->n_pad * b->NB_pad * es, "cudaMalloc tmp"))) return st;
  if ((st = dmalloc(&b->scratch, (size_t)b->n_pad * b->s_max * es, "cudaMalloc scratch"))) return st;
  const long long inf_len = std::max(b->NB_pad, b->s_max);
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
  if ((st = dupload<int>(h, K, &b->d_rowcomp, rowcomp.data(), rowcomp.size()))) return st;
  if ((st = dupload<int>(h, K, &b->d_rowcomp_b, rowcomp_b.data(), rowcomp_b.size()))) return st;
  if ((st = dupload<long long>(h, K, &b->d_off, b->off.data(), k))) return st;
  if ((st = dupload<long long>(h, K, &b->d_boff, b->boff.data(), k))) return st;
  if ((st = dupload<long long>(h, K, &b->d_spad, b->s_pad.data(), k))) return st;
  if ((st = dupload<long long>(h, K, &b->d_nbpad, b->nb_pad.data(), k))) return st;
  if ((st = h->cuda(cudaStreamSynchronize(h->stream), "boundary alloc sync"))) return st;

  // ---- batched min-plus descriptors -------------------------------------------------
  T* D = static_cast<T*>(b->D);
  T* bound = static_cast<T*>(b->bound);
  T* tmp = static_cast<T*>(b->tmp);
  T* scr = static_cast<T*>(b->scratch);
  const T* infr = static_cast<const T*>(b->inf_row);
  const long long ld = b->n_pad, NB = b->NB_pad;
  Builder<T> bl;
  const long long R = b->s_max / kTile;
  for (long long r = 0; r < R; ++r) {
    std::vector<T*> piv;
    Launch L2 = bl.begin(1);
    for (int c = 0; c < k; ++c) {
      const long long nbc = b->s_pad[c] / kTile;
      if (r >= nbc) continue;
      T* base = D + b->off[c] * ld + b->off[c];
      T* band = base + r * kTile * ld;
      piv.push_back(band + r * kTile);
      MinPlusDesc<T> d0 = mkdesc<T>(band, band, band + r * kTile, band, ld, ld, ld, 1, (int)(nbc - 1), -1, (int)r);
      MinPlusDesc<T> d1 = mkdesc<T>(base + r * kTile, base + r * kTile, base + r * kTile, band + r * kTile, ld, ld,
                                    ld, (int)(nbc - 1), 1, (int)r, -1);
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
      T* base = D + b->off[c] * ld + b->off[c];
      MinPlusDesc<T> d = mkdesc<T>(base, base, base + r * kTile, base + r * kTile * ld, ld, ld, ld, (int)(nbc - 1),
                                   (int)(nbc - 1), (int)r, (int)r);
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
  // step 4, product 1: tmp(C_i, :) = C2B[i] (x) bound(B_i, :)  (every row of Cin = +inf: ldc_in 0)
  b->prod1 = bl.begin(2);
  for (int c = 0; c < k; ++c) {
    MinPlusDesc<T> d = mkdesc<T>(tmp + b->off[c] * NB, infr, D + b->off[c] * ld + b->off[c], bound + b->boff[c] * NB,
                                 NB, ld, NB, (int)(b->s_pad[c] / kTile), (int)(NB / kTile), -1, -1);
    d.ldc_in = 0;
    d.K = (int)b->nb_pad[c];
    bl.add(b->prod1, d);
  }
  bl.end(b->prod1);
  // product 2, off-diagonal blocks: A(i,j) = tmp(C_i, B_j) (x) B2C[j]
  b->prod2 = bl.begin(2);
  for (int i = 0; i < k; ++i)
    for (int j = 0; j < k; ++j) {
      if (i == j) continue;
      MinPlusDesc<T> d = mkdesc<T>(D + b->off[i] * ld + b->off[j], infr, tmp + b->off[i] * NB + b->boff[j],
                                   D + b->off[j] * ld + b->off[j], ld, NB, ld, (int)(b->s_pad[i] / kTile),
                                   (int)(b->s_pad[j] / kTile), -1, -1);
      d.ldc_in = 0;
      d.K = (int)b->nb_pad[j];
      bl.add(b->prod2, d);
    }
  bl.end(b->prod2);
  // product 2, diagonal blocks, out of place: scratch(C_i) = min(dist2(i,i), tmp(C_i, B_i) (x) B2C[i])
  b->prodd = bl.begin(2);
  for (int c = 0; c < k; ++c) {
    T* blk = D + b->off[c] * ld + b->off[c];
    MinPlusDesc<T> d = mkdesc<T>(scr + b->off[c] * b->s_max, blk, tmp + b->off[c] * NB + b->boff[c], blk, b->s_max,
                                 NB, ld, (int)(b->s_pad[c] / kTile), (int)(b->s_pad[c] / kTile), -1, -1);
    d.ldc_in = ld;
    d.K = (int)b->nb_pad[c];
    bl.add(b->prodd, d);
  }
  bl.end(b->prodd);
  {
    MinPlusDesc<T>* dd = nullptr;
    if ((st = dupload<MinPlusDesc<T>>(h, K, &dd, bl.descs.data(), bl.descs.size()))) return st;
    b->d_desc = dd;
  }
  if ((st = dupload<long long>(h, K, &b->d_pref, bl.pref.data(), bl.pref.size()))) return st;
  if ((st = h->cuda(launch_fill<T>(static_cast<T*>(b->inf_row), inf_len, inf_value<T>(), h->stream), "fill inf")))
    return st;
  // rows of components without boundary nodes are never produced by product 1: keep them infinite
  return h->cuda(launch_fill<T>(tmp, b->n_pad * NB, inf_value<T>(), h->stream), "fill tmp");
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
  const long long ld = b->n_pad;
  T* D = static_cast<T*>(b->D);
  // blocks (i, j) into a component without boundary nodes are never produced: +inf
  if ((st = h->cuda(launch_fill<T>(D, b->n_pad * b->n_pad, inf_value<T>(), h->stream), "fill dist")))
    return st;
  // dist2 init: each diagonal block from the intra-component arcs
  for (int c = 0; c < b->k; ++c) {
    const long long o = b->off[c];
    if ((st = h->cuda(launch_init_rows<T>(D + o * ld + o, ld, b->s_pad[c], 0, b->s_pad[c], b->s_pad[c], b->d_irp + o,
                                          0, b->d_icol, static_cast<const T*>(b->d_iw), h->stream),
                      "init dist2")))
      return st;
  }
  return h->cuda(cudaMemsetAsync(h->d_flag, 0, sizeof(int), h->stream), "memset flag");
}

template <typename T>
apsp_status run_t(Handle* h) {
  Bnd* b = B_(h);
  apsp_status st;
  cudaStream_t s = h->stream;
  const long long ld = b->n_pad, NB = b->NB_pad;
  T* D = static_cast<T*>(b->D);
  T* bound = static_cast<T*>(b->bound);
  // ---- step 2: dist2, all components one round per launch -----------------
  for (size_t r = 0; r < b->p2.size(); ++r) {
    h->ev_begin(0, s);
    if ((st = h->cuda(launch_phase1_batched<T>(static_cast<T* const*>(b->p1_tiles[r]), b->p1_count[r], ld, h->d_flag,
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
  bound_merge_kernel<T><<<(unsigned)NB, 128, 0, s>>>(bound, NB, D, ld, b->d_rowcomp_b, b->d_off, b->d_boff,
                                                     b->d_nbpad);
  if ((st = h->cuda(cudaGetLastError(), "bound merge"))) return st;
  h->ev_end(0, s);
  if ((st = fw_closure<T>(h, bound, NB, NB, 0, NB / kTile, s))) return st;
  // ---- step 4: dist4 ------------------------------------------------------------------
  if ((st = batched<T>(h, b->prod1, s))) return st;
  if ((st = batched<T>(h, b->prod2, s))) return st;
  if ((st = batched<T>(h, b->prodd, s))) return st;
  h->ev_begin(3, s);
  diag_copy_kernel<T><<<(unsigned)b->n_pad, 128, 0, s>>>(D, ld, static_cast<const T*>(b->scratch), b->s_max,
                                                        b->d_rowcomp, b->d_off, b->d_spad, b->d_nbpad);
  h->ev_end(0, s);
  return h->cuda(cudaGetLastError(), "diag copy");
}

}  // namespace

apsp_status bnd_setup(Handle* h, const int64_t* row_ptr, const int32_t* col, const void* w, const int32_t* comp,
                      int k) {
  h->bnd = new Bnd();
  apsp_status st = h->dtype == APSP_I32
                       ? setup_t<int>(h, row_ptr, col, static_cast<const int*>(w), comp, k)
                       : setup_t<float>(h, row_ptr, col, static_cast<const float*>(w), comp, k);
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

apsp_status bnd_get_rows(Handle* h, long long r0, long long cnt, void* out, long long ld_out) {
  Bnd* b = B_(h);
  apsp_status st;
  const long long n = h->n;
  const long long blk = std::max<long long>(1, std::min<long long>(cnt, (64ll << 20) / (n * (long long)h->elem)));
  if (b->stage_rows < blk) {
    cudaFree(b->d_stage);
    cudaFree(b->d_rowmap);
    b->d_stage = nullptr;
    b->d_rowmap = nullptr;
    if ((st = h->cuda(cudaMalloc(&b->d_stage, blk * n * h->elem), "cudaMalloc stage"))) return st;
    if ((st = h->cuda(cudaMalloc(&b->d_rowmap, blk * sizeof(int)), "cudaMalloc rowmap"))) return st;
    b->stage_rows = blk;
  }
  for (long long r = r0; r < r0 + cnt; r += blk) {
    const long long rr = std::min(blk, r0 + cnt - r);
    if ((st = h->cuda(cudaMemcpyAsync(b->d_rowmap, b->new_id.data() + r, rr * sizeof(int), cudaMemcpyHostToDevice,
                                      h->stream),
                      "H2D rowmap")))
      return st;
    cudaError_t e = h->dtype == APSP_I32
                        ? launch_gather<int>(static_cast<const int*>(b->D), b->n_pad, b->d_rowmap, b->d_new_id,
                                             static_cast<int*>(b->d_stage), n, rr, n, h->stream)
                        : launch_gather<float>(static_cast<const float*>(b->D), b->n_pad, b->d_rowmap, b->d_new_id,
                                               static_cast<float*>(b->d_stage), n, rr, n, h->stream);
    if ((st = h->cuda(e, "gather"))) return st;
    if ((st = h->cuda(cudaMemcpy2DAsync(static_cast<char*>(out) + (r - r0) * ld_out * h->elem, ld_out * h->elem,
                                        b->d_stage, n * h->elem, n * h->elem, rr, cudaMemcpyDeviceToHost, h->stream),
                      "D2H dist")))
      return st;
    if ((st = h->cuda(cudaStreamSynchronize(h->stream), "get_dist sync"))) return st;  // rowmap / stage reuse
  }
  return APSP_OK;
}

void bnd_free(Handle* h) {
  Bnd* b = B_(h);
  if (!b) return;
  if (h->stream) {
    for (void* p : {b->D, b->bound, b->tmp, b->scratch, b->inf_row})
      if (p) cudaFreeAsync(p, h->stream);
    cudaStreamSynchronize(h->stream);
  }
  for (void* p : b->dev) cudaFree(p);
  cudaFree(b->d_stage);
  cudaFree(b->d_rowmap);
  delete b;
  h->bnd = nullptr;
}

}  // namespace apsp
