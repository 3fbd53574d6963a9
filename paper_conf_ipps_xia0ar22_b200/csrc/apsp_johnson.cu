// apsp_johnson.cu — Johnson's algorithm with batched Near-Far SSSP (PAPER.md:66,
// §II-B; Near-Far; out-of-core batches, Algorithm 2) on one B200.
//
// APSP = one single-source shortest-path (SSSP) run per source vertex
// (Johnson). Every SSSP instance belongs to ONE thread block (P:115:
// "We assign each SSSP instance to one thread block so that we are able to
// synchronize threads within one thread block"); a persistent grid of blocks
// walks the sources of a batch (Alg. 2 l.1-5: source_id = block_id; source_id <
// bat; source_id += num_blocks), and batch results go back to the host while
// the next batch runs (Alg. 2 l.7-11, "Transfer results back to CPU").
//
// Near-Far: the work queue is split into a Near queue (distances below
// the threshold T) and a Far queue. One iteration expands every Near vertex u:
// each arc (u,v,w) is relaxed with atomicMin on dist[v]; an improved v goes to
// the next Near queue if its distance is < T, else to the Far queue. When Near
// runs empty, T advances by Delta and the Far queue is split the same way.
// (Here T restarts at min(Far) + Delta, so an empty bucket costs nothing.)
//
// B200 design choices (not the paper's code):
//  - the SSSP's distance array IS the output row (no copy), relaxed with
//    L2 atomics; reads of dist go through ld.cg (never a stale L1 line, so a
//    vertex improved after its queue entry was cleared is always re-expanded)
//  - "already queued" flags are bitmaps in shared memory (2 x n/8 bytes) when
//    they fit, otherwise in a per-block global slice; queue entries are
//    deduplicated with them, so each queue holds at most n entries
//  - a frontier vertex is expanded by G lanes (G = the average out-degree
//    rounded to a power of two, <= 32), which keeps the lanes of a warp busy on
//    both road-like (degree ~4) and denser (degree 256) graphs without the
//    paper's dynamic-parallelism child kernels
//  - queue appends are warp-aggregated (one shared atomic per coalesced group)
//  - negative int32 weights: Johnson's reweighting (the classic
//    algorithm) — potentials p from a Bellman–Ford pass over a virtual source
//    (P:68), w'(u,v) = w + p(u) - p(v) >= 0, and the row epilogue restores
//    dist(s,t) = dist'(s,t) - p(s) + p(t); a negative cycle -> APSP_ENEGCYCLE.
#include "apsp_internal.h"

#include <cooperative_groups.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>

namespace cg = cooperative_groups;

namespace apsp {

namespace {

constexpr int kJThreads = 256;

template <typename T> struct JV;
template <> struct JV<int> {
  static __device__ __forceinline__ int inf() { return APSP_INF_I32; }
  // d + w with the int32 "no path" guard (d < INF on entry)
  static __device__ __forceinline__ int add(int d, int w) {
    const long long s = (long long)d + w;
    return s < APSP_INF_I32 ? (int)s : APSP_INF_I32;
  }
  static __device__ __forceinline__ int amin(int* p, int v) { return atomicMin(p, v); }
  static __device__ __forceinline__ int load(const int* p) { return __ldcg(p); }
  static __device__ __forceinline__ int plus_delta(int d, int delta) {
    const long long s = (long long)d + delta;
    return s < APSP_INF_I32 ? (int)s : APSP_INF_I32;
  }
};
template <> struct JV<float> {
  static __device__ __forceinline__ float inf() { return __int_as_float(0x7f800000); }
  static __device__ __forceinline__ float add(float d, float w) { return __fadd_rn(d, w); }
  // non-negative floats order like their bit patterns (Johnson fp32: weights >= 0)
  static __device__ __forceinline__ float amin(float* p, float v) {
    return __int_as_float(atomicMin(reinterpret_cast<int*>(p), __float_as_int(v)));
  }
  static __device__ __forceinline__ float load(const float* p) { return __ldcg(p); }
  static __device__ __forceinline__ float plus_delta(float d, float delta) { return __fadd_rn(d, delta); }
};

template <typename T>
struct MsspArgs {
  long long n;
  const long long* rp;
  const int* col;
  const T* w;           // (reweighted) arc weights, >= 0
  long long src_begin, src_end;  // sources of this launch
  T* out;               // row of source s at out + (s - row_base) * ld
  long long row_base, ld;
  int* work;            // per block: 4 queues of n entries
  unsigned* gbits;      // per block: 2 bitmaps of nwords (when not in shared memory)
  long long nwords;     // ceil(n / 32)
  int smem_bits;        // 1: bitmaps in dynamic shared memory
  T delta;
  const long long* pot; // Johnson potentials (negative weights) or nullptr
  unsigned long long* edges;  // arcs scanned (statistics)
};

// test-and-set of bit v; true if this call set it
__device__ __forceinline__ bool tas(unsigned* bits, int v) {
  const unsigned m = 1u << (v & 31);
  return (atomicOr(bits + (v >> 5), m) & m) == 0;
}
__device__ __forceinline__ void clr(unsigned* bits, int v) { atomicAnd(bits + (v >> 5), ~(1u << (v & 31))); }

// warp-aggregated append of v to q (counter in shared memory)
__device__ __forceinline__ void append(int* q, int* cnt, int v) {
  cg::coalesced_group g = cg::coalesced_threads();
  int base = 0;
  if (g.thread_rank() == 0) base = atomicAdd(cnt, (int)g.size());
  base = g.shfl(base, 0);
  q[base + g.thread_rank()] = v;
}

// NT threads per block, G lanes per frontier vertex (power of two <= 32)
template <typename T, int NT, int G>
__global__ void __launch_bounds__(NT) mssp_kernel(MsspArgs<T> a) {
  extern __shared__ __align__(16) unsigned jsm[];
  __shared__ int s_qn, s_qn2, s_fn, s_fn2;
  __shared__ T s_T, s_min;
  const int tid = threadIdx.x;
  const long long n = a.n;
  unsigned* nearb = a.smem_bits ? jsm : a.gbits + (size_t)blockIdx.x * 2 * a.nwords;
  unsigned* farb = nearb + a.nwords;
  int* Q = a.work + (size_t)blockIdx.x * 4 * n;
  int* Q2 = Q + n;
  int* F = Q2 + n;
  int* F2 = F + n;
  const int lane_g = tid % G;
  const int grp = tid / G;
  constexpr int NG = NT / G;
  unsigned long long scanned = 0;

  for (long long s = a.src_begin + blockIdx.x; s < a.src_end; s += gridDim.x) {
    T* const row = a.out + (s - a.row_base) * a.ld;
    for (long long v = tid; v < n; v += NT) row[v] = JV<T>::inf();
    for (long long x = tid; x < 2 * a.nwords; x += NT) nearb[x] = 0u;
    __syncthreads();
    if (tid == 0) {
      row[s] = T(0);
      Q[0] = (int)s;
      s_qn = 1;
      s_fn = 0;
      s_T = a.delta;
    }
    __syncthreads();
    for (;;) {
      int qn = s_qn;
      if (qn == 0) {
        // Near queue empty: advance the threshold past the smallest Far distance
        // and split the Far queue ("swap Near Queue and Far Queue ... (i+1)Delta")
        const int fn = s_fn;
        if (fn == 0) break;
        if (tid == 0) {
          s_min = JV<T>::inf();
          s_qn2 = 0;
          s_fn2 = 0;
        }
        __syncthreads();
        // every vertex below the old threshold told is settled (weights >= 0 and the
        // Near queue of that bucket ran empty), so Far entries below it are stale
        const T told = s_T;
        T mn = JV<T>::inf();
        for (int i = tid; i < fn; i += NT) {
          const int v = F[i];
          clr(farb, v);
          const T d = JV<T>::load(row + v);
          if (d >= told) mn = d < mn ? d : mn;
        }
        for (int o = 16; o; o >>= 1) {
          const T x = __shfl_xor_sync(0xffffffffu, mn, o);
          mn = x < mn ? x : mn;
        }
        if ((tid & 31) == 0) JV<T>::amin(&s_min, mn);
        __syncthreads();
        const T thr = JV<T>::plus_delta(s_min, a.delta);
        for (int i = tid; i < fn; i += NT) {
          const int v = F[i];
          const T d = JV<T>::load(row + v);
          if (d < told) {
            // stale: improved below the old threshold later and expanded then
          } else if (d < thr) {
            if (tas(nearb, v)) append(Q, &s_qn2, v);
          } else if (tas(farb, v)) {
            append(F2, &s_fn2, v);
          }
        }
        __syncthreads();
        if (tid == 0) {
          s_T = thr;
          s_qn = s_qn2;
          s_fn = s_fn2;
        }
        int* t = F;
        F = F2;
        F2 = t;
        __syncthreads();
        continue;
      }
      // expand the Near queue; its entries' flags are cleared first so that a
      // vertex improved during this iteration is queued again
      for (int i = tid; i < qn; i += NT) clr(nearb, Q[i]);
      if (tid == 0) s_qn2 = 0;
      __syncthreads();
      const T thr = s_T;
      for (int i = grp; i < qn; i += NG) {
        const int u = Q[i];
        const T du = JV<T>::load(row + u);
        const long long e0 = a.rp[u], e1 = a.rp[u + 1];
        scanned += (unsigned long long)((e1 - e0 + G - 1 - lane_g) / G);
        for (long long e = e0 + lane_g; e < e1; e += G) {
          const int v = a.col[e];
          const T nd = JV<T>::add(du, a.w[e]);
          if (nd < JV<T>::load(row + v)) {
            const T old = JV<T>::amin(row + v, nd);
            if (nd < old) {
              if (nd < thr) {
                if (tas(nearb, v)) append(Q2, &s_qn2, v);
              } else if (tas(farb, v)) {
                append(F, &s_fn, v);
              }
            }
          }
        }
      }
      __syncthreads();
      if (tid == 0) s_qn = s_qn2;
      int* t = Q;
      Q = Q2;
      Q2 = t;
      __syncthreads();
    }
    // Johnson epilogue: undo the reweighting, dist(s,t) = dist'(s,t) - p(s) + p(t)
    if (a.pot) {
      const long long ps = a.pot[s];
      for (long long v = tid; v < n; v += NT) {
        const T d = row[v];
        if (d < JV<T>::inf()) row[v] = (T)((long long)d - ps + a.pot[v]);
      }
    }
    __syncthreads();
  }
  for (int o = 16; o; o >>= 1) scanned += __shfl_xor_sync(0xffffffffu, scanned, o);
  if ((tid & 31) == 0 && a.edges) atomicAdd(a.edges, scanned);
}

// ---- Johnson reweighting: Bellman–Ford from a virtual source ----
__global__ void bf_sweep_kernel(long long n, const long long* rp, const int* col, const int* w, long long* p,
                                int* changed) {
  for (long long u = blockIdx.x * (long long)blockDim.x + threadIdx.x; u < n; u += (long long)gridDim.x * blockDim.x) {
    const long long pu = __ldcg(p + u);
    for (long long e = rp[u]; e < rp[u + 1]; ++e) {
      const int v = col[e];
      const long long nv = pu + w[e];
      if (nv < __ldcg(p + v) && nv < (long long)atomicMin((long long*)(p + v), nv)) *changed = 1;
    }
  }
}

__global__ void reweight_kernel(long long n, const long long* rp, const int* col, const int* w, const long long* p,
                                int* w2) {
  for (long long u = blockIdx.x * (long long)blockDim.x + threadIdx.x; u < n; u += (long long)gridDim.x * blockDim.x)
    for (long long e = rp[u]; e < rp[u + 1]; ++e) w2[e] = (int)(w[e] + p[u] - p[col[e]]);
}

struct Jn {
  long long m = 0;
  long long* d_rp = nullptr;
  int* d_col = nullptr;
  void* d_w = nullptr;       // weights as given
  int* d_w2 = nullptr;       // reweighted (negative int32 weights only)
  long long* d_pot = nullptr;
  int* d_changed = nullptr;
  unsigned long long* d_edges = nullptr;
  void* D = nullptr;         // in core: n x n result (ld = n)
  void* buf[2] = {nullptr, nullptr};  // out of core: batch buffers (bat x n)
  void* h_D = nullptr;       // out of core: pinned n x n host result
  int* work = nullptr;
  unsigned* gbits = nullptr;
  long long nwords = 0;
  int grid = 0, G = 1, smem_bits = 0, nt = 256;
  size_t smem = 0;
  long long bat = 0;         // sources per batch (Alg. 2's bat)
  double delta = 0;
  bool ooc = false;
  long long r0 = 0, rc = 0;  // this rank's sources = result rows [r0, r0 + rc)
  bool sample = false;       // apsp_select's estimation handle (no result matrix)
  unsigned long long edges_last = 0;
  cudaStream_t d2h = nullptr;
  cudaEvent_t computed[2] = {nullptr, nullptr}, stored[2] = {nullptr, nullptr};
};

Jn* J_(Handle* h) { return static_cast<Jn*>(h->jn); }

template <typename T, int NT, int G>
cudaError_t launch_v(const MsspArgs<T>& a, int grid, size_t smem, cudaStream_t s) {
  auto k = mssp_kernel<T, NT, G>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k<<<grid, NT, smem, s>>>(a);
  return cudaGetLastError();
}

template <typename T, int NT, int G>
int occ_v(size_t smem) {
  auto k = mssp_kernel<T, NT, G>;
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) return 0;
  int nb = 0;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k, NT, smem) == cudaSuccess ? nb : 0;
}

// one (NT, G) instantiation: launch it (grid > 0) or report its occupancy (grid == 0)
template <typename T, int NT>
int dispatch_g(const MsspArgs<T>* a, int G, int grid, size_t smem, cudaStream_t s, cudaError_t* err) {
#define JN_CASE(g)                                                   \
  case g:                                                            \
    if (grid == 0) return occ_v<T, NT, g>(smem);                     \
    *err = launch_v<T, NT, g>(*a, grid, smem, s);                    \
    return 0;
  switch (G) {
    JN_CASE(1) JN_CASE(2) JN_CASE(4) JN_CASE(8) JN_CASE(16) default: JN_CASE(32)
  }
#undef JN_CASE
}

template <typename T>
cudaError_t launch_mssp(const MsspArgs<T>& a, int nt, int G, int grid, size_t smem, cudaStream_t s) {
  cudaError_t e = cudaSuccess;
  if (nt == 1024) dispatch_g<T, 1024>(&a, G, grid, smem, s, &e);
  else dispatch_g<T, 256>(&a, G, grid, smem, s, &e);
  return e;
}

template <typename T>
int occupancy(int nt, int G, size_t smem) {
  cudaError_t e = cudaSuccess;
  return nt == 1024 ? dispatch_g<T, 1024>(nullptr, G, 0, smem, nullptr, &e)
                    : dispatch_g<T, 256>(nullptr, G, 0, smem, nullptr, &e);
}

template <typename T>
MsspArgs<T> make_args(Handle* h, long long s0, long long s1, T* out, long long row_base) {
  Jn* j = J_(h);
  MsspArgs<T> a;
  a.n = h->n;
  a.rp = j->d_rp;
  a.col = j->d_col;
  a.w = j->d_w2 ? reinterpret_cast<const T*>(j->d_w2) : static_cast<const T*>(j->d_w);
  a.src_begin = s0;
  a.src_end = s1;
  a.out = out;
  a.row_base = row_base;
  a.ld = h->n;
  a.work = j->work;
  a.gbits = j->gbits;
  a.nwords = j->nwords;
  a.smem_bits = j->smem_bits;
  a.delta = (T)j->delta;
  a.pot = j->d_pot;
  a.edges = j->d_edges;
  return a;
}

apsp_status reweight(Handle* h) {
  Jn* j = J_(h);
  apsp_status st;
  const long long n = h->n;
  if ((st = h->cuda(cudaMemsetAsync(j->d_pot, 0, n * sizeof(long long), h->stream), "memset pot"))) return st;
  const int grid = (int)std::min<long long>((n + 255) / 256, 148 * 8);
  // Bellman–Ford from a virtual source joined to every vertex by 0-weight arcs:
  // without a negative cycle it settles within n sweeps; a change in sweep n+1 means a cycle
  int changed = 1;
  long long sweeps = 0;
  h->ev_begin(1);
  while (changed) {
    if (sweeps > n) {
      h->ev_end(0);
      return h->fail(APSP_ENEGCYCLE, "negative cycle detected (Bellman-Ford reweighting): distances are unspecified");
    }
    if ((st = h->cuda(cudaMemsetAsync(j->d_changed, 0, sizeof(int), h->stream), "memset"))) return st;
    bf_sweep_kernel<<<grid, 256, 0, h->stream>>>(n, j->d_rp, j->d_col, static_cast<const int*>(j->d_w), j->d_pot,
                                                 j->d_changed);
    if ((st = h->cuda(cudaGetLastError(), "bf_sweep"))) return st;
    if ((st = h->cuda(cudaMemcpyAsync(&changed, j->d_changed, sizeof(int), cudaMemcpyDeviceToHost, h->stream),
                      "D2H changed")))
      return st;
    if ((st = h->cuda(cudaStreamSynchronize(h->stream), "bf sync"))) return st;
    ++sweeps;
  }
  reweight_kernel<<<grid, 256, 0, h->stream>>>(n, j->d_rp, j->d_col, static_cast<const int*>(j->d_w), j->d_pot,
                                               j->d_w2);
  h->ev_end(0);
  return h->cuda(cudaGetLastError(), "reweight");
}

template <typename T>
apsp_status run_t(Handle* h) {
  Jn* j = J_(h);
  apsp_status st;
  const long long n = h->n;
  if (j->d_w2 && (st = reweight(h))) return st;
  if ((st = h->cuda(cudaMemsetAsync(j->d_edges, 0, sizeof(unsigned long long), h->stream), "memset"))) return st;
  if (!j->ooc) {
    MsspArgs<T> a = make_args<T>(h, j->r0, j->r0 + j->rc, static_cast<T*>(j->D), j->r0);
    h->ev_begin(2);
    if ((st = h->cuda(launch_mssp<T>(a, j->nt, j->G, j->grid, j->smem, h->stream), "mssp"))) return st;
    h->ev_end(0);
  } else {
    // Algorithm 2: batches of `bat` sources; batch b+1 runs while batch b is copied back
    const long long nb = (j->rc + j->bat - 1) / j->bat;
    for (long long b = 0; b < nb; ++b) {
      const int sl = (int)(b & 1);
      const long long s0 = j->r0 + b * j->bat, s1 = std::min(j->r0 + j->rc, s0 + j->bat);
      if ((st = h->cuda(cudaStreamWaitEvent(h->stream, j->stored[sl], 0), "wait"))) return st;
      MsspArgs<T> a = make_args<T>(h, s0, s1, static_cast<T*>(j->buf[sl]), s0);
      h->ev_begin(2);
      if ((st = h->cuda(launch_mssp<T>(a, j->nt, j->G, j->grid, j->smem, h->stream), "mssp"))) return st;
      h->ev_end(0);
      if ((st = h->cuda(cudaEventRecord(j->computed[sl], h->stream), "event"))) return st;
      if ((st = h->cuda(cudaStreamWaitEvent(j->d2h, j->computed[sl], 0), "wait"))) return st;
      h->ev_begin(3, j->d2h);
      if ((st = h->cuda(cudaMemcpyAsync(static_cast<char*>(j->h_D) + (size_t)(s0 - j->r0) * n * sizeof(T), j->buf[sl],
                                        (size_t)(s1 - s0) * n * sizeof(T), cudaMemcpyDeviceToHost, j->d2h),
                        "D2H batch")))
        return st;
      h->ev_end(0, j->d2h);
      if ((st = h->cuda(cudaEventRecord(j->stored[sl], j->d2h), "event"))) return st;
    }
    if ((st = h->cuda(cudaStreamSynchronize(j->d2h), "d2h sync"))) return st;
  }
  unsigned long long edges = 0;
  if ((st = h->cuda(cudaMemcpyAsync(&edges, j->d_edges, sizeof(edges), cudaMemcpyDeviceToHost, h->stream), "D2H")))
    return st;
  if ((st = h->cuda(cudaStreamSynchronize(h->stream), "mssp sync"))) return st;
  j->edges_last = edges;
  return APSP_OK;
}

}  // namespace

apsp_status jn_setup(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col, const void* w,
                     double delta, long long batch, bool sample) {
  apsp_status st;
  Jn* j = new Jn();
  h->jn = j;
  const long long n = h->n;
  const long long m = row_ptr[n];
  j->m = m;
  if (h->dtype == APSP_F32 && h->has_neg)
    return h->fail(APSP_EINVAL, "Johnson's algorithm takes fp32 weights >= 0 only (int32 negatives are reweighted)");
  // graph on the device ("the memory required for storing the graph be S")
  if ((st = h->cuda(cudaMalloc(&j->d_rp, (n + 1) * sizeof(long long)), "cudaMalloc csr"))) return st;
  if ((st = h->cuda(cudaMemcpy(j->d_rp, row_ptr, (n + 1) * sizeof(long long), cudaMemcpyHostToDevice), "H2D csr")))
    return st;
  const long long mm = std::max<long long>(m, 1);
  if ((st = h->cuda(cudaMalloc(&j->d_col, mm * sizeof(int)), "cudaMalloc csr"))) return st;
  if ((st = h->cuda(cudaMalloc(&j->d_w, mm * h->elem), "cudaMalloc csr"))) return st;
  if (m > 0) {
    if ((st = h->cuda(cudaMemcpy(j->d_col, col, m * sizeof(int), cudaMemcpyHostToDevice), "H2D csr"))) return st;
    if ((st = h->cuda(cudaMemcpy(j->d_w, w, m * h->elem, cudaMemcpyHostToDevice), "H2D csr"))) return st;
  }
  if (h->has_neg) {
    if ((st = h->cuda(cudaMalloc(&j->d_w2, mm * sizeof(int)), "cudaMalloc w2"))) return st;
    if ((st = h->cuda(cudaMalloc(&j->d_pot, n * sizeof(long long)), "cudaMalloc pot"))) return st;
  }
  if ((st = h->cuda(cudaMalloc(&j->d_changed, sizeof(int)), "cudaMalloc"))) return st;
  if ((st = h->cuda(cudaMalloc(&j->d_edges, sizeof(unsigned long long)), "cudaMalloc"))) return st;
  long long graph_bytes = (n + 1) * 8 + mm * (4 + (long long)h->elem) * (h->has_neg ? 2 : 1);

  // lanes per frontier vertex: average out-degree rounded up to a power of two
  const double avg_deg = n > 0 ? (double)m / n : 0.0;
  j->G = 1;
  while (j->G < 32 && j->G < avg_deg) j->G *= 2;
  // Delta: default = mean |weight| x 64 / degree^2, clamped to [mean/4, 4 mean]
  // (measured optimum: 4 x mean on the degree-4 grid of config 2, mean/4 on the
  // degree-16 ER graph of config 3; larger degrees favour narrower buckets because
  // every expansion already exposes many arcs)
  if (delta > 0) {
    j->delta = delta;
  } else {
    double sum = 0;
    if (h->dtype == APSP_I32) {
      for (long long e = 0; e < m; ++e) sum += std::fabs((double)static_cast<const int32_t*>(w)[e]);
    } else {
      for (long long e = 0; e < m; ++e) sum += std::fabs((double)static_cast<const float*>(w)[e]);
    }
    const double mean = m > 0 ? sum / m : 1.0;
    const double d = std::max(1.0, avg_deg);
    j->delta = std::max(1.0, mean * std::min(4.0, std::max(0.25, 64.0 / (d * d))));
    if (h->has_neg) j->delta *= 2;  // reweighted arcs are longer on average
  }
  if (h->dtype == APSP_I32) j->delta = std::floor(std::min(j->delta, (double)(1 << 29)));

  // flags: two bitmaps per block, in shared memory when they fit
  j->nwords = (n + 31) / 32;
  const size_t bits_bytes = 2 * (size_t)j->nwords * sizeof(unsigned);
  const size_t row_bytes = (size_t)n * h->elem;
  j->smem_bits = bits_bytes <= 96 * 1024 ? 1 : 0;
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->device);
  // threads per block: 256 (8 sources per SM in flight: small frontiers, e.g. road
  // graphs, need many concurrent sources) unless those 8 x 148 rows overflow ~96 MB
  // of the 126 MB L2 — relaxations are random atomics into the rows — then 1024
  // (2 per SM); measured on configs 2 and 3
  j->nt = (long long)sms * 8 * (long long)row_bytes > (96ll << 20) ? 1024 : 256;
  if (const char* e = std::getenv("APSP_JN_THREADS")) j->nt = std::atoi(e) == 1024 ? 1024 : 256;
  if (std::getenv("APSP_TEST_JN_GLOBAL_BITS")) j->smem_bits = 0;  // test hook (tests/test_gpu_johnson.py)
  j->smem = j->smem_bits ? bits_bytes : 0;
  int per_sm = h->dtype == APSP_I32 ? occupancy<int>(j->nt, j->G, j->smem) : occupancy<float>(j->nt, j->G, j->smem);
  if (per_sm < 1) return h->fail(APSP_ECUDA, "mssp kernel cannot be resident (smem %zu B)", j->smem);
  if (const char* e = std::getenv("APSP_JN_CTAS_PER_SM")) per_sm = std::max(1, std::min(per_sm, std::atoi(e)));
  j->grid = (int)std::max<long long>(1, std::min<long long>((long long)sms * per_sm, n));
  // per-block queues (4 x n) and global bitmaps
  const size_t work_bytes = (size_t)j->grid * 4 * std::max<long long>(n, 1) * sizeof(int);
  if ((st = h->cuda(cudaMalloc(&j->work, work_bytes), "cudaMalloc queues"))) return st;
  if (!j->smem_bits && (st = h->cuda(cudaMalloc(&j->gbits, (size_t)j->grid * bits_bytes), "cudaMalloc bits")))
    return st;
  graph_bytes += (long long)work_bytes + (j->smem_bits ? 0 : (long long)j->grid * bits_bytes);

  const long long avail = device_free_bytes(h->device, (long long)n * n * h->elem);
  if (avail < 0) return h->fail(APSP_ECUDA, "cudaMemGetInfo failed");
  const long long budget = cfg.device_budget_bytes > 0 ? cfg.device_budget_bytes - graph_bytes
                                                       : avail - (1ll << 30);
  // sources of this rank (world_size > 1): a contiguous block of result rows; the
  // SSSP instances are independent, so ranks need no communication at all
  {
    const long long per = (n + h->world - 1) / h->world;
    j->r0 = std::min<long long>(n, (long long)h->rank * per);
    j->rc = std::min<long long>(n, j->r0 + per) - j->r0;
  }
  const long long mat = j->rc * n * (long long)h->elem;
  j->ooc = cfg.force_out_of_core || mat > budget;
  h->n_pad = n;
  h->ld = n;
  h->rows_per_rank = n;
  if (sample) {
    // selector cost model (apsp_select): room for one batch of `grid` sources only
    j->sample = true;
    j->bat = j->grid;
    if ((st = h->cuda(cudaMalloc(&j->buf[0], (size_t)j->bat * n * h->elem), "cudaMalloc sample"))) return st;
    h->device_bytes = graph_bytes + (long long)j->bat * n * (long long)h->elem;
  } else if (!j->ooc) {
    if ((st = h->cuda(cudaMallocAsync(&j->D, std::max<long long>(mat, 4), h->stream), "cudaMalloc dist"))) return st;
    h->device_bytes = graph_bytes + mat;
  } else {
    // Alg. 2: bat sources per batch; two batch buffers (compute / copy back)
    const long long row = n * (long long)h->elem;
    long long bat = batch > 0 ? batch : std::max<long long>(1, std::min<long long>(budget / 2, 4ll << 30) / row);
    bat = std::max<long long>(1, std::min(bat, j->rc));
    j->bat = bat;
    for (int i = 0; i < 2; ++i)
      if ((st = h->cuda(cudaMalloc(&j->buf[i], bat * row), "cudaMalloc batch"))) return st;
    if ((st = h->cuda(cudaHostAlloc(&j->h_D, std::max<long long>(mat, 4), cudaHostAllocDefault), "cudaHostAlloc dist")))
      return st;
    h->host_bytes = mat;
    h->device_bytes = graph_bytes + 2 * bat * row;
    if ((st = h->cuda(cudaStreamCreateWithFlags(&j->d2h, cudaStreamNonBlocking), "stream"))) return st;
    for (int i = 0; i < 2; ++i) {
      cudaEventCreateWithFlags(&j->computed[i], cudaEventDisableTiming);
      cudaEventCreateWithFlags(&j->stored[i], cudaEventDisableTiming);
    }
  }
  return h->cuda(cudaStreamSynchronize(h->stream), "johnson setup sync");
}

// The paper's Johnson cost model (§IV-B-2): run k randomly chosen
// batches, T_comp = (n_b / k) * T. One batch = one wave of `grid` sources.
apsp_status jn_sample_seconds(Handle* h, int k, unsigned long long seed, double* seconds) {
  Jn* j = J_(h);
  apsp_status st;
  if (!j->sample) return h->fail(APSP_ESTATE, "not a sampling handle");
  const long long n = h->n;
  if (j->d_w2 && (st = reweight(h))) return st;
  const long long nb = (n + j->bat - 1) / j->bat;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  double total_ms = 0;
  unsigned long long x = seed * 6364136223846793005ull + 1442695040888963407ull;
  for (int i = 0; i <= k; ++i) {  // i = 0 is a warm-up batch (not counted)
    x = x * 6364136223846793005ull + 1442695040888963407ull;
    const long long b = (long long)((x >> 33) % (unsigned long long)nb);
    const long long s0 = b * j->bat, s1 = std::min(n, s0 + j->bat);
    cudaEventRecord(e0, h->stream);
    cudaError_t e = h->dtype == APSP_I32
        ? launch_mssp<int>(make_args<int>(h, s0, s1, static_cast<int*>(j->buf[0]), s0), j->nt, j->G, j->grid,
                           j->smem, h->stream)
        : launch_mssp<float>(make_args<float>(h, s0, s1, static_cast<float*>(j->buf[0]), s0), j->nt, j->G, j->grid,
                             j->smem, h->stream);
    if ((st = h->cuda(e, "mssp sample"))) return st;
    cudaEventRecord(e1, h->stream);
    if ((st = h->cuda(cudaEventSynchronize(e1), "sample sync"))) return st;
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    if (i > 0) total_ms += ms * (double)j->bat / (double)(s1 - s0);  // a ragged last batch counts as a full one
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  *seconds = (double)nb / k * total_ms * 1e-3;
  return APSP_OK;
}

apsp_status jn_reinit(Handle* h) {
  h->fw_done = false;
  h->canonical = true;
  return APSP_OK;
}

apsp_status jn_run(Handle* h) { return h->dtype == APSP_I32 ? run_t<int>(h) : run_t<float>(h); }

apsp_status jn_get_rows(Handle* h, long long r0, long long cnt, void* out, long long ld_out) {
  Jn* j = J_(h);
  if (!h->fw_done) return h->fail(APSP_ESTATE, "Johnson handle: apsp_solve first");
  if (r0 < j->r0 || r0 + cnt > j->r0 + j->rc)
    return h->fail(APSP_EINVAL, "get_dist: rows [%lld, %lld) are not this rank's [%lld, %lld)", r0, r0 + cnt, j->r0,
                   j->r0 + j->rc);
  r0 -= j->r0;
  const size_t es = h->elem;
  if (j->ooc) {
    for (long long r = 0; r < cnt; ++r)
      memcpy(static_cast<char*>(out) + (size_t)r * ld_out * es,
             static_cast<const char*>(j->h_D) + (size_t)(r0 + r) * h->n * es, (size_t)h->n * es);
    return APSP_OK;
  }
  apsp_status st;
  if ((st = h->cuda(cudaMemcpy2DAsync(out, ld_out * es, static_cast<const char*>(j->D) + (size_t)r0 * h->n * es,
                                      h->n * es, h->n * es, cnt, cudaMemcpyDeviceToHost, h->stream),
                    "get rows")))
    return st;
  return h->cuda(cudaStreamSynchronize(h->stream), "get rows sync");
}

void jn_local_rows(const Handle* h, long long* r0, long long* rc) {
  const Jn* j = static_cast<const Jn*>(h->jn);
  *r0 = j ? j->r0 : 0;
  *rc = j ? j->rc : h->n;
}

long long jn_edges(const Handle* h) { return h->jn ? (long long)static_cast<const Jn*>(h->jn)->edges_last : 0; }

void jn_free(Handle* h) {
  Jn* j = J_(h);
  if (!j) return;
  if (j->d2h) cudaStreamSynchronize(j->d2h);
  if (h->stream && j->D) {
    cudaFreeAsync(j->D, h->stream);
    cudaStreamSynchronize(h->stream);
  }
  for (int i = 0; i < 2; ++i) {
    if (j->computed[i]) cudaEventDestroy(j->computed[i]);
    if (j->stored[i]) cudaEventDestroy(j->stored[i]);
    cudaFree(j->buf[i]);
  }
  if (j->d2h) cudaStreamDestroy(j->d2h);
  if (j->h_D) cudaFreeHost(j->h_D);
  for (void* p : {(void*)j->d_rp, (void*)j->d_col, j->d_w, (void*)j->d_w2, (void*)j->d_pot, (void*)j->d_changed,
                  (void*)j->d_edges, (void*)j->work, (void*)j->gbits})
    cudaFree(p);
  delete j;
  h->jn = nullptr;
}

}  // namespace apsp
