// apsp_fw_dataflow.cu — the whole single-GPU blocked Floyd–Warshall (every
// round, all three phases of PAPER.md:62) as ONE persistent dataflow kernel.
//
// Why: with one launch per phase the chip idles at every launch boundary
// (wave tail, the partial wave of the next round's panels, launch gaps, the
// phase-1 tile on the critical path of every round). Here 2 CTAs of 256
// threads per SM pull tasks (one 128x128 tile update each) from a global
// queue in a fixed dependency-respecting order and wait on per-tile flags, so
// rounds overlap (round k+1's panels are computed while round k's phase 3
// drains) and no SM waits for a wave to finish.
// Measured on cfg2 (n=16384, int32): 0.887 of the DPX peak vs 0.846 for the
// launch-per-phase schedule (profiles/). Two CTAs per SM of one
// 256-thread group each measured far better than one CTA of two groups
// (0.825; DF_GROUPS=2 keeps that variant compilable for experiments).
//
// Tasks of round k (nb = n/128 tile rows):
//   P1(k)       closure of A(k,k) (phase 1, Alg. 1 l.3)
//   P2(k; k,j)  A(k,j) = D (x) A(k,j), j != k  (phase 2 row panel, Alg. 1 l.7)
//   P2(k; i,k)  A(i,k) = A(i,k) (x) D, i != k  (phase 2 column panel, l.11)
//   P3(k; i,j)  A(i,j) = min(A(i,j), A(i,k) (x) A(k,j)), i,j != k  (phase 3, l.17)
// P1 and P2 also write their result to a panel buffer pbuf[k % 2] (diagonal,
// row-panel and column-panel tiles, 128x128 each, ld 128); P2 and P3 read the
// panels from there, so a later round may update A(i,k) in place while round
// k's readers still run (write-after-read on the matrix never arises).
//
// Flags (device ints, monotone within one solve, zeroed before the launch):
//   ver[i*nb+j]      rounds applied to tile (i,j)
//   diagready[p]     k+1 once P1(k) wrote pbuf[p] (p = k % 2)
//   rowready[p][j]   k+1 once P2(k; k,j) wrote pbuf[p]
//   colready[p][i]   k+1 once P2(k; i,k) wrote pbuf[p]
//   done2[k], done3[k]  completed P2 / P3 tasks of round k
// Dependencies: P1(k): ver(k,k) >= k and (k >= 2) done2[k-2] complete (pbuf
// diagonal reuse); P2(k): ver >= k, diagready >= k+1, (k >= 2) done3[k-2]
// complete (pbuf panel reuse); P3(k): ver >= k, rowready/colready >= k+1.
//
// Queue order (one global counter): P1(0), seg(0), ..., seg(nb-1), tail, where
//   seg(k) = [G3R(k-1)[0:delay], G2(k), G3R(k-1)[delay:], G3L(k)[0], P1(k+1), G3L(k)[1:]]
//   G2(k)  = the 2(nb-1) panel tasks of round k
//   G3L(k) = round-k phase 3 on row/column k+1, tile (k+1,k+1) first
//   G3R(k) = the other round-k phase-3 tiles, row/column k+2 first
//   tail   = G3R(nb-1)  (the last round's whole phase 3)
// Every task's dependencies are earlier in this order and a group finishes a
// task before it takes the next one, so the task with the smallest index
// that is not done always has its dependencies met and a running group:
// the kernel cannot deadlock, whatever the number of resident CTAs.
//
// The tile engine is the min-plus kernel's (apsp_kernels.cu): 8x8 outputs per
// thread, 32-deep chunks through a 3-stage cp.async pipeline with full/empty
// mbarriers; here the chunk stream of a CTA is continuous across its tasks
// (stage and barrier parity carry over), and the C tile is fetched into the
// two free stages during the last chunk.
// Bookkeeping per task: the SCH thread dequeues the next task, decodes it and
// checks its flags (relaxed loads + fence.acquire) during chunk 1, so the next
// task usually starts without waiting; the SIG thread publishes a finished
// task (fence.release, then the flags) right after the task's last barrier.
#include "apsp_kernels.cuh"
#include "apsp_df_common.cuh"

#include <cuda_runtime.h>
#include <climits>
#include <cstdlib>
#include <cstdint>
#include <cstring>
#include <vector>

namespace apsp {
namespace {

#ifndef DF_GROUPS
#define DF_GROUPS 1
#endif
constexpr int BM = 128, BN = 128, BK = 32, GNT = 256, GROUPS = DF_GROUPS, STAGES = 3;
constexpr int CTAS_PER_SM = 2 / GROUPS;  // two groups per SM either way
// single GPU: the two-round (pair) queue by default for int32 from nb = kPairMinNb tile rows
// (decode2). Measured against the one-round kernel (profiles/r02_pair_ab.txt): nb = 128 -1.8 %,
// nb = 256 +0.1 %, nb = 512 (config 3) +0.8 %; fp32 nb = 256 -0.8 % (one-round kept)
constexpr bool kPairDefault = true;
constexpr int kPairMinNb = 384;
// Stage = A chunk stored transposed, As[kk][r] (32 x 128), then B chunk
// Bs[kk][c] (32 x 128): every operand read is one 16-byte vector per 4 rows or
// columns (4 shared loads per 64 relaxations); a C half-tile (64 x 128) fits too.
constexpr int ALD = BM, BLD = BN, CLD = BN;
constexpr int STAGE_ELEMS = BK * ALD + BK * BLD;  // 8192 words
constexpr int TILE_ELEMS = BM * BN;
// Bookkeeping is spread over lanes 0 of three warps of a group, so no warp
// carries more than one latency (a warp that lags delays the group's barriers):
constexpr int SIG = 32;  // publishes the group's finished task (release fence + flags)
constexpr int SCH = 64;  // dequeues the next task, decodes it, reads its flags, fills its slot
static_assert(64 * CLD <= STAGE_ELEMS, "half a C tile must fit one stage");

template <typename T> struct DV;
template <> struct DV<int> {
  using V4 = int4;
  static __device__ __forceinline__ int inf() { return 0x3FFFFFFF; }
  static __device__ __forceinline__ int relax(int a, int b, int c) { return __viaddmin_s32(a, b, c); }
  static __device__ __forceinline__ int vmin(int a, int b) { return min(a, b); }
};
template <> struct DV<float> {
  using V4 = float4;
  static __device__ __forceinline__ float inf() { return __int_as_float(0x7f800000); }
  static __device__ __forceinline__ float relax(float a, float b, float c) { return fminf(c, __fadd_rn(a, b)); }
  static __device__ __forceinline__ float vmin(float a, float b) { return fminf(a, b); }
};

// named barrier of one 256-thread group (id 0 is __syncthreads)
__device__ __forceinline__ void gbar(int g) { asm volatile("bar.sync %0, %1;" ::"r"(g + 1), "r"(GNT) : "memory"); }

constexpr int kMaxRanks = 8;  // one node

template <typename T>
struct DFArgs {
  T* D;            // this rank's rows (all n_pad rows on one GPU), row-major, ld
  long long ld;
  int nb;          // tile rows / columns of the whole matrix
  T* pbuf;         // 2 parities x (2 + nb + nl) tiles of 128x128: [0] diagonal, [1] its transpose,
                   // [2 + j] row panel, [2 + nb + il] column panel of local tile row il (transposed)
  int* ver;        // [nl][nb] rounds applied to each local tile
  int* diagready;  // [2]
  int* rowready;   // [2][nb]
  int* colready;   // [2][nl]
  int* done2;      // [nb]
  int* done3;      // [nb]
  unsigned long long* counter;
  int* negflag;
  long long total;   // tasks in this rank's queue (nb^3 on one GPU)
  long long delay;   // G3R tasks placed before G2 in a segment
  long long stagger; // clock cycles group 1 waits before its first task
  unsigned long long* prof;  // optional [CTAs x GROUPS x 8] cycle counters (thread 0 of each group)
  // 1-D block-row shard over P ranks (sharded kernel only; P = 1, q = 0, nl = nb otherwise):
  // rank q owns tile rows [q*nl, (q+1)*nl); the owner of round k writes the closed diagonal
  // block and the row panel straight into every rank's pbuf (peer stores over NVLink) and
  // raises their flags; owners read every rank's done2/done3 before reusing a parity.
  int P, q, nl;
  int npar;   // panel-copy parities: 2 (sharded kernel), 4 (single GPU: the pair schedule needs them)
  int pairq;  // single GPU: 1 = the two-round queue (decode2, T_PAIR tasks), 0 = decode
  const long long* segstart;  // [nb + 1] queue position of segment k (k = nb: the last round's phase 3)
  T* peer_pbuf[kMaxRanks];    // pbuf of every rank (peer_pbuf[q] == pbuf)
  int* peer_base[kMaxRanks];  // flag block of every rank (== its counter address)
};

// panel copies of round k (parity k % npar), 128x128 tiles with ld 128:
//   D = A(k,k) closed, D^T, row panel A(k,j), column panel A(i,k) transposed
template <typename T>
__device__ __forceinline__ T* pb_diag(const DFArgs<T>& a, int k) {
  return a.pbuf + (long long)(k & (a.npar - 1)) * (2 + a.nb + a.nl) * TILE_ELEMS;
}
template <typename T>
__device__ __forceinline__ T* pb_diagT(const DFArgs<T>& a, int k) {
  return pb_diag(a, k) + TILE_ELEMS;
}
template <typename T>
__device__ __forceinline__ T* pb_row(const DFArgs<T>& a, int k, int j) {
  return pb_diag(a, k) + (long long)(2 + j) * TILE_ELEMS;
}
template <typename T>
__device__ __forceinline__ T* pb_colT(const DFArgs<T>& a, int k, int i) {  // i: global tile row (local to q)
  return pb_diag(a, k) + (long long)(2 + a.nb + (i - a.q * a.nl)) * TILE_ELEMS;
}
// the same address in rank r's flag block / pbuf
template <typename T>
__device__ __forceinline__ int* peer_flag(const DFArgs<T>& a, int r, const int* local) {
  return a.peer_base[r] + (local - reinterpret_cast<const int*>(a.counter));
}
template <typename T>
__device__ __forceinline__ T* peer_pb(const DFArgs<T>& a, int r, const T* local) {
  return a.peer_pbuf[r] + (local - a.pbuf);
}

// ---- sharded queue (rank q of P): segments as in decode() (apsp_df_common.cuh), restricted to
// the local tile rows; segment starts come from the host (fw_dataflow_sharded_segments).
//   pre        P1(0) if q owns row 0
//   seg(k)     [G3R(k-1)[0:d], G2(k), G3R(k-1)[d:], G3Lx(k)]   (k >= 1 parts exist only if defined)
//   tail       round nb-1's phase 3
//   G2(k)      owner: P2R(k, j != k); every rank: P2C(k, local i != k)
//   G3Lx(k)    owner of k+1: (k+1,k+1), P1(k+1), row k+1 (j not in {k,k+1}), local column k+1;
//              others: local column k+1 (i != k)
//   G3R(k)     local rows not in {k,k+1} x columns not in {k,k+1}, banded
// Every cross-rank dependency points to an earlier segment or, inside segment k, from G3Lx(k)
// to G2(k): with the same part order on every rank no cycle exists.
__host__ __device__ __forceinline__ int loc_of(int k, int q, int nl) { return (k / nl) == q ? k - q * nl : -1; }
__host__ __device__ __forceinline__ int lrow(int x, int e0, int e1) {  // x-th local row skipping local e0, e1 (-1 none)
  const int s0 = (e0 >= 0 && e1 >= 0) ? (e0 < e1 ? e0 : e1) : (e0 >= 0 ? e0 : e1);
  const int s1 = (e0 >= 0 && e1 >= 0) ? (e0 < e1 ? e1 : e0) : -1;
  return skip3(x, s0, s1, -1);
}
__host__ __device__ __forceinline__ long long g3r_size_sh(int nb, int nl, int q, int k) {
  const int l0 = loc_of(k, q, nl) >= 0, l1 = loc_of(k + 1, q, nl) >= 0;
  return (long long)(nl - l0 - l1) * (nb - 2);
}
__host__ __device__ __forceinline__ long long g2_size_sh(int nb, int nl, int q, int k) {
  const int l0 = loc_of(k, q, nl) >= 0;
  return (long long)l0 * (nb - 1) + (nl - l0);
}
__host__ __device__ Task decode_sh(long long g, int nb, int nl, int q, long long delay, const long long* segstart) {
  Task t;
  const int base = q * nl;
  if (g < segstart[0]) { t.type = T_P1; t.k = 0; t.i = t.j = 0; return t; }
  int lo = 0, hi = nb;  // largest k with segstart[k] <= g
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (segstart[mid] <= g) lo = mid; else hi = mid - 1;
  }
  const int k = lo;
  long long x = g - segstart[k];
  t.type = T_P3;
  if (k == nb) {  // tail: round nb-1, local rows != nb-1 x columns != nb-1
    const int kl = loc_of(nb - 1, q, nl);
    int r, c;
    banded(x, nl - (kl >= 0), nb - 1, r, c);
    t.k = nb - 1; t.i = base + lrow(r, kl, -1); t.j = c;
    return t;
  }
  auto g3r = [&](int kk, long long y) {  // G3R(kk)
    const int l0 = loc_of(kk, q, nl), l1 = loc_of(kk + 1, q, nl);
    int r, c;
    banded(y, nl - (l0 >= 0) - (l1 >= 0), nb - 2, r, c);
    Task u;
    u.type = T_P3; u.k = kk; u.i = base + lrow(r, l0, l1); u.j = skip3(c, kk, kk + 1, -1);
    return u;
  };
  long long r3 = 0, d = 0;
  if (k >= 1) {
    r3 = g3r_size_sh(nb, nl, q, k - 1);
    d = delay < r3 ? delay : r3;
    if (x < d) return g3r(k - 1, x);
    x -= d;
  }
  const long long n2 = g2_size_sh(nb, nl, q, k);
  if (x < n2) {
    const int l0 = loc_of(k, q, nl);
    t.k = k;
    if (l0 >= 0) {
      if (x < nb - 1) { t.type = T_P2R; t.i = k; t.j = skip3((int)x, k, -1, -1); return t; }
      x -= nb - 1;
    }
    t.type = T_P2C; t.i = base + lrow((int)x, l0, -1); t.j = k;
    return t;
  }
  x -= n2;
  if (k >= 1) {
    if (x < r3 - d) return g3r(k - 1, d + x);
    x -= r3 - d;
  }
  // G3Lx(k), k <= nb-2
  const int l0 = loc_of(k, q, nl), l1 = loc_of(k + 1, q, nl);
  t.k = k;
  if (l1 >= 0) {
    if (x == 0) { t.i = k + 1; t.j = k + 1; return t; }
    if (x == 1) { t.type = T_P1; t.k = k + 1; t.i = t.j = k + 1; return t; }
    x -= 2;
    if (x < nb - 2) { t.i = k + 1; t.j = skip3((int)x, k, k + 1, -1); return t; }
    x -= nb - 2;
    t.i = base + lrow((int)x, l0, l1); t.j = k + 1;
    return t;
  }
  t.i = base + lrow((int)x, l0, -1); t.j = k + 1;
  return t;
}

// completed P2 / P3 tasks rank r runs in round k
__device__ __forceinline__ int cnt2_sh(int nb, int nl, int r, int k) {
  const int l0 = (k / nl) == r;
  return l0 * (nb - 1) + (nl - l0);
}
__device__ __forceinline__ int cnt3_sh(int nb, int nl, int r, int k) {
  const int l0 = (k / nl) == r;
  return (nl - l0) * (nb - 1);
}

// Dependencies of task t on rank q (one thread). Local flags, some of them written by the
// owner of the round over NVLink (diagready, rowready), plus for the owner's P1 / P2R the
// done counters of round k-2 on every rank (parity reuse of the panels it broadcasts).
template <typename T>
__device__ bool deps_met_sh(const DFArgs<T>& a, const Task& t) {
  const int nb = a.nb, nl = a.nl, k = t.k, p = k & 1;
  if (ld_relaxed_sys(a.ver + (long long)(t.i - a.q * nl) * nb + t.j) < k) return false;
  if (t.type == T_P3) {
    if (ld_relaxed_sys(a.rowready + p * nb + t.j) < k + 1) return false;
    if (ld_relaxed_sys(a.colready + p * nl + (t.i - a.q * nl)) < k + 1) return false;
  } else if (t.type == T_P2C) {
    if (ld_relaxed_sys(a.diagready + p) < k + 1) return false;
    if (k >= 2 && ld_relaxed_sys(a.done3 + k - 2) < cnt3_sh(nb, nl, a.q, k - 2)) return false;
  } else {
    if (t.type == T_P2R && ld_relaxed_sys(a.diagready + p) < k + 1) return false;
    if (k >= 2) {
      for (int r = 0; r < a.P; ++r) {
        const int* f = t.type == T_P1 ? a.done2 + k - 2 : a.done3 + k - 2;
        const int need = t.type == T_P1 ? cnt2_sh(nb, nl, r, k - 2) : cnt3_sh(nb, nl, r, k - 2);
        if (ld_relaxed_sys(peer_flag(a, r, f)) < need) return false;
      }
    }
  }
  asm volatile("fence.acquire.sys;" ::: "memory");  // (an acquire: no wait for this thread's own stores)
  return true;
}

// Publish task t on rank q (one thread, after the group barrier that follows its stores,
// including the peer stores of P1 / P2R): a system-scope fence, then the flags.
template <typename T>
__device__ void signal_done_sh(const DFArgs<T>& a, const Task& t) {
  const int nb = a.nb, nl = a.nl, k = t.k, p = k & 1;
  asm volatile("fence.release.sys;" ::: "memory");
  st_relaxed_sys(a.ver + (long long)(t.i - a.q * nl) * nb + t.j, k + 1);
  switch (t.type) {
    case T_P1:
      for (int r = 0; r < a.P; ++r) st_relaxed_sys(peer_flag(a, r, a.diagready + p), k + 1);
      break;
    case T_P2R:
      for (int r = 0; r < a.P; ++r) st_relaxed_sys(peer_flag(a, r, a.rowready + p * nb + t.j), k + 1);
      red_relaxed_sys_add(a.done2 + k, 1);
      break;
    case T_P2C:
      st_relaxed_sys(a.colready + p * nl + (t.i - a.q * nl), k + 1);
      red_relaxed_sys_add(a.done2 + k, 1);
      break;
    default: red_relaxed_sys_add(a.done3 + k, 1); break;
  }
}

// Single-GPU dependencies / publication with npar parities (the per-round panel copies of
// round k are rewritten by round k + npar) and the pair task T_PAIR (rounds k, k+1 of one tile).
template <typename T>
__device__ bool deps_single(const DFArgs<T>& a, const Task& t) {
  const int nb = a.nb, k = t.k, np = a.npar, p = k & (np - 1);
  // up to five flags: independent relaxed loads first (one round trip), then the tests
  const int* f0 = a.ver + (long long)t.i * nb + t.j;
  const int* f1;
  const int* f2;
  const int* f3 = f0;
  const int* f4 = f0;
  int v1, v2, v3 = INT_MIN, v4 = INT_MIN;
  if (t.type == T_P1) {
    f1 = a.done2 + (k >= np ? k - np : 0); v1 = k >= np ? 2 * (nb - 1) : INT_MIN;
    f2 = f1; v2 = v1;
  } else if (t.type == T_P3 || t.type == T_PAIR) {
    f1 = a.rowready + p * nb + t.j; v1 = k + 1;
    f2 = a.colready + p * nb + t.i; v2 = k + 1;
    if (t.type == T_PAIR) {
      const int p1 = (k + 1) & (np - 1);
      f3 = a.rowready + p1 * nb + t.j; v3 = k + 2;
      f4 = a.colready + p1 * nb + t.i; v4 = k + 2;
    }
  } else {
    f1 = a.diagready + p; v1 = k + 1;
    f2 = a.done3 + (k >= np ? k - np : 0); v2 = k >= np ? (nb - 1) * (nb - 1) : INT_MIN;
  }
  const int x0 = ld_relaxed(f0), x1 = ld_relaxed(f1), x2 = ld_relaxed(f2), x3 = ld_relaxed(f3), x4 = ld_relaxed(f4);
  if (x0 >= k && x1 >= v1 && x2 >= v2 && x3 >= v3 && x4 >= v4) {
    asm volatile("fence.acquire.gpu;" ::: "memory");  // (see deps_met)
    return true;
  }
  return false;
}
template <typename T>
__device__ void signal_single(const DFArgs<T>& a, const Task& t) {
  const int nb = a.nb, k = t.k, p = k & (a.npar - 1);
  asm volatile("fence.release.gpu;" ::: "memory");
  st_relaxed(a.ver + (long long)t.i * nb + t.j, t.type == T_PAIR ? k + 2 : k + 1);
  switch (t.type) {
    case T_P1: st_relaxed(a.diagready + p, k + 1); break;
    case T_P2R: st_relaxed(a.rowready + p * nb + t.j, k + 1); red_relaxed_add(a.done2 + k, 1); break;
    case T_P2C: st_relaxed(a.colready + p * nb + t.i, k + 1); red_relaxed_add(a.done2 + k, 1); break;
    case T_PAIR: red_relaxed_add(a.done3 + k, 1); red_relaxed_add(a.done3 + k + 1, 1); break;
    default: red_relaxed_add(a.done3 + k, 1); break;
  }
}

template <bool SH, bool PQ, typename T>
__device__ __forceinline__ Task decode_any(const DFArgs<T>& a, long long g) {
  // sharded: the segment starts are binary-searched in a shared-memory copy (the kernel
  // fills it after its stages): from global memory the ~log2(nb) dependent loads went to
  // L2 every time (each dependency check's acquire fence invalidates L1) and delayed the
  // decoding warp, and with it its CTA, by thousands of cycles per task
  extern __shared__ __align__(16) unsigned char smem_raw[];
  if constexpr (SH)
    return decode_sh(g, a.nb, a.nl, a.q, a.delay,
                     reinterpret_cast<const long long*>(smem_raw + GROUPS * STAGES * STAGE_ELEMS * sizeof(T)));
  else if constexpr (PQ) return decode2(g, a.nb, a.delay);  // the two-round queue
  else return decode(g, a.nb, a.delay);
}
template <bool SH, bool PQ, typename T>
__device__ __forceinline__ bool deps_any(const DFArgs<T>& a, const Task& t) {
  if constexpr (SH) return deps_met_sh(a, t);
  else if constexpr (PQ) return deps_single(a, t);  // 4 parities, T_PAIR
  else return deps_met(a, t);
}
// Phase 1 inside a group: in-place FW closure of one 128x128 tile (the same
// register blocking as phase1_kernel in apsp_kernels.cu); result also to out2.
// Sharded kernel: `peers` (npeer entries) also receive D at the same offset (peer stores).
template <typename T>
__device__ __noinline__ void group_phase1(T* tile, long long ld, T* out2, T* out2t, int* negflag, T* scratch, int g,
                                         int gtid, T* const* peers = nullptr, int npeer = 0) {
  using V4 = typename DV<T>::V4;
  T* rowbuf = scratch;            // [2][128]
  T* colbuf = scratch + 2 * 128;  // [2][128]
  const int tx = gtid & 15, ty = gtid >> 4;
  T acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    const V4 v0 = __ldcg(reinterpret_cast<const V4*>(tile + r * ld + tx * 4));
    const V4 v1 = __ldcg(reinterpret_cast<const V4*>(tile + r * ld + 64 + tx * 4));
    acc[i][0] = v0.x; acc[i][1] = v0.y; acc[i][2] = v0.z; acc[i][3] = v0.w;
    acc[i][4] = v1.x; acc[i][5] = v1.y; acc[i][6] = v1.z; acc[i][7] = v1.w;
  }
  bool neg = false;
#pragma unroll
  for (int half = 0; half < 2; ++half) {
    for (int q = 0; q < 16; ++q) {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int kk = half * 64 + q * 4 + u;
        const int p = u & 1;
        const int io = half * 4 + u;
        if (ty == q) {
          V4 x0, x1;
          x0.x = acc[io][0]; x0.y = acc[io][1]; x0.z = acc[io][2]; x0.w = acc[io][3];
          x1.x = acc[io][4]; x1.y = acc[io][5]; x1.z = acc[io][6]; x1.w = acc[io][7];
          *reinterpret_cast<V4*>(&rowbuf[p * 128 + tx * 4]) = x0;
          *reinterpret_cast<V4*>(&rowbuf[p * 128 + 64 + tx * 4]) = x1;
        }
        if (tx == q) {
          V4 y0, y1;
          y0.x = acc[0][io]; y0.y = acc[1][io]; y0.z = acc[2][io]; y0.w = acc[3][io];
          y1.x = acc[4][io]; y1.y = acc[5][io]; y1.z = acc[6][io]; y1.w = acc[7][io];
          *reinterpret_cast<V4*>(&colbuf[p * 128 + ty * 4]) = y0;
          *reinterpret_cast<V4*>(&colbuf[p * 128 + 64 + ty * 4]) = y1;
        }
        gbar(g);
        if (gtid == 0 && rowbuf[p * 128 + kk] < T(0)) neg = true;
        const V4 a0 = *reinterpret_cast<const V4*>(&colbuf[p * 128 + ty * 4]);
        const V4 a1 = *reinterpret_cast<const V4*>(&colbuf[p * 128 + 64 + ty * 4]);
        const V4 b0 = *reinterpret_cast<const V4*>(&rowbuf[p * 128 + tx * 4]);
        const V4 b1 = *reinterpret_cast<const V4*>(&rowbuf[p * 128 + 64 + tx * 4]);
        const T av[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const T bv[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[i][j] = DV<T>::relax(av[i], bv[j], acc[i][j]);
      }
    }
  }
  if (neg) *negflag = 1;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    V4 v0, v1;
    v0.x = acc[i][0]; v0.y = acc[i][1]; v0.z = acc[i][2]; v0.w = acc[i][3];
    v1.x = acc[i][4]; v1.y = acc[i][5]; v1.z = acc[i][6]; v1.w = acc[i][7];
    *reinterpret_cast<V4*>(tile + r * ld + tx * 4) = v0;
    *reinterpret_cast<V4*>(tile + r * ld + 64 + tx * 4) = v1;
    *reinterpret_cast<V4*>(out2 + r * BN + tx * 4) = v0;
    *reinterpret_cast<V4*>(out2 + r * BN + 64 + tx * 4) = v1;
    for (int e = 0; e < npeer; ++e) {
      *reinterpret_cast<V4*>(peers[e] + r * BN + tx * 4) = v0;
      *reinterpret_cast<V4*>(peers[e] + r * BN + 64 + tx * 4) = v1;
    }
  }
#pragma unroll
  for (int j = 0; j < 8; ++j) {  // D^T: column c of the block = 4 + 4 consecutive rows
    const int c = (j < 4) ? (tx * 4 + j) : (64 + tx * 4 + j - 4);
    V4 w0, w1;
    w0.x = acc[0][j]; w0.y = acc[1][j]; w0.z = acc[2][j]; w0.w = acc[3][j];
    w1.x = acc[4][j]; w1.y = acc[5][j]; w1.z = acc[6][j]; w1.w = acc[7][j];
    *reinterpret_cast<V4*>(out2t + c * BM + ty * 4) = w0;
    *reinterpret_cast<V4*>(out2t + c * BM + 64 + ty * 4) = w1;
  }
}

// Operands of a group's current min-plus task, written by the group's thread 0
// before the task-start barrier (kept in shared memory, not in registers).
template <typename T>
struct GDesc {
  const T* A;  // a_rows = 0: A^T as 128 rows kk of 128 r (ld lda); 1: A itself, rows r (transposed on load)
  const T* B;  // rows kk of 128 c (ld ldb)
  const T* Cin;
  T* Cout;
  T* Cout2;  // panel copy (ld 128) or nullptr; c2t = 1: written transposed
  int lda, ldb, ldc;
  int a_rows, c2t;
  int bulk;  // 1: A and B chunks are contiguous 16 KB blocks (panel copies): one thread copies them
  int bcast; // sharded P2R: Cout2 also goes to every other rank's pbuf (same offset)
};

// The second round of a pair task (kept out of GDesc: the engine's shared-memory descriptor
// layout is performance-sensitive, measured -2 % when these fields sat inside it)
template <typename T>
struct GPair {
  const T* A2;  // round k+1's operands (chunks 4..7), same layout as GDesc::A / B
  const T* B2;
  int nk;       // chunks of depth 32: 4 (one round), 8 (pair task: rounds k and k+1)
};


// A group's task slot (shared memory, double-buffered by iteration parity):
// the task index, its decoded form, the operands of a min-plus task and
// whether its dependencies were already seen met. Thread 0 fills the slot of
// the next iteration while the current task runs.
template <typename T, bool PQ>
struct Slot {
  long long t;
  Task tk;
  GDesc<T> d;
  int ready;
  int pref;  // fp32: chunk 0 already issued by the previous task (during its last chunk)
};
template <typename T>
struct Slot<T, true> {  // the pair kernel's slot: + the second round of a pair task
  long long t;
  Task tk;
  GDesc<T> d;
  int ready;
  int pref;
  GPair<T> p2;
};

// the pair data of a slot (nullptr in the one-round kernels)
template <typename T>
__device__ __forceinline__ GPair<T>* slot_p2(Slot<T, true>* s) { return &s->p2; }
template <typename T>
__device__ __forceinline__ GPair<T>* slot_p2(Slot<T, false>*) { return nullptr; }


template <typename T>
__device__ void fill_desc(const DFArgs<T>& a, const Task& tk, GDesc<T>& d, GPair<T>* p2 = nullptr) {
  const int k = tk.k;
  T* const tile = a.D + (long long)(tk.i - a.q * a.nl) * BM * a.ld + (long long)tk.j * BN;
  d.Cin = tile; d.Cout = tile; d.ldc = (int)a.ld;
  d.a_rows = 0; d.c2t = 0; d.bulk = 0; d.bcast = 0;
  if (p2) p2->nk = BM / BK;
  if (tk.type == T_P2R) {         // A(k,j) = D (x) A(k,j)
    d.A = pb_diagT(a, k); d.lda = BM; d.B = tile; d.ldb = (int)a.ld; d.Cout2 = pb_row(a, k, tk.j);
    d.bcast = a.P > 1;
  } else if (tk.type == T_P2C) {  // A(i,k) = A(i,k) (x) D; the copy goes to the transposed column panel
    d.A = tile; d.lda = (int)a.ld; d.a_rows = 1; d.B = pb_diag(a, k); d.ldb = BN;
    d.Cout2 = pb_colT(a, k, tk.i); d.c2t = 1;
  } else {                        // A(i,j) = min(A(i,j), A(i,k) (x) A(k,j)) from the panel copies
    d.A = pb_colT(a, k, tk.i); d.lda = BM; d.B = pb_row(a, k, tk.j); d.ldb = BN; d.Cout2 = nullptr;
    if (p2 && tk.type == T_PAIR) {  // then round k+1: min(., A(i,k+1) (x) A(k+1,j)) (min is order-free)
      p2->A2 = pb_colT(a, k + 1, tk.i); p2->B2 = pb_row(a, k + 1, tk.j); p2->nk = 2 * (BM / BK);
    }
#ifndef DF_NOBULK
    d.bulk = 1;
#endif
  }
}

// One 128x128 min-plus tile update of depth 128 by a group:
//   Cout = min(Cin, A (x) B)  (and Cout2 = the same, ld 128, if non-null)
// `c0` is the group's running chunk counter (stage = chunk % 3, barrier
// parity = (chunk / 3) & 1); the task uses chunks c0 .. c0+3.
// The SCH thread also prepares the slot of the next task `nxt` during chunk 1:
// decoded, operands filled, dependencies checked once.
// Inlined into the kernel (default): ptxas then schedules the shared-memory operand
// loads a step ahead across the whole loop (measured: fp32 +2.4 %, int32 neutral;
// packed16 +8 % in apsp_fw_dataflow16.cu). -DDF_NOINLINE keeps it a separate function.
#ifndef DF_NOINLINE
#define DF_MP_INLINE __forceinline__
#else
#define DF_MP_INLINE __noinline__
#endif
template <bool SH, bool PQ, typename T, int NK>
__device__ DF_MP_INLINE void group_minplus(const GDesc<T>* d, const GPair<T>* p2, T* stage0, unsigned full0,
                                           unsigned empty0, unsigned c0,
                                           int gtid, int g, const DFArgs<T>* args, long long nxt,
                                           Slot<T, PQ>* ns, int pref) {
  using V4 = typename DV<T>::V4;
  // NK = 4 chunks of depth 32 (one round), 8 for a pair task (compile-time: two instantiations);
  // NK = 0: the pair task's runtime depth (one engine copy, APSP_DF_PQ_ONE_ENGINE A/B builds)
  const int nkc = NK ? NK : p2->nk;
#define NK nkc
  // fp32: fold the top half of C before the last chunk and issue the next phase-3 task's
  // chunk 0 into the freed stage (measured +1.2 % for fp32, -1.7 % for int32, so int32 keeps
  // the C fetch into both free stages during the last chunk and the fold at the end)
#ifdef DF_XPREF_ALL
  constexpr bool kXpref = true;
#else
  constexpr bool kXpref = sizeof(T) == 4 && T(0.5) != T(0);
#endif
  const int lane = gtid & 31;
  const int tx = gtid & 15, ty = gtid >> 4;
  // Chunk c of A and B into stage `stage`, completing one phase of full[stage]
  // (one arrival + transaction bytes). Panel-copy tasks (phase 3, 62 in 64
  // tasks): thread 0 issues two 16 KB bulk copies, after waiting for the
  // stage's previous chunk to be released (wait_G: that chunk, or -1). Phase-2
  // tasks: every thread copies its share (the column-panel task transposes A
  // through registers), then one barrier and one arrival.
  const bool bulk = d->bulk;
  auto load_chunk = [&](int stage, int c, long long wait_G) {
    T* st = stage0 + stage * STAGE_ELEMS;
    if (bulk) {
      if (gtid == 0) {
        if (wait_G >= 0) mb_wait(empty0 + 8 * stage, ((unsigned)wait_G / STAGES) & 1);
        // generic-proxy -> async-proxy ordering: the stage was last read by generic loads
        // (shared::cta), and the panel copies were written by other CTAs (or peer GPUs) with
        // generic stores that this CTA acquired before the task started (global; once per task)
        if (c == 0) asm volatile("fence.proxy.async.global;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        const unsigned bytes = BK * BM * (unsigned)sizeof(T);
        mb_expect_tx(full0 + 8 * stage, 2 * bytes);
        const int cr = c & 3;  // chunk within its round (pair tasks: chunks 4..7 from round k+1)
        const T* const Ar = (NK == 4 || c < 4) ? d->A : p2->A2;
        const T* const Br = (NK == 4 || c < 4) ? d->B : p2->B2;
        bulk_g2s(saddr(st), Ar + (long long)cr * BK * BM, bytes, full0 + 8 * stage);
        bulk_g2s(saddr(st + BK * ALD), Br + (long long)cr * BK * BN, bytes, full0 + 8 * stage);
      }
      return;
    }
    if (wait_G >= 0) mb_wait(empty0 + 8 * stage, ((unsigned)wait_G / STAGES) & 1);
    const int ldb = d->ldb;
    const T* bg = d->B + ((gtid >> 5) + c * BK) * (long long)ldb + (gtid & 31) * 4;
    T* const bdst = st + BK * ALD + (gtid >> 5) * BLD + (gtid & 31) * 4;
    if (!d->a_rows) {  // A^T rows (panel copies): a 32 x 128 block, like B
      const int lda = d->lda;
      const T* ag = d->A + ((gtid >> 5) + c * BK) * (long long)lda + (gtid & 31) * 4;
      T* const adst = st + (gtid >> 5) * ALD + (gtid & 31) * 4;
#pragma unroll
      for (int q = 0; q < 4; ++q) cp16(adst + q * 8 * ALD, ag + q * 8 * lda);
#pragma unroll
      for (int q = 0; q < 4; ++q) cp16(bdst + q * 8 * BLD, bg + q * 8 * ldb);
      mb_cp_arrive_inc(full0 + 8 * stage);  // the phase also waits for these copies
    } else {  // A rows r (column-panel tasks): transpose through registers
      const int r = gtid & (BM - 1), h = gtid >> 7;
      const T* ag = d->A + (long long)r * d->lda + c * BK + h * 16;
      V4 v[4];
#pragma unroll
      for (int m = 0; m < 4; ++m) v[m] = __ldcg(reinterpret_cast<const V4*>(ag + 4 * m));
      V4 w[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) w[q] = __ldcg(reinterpret_cast<const V4*>(bg + q * 8 * ldb));
#pragma unroll
      for (int m = 0; m < 4; ++m) {
        st[(h * 16 + 4 * m + 0) * ALD + r] = v[m].x;
        st[(h * 16 + 4 * m + 1) * ALD + r] = v[m].y;
        st[(h * 16 + 4 * m + 2) * ALD + r] = v[m].z;
        st[(h * 16 + 4 * m + 3) * ALD + r] = v[m].w;
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) *reinterpret_cast<V4*>(bdst + q * 8 * BLD) = w[q];
    }
    gbar(g);
    if (gtid == 0) mb_arrive(full0 + 8 * stage);
  };
  if (!pref) load_chunk((int)(c0 % STAGES), 0, -1);  // (the previous task ended with a barrier)
  load_chunk((int)((c0 + 1) % STAGES), 1, -1);

  T acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = DV<T>::inf();
  // the C tile goes to the stages of chunks c0+NK-3 and c0+NK-2 (free during the last chunk)
  const unsigned g_lo = c0 + NK - 3, g_hi = c0 + NK - 2;
  const int s_lo = (int)(g_lo % STAGES), s_hi = (int)(g_hi % STAGES);

#pragma unroll 1
  for (int c = 0; c < NK; ++c) {
    const unsigned G = c0 + c;
    const int s = (int)(G % STAGES);
    if (!kXpref && c == NK - 1) {
      // C goes to the stages of chunks c0+1 and c0+2 once every warp released them
      mb_wait(empty0 + 8 * s_lo, (g_lo / STAGES) & 1);
      mb_wait(empty0 + 8 * s_hi, (g_hi / STAGES) & 1);
      const int ldc = d->ldc;
      const T* cg = d->Cin + (gtid >> 5) * ldc + (gtid & 31) * 4;
      const int cd = (gtid >> 5) * CLD + (gtid & 31) * 4;
      T* const cs_lo = stage0 + s_lo * STAGE_ELEMS;
      T* const cs_hi = stage0 + s_hi * STAGE_ELEMS;
#pragma unroll
      for (int q = 0; q < 8; ++q) cp16(cs_lo + cd + q * 8 * CLD, cg + q * 8 * ldc);
#pragma unroll
      for (int q = 0; q < 8; ++q) cp16(cs_hi + cd + q * 8 * CLD, cg + (64 + q * 8) * ldc);
      cp_commit();
    }
    // fp32 (kXpref): C rows 0-63 go to stage s_lo as soon as chunk g_lo released it (start of chunk NK-2),
    // rows 64-127 to s_hi at the start of the last chunk. The top half is folded into the
    // accumulators right before the last chunk (min is order-free), which frees s_lo for the
    // NEXT task's chunk 0 (stage of chunk c0+4): thread 0 issues it then, if that task is a
    // phase-3 task whose dependencies were seen met, so its latency hides under this chunk.
    if (kXpref && c >= NK - 2) {
      const int sC = c == NK - 2 ? s_lo : s_hi;
      mb_wait(empty0 + 8 * sC, ((c == NK - 2 ? g_lo : g_hi) / STAGES) & 1);
      const int ldc = d->ldc;
      const T* cg = d->Cin + ((gtid >> 5) + (c == NK - 2 ? 0 : 64)) * (long long)ldc + (gtid & 31) * 4;
      const int cd = (gtid >> 5) * CLD + (gtid & 31) * 4;
      T* const cs = stage0 + sC * STAGE_ELEMS;
#pragma unroll
      for (int q = 0; q < 8; ++q) cp16(cs + cd + q * 8 * CLD, cg + q * 8 * ldc);
      cp_commit();
    }
    if (c == 1 && gtid == SCH) {  // the next task's slot
      ns->t = nxt;
      if (nxt < args->total) {
        const Task tn = decode_any<SH, PQ>(*args, nxt);
        ns->tk = tn;
        if (tn.type != T_P1) fill_desc(*args, tn, ns->d, slot_p2(ns));
        ns->ready = deps_any<SH, PQ>(*args, tn) ? 1 : 0;
      }
    }
    if (kXpref && c == NK - 1) {
      asm volatile("cp.async.wait_group 1;\n" ::: "memory");  // this thread's C-top copies
      gbar(g);
      const T* const cs_lo = stage0 + s_lo * STAGE_ELEMS;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const T* crow = cs_lo + (ty * 4 + i) * CLD;
        const V4 x0 = *reinterpret_cast<const V4*>(crow + tx * 4);
        const V4 x1 = *reinterpret_cast<const V4*>(crow + 64 + tx * 4);
        acc[i][0] = DV<T>::vmin(acc[i][0], x0.x); acc[i][1] = DV<T>::vmin(acc[i][1], x0.y);
        acc[i][2] = DV<T>::vmin(acc[i][2], x0.z); acc[i][3] = DV<T>::vmin(acc[i][3], x0.w);
        acc[i][4] = DV<T>::vmin(acc[i][4], x1.x); acc[i][5] = DV<T>::vmin(acc[i][5], x1.y);
        acc[i][6] = DV<T>::vmin(acc[i][6], x1.z); acc[i][7] = DV<T>::vmin(acc[i][7], x1.w);
      }
      gbar(g);  // s_lo read by every thread: free for the next task's chunk 0
      if (gtid == 0) {
        int pf = 0;
        if (ns->t < args->total && ns->ready && (ns->tk.type == T_P3 || (PQ && ns->tk.type == T_PAIR)) &&
            ns->d.bulk) {
          asm volatile("fence.proxy.async.global;" ::: "memory");  // acquired panel copies (see load_chunk)
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          const unsigned bytes = BK * BM * (unsigned)sizeof(T);
          T* const dst = stage0 + s_lo * STAGE_ELEMS;
          mb_expect_tx(full0 + 8 * s_lo, 2 * bytes);
          bulk_g2s(saddr(dst), ns->d.A, bytes, full0 + 8 * s_lo);
          bulk_g2s(saddr(dst + BK * ALD), ns->d.B, bytes, full0 + 8 * s_lo);
          pf = 1;
        }
        ns->pref = pf;
      }
    }
    mb_wait(full0 + 8 * s, (G / STAGES) & 1);
    const T* as = stage0 + s * STAGE_ELEMS;  // As[kk][r]
    const T* bs = as + BK * ALD;             // Bs[kk][c]
    if constexpr (sizeof(T) == 4 && T(0.5) != T(0)) {
      // fp32: two depth steps per accumulator update, FADD2 (a scalar broadcast
      // against a column pair) + FMNMX3 = 1 instruction per relaxation instead of
      // FADD + FMNMX. Every candidate a + b is still one RN add and min is exact,
      // so the result is bit-identical to the one-step update.
#pragma unroll
      for (int kk = 0; kk < BK; kk += 2) {
        const V4 b00 = *reinterpret_cast<const V4*>(bs + kk * BLD + tx * 4);
        const V4 b01 = *reinterpret_cast<const V4*>(bs + kk * BLD + 64 + tx * 4);
        const V4 b10 = *reinterpret_cast<const V4*>(bs + (kk + 1) * BLD + tx * 4);
        const V4 b11 = *reinterpret_cast<const V4*>(bs + (kk + 1) * BLD + 64 + tx * 4);
        const float2 p0[4] = {make_float2(b00.x, b00.y), make_float2(b00.z, b00.w), make_float2(b01.x, b01.y),
                              make_float2(b01.z, b01.w)};
        const float2 p1[4] = {make_float2(b10.x, b10.y), make_float2(b10.z, b10.w), make_float2(b11.x, b11.y),
                              make_float2(b11.z, b11.w)};
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const V4 a0 = *reinterpret_cast<const V4*>(as + kk * ALD + 64 * h + ty * 4);
          const V4 a1 = *reinterpret_cast<const V4*>(as + (kk + 1) * ALD + 64 * h + ty * 4);
          const float x0[4] = {a0.x, a0.y, a0.z, a0.w};
          const float x1[4] = {a1.x, a1.y, a1.z, a1.w};
#ifndef APSP_F32_JP_OUTER
#define APSP_F32_JP_OUTER 2
#endif
          // column pair outer, the four sums of each depth step first: the FADD2s of one pair
          // operand run back to back, so its 64-bit operand comes from the operand reuse cache
          // (fewer register-file reads, which bound this instruction stream: DESIGN.md §5 pipe
          // decomposition). Measured at n = 16384 / 32768 (fp32 ER, profiles/r02_f32_order_ab.txt):
          // row outer (0) 1.849e13, pair outer (1) 1.861e13, pair outer with the sums grouped (2,
          // default) 1.876-1.880e13.
#pragma unroll
          for (int u = 0; u < 16; u += (APSP_F32_JP_OUTER == 2 ? 4 : 1)) {
            if constexpr (APSP_F32_JP_OUTER == 2) {
              const int jp = u >> 2;
              float2 s0[4], s1[4];
#pragma unroll
              for (int i = 0; i < 4; ++i) s0[i] = __fadd2_rn(make_float2(x0[i], x0[i]), p0[jp]);
#pragma unroll
              for (int i = 0; i < 4; ++i) s1[i] = __fadd2_rn(make_float2(x1[i], x1[i]), p1[jp]);
#pragma unroll
              for (int i = 0; i < 4; ++i) {
                float& c0 = acc[4 * h + i][2 * jp];
                float& c1 = acc[4 * h + i][2 * jp + 1];
                c0 = fminf(fminf(c0, s0[i].x), s1[i].x);
                c1 = fminf(fminf(c1, s0[i].y), s1[i].y);
              }
            } else {
              const int i = APSP_F32_JP_OUTER ? (u & 3) : (u >> 2), jp = APSP_F32_JP_OUTER ? (u >> 2) : (u & 3);
              const float2 s0 = __fadd2_rn(make_float2(x0[i], x0[i]), p0[jp]);
              const float2 s1 = __fadd2_rn(make_float2(x1[i], x1[i]), p1[jp]);
              float& c0 = acc[4 * h + i][2 * jp];
              float& c1 = acc[4 * h + i][2 * jp + 1];
              c0 = fminf(fminf(c0, s0.x), s1.x);
              c1 = fminf(fminf(c1, s0.y), s1.y);
            }
          }
        }
      }
    } else {
#pragma unroll
      for (int kk = 0; kk < BK; ++kk) {
        const V4 a0 = *reinterpret_cast<const V4*>(as + kk * ALD + ty * 4);
        const V4 a1 = *reinterpret_cast<const V4*>(as + kk * ALD + 64 + ty * 4);
        const V4 b0 = *reinterpret_cast<const V4*>(bs + kk * BLD + tx * 4);
        const V4 b1 = *reinterpret_cast<const V4*>(bs + kk * BLD + 64 + tx * 4);
        const T av[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const T bv[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[i][j] = DV<T>::relax(av[i], bv[j], acc[i][j]);
      }
    }
    __syncwarp();
    if (lane == 0) mb_arrive(empty0 + 8 * s);
    if (c + 2 < NK) {  // refill the stage of chunk G-1 with chunk c+2
      const unsigned Gn = G + 2;
      load_chunk((int)(Gn % STAGES), c + 2, Gn >= STAGES ? (long long)(Gn - STAGES) : -1ll);
    }
  }
  cp_wait_all();
  gbar(g);
  {
    T* const Cout = d->Cout;
    T* const Cout2 = d->Cout2;
    const int ldc = d->ldc;
    const T* const cs_lo = stage0 + s_lo * STAGE_ELEMS;
    const T* const cs_hi = stage0 + s_hi * STAGE_ELEMS;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
      if (!kXpref || i >= 4) {  // (kXpref: the top half was folded before the last chunk)
        const T* crow = (i < 4 ? cs_lo : cs_hi) + (ty * 4 + (i & 3)) * CLD;
        const V4 x0 = *reinterpret_cast<const V4*>(crow + tx * 4);
        const V4 x1 = *reinterpret_cast<const V4*>(crow + 64 + tx * 4);
        acc[i][0] = DV<T>::vmin(acc[i][0], x0.x); acc[i][1] = DV<T>::vmin(acc[i][1], x0.y);
        acc[i][2] = DV<T>::vmin(acc[i][2], x0.z); acc[i][3] = DV<T>::vmin(acc[i][3], x0.w);
        acc[i][4] = DV<T>::vmin(acc[i][4], x1.x); acc[i][5] = DV<T>::vmin(acc[i][5], x1.y);
        acc[i][6] = DV<T>::vmin(acc[i][6], x1.z); acc[i][7] = DV<T>::vmin(acc[i][7], x1.w);
      }
      V4 v0, v1;
      v0.x = acc[i][0]; v0.y = acc[i][1]; v0.z = acc[i][2]; v0.w = acc[i][3];
      v1.x = acc[i][4]; v1.y = acc[i][5]; v1.z = acc[i][6]; v1.w = acc[i][7];
      *reinterpret_cast<V4*>(Cout + (long long)r * ldc + tx * 4) = v0;
      *reinterpret_cast<V4*>(Cout + (long long)r * ldc + 64 + tx * 4) = v1;
      if (Cout2 && !d->c2t) {
        *reinterpret_cast<V4*>(Cout2 + r * BN + tx * 4) = v0;
        *reinterpret_cast<V4*>(Cout2 + r * BN + 64 + tx * 4) = v1;
        if constexpr (SH) {
          if (d->bcast) {  // the row panel tile into every other rank's pbuf (NVLink peer stores)
            for (int e = 0; e < args->P; ++e) {
              if (e == args->q) continue;
              T* const o = peer_pb(*args, e, Cout2);
              *reinterpret_cast<V4*>(o + r * BN + tx * 4) = v0;
              *reinterpret_cast<V4*>(o + r * BN + 64 + tx * 4) = v1;
            }
          }
        }
      }
    }
    if (Cout2 && d->c2t) {  // transposed copy: column c of the block = 4 + 4 consecutive rows
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const int cc = (j < 4) ? (tx * 4 + j) : (64 + tx * 4 + j - 4);
        V4 w0, w1;
        w0.x = acc[0][j]; w0.y = acc[1][j]; w0.z = acc[2][j]; w0.w = acc[3][j];
        w1.x = acc[4][j]; w1.y = acc[5][j]; w1.z = acc[6][j]; w1.w = acc[7][j];
        *reinterpret_cast<V4*>(Cout2 + cc * BM + ty * 4) = w0;
        *reinterpret_cast<V4*>(Cout2 + cc * BM + 64 + ty * 4) = w1;
      }
    }
  }
}

// Launch parameters: one argument block per rank run by this launch (nv > 1 only for
// virtual ranks, i.e. several shards on one GPU in one launch: CTA b serves rank b % nv).
template <typename T>
struct DFLaunch {
  DFArgs<T> r[kMaxRanks];
  int nv;
};

#undef NK

// SH: the sharded kernel; PQ: the single-GPU kernel on the two-round (pair) queue. The one-round
// single-GPU kernel (PQ = false) keeps exactly the pre-pair code (measured: the pair engine's
// extra code costs the one-round path ~2-3 %, so each queue gets its own instantiation).
template <bool SH, bool PQ, typename T>
__global__ void __launch_bounds__(GNT * GROUPS, CTAS_PER_SM) fw_dataflow_kernel(const __grid_constant__ DFLaunch<T> L) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ __align__(8) unsigned long long bars[GROUPS][2 * STAGES];
  __shared__ Slot<T, PQ> slots[GROUPS][2];
  const DFArgs<T>& a = L.r[SH ? blockIdx.x % L.nv : 0];
  const int g = threadIdx.x / GNT, gtid = threadIdx.x % GNT;
  T* const stage0 = reinterpret_cast<T*>(smem_raw) + g * STAGES * STAGE_ELEMS;
  const unsigned full0 = saddr(&bars[g][0]), empty0 = full0 + 8 * STAGES;
  if constexpr (SH) {  // segment starts -> shared memory (decode_any), before the first decode
    long long* const seg = reinterpret_cast<long long*>(smem_raw + GROUPS * STAGES * STAGE_ELEMS * sizeof(T));
    for (int x = threadIdx.x; x <= a.nb; x += blockDim.x) seg[x] = a.segstart[x];
    __syncthreads();
  }
  if (gtid == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mb_init(full0 + 8 * s, 1);  // one arrival per chunk (+ transaction bytes of bulk copies)
      mb_init(empty0 + 8 * s, GNT / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (gtid == SCH) {
    if (!SH && (GROUPS > 1 ? g > 0 : blockIdx.x >= gridDim.x / 2) && a.stagger > 0) {  // half the groups start later
      const long long t0 = clock64();
      while (clock64() - t0 < a.stagger) __nanosleep(256);
    }
    Slot<T, PQ>& s0 = slots[g][0];
    s0.t = (long long)atomicAdd(a.counter, 1ull);
    s0.ready = 0;
    s0.pref = 0;
    slots[g][1].pref = 0;
    if (s0.t < a.total) {
      s0.tk = decode_any<SH, PQ>(a, s0.t);
      if (s0.tk.type != T_P1) fill_desc(a, s0.tk, s0.d, slot_p2(&s0));
    }
  }
  gbar(g);
  unsigned chunk = 0;
  unsigned long long pr[6] = {0, 0, 0, 0, 0, 0};  // wait, body, tail, tasks, p1 cycles, waits that blocked
  long long tc0 = clock64();
  for (int it = 0;; ++it) {
    Slot<T, PQ>& S = slots[g][it & 1];
    Slot<T, PQ>* N = &slots[g][(it + 1) & 1];
    const long long t = S.t;
    if (t >= a.total) break;
    const Task tk = S.tk;
    if (!S.ready) {  // uniform: the slot was published by the last barrier
      if (gtid == SCH && !deps_any<SH, PQ>(a, tk)) {
        const long long w0 = clock64();
        while (!deps_any<SH, PQ>(a, tk)) {
          __nanosleep(64);
          // sharded: a peer that never delivers (a dead rank) must not hang the GPU: after
          // ~30 s of waiting the kernel traps (the launch fails, the handle reports APSP_ECUDA)
          if (SH && clock64() - w0 > 60000000000ll) __trap();
        }
        pr[5]++;
      }
      gbar(g);
    }
    long long nxt = 0;
    if (gtid == SCH) nxt = (long long)atomicAdd(a.counter, 1ull);  // the result is needed in chunk 1
    const long long tc1 = clock64();
    pr[0] += tc1 - tc0;
    if (tk.type == T_P1) {
      T* const tile = a.D + (long long)(tk.i - a.q * a.nl) * BM * a.ld + (long long)tk.j * BN;
      if constexpr (SH) {  // D also into every other rank's pbuf
        T* peers[kMaxRanks];
        int np = 0;
        for (int e = 0; e < a.P; ++e)
          if (e != a.q) peers[np++] = peer_pb(a, e, pb_diag(a, tk.k));
        group_phase1<T>(tile, a.ld, pb_diag(a, tk.k), pb_diagT(a, tk.k), a.negflag, stage0, g, gtid, peers, np);
      } else {
        group_phase1<T>(tile, a.ld, pb_diag(a, tk.k), pb_diagT(a, tk.k), a.negflag, stage0, g, gtid);
      }
      if (gtid == SCH) {
        N->t = nxt;
        N->pref = 0;
        if (nxt < a.total) {
          N->tk = decode_any<SH, PQ>(a, nxt);
          N->ready = 0;
          if (N->tk.type != T_P1) fill_desc(a, N->tk, N->d, slot_p2(N));
        }
      }
    } else {
      if constexpr (PQ) {
#ifdef APSP_DF_PQ_ONE_ENGINE
        group_minplus<SH, PQ, T, 0>(&S.d, &S.p2, stage0, full0, empty0, chunk, gtid, g, &a, nxt, N, S.pref);
#else
        if (S.p2.nk == 2 * (BM / BK)) {
          group_minplus<SH, PQ, T, 2 * (BM / BK)>(&S.d, &S.p2, stage0, full0, empty0, chunk, gtid, g, &a, nxt, N,
                                                  S.pref);
        } else {
          group_minplus<SH, PQ, T, BM / BK>(&S.d, &S.p2, stage0, full0, empty0, chunk, gtid, g, &a, nxt, N, S.pref);
        }
#endif
        chunk += S.p2.nk;
      } else {
        group_minplus<SH, PQ, T, BM / BK>(&S.d, nullptr, stage0, full0, empty0, chunk, gtid, g, &a, nxt, N, S.pref);
        chunk += BM / BK;
      }
    }
    const long long tc2 = clock64();
    pr[1] += tc2 - tc1;
    if (tk.type == T_P1) pr[4] += tc2 - tc1;
    pr[3]++;
    gbar(g);  // every thread's stores of this task are issued; the next slot is published
    // published right away by the SIG thread (its warp absorbs the fence; measured
    // better than deferring it under the next task's first loads)
    if (gtid == SIG) {
      if constexpr (SH) signal_done_sh(a, tk);
      else if constexpr (PQ) signal_single(a, tk);
      else signal_done(a, tk);
    }
    tc0 = clock64();
    pr[2] += tc0 - tc2;
  }
  if (a.prof && gtid == SCH) {
    unsigned long long* o = a.prof + ((long long)blockIdx.x * GROUPS + g) * 8;
    for (int i = 0; i < 6; ++i) o[i] = pr[i];
  }
}

}  // namespace

// Work-buffer layout of one rank: pbuf (npar parities x (2 + nb + nl) tiles), then the
// flag block (sized for 4 parities), then (sharded) the nb + 1 segment starts.
template <typename T>
static void df_layout(DFArgs<T>& a, void* work, int nb, int nl, int npar) {
  a.nb = nb;
  a.nl = nl;
  a.npar = npar;
  a.pbuf = static_cast<T*>(work);
  char* const fb = static_cast<char*>(work) + fw_dataflow_pbuf_bytes(nb, nl, sizeof(T), npar);
  int* f = reinterpret_cast<int*>(fb);
  a.counter = reinterpret_cast<unsigned long long*>(f); f += 2;  // first: 8-byte aligned
  a.ver = f; f += (long long)nl * nb;
  a.diagready = f; f += 4;
  a.rowready = f; f += 4 * nb;
  a.colready = f; f += 4 * nl;
  a.done2 = f; f += nb;
  a.done3 = f; f += nb;
  a.segstart = reinterpret_cast<const long long*>(fb + fw_dataflow_flag_bytes(nb, nl));
}

template <typename T>
cudaError_t launch_fw_dataflow(T* D, long long ld, int nb, void* work, int* negflag, long long delay,
                               long long stagger, cudaStream_t s, unsigned long long* prof, int* used_pair) {
  if (nb <= 0) return cudaSuccess;
  const int smem = GROUPS * STAGES * STAGE_ELEMS * (int)sizeof(T);
  cudaError_t e = cudaFuncSetAttribute(fw_dataflow_kernel<false, false, T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(fw_dataflow_kernel<false, true, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  DFLaunch<T> L;
  memset(&L, 0, sizeof(L));
  L.nv = 1;
  DFArgs<T>& a = L.r[0];
  // the two-round (pair) queue: APSP_DF_PAIR=0/1 overrides the default (tuning experiments)
  int pairq = kPairDefault && sizeof(T) == 4 && T(0.5) == T(0) && nb >= kPairMinNb;  // int32
  if (const char* e = getenv("APSP_DF_PAIR")) pairq = atoi(e) != 0 && nb >= 2;
  df_layout(a, work, nb, nb, pairq ? 4 : 2);  // the pair queue keeps 4 rounds of panel copies
  a.pairq = pairq;
  if (used_pair) *used_pair = pairq;
  a.D = D; a.ld = ld;
  a.negflag = negflag;
  a.total = a.pairq ? pair_total(nb) : (long long)nb * nb * nb;
  a.delay = delay;
  a.stagger = stagger;
  a.prof = prof;
  a.P = 1; a.q = 0;
  a.peer_pbuf[0] = a.pbuf;
  a.peer_base[0] = reinterpret_cast<int*>(a.counter);
  e = cudaMemsetAsync(a.counter, 0, fw_dataflow_flag_bytes(nb, nb), s);
  if (e != cudaSuccess) return e;
  long long grid = (long long)sms * CTAS_PER_SM;
  if (grid > a.total) grid = a.total;
  if (a.pairq) fw_dataflow_kernel<false, true, T><<<(unsigned)grid, GNT * GROUPS, smem, s>>>(L);
  else fw_dataflow_kernel<false, false, T><<<(unsigned)grid, GNT * GROUPS, smem, s>>>(L);
  return cudaGetLastError();
}

// Queue of rank q (segment starts and length): the host mirror of decode_sh.
long long fw_dataflow_sharded_segments(int nb, int nl, int q, long long* segstart) {
  auto loc = [&](int k) { return (k / nl) == q ? 1 : 0; };
  long long pos = loc(0);
  for (int k = 0; k < nb; ++k) {
    segstart[k] = pos;
    long long sz = (long long)loc(k) * (nb - 1) + (nl - loc(k));          // G2(k)
    if (k >= 1) sz += (long long)(nl - loc(k - 1) - loc(k)) * (nb - 2);    // G3R(k-1)
    if (k <= nb - 2)                                                         // G3Lx(k)
      sz += loc(k + 1) ? 2 + (nb - 2) + (nl - 1 - loc(k)) : (nl - loc(k));
    pos += sz;
  }
  segstart[nb] = pos;
  return pos + (long long)(nl - loc(nb - 1)) * (nb - 1);  // + the last round's phase 3
}

template <typename T>
cudaError_t launch_fw_dataflow_sharded(const DFShard* ranks, int nv, int P, int nb, long long ld, int* negflag,
                                       long long delay, cudaStream_t s) {
  if (nb <= 0 || nv < 1 || nv > kMaxRanks || P < 1 || P > kMaxRanks || nb % P) return cudaErrorInvalidValue;
  const int nl = nb / P;
  const int smem = GROUPS * STAGES * STAGE_ELEMS * (int)sizeof(T) + 8 * (nb + 1);  // + segment starts
  cudaError_t e = cudaFuncSetAttribute(fw_dataflow_kernel<true, false, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  DFLaunch<T> L;
  memset(&L, 0, sizeof(L));
  L.nv = nv;
  std::vector<long long> seg((size_t)nb + 1);
  for (int v = 0; v < nv; ++v) {
    DFArgs<T>& a = L.r[v];
    const DFShard& sh = ranks[v];
    df_layout(a, sh.work, nb, nl, 2);
    a.pairq = 0;
    a.D = static_cast<T*>(sh.D); a.ld = ld;
    a.negflag = negflag;
    a.P = P; a.q = sh.rank;
    a.total = fw_dataflow_sharded_segments(nb, nl, sh.rank, seg.data());
    a.delay = delay;
    a.stagger = 0;
    a.prof = nullptr;
    for (int r = 0; r < P; ++r) {
      a.peer_pbuf[r] = static_cast<T*>(sh.peer_work[r]);
      a.peer_base[r] = reinterpret_cast<int*>(static_cast<char*>(sh.peer_work[r]) +
                                              fw_dataflow_pbuf_bytes(nb, nl, sizeof(T), 2));
    }
    // blocking copy: `seg` is reused for the next rank (a few KB)
    if ((e = cudaMemcpyAsync(const_cast<long long*>(a.segstart), seg.data(), seg.size() * sizeof(long long),
                             cudaMemcpyHostToDevice, s)) != cudaSuccess)
      return e;
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
  }
  // a persistent grid must be fully resident (tasks wait on each other): CTAs per SM as the
  // occupancy calculator allows with this launch's shared memory (the segment starts grow it)
  int occ = 0;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fw_dataflow_kernel<true, false, T>, GNT * GROUPS, smem)) !=
      cudaSuccess)
    return e;
  if (occ < 1) return cudaErrorInvalidConfiguration;
  long long grid = (long long)sms * (occ < CTAS_PER_SM ? occ : CTAS_PER_SM);
  grid -= grid % nv;
  if (grid < nv) return cudaErrorInvalidConfiguration;
  fw_dataflow_kernel<true, false, T><<<(unsigned)grid, GNT * GROUPS, smem, s>>>(L);
  return cudaGetLastError();
}

long long fw_dataflow_pbuf_bytes(int nb, int nl, size_t elem, int npar) {
  return (long long)npar * (2 + nb + nl) * TILE_ELEMS * (long long)elem;  // (kept a multiple of 8 bytes)
}
long long fw_dataflow_flag_bytes(int nb, int nl) {  // 4 parities; rounded to 16 B: the segment starts follow
  return ((((long long)nl * nb + 6ll * nb + 4ll * nl + 6) * 4 + 15) / 16) * 16;
}
long long fw_dataflow_work_bytes(int nb, int nl, size_t elem) {  // sharded kernel: 2 parities
  return fw_dataflow_pbuf_bytes(nb, nl, elem, 2) + fw_dataflow_flag_bytes(nb, nl) + 8ll * (nb + 1);
}
long long fw_dataflow_pbuf_bytes(int nb, size_t elem) { return fw_dataflow_pbuf_bytes(nb, nb, elem, 4); }
long long fw_dataflow_flag_bytes(int nb) { return fw_dataflow_flag_bytes(nb, nb); }
long long fw_dataflow_work_bytes(int nb, size_t elem) {  // single GPU: 4 parities (pair schedule)
  return fw_dataflow_pbuf_bytes(nb, nb, elem, 4) + fw_dataflow_flag_bytes(nb, nb) + 8ll * (nb + 1);
}

}  // namespace apsp

// Test hook (declared in include/apsp.h): the task queue the dataflow kernel decodes, on the
// host. P = 0: the single-GPU queue (decode); P >= 1: rank q's sharded queue (decode_sh).
extern "C" int64_t apsp_debug_queue(int32_t nb, int32_t P, int32_t q, int64_t delay, int32_t* out, int64_t cap) {
  using namespace apsp;
  if (P == -2) {  // the two-round ("pair") queue of the single-GPU kernel (decode2)
    if (nb <= 0) return -1;
    const long long total = pair_total(nb);
    for (long long g = 0; g < total && g < cap; ++g) {
      const Task t = decode2(g, nb, delay);
      out[4 * g] = t.type; out[4 * g + 1] = t.k; out[4 * g + 2] = t.i; out[4 * g + 3] = t.j;
    }
    return total;
  }
  if (P == -1) {  // the small-n kernel's queue (apsp_fw_small.cu), nb 64-wide tile rows
    if (nb <= 0) return -1;
    if (!out || cap <= 0) return small_queue(nb, delay, nullptr);  // the launch path's closed-form length
    std::vector<int4> sq;
    const long long total = small_queue(nb, delay, &sq);
    for (long long g = 0; g < total && g < cap; ++g) {
      out[4 * g] = sq[g].x; out[4 * g + 1] = sq[g].y; out[4 * g + 2] = sq[g].z; out[4 * g + 3] = sq[g].w;
    }
    return total;
  }
  if (nb <= 0 || P < 0 || (P > 0 && (nb % P || q < 0 || q >= P))) return -1;
  const int nl = P > 0 ? nb / P : nb;
  std::vector<long long> seg((size_t)nb + 1);
  const long long total = P > 0 ? fw_dataflow_sharded_segments(nb, nl, q, seg.data()) : (long long)nb * nb * nb;
  for (long long g = 0; g < total && g < cap; ++g) {
    const Task t = P > 0 ? decode_sh(g, nb, nl, q, delay, seg.data()) : decode(g, nb, delay);
    out[4 * g] = t.type; out[4 * g + 1] = t.k; out[4 * g + 2] = t.i; out[4 * g + 3] = t.j;
  }
  return total;
}

namespace apsp {

template cudaError_t launch_fw_dataflow_sharded<int>(const DFShard*, int, int, int, long long, int*, long long,
                                                     cudaStream_t);
template cudaError_t launch_fw_dataflow_sharded<float>(const DFShard*, int, int, int, long long, int*, long long,
                                                       cudaStream_t);
template cudaError_t launch_fw_dataflow<int>(int*, long long, int, void*, int*, long long, long long, cudaStream_t,
                                             unsigned long long*, int*);
template cudaError_t launch_fw_dataflow<float>(float*, long long, int, void*, int*, long long, long long,
                                               cudaStream_t, unsigned long long*, int*);

}  // namespace apsp
