// apsp_fw_small.cu — the whole single-GPU blocked Floyd–Warshall (PAPER.md:62,
// every round and phase) for SMALL n as one persistent dataflow launch with
// 64 x 64 tiles (b = 64).
//
// Why a second kernel: at small n (config 1, n = 1024) the 128-tile dataflow
// kernel is latency bound. Each round's critical path is three dependent
// 128^3 tasks, phase 1 (k) -> panel tiles (k, k+1) / (k+1, k) -> phase-3 tile
// (k+1, k+1) -> phase 1 (k+1), each ~2.1M relaxations on ONE SM (>= 17 us at
// 64 DPX lanes/clk), while only 49 of 296 CTAs have phase-3 work per round
// (8 rounds: 0.77 ms = 0.075 of the DPX peak). With b = 64 a
// task is 262K relaxations (2.1 us on one SM), so the chain per round shrinks
// ~8x while the rounds double (16 at n = 1024), and a round has 16^2 = 256
// tasks for the 148 SMs instead of 64. The blocked FW is the same for any b
// (R7 pads n to a multiple of 128, hence of 64).
//
// Structure: the flag protocol of apsp_fw_dataflow.cu (apsp_df_common.cuh: per-tile
// versions, diagonal / panel readiness, double-buffered panel copies, deps_met /
// signal_done) with a queue ordered for the critical path and a simpler engine:
//   * the queue is built on the host (small_queue, at most 32^3 + 186 entries): the
//     128-tile kernel's segment order (decode), so round k+1's diagonal and panels
//     come right after the round-k tiles they need; every dependency of an entry lies
//     earlier in the queue (tests/test_schedule.py simulates it), so a CTA that
//     finishes its task before taking the next cannot deadlock (a critical-path list
//     order is kept as a tuning variant: measured slower);
//   * the two panel tiles next to the diagonal, P2R(k; k,k+1) and P2C(k; k+1,k), which
//     every round's chain waits for, run as 16, 8 or 4 parts on as many CTAs (column / row
//     ranges; small_split_for);
//   * F(k) fuses P3(k; k+1,k+1) with P1(k+1): the CTA that updates the next
//     diagonal tile closes it in registers right away (one flag hop and one
//     tile load less on the chain of every round);
//   * one CTA of 256 threads per task (one CTA per SM by default), thread
//     (tx, ty) owns rows 4ty..4ty+3 x columns 4tx..4tx+3 of the 64x64 tile;
//   * the task's whole depth (64) is staged at once: A^T as As[kk][r] and B as
//     Bs[kk][c] (16 KB each, cp.async from the L2-resident panel copies; the
//     column-panel task transposes its own tile through registers); per depth
//     step 2 LDS.128 feed 16 relaxations (VIADDMNMX for int32);
//   * C is loaded into the accumulators first (min is exact, any order) and
//     stored once (out of place per tile, so phase 2, where an operand aliases
//     C, is exact);
//   * phase 1: the tile in registers, 64 steps, each publishing row / column kk
//     through a double-buffered shared copy (one barrier per step), the R6
//     negative-cycle check at the start of every step;
//   * thread 0 fetches the next queue entry and the index after it while the CTA
//     computes the current task, and checks the next task's flags right after
//     publishing the current one;
//   * the last CTA to finish zeroes the flags for the next launch (no memset in the
//     launch's critical path).
#include "apsp_kernels.cuh"
#include "apsp_df_common.cuh"

#include <cuda_runtime.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

namespace apsp {
namespace {

constexpr int SB = 64;          // tile edge (round depth b)
constexpr int SNT = 256;        // threads per CTA (one task at a time)
constexpr int STE = SB * SB;    // elements per tile

template <typename T> struct SV;
template <> struct SV<int> {
  using V4 = int4;
  using V2 = int2;
  static __device__ __forceinline__ int relax(int a, int b, int c) { return __viaddmin_s32(a, b, c); }
};
template <> struct SV<float> {
  using V4 = float4;
  using V2 = float2;
  static __device__ __forceinline__ float relax(float a, float b, float c) { return fminf(c, __fadd_rn(a, b)); }
};

template <typename T>
struct SmArgs {
  T* D;            // n_pad x n_pad, row-major, ld
  long long ld;
  int nb;          // n_pad / 64
  T* pbuf;         // 2 parities x (2 + 2 nb) tiles of 64x64: diag, diag^T, row panel [nb], column panel^T [nb]
  int* ver;        // [nb][nb]
  int* diagready;  // [2]
  int* rowready;   // [2][nb]
  int* colready;   // [2][nb]
  int* done2;      // [nb]
  int* done3;      // [nb]
  unsigned long long* counter;
  int* negflag;
  long long total;   // queue entries
  const int4* queue; // [total] (type, k, i, j), built on the host (small_queue)
  unsigned long long* prof;  // optional [CTAs][16] cycle counters (tuning: APSP_SMALL_PROFILE)
  int close_v;               // phase-1 variant: 1 small_close_defer, 0 small_close (APSP_SMALL_CLOSE)
  int split;                 // parts of each chain panel tile (small_split(); 1 = whole tasks)
  int* rsplit;               // [nb] finished parts of P2R(j-1; j-1, j), the row-panel tile next to the diagonal
  int* csplit;               // [nb] finished parts of P2C(i-1; i, i-1)
  int early_pub;             // F(k): diagready published before the matrix tile is stored (APSP_SMALL_EARLYPUB)
  int spin;                  // dependency polls back to back, no __nanosleep between them (APSP_SMALL_SPIN)
  int* exitc;                // CTAs past their last task: the last one zeroes every flag for the next launch
  long long flag_words;      // 32-bit words from counter to exitc inclusive
};

template <typename T>
__device__ __forceinline__ T* sp_diag(const SmArgs<T>& a, int k) {
  return a.pbuf + (long long)(k & 1) * (2 + 2 * a.nb) * STE;
}
template <typename T>
__device__ __forceinline__ T* sp_diagT(const SmArgs<T>& a, int k) { return sp_diag(a, k) + STE; }
template <typename T>
__device__ __forceinline__ T* sp_row(const SmArgs<T>& a, int k, int j) { return sp_diag(a, k) + (2ll + j) * STE; }
template <typename T>
__device__ __forceinline__ T* sp_colT(const SmArgs<T>& a, int k, int i) {
  return sp_diag(a, k) + (2ll + a.nb + i) * STE;
}

enum { T_P3P1 = 4 };  // fused P3(k; k+1,k+1) + P1(k+1)
// Split chain panel tasks: queue entry type = base (T_P2R / T_P2C) + 16 * (part + 1). The two panel
// tiles next to the diagonal, P2R(k; k,k+1) and P2C(k; k+1,k), sit on every round's critical path
// (F(k) waits for both); each is cut into `split` parts run by as many CTAs: P2R by column ranges
// (a part reads only its columns of the tile it updates, B = A(k,k+1)), P2C by row ranges (a part
// reads only its rows, A = A(k+1,k)), so no part reads what another writes. The parts count into
// rsplit / csplit instead of the tile's version and panel flags (PAPER.md:62 phase 2, unchanged).
constexpr int kPartShift = 4;
__host__ __device__ __forceinline__ int part_of(int type) { return (type >> kPartShift) - 1; }
__host__ __device__ __forceinline__ int base_of(int type) { return type & 15; }

// queue variant: 3 (default) the 128-tile kernel's segment order with F(k) fused; tuning
// experiments only: APSP_SMALL_QUEUE=decode (1: no fusion), bl_nofuse (2: list order without
// fused entries), anything else (0: list order + F(k))
static int small_variant() {
  const char* qv = getenv("APSP_SMALL_QUEUE");
  return !qv                               ? 3
         : strcmp(qv, "decode") == 0      ? 1
         : strcmp(qv, "bl_nofuse") == 0   ? 2
         : strcmp(qv, "decode_fuse") == 0 ? 3
                                          : 0;
}

// parts per chain panel tile, by size (measured, device time of 30 runs, three alternations,
// profiles/r02_small_split_ab.txt / r02_small_split8.txt / r02_small_split16.txt):
//   n = 1024 (nb 16): whole 0.265, 2 parts 0.248, 4 0.239, 8 0.230, 16 0.228 ms
//   n = 1536 (nb 24): 4 parts 0.436, 8 0.428, 16 0.435 ms;  n = 2048 (nb 32): 4 0.750, 8 0.758, 16 0.778 ms
// APSP_SMALL_SPLIT=1|2|4|8|16 overrides (tuning A/B); the fused segment-order queue only (variant 3)
static int small_split_for(int variant, int nb) {
  if (variant != 3) return 1;
  if (const char* e = getenv("APSP_SMALL_SPLIT")) {
    const int v = atoi(e);
    return v == 1 || v == 2 || v == 4 || v == 8 || v == 16 ? v : 8;
  }
  return nb <= 16 ? 16 : nb <= 24 ? 8 : 4;
}

struct SmSlot {
  long long t;
  Task tk;
  int ready;
};

// Phase 1 on a tile held in registers (thread: rows 4ty.., columns 4tx..): in-place FW
// closure of the 64x64 block (P:60 restricted to it), 64 steps, row / column kk published
// through a double-buffered shared copy, one barrier per step; R6 check at every step.
template <typename T>
__device__ __forceinline__ void small_close(T (&acc)[4][4], T* rowbuf, T* colbuf, int* negflag) {
  using V4 = typename SV<T>::V4;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  bool neg = false;
  for (int q = 0; q < 16; ++q) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int kk = q * 4 + u, p = u & 1;
      if (ty == q) {  // row kk
        V4 x;
        x.x = acc[u][0]; x.y = acc[u][1]; x.z = acc[u][2]; x.w = acc[u][3];
        *reinterpret_cast<V4*>(&rowbuf[p * SB + tx * 4]) = x;
      }
      if (tx == q) {  // column kk
        V4 y;
        y.x = acc[0][u]; y.y = acc[1][u]; y.z = acc[2][u]; y.w = acc[3][u];
        *reinterpret_cast<V4*>(&colbuf[p * SB + ty * 4]) = y;
      }
      __syncthreads();
      if (tid == 0 && rowbuf[p * SB + kk] < T(0)) neg = true;  // R6: D[kk][kk] < 0 -> negative cycle
      const V4 av = *reinterpret_cast<const V4*>(&colbuf[p * SB + ty * 4]);
      const V4 bv = *reinterpret_cast<const V4*>(&rowbuf[p * SB + tx * 4]);
      const T A4[4] = {av.x, av.y, av.z, av.w}, B4[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = SV<T>::relax(A4[i], B4[j], acc[i][j]);
    }
  }
  if (neg) *negflag = 1;
}

// The closure with the bulk of each step deferred past the next barrier: in step kk a thread
// relaxes only its elements of row / column kk+1 (the owners store them into the other buffer
// for step kk+1), and the rest of its 4x4 block for step kk right after the barrier of step
// kk+1, while that step's row / column loads are in flight. The per-step chain is then barrier
// -> loads -> 7 relaxations -> stores; per element the steps still apply in order (the deferred
// rest of step kk precedes step kk+1's relaxations of the same registers). One barrier per step:
// the other buffer was last read before this step's barrier (WAR) and is read after the next.
// Steps are a template on kk mod 4 with the first and last steps peeled, so a step body has no
// branch and ptxas schedules across it.
template <typename T, int U, bool REST, bool CRIT>
__device__ __forceinline__ void close_step(T (&acc)[4][4], T (&pa)[4], T (&pb)[4], T* rowbuf, T* colbuf, int kk,
                                           bool& neg) {
  using V4 = typename SV<T>::V4;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  constexpr int p = U & 1, nu = (U + 1) & 3;  // buffer; row / column kk+1 within a 4x4 block
  __syncthreads();
  const V4 av = *reinterpret_cast<const V4*>(&colbuf[p * SB + ty * 4]);
  const V4 bv = *reinterpret_cast<const V4*>(&rowbuf[p * SB + tx * 4]);
  const T dkk = rowbuf[p * SB + kk];
  if (REST) {  // rest of step kk-1: every element outside row / column U (= (kk-1)+1 mod 4)
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j)
        if (i != U && j != U) acc[i][j] = SV<T>::relax(pa[i], pb[j], acc[i][j]);
  }
  const T A4[4] = {av.x, av.y, av.z, av.w}, B4[4] = {bv.x, bv.y, bv.z, bv.w};
  if (CRIT) {
    const int owner = (kk + 1) >> 2;  // ty (row kk+1) / tx (column kk+1) of its owners
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[nu][j] = SV<T>::relax(A4[nu], B4[j], acc[nu][j]);
#pragma unroll
    for (int i = 0; i < 4; ++i)
      if (i != nu) acc[i][nu] = SV<T>::relax(A4[i], B4[nu], acc[i][nu]);
    if (ty == owner) {
      V4 x;
      x.x = acc[nu][0]; x.y = acc[nu][1]; x.z = acc[nu][2]; x.w = acc[nu][3];
      *reinterpret_cast<V4*>(&rowbuf[(p ^ 1) * SB + tx * 4]) = x;
    }
    if (tx == owner) {
      V4 y;
      y.x = acc[0][nu]; y.y = acc[1][nu]; y.z = acc[2][nu]; y.w = acc[3][nu];
      *reinterpret_cast<V4*>(&colbuf[(p ^ 1) * SB + ty * 4]) = y;
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      pa[i] = A4[i];
      pb[i] = B4[i];
    }
  } else {
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = SV<T>::relax(A4[i], B4[j], acc[i][j]);
  }
  neg |= dkk < T(0);  // R6: D[kk][kk] < 0 -> negative cycle (every thread reads it: a broadcast)
}

template <typename T>
__device__ __forceinline__ void small_close_defer(T (&acc)[4][4], T* rowbuf, T* colbuf, int* negflag) {
  using V4 = typename SV<T>::V4;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  bool neg = false;
  if (ty == 0) {
    V4 x;
    x.x = acc[0][0]; x.y = acc[0][1]; x.z = acc[0][2]; x.w = acc[0][3];
    *reinterpret_cast<V4*>(&rowbuf[tx * 4]) = x;
  }
  if (tx == 0) {
    V4 y;
    y.x = acc[0][0]; y.y = acc[1][0]; y.z = acc[2][0]; y.w = acc[3][0];
    *reinterpret_cast<V4*>(&colbuf[ty * 4]) = y;
  }
  T pa[4], pb[4];  // step kk-1's column / row values for its deferred rest
  close_step<T, 0, false, true>(acc, pa, pb, rowbuf, colbuf, 0, neg);
  for (int q = 0; q < 15; ++q) {  // steps 1 .. 60
    const int kk = 4 * q + 1;
    close_step<T, 1, true, true>(acc, pa, pb, rowbuf, colbuf, kk, neg);
    close_step<T, 2, true, true>(acc, pa, pb, rowbuf, colbuf, kk + 1, neg);
    close_step<T, 3, true, true>(acc, pa, pb, rowbuf, colbuf, kk + 2, neg);
    close_step<T, 0, true, true>(acc, pa, pb, rowbuf, colbuf, kk + 3, neg);
  }
  close_step<T, 1, true, true>(acc, pa, pb, rowbuf, colbuf, 61, neg);
  close_step<T, 2, true, true>(acc, pa, pb, rowbuf, colbuf, 62, neg);
  close_step<T, 3, true, false>(acc, pa, pb, rowbuf, colbuf, 63, neg);
  if (neg) *negflag = 1;
}

// phase 1 of the tile in registers: small_close_defer (default) or small_close (APSP_SMALL_CLOSE=0)
template <typename T>
__device__ __forceinline__ void small_close_any(const SmArgs<T>& a, T (&acc)[4][4], T* rowbuf, T* colbuf) {
  if (a.close_v) small_close_defer(acc, rowbuf, colbuf, a.negflag);
  else small_close(acc, rowbuf, colbuf, a.negflag);
}

// a thread's 4x4 block of a tile of the matrix (ld elements per row)
template <typename T>
__device__ __forceinline__ void small_store_tile(T* tile, long long ld, const T (&acc)[4][4]) {
  using V4 = typename SV<T>::V4;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    V4 v;
    v.x = acc[i][0]; v.y = acc[i][1]; v.z = acc[i][2]; v.w = acc[i][3];
    *reinterpret_cast<V4*>(tile + (long long)(ty * 4 + i) * ld + tx * 4) = v;
  }
}

// the closed diagonal block of round k: into the matrix (tile != nullptr), D and D^T into the panel copy
template <typename T>
__device__ __forceinline__ void small_store_diag(const SmArgs<T>& a, int k, T* tile, const T (&acc)[4][4]) {
  using V4 = typename SV<T>::V4;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  T* const d = sp_diag(a, k);
  T* const dt = sp_diagT(a, k);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    V4 v;
    v.x = acc[i][0]; v.y = acc[i][1]; v.z = acc[i][2]; v.w = acc[i][3];
    if (tile) *reinterpret_cast<V4*>(tile + (long long)(ty * 4 + i) * a.ld + tx * 4) = v;
    *reinterpret_cast<V4*>(d + (ty * 4 + i) * SB + tx * 4) = v;
  }
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    V4 w;
    w.x = acc[0][j]; w.y = acc[1][j]; w.z = acc[2][j]; w.w = acc[3][j];
    *reinterpret_cast<V4*>(dt + (tx * 4 + j) * SB + ty * 4) = w;
  }
}

// Phase 1 task P1(k): close A(k,k) (PAPER.md:62 step 1)
template <typename T>
__device__ __forceinline__ void small_phase1(const SmArgs<T>& a, const Task& tk, T* rowbuf, T* colbuf) {
  using V4 = typename SV<T>::V4;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  T* const tile = a.D + (long long)tk.i * SB * a.ld + (long long)tk.j * SB;
  T acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const V4 v = __ldcg(reinterpret_cast<const V4*>(tile + (long long)(ty * 4 + i) * a.ld + tx * 4));
    acc[i][0] = v.x; acc[i][1] = v.y; acc[i][2] = v.z; acc[i][3] = v.w;
  }
  small_close_any(a, acc, rowbuf, colbuf);
  small_store_diag(a, tk.k, tile, acc);
}

// Phase 2 / phase 3 task: C = min(C, A (x) B) with the depth-64 operands of round k.
//   P2R(k; k,j): A = D (panel copy D^T), B = A(k,j) itself; result also -> row panel copy
//   P2C(k; i,k): A = A(i,k) itself (transposed on load), B = D; result also -> column panel^T
//   P3(k; i,j):  A = column panel^T (i), B = row panel (j)
//   F(k) = P3(k; k+1,k+1) then P1(k+1) on the same registers (fused: closes the tile right away)
template <typename T>
__device__ __forceinline__ void small_minplus(const SmArgs<T>& a, const Task& tk, T* As, T* Bs, T* rowbuf,
                                              T* colbuf) {
  using V4 = typename SV<T>::V4;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  T* const C = a.D + (long long)tk.i * SB * a.ld + (long long)tk.j * SB;
  // operands -> shared memory: 64 rows of 256 B each, 16 B per cp.async, 4 per thread per operand
  const bool fused = tk.type == T_P3P1;
  const T* Bsrc;
  long long ldb;
  if (tk.type == T_P2R) { Bsrc = C; ldb = a.ld; }
  else if (tk.type == T_P2C) { Bsrc = sp_diag(a, tk.k); ldb = SB; }
  else { Bsrc = sp_row(a, tk.k, tk.j); ldb = SB; }
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    const int x = tid + e * SNT;  // 0..1023: row x/16, 16-byte column x%16
    const int r = x >> 4, c4 = (x & 15) * 4;
    cp16(Bs + r * SB + c4, Bsrc + r * ldb + c4);
  }
  if (tk.type == T_P2C) {  // A(i,k) rows r, depth kk -> As[kk][r]: a 4x4 block per thread,
    // transposed in registers, so every shared store is a conflict-free 16-byte vector
    // (scalar column stores were 16-way bank conflicts: +2.3K cycles on the chain's P2C task)
    const int r0 = (tid & 15) * 4, c0 = (tid >> 4) * 4;
    V4 v[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) v[q] = __ldcg(reinterpret_cast<const V4*>(C + (long long)(r0 + q) * a.ld + c0));
    V4 w;
    w.x = v[0].x; w.y = v[1].x; w.z = v[2].x; w.w = v[3].x;
    *reinterpret_cast<V4*>(As + (c0 + 0) * SB + r0) = w;
    w.x = v[0].y; w.y = v[1].y; w.z = v[2].y; w.w = v[3].y;
    *reinterpret_cast<V4*>(As + (c0 + 1) * SB + r0) = w;
    w.x = v[0].z; w.y = v[1].z; w.z = v[2].z; w.w = v[3].z;
    *reinterpret_cast<V4*>(As + (c0 + 2) * SB + r0) = w;
    w.x = v[0].w; w.y = v[1].w; w.z = v[2].w; w.w = v[3].w;
    *reinterpret_cast<V4*>(As + (c0 + 3) * SB + r0) = w;
  } else {
    const T* Asrc = tk.type == T_P2R ? sp_diagT(a, tk.k) : sp_colT(a, tk.k, tk.i);
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int x = tid + e * SNT;
      cp16(As + x * 4, Asrc + x * 4);
    }
  }
  cp_commit();
  T acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const V4 v = __ldcg(reinterpret_cast<const V4*>(C + (long long)(ty * 4 + i) * a.ld + tx * 4));
    acc[i][0] = v.x; acc[i][1] = v.y; acc[i][2] = v.z; acc[i][3] = v.w;
  }
  cp_wait_all();
  __syncthreads();
#pragma unroll 8
  for (int kk = 0; kk < SB; ++kk) {
    const V4 av = *reinterpret_cast<const V4*>(&As[kk * SB + ty * 4]);
    const V4 bv = *reinterpret_cast<const V4*>(&Bs[kk * SB + tx * 4]);
    const T A4[4] = {av.x, av.y, av.z, av.w}, B4[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = SV<T>::relax(A4[i], B4[j], acc[i][j]);
  }
  if (fused) {  // tile (k+1,k+1) after round k: close it as P1(k+1) (R6 check included)
    small_close_any(a, acc, rowbuf, colbuf);
    if (a.early_pub) {
      // round k+1's panel tasks need only the panel copies D / D^T: publish them before the
      // matrix tile is stored, so the release fence does not wait for those 16 KB (the
      // kernel loop's publication after the task repeats diagready with ver and done3)
      small_store_diag(a, tk.k + 1, static_cast<T*>(nullptr), acc);
      __syncthreads();
      if (threadIdx.x == 32) {
        asm volatile("fence.release.gpu;" ::: "memory");
        st_relaxed(a.diagready + ((tk.k + 1) & 1), tk.k + 2);
      }
      small_store_tile(C, a.ld, acc);
      return;
    }
    small_store_diag(a, tk.k + 1, C, acc);
    return;
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    V4 v;
    v.x = acc[i][0]; v.y = acc[i][1]; v.z = acc[i][2]; v.w = acc[i][3];
    *reinterpret_cast<V4*>(C + (long long)(ty * 4 + i) * a.ld + tx * 4) = v;
    if (tk.type == T_P2R) *reinterpret_cast<V4*>(sp_row(a, tk.k, tk.j) + (ty * 4 + i) * SB + tx * 4) = v;
  }
  if (tk.type == T_P2C) {
    T* const ct = sp_colT(a, tk.k, tk.i);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      V4 w;
      w.x = acc[0][j]; w.y = acc[1][j]; w.z = acc[2][j]; w.w = acc[3][j];
      *reinterpret_cast<V4*>(ct + (tx * 4 + j) * SB + ty * 4) = w;
    }
  }
}

// N consecutive elements (N = 1, 2, 4; the address is N-element aligned) in one store
template <typename T, int N>
__device__ __forceinline__ void st_vec(T* dst, const T* v) {
  if constexpr (N == 4) {
    typename SV<T>::V4 x;
    x.x = v[0]; x.y = v[1]; x.z = v[2]; x.w = v[3];
    *reinterpret_cast<typename SV<T>::V4*>(dst) = x;
  } else if constexpr (N == 2) {
    typename SV<T>::V2 x;
    x.x = v[0]; x.y = v[1];
    *reinterpret_cast<typename SV<T>::V2*>(dst) = x;
  } else {
    dst[0] = v[0];
  }
}

// One part of a split chain panel task (see kPartShift): P2R(k; k,j) part q updates columns
// [q*C, (q+1)*C) of A(k,j) (C = 64/split; A = D via the panel copy D^T, B = those columns of A(k,j));
// P2C(k; i,k) part q updates rows [q*R, (q+1)*R) (A = those rows of A(i,k), transposed on load;
// B = D). 256 threads in a GX x (256 / GX) grid; thread (tx, ty) owns TR x TC outputs.
template <typename T, bool COLS, int TR, int TC, int GX = 16>
__device__ __forceinline__ void small_part(const SmArgs<T>& a, const Task& tk, int q, T* As, T* Bs) {
  constexpr int GY = SNT / GX;
  constexpr int R = GY * TR, CC = GX * TC;  // part rows / columns
  const int tid = threadIdx.x, tx = tid % GX, ty = tid / GX;
  const int r_off = COLS ? 0 : q * R, c_off = COLS ? q * CC : 0;
  T* const C = a.D + (long long)tk.i * SB * a.ld + (long long)tk.j * SB;
  if (COLS) {  // As[kk][r] = D^T (whole), Bs[kk][c] = A(k,j)[kk][c_off + c]
    const T* dt = sp_diagT(a, tk.k);
#pragma unroll
    for (int e = 0; e < 4; ++e) cp16(As + (tid + e * SNT) * 4, dt + (tid + e * SNT) * 4);
    constexpr int CH = CC / 4;  // 16-byte chunks per row
#pragma unroll
    for (int e = 0; e < (SB * CH + SNT - 1) / SNT; ++e) {
      const int x = tid + e * SNT;
      if (SB * CH % SNT == 0 || x < SB * CH) cp16(Bs + (x / CH) * CC + (x % CH) * 4, C + (long long)(x / CH) * a.ld + c_off + (x % CH) * 4);
    }
  } else {  // As[kk][r] = A(i,k)[r_off + r][kk] (4x4 register transpose), Bs = D (whole)
    const T* d = sp_diag(a, tk.k);
#pragma unroll
    for (int e = 0; e < 4; ++e) cp16(Bs + (tid + e * SNT) * 4, d + (tid + e * SNT) * 4);
    constexpr int RB = R / 4;  // 4x4 blocks per column strip
    if (tid < RB * 16) {
      using V4 = typename SV<T>::V4;
      const int r0 = (tid % RB) * 4, c0 = (tid / RB) * 4;
      V4 v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u)
        v[u] = __ldcg(reinterpret_cast<const V4*>(C + (long long)(r_off + r0 + u) * a.ld + c0));
      V4 w;
      w.x = v[0].x; w.y = v[1].x; w.z = v[2].x; w.w = v[3].x;
      *reinterpret_cast<V4*>(As + (c0 + 0) * R + r0) = w;
      w.x = v[0].y; w.y = v[1].y; w.z = v[2].y; w.w = v[3].y;
      *reinterpret_cast<V4*>(As + (c0 + 1) * R + r0) = w;
      w.x = v[0].z; w.y = v[1].z; w.z = v[2].z; w.w = v[3].z;
      *reinterpret_cast<V4*>(As + (c0 + 2) * R + r0) = w;
      w.x = v[0].w; w.y = v[1].w; w.z = v[2].w; w.w = v[3].w;
      *reinterpret_cast<V4*>(As + (c0 + 3) * R + r0) = w;
    }
  }
  cp_commit();
  T acc[TR][TC];
#pragma unroll
  for (int i = 0; i < TR; ++i)
#pragma unroll
    for (int j = 0; j < TC; ++j) acc[i][j] = __ldcg(C + (long long)(r_off + ty * TR + i) * a.ld + c_off + tx * TC + j);
  cp_wait_all();
  __syncthreads();
#pragma unroll 8
  for (int kk = 0; kk < SB; ++kk) {
    T A[TR], B[TC];
#pragma unroll
    for (int i = 0; i < TR; ++i) A[i] = As[kk * R + ty * TR + i];
#pragma unroll
    for (int j = 0; j < TC; ++j) B[j] = Bs[kk * CC + tx * TC + j];
#pragma unroll
    for (int i = 0; i < TR; ++i)
#pragma unroll
      for (int j = 0; j < TC; ++j) acc[i][j] = SV<T>::relax(A[i], B[j], acc[i][j]);
  }
  const int r0 = r_off + ty * TR, c0 = c_off + tx * TC;
#pragma unroll
  for (int i = 0; i < TR; ++i) {
    st_vec<T, TC>(C + (long long)(r0 + i) * a.ld + c0, acc[i]);
    if (COLS) st_vec<T, TC>(sp_row(a, tk.k, tk.j) + (r0 + i) * SB + c0, acc[i]);
  }
  if (!COLS) {
    T* const ct = sp_colT(a, tk.k, tk.i);
#pragma unroll
    for (int j = 0; j < TC; ++j) {
      T col[TR];
#pragma unroll
      for (int i = 0; i < TR; ++i) col[i] = acc[i][j];
      st_vec<T, TR>(ct + (c0 + j) * SB + r0, col);
    }
  }
}

template <typename T>
__device__ __forceinline__ void small_part_any(const SmArgs<T>& a, const Task& tk, T* As, T* Bs) {
  const int q = part_of(tk.type);
  Task w = tk;
  w.type = base_of(tk.type);
  if (w.type == T_P2R) {
    if (a.split == 16) small_part<T, true, 1, 1, 4>(a, w, q, As, Bs);       // 64 rows x 4 columns
    else if (a.split == 8) small_part<T, true, 2, 1, 8>(a, w, q, As, Bs);   // 64 rows x 8 columns
    else if (a.split == 4) small_part<T, true, 4, 1>(a, w, q, As, Bs);
    else small_part<T, true, 4, 2>(a, w, q, As, Bs);
  } else {
    if (a.split == 16) small_part<T, false, 1, 1, 64>(a, w, q, As, Bs);     // 4 rows x 64 columns
    else if (a.split == 8) small_part<T, false, 1, 2, 32>(a, w, q, As, Bs); // 8 rows x 64 columns
    else if (a.split == 4) small_part<T, false, 1, 4>(a, w, q, As, Bs);
    else small_part<T, false, 2, 4>(a, w, q, As, Bs);
  }
}

__device__ __forceinline__ Task small_task(const int4 e) {
  Task t;
  t.type = e.x; t.k = e.y; t.i = e.z; t.j = e.w;
  return t;
}

// Dependencies of a queue entry (one thread): deps_met's flags (own tile's version, the panel
// tiles / diagonal it reads, panel-copy parity reuse) with the split chain tiles read through
// their part counters, all loaded at once (one round trip), then an acquire fence once met.
// A fused F(k) needs those of P3(k; k+1,k+1) and of P1(k+1) (the panel copy of parity (k+1) % 2
// may be rewritten once round k-1's panel tasks, every part counted, are done).
template <typename T>
__device__ __forceinline__ bool small_deps(const SmArgs<T>& a, const Task& t) {
  const int type = base_of(t.type), nb = a.nb, k = t.k, p = k & 1, S = a.split;
  const bool sp = S > 1;
  const int* f[4];
  int v[4];
  // own tile: the chain tiles of round k-1 (P2R(k-1; k-1,k) / P2C(k-1; k,k-1)) finish as parts
  if (sp && k >= 1 && t.i == k - 1 && t.j == k) { f[0] = a.rsplit + k; v[0] = S; }
  else if (sp && k >= 1 && t.i == k && t.j == k - 1) { f[0] = a.csplit + k; v[0] = S; }
  else { f[0] = a.ver + (long long)t.i * nb + t.j; v[0] = k; }
  f[3] = f[0]; v[3] = v[0];
  if (type == T_P1) {
    f[1] = a.done2 + (k >= 2 ? k - 2 : 0); v[1] = k >= 2 ? 2 * (nb - 1) + 2 * (S - 1) : INT_MIN;
    f[2] = f[1]; v[2] = v[1];
  } else if (type == T_P3 || type == T_P3P1) {
    if (sp && t.j == k + 1) { f[1] = a.rsplit + t.j; v[1] = S; }
    else { f[1] = a.rowready + p * nb + t.j; v[1] = k + 1; }
    if (sp && t.i == k + 1) { f[2] = a.csplit + t.i; v[2] = S; }
    else { f[2] = a.colready + p * nb + t.i; v[2] = k + 1; }
    if (type == T_P3P1 && k >= 1) { f[3] = a.done2 + k - 1; v[3] = 2 * (nb - 1) + 2 * (S - 1); }
  } else {
    f[1] = a.diagready + p; v[1] = k + 1;
    f[2] = a.done3 + (k >= 2 ? k - 2 : 0); v[2] = k >= 2 ? (nb - 1) * (nb - 1) : INT_MIN;
  }
  const int x0 = ld_relaxed(f[0]), x1 = ld_relaxed(f[1]), x2 = ld_relaxed(f[2]), x3 = ld_relaxed(f[3]);
  if (x0 >= v[0] && x1 >= v[1] && x2 >= v[2] && x3 >= v[3]) {
    asm volatile("fence.acquire.gpu;" ::: "memory");
    return true;
  }
  return false;
}

template <typename T>
__device__ __forceinline__ void small_signal(const SmArgs<T>& a, const Task& t) {
  const int k = t.k, nb = a.nb;
  if (t.type >= (1 << kPartShift)) {  // a part of a split chain panel tile: count it
    asm volatile("fence.release.gpu;" ::: "memory");
    red_relaxed_add(base_of(t.type) == T_P2R ? a.rsplit + t.j : a.csplit + t.i, 1);
    red_relaxed_add(a.done2 + k, 1);
    return;
  }
  if (t.type != T_P3P1) {
    signal_done(a, t);
    return;
  }
  // F(k): tile (k+1,k+1) has rounds 0..k+1 applied; round k+1's diagonal is in the panel copy
  asm volatile("fence.release.gpu;" ::: "memory");
  st_relaxed(a.ver + (long long)t.i * nb + t.j, k + 2);
  st_relaxed(a.diagready + ((k + 1) & 1), k + 2);
  red_relaxed_add(a.done3 + k, 1);
}

template <typename T>
__global__ void __launch_bounds__(SNT) fw_small_kernel(const __grid_constant__ SmArgs<T> a) {
  __shared__ __align__(16) T As[STE];
  __shared__ __align__(16) T Bs[STE];
  __shared__ __align__(16) T rowbuf[2 * SB];
  __shared__ __align__(16) T colbuf[2 * SB];
  __shared__ SmSlot slot[2];
  const int tid = threadIdx.x;
  long long idx_next = 0;  // thread 0: queue index of the slot after N (fetched one task ahead)
  if (tid == 0) {
    const long long t0 = (long long)atomicAdd(a.counter, 1ull);
    slot[0].t = t0;
    slot[0].ready = 0;
    if (t0 < a.total) slot[0].tk = small_task(a.queue[t0]);
    slot[1].t = (long long)atomicAdd(a.counter, 1ull);
    slot[1].ready = 0;
  }
  __syncthreads();
  // thread 0's cycle counters (a.prof): [0] dependency waits, [1 + type] task bodies, [6 + type]
  // task counts, [11] publication
  unsigned long long pr[12] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  long long c0 = clock64();
  for (int it = 0;; ++it) {
    SmSlot& S = slot[it & 1];
    SmSlot& N = slot[(it + 1) & 1];
    if (S.t >= a.total) break;
    const Task tk = S.tk;
    int4 nq = make_int4(0, 0, 0, 0);
    if (tid == 0) {
      if (!S.ready)
        while (!small_deps(a, tk))
          if (!a.spin) __nanosleep(32);
      if (a.prof) {
        const long long c1 = clock64();
        pr[0] += c1 - c0;
        c0 = c1;
      }
      // N's entry and the next queue index: issued now, consumed after this task's work, so
      // their latency hides under it
      if (N.t < a.total) nq = a.queue[N.t];
      idx_next = (long long)atomicAdd(a.counter, 1ull);
    }
    __syncthreads();  // dependencies met (acquired by thread 0)
    if (tk.type == T_P1) small_phase1(a, tk, rowbuf, colbuf);
    else if (tk.type >= (1 << kPartShift)) small_part_any(a, tk, As, Bs);
    else small_minplus(a, tk, As, Bs, rowbuf, colbuf);
    if (tid == 0 && N.t < a.total) N.tk = small_task(nq);
    __syncthreads();  // every thread's stores of this task are issued; As / Bs free; N.tk published
    // publication (release fence + flags) by warp 1 while thread 0 checks the next task's flags:
    // two L2 round trips in parallel instead of one after the other
    if (tid == 32) small_signal(a, tk);
    if (tid == 0) {
      if (a.prof) {
        const long long c1 = clock64();
        pr[1 + base_of(tk.type)] += c1 - c0;
        pr[6 + base_of(tk.type)] += 1;
        c0 = c1;
      }
      // the next task's flags, once: if met, it starts without another wait
      N.ready = N.t < a.total && small_deps(a, N.tk);
      S.t = idx_next;  // this slot becomes the one after N (read by the others only after the
      S.ready = 0;     // next iteration's first barrier)
      if (a.prof) {
        const long long c1 = clock64();
        pr[11] += c1 - c0;
        c0 = c1;
      }
    }
  }
  if (a.prof && tid == 0)
    for (int x = 0; x < 12; ++x) a.prof[(long long)blockIdx.x * 16 + x] = pr[x];
  // The flags start every launch at zero: the last CTA to leave its task loop (no CTA reads a flag
  // after that) zeroes them, so a launch needs no memset in front of it (only the first one on a
  // work buffer: launch_fw_small).
  __shared__ int last;
  __syncthreads();
  if (tid == 0) last = atomicAdd(a.exitc, 1) == (int)gridDim.x - 1;
  __syncthreads();
  if (last) {
    int* const fw = reinterpret_cast<int*>(a.counter);
    for (long long x = tid; x < a.flag_words; x += SNT) fw[x] = 0;
  }
}

}  // namespace

// The small kernel's queue: critical-path list scheduling. Every task (k, i, j) of the blocked
// FW (P1 / P2R / P2C / P3 by position) is a node of the dependency graph the kernel waits on
// (previous round of the same tile; the diagonal / panel tiles it reads; the panel copies'
// parity reuse two rounds later); its bottom level = its duration + the longest chain of
// (hop + duration) after it. Entries are sorted by decreasing bottom level, which is a
// topological order (every edge strictly decreases it), so the queue is deadlock-free, and the
// chain phase 1 -> panel tiles -> next diagonal tile is always served first with the bulk
// filling the gaps. F(k) = P3(k; k+1,k+1) fused with P1(k+1) (one entry, type 4). Durations
// are model units (a 64^3 min-plus task ~3 us on one SM, phase 1 ~5 us, a flag hop ~1.5 us).
// Host and test hook (apsp_debug_queue, P = -1).
long long small_queue(int nb, long long delay, std::vector<int4>* q) {
  if (nb <= 0) return 0;
  // tuning experiments only: APSP_SMALL_QUEUE=decode (the 128-tile kernel's segment order,
  // no fusion) or bl_nofuse (list order without fused entries); default: list order + F(k)
  const int variant = small_variant();
  const int S = small_split_for(variant, nb);
  if (!q)  // the length alone (every launch asks for it): P1(k >= 1) lives inside F(k-1) when fused;
           // each round but the last has two chain panel tiles of S parts
    return (long long)nb * nb * nb - (variant == 1 || variant == 2 ? 0 : nb - 1) + 2ll * (S - 1) * (nb - 1);
  if (variant == 1 || variant == 3) {
    // the 128-tile kernel's segment order (decode with this queue delay); variant 3 fuses the tile (k+1,k+1)
    // of round k with the P1(k+1) that follows it
    std::vector<int4> v;
    const long long total = (long long)nb * nb * nb;
    for (long long g = 0; g < total; ++g) {
      const Task t = decode(g, nb, delay);
      if (variant == 3 && t.type == T_P1 && t.k >= 1) continue;  // inside F(k-1)
      if (variant == 3 && t.type == T_P3 && t.i == t.k + 1 && t.j == t.k + 1)
        v.push_back(make_int4(T_P3P1, t.k, t.i, t.j));
      else if (S > 1 && ((t.type == T_P2R && t.j == t.k + 1) || (t.type == T_P2C && t.i == t.k + 1)))
        for (int part = 0; part < S; ++part) v.push_back(make_int4(t.type + ((part + 1) << kPartShift), t.k, t.i, t.j));
      else
        v.push_back(make_int4(t.type, t.k, t.i, t.j));
    }
    if (q) *q = v;
    return (long long)v.size();
  }
  const double d13 = 3.0, d1 = 5.0, hop = 1.5;
  const long long N = (long long)nb * nb * nb;
  auto id = [&](int k, int i, int j) { return ((long long)k * nb + i) * nb + j; };
  std::vector<double> bl(N, 0.0);
  std::vector<double> maxP2(nb + 2, -1.0), maxP1(nb + 2, -1.0);
  auto dur = [&](int k, int i, int j) { return (i == k && j == k) ? d1 : d13; };
  for (int k = nb - 1; k >= 0; --k) {
    auto finish = [&](int i, int j) {  // bl of (k, i, j) from its successors
      double m = -1.0;
      if (k + 1 < nb) m = std::max(m, bl[id(k + 1, i, j)]);  // the tile's next round
      const bool p1 = i == k && j == k, p2r = i == k && j != k, p2c = j == k && i != k;
      if (p1)
        for (int x = 0; x < nb; ++x)
          if (x != k) m = std::max({m, bl[id(k, k, x)], bl[id(k, x, k)]});
      if (p2r)
        for (int x = 0; x < nb; ++x)
          if (x != k) m = std::max(m, bl[id(k, x, j)]);
      if (p2c)
        for (int x = 0; x < nb; ++x)
          if (x != k) m = std::max(m, bl[id(k, i, x)]);
      if ((p2r || p2c) && k + 2 < nb) m = std::max(m, maxP1[k + 2]);  // done2[k] -> P1(k+2)
      if (!p1 && !p2r && !p2c && k + 2 < nb) m = std::max(m, maxP2[k + 2]);  // done3[k] -> P2(k+2)
      bl[id(k, i, j)] = dur(k, i, j) + (m >= 0 ? hop + m : 0.0);
    };
    for (int i = 0; i < nb; ++i)
      for (int j = 0; j < nb; ++j)
        if (i != k && j != k) finish(i, j);
    for (int x = 0; x < nb; ++x)
      if (x != k) {
        finish(k, x);
        finish(x, k);
        maxP2[k] = std::max({maxP2[k], bl[id(k, k, x)], bl[id(k, x, k)]});
      }
    finish(k, k);
    maxP1[k] = bl[id(k, k, k)];
  }
  struct E {
    double key;
    int4 t;
  };
  std::vector<E> e;
  e.reserve(N);
  for (int k = 0; k < nb; ++k)
    for (int i = 0; i < nb; ++i)
      for (int j = 0; j < nb; ++j) {
        if (i == k && j == k) {
          if (k == 0 || variant == 2) e.push_back({bl[id(k, k, k)], make_int4(T_P1, k, k, k)});
          continue;  // P1(k >= 1) is fused into F(k-1)
        }
        if (variant != 2 && k + 1 < nb && i == k + 1 && j == k + 1) {  // F(k): P3 then P1(k+1), no hop
          e.push_back({d13 + bl[id(k + 1, k + 1, k + 1)], make_int4(T_P3P1, k, i, j)});
          continue;
        }
        const int type = i == k ? T_P2R : (j == k ? T_P2C : T_P3);
        e.push_back({bl[id(k, i, j)], make_int4(type, k, i, j)});
      }
  std::stable_sort(e.begin(), e.end(), [](const E& a, const E& b) { return a.key > b.key; });
  if (q) {
    q->resize(e.size());
    for (size_t x = 0; x < e.size(); ++x) (*q)[x] = e[x].t;
  }
  return (long long)e.size();
}

static long long small_pbuf_bytes(int nb, size_t elem) { return 2ll * (2 + 2 * nb) * STE * (long long)elem; }
static long long small_flag_bytes(int nb) {
  return ((2 + (long long)nb * nb + 2 + 4ll * nb + 2ll * nb + 2ll * nb + 1) * 4 + 15) / 16 * 16;
}

long long fw_small_work_bytes(int nb, size_t elem) {  // the queue is at most nb^3 + 30 (nb - 1) entries (split 16)
  return small_pbuf_bytes(nb, elem) + small_flag_bytes(nb) + ((long long)nb * nb * nb + 30ll * nb) * (long long)sizeof(int4);
}

template <typename T>
cudaError_t launch_fw_small(T* D, long long ld, int nb, void* work, int* negflag, long long delay, long long* queue_key,
                            int ctas_per_sm, cudaStream_t s) {
  if (nb <= 0) return cudaSuccess;
  int dev = 0, sms = 0;
  cudaError_t e;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  SmArgs<T> a;
  memset(&a, 0, sizeof(a));
  a.D = D;
  a.ld = ld;
  a.nb = nb;
  a.pbuf = static_cast<T*>(work);
  char* const fb = static_cast<char*>(work) + small_pbuf_bytes(nb, sizeof(T));
  int* f = reinterpret_cast<int*>(fb);
  a.counter = reinterpret_cast<unsigned long long*>(f); f += 2;
  a.ver = f; f += (long long)nb * nb;
  a.diagready = f; f += 2;
  a.rowready = f; f += 2 * nb;
  a.colready = f; f += 2 * nb;
  a.done2 = f; f += nb;
  a.done3 = f; f += nb;
  a.rsplit = f; f += nb;
  a.csplit = f; f += nb;
  a.exitc = f; f += 1;
  a.flag_words = f - reinterpret_cast<int*>(fb);
  const int variant = small_variant();
  a.split = small_split_for(variant, nb);
  // the queue in the work buffer was built for (variant, split, delay) = *queue_key (-1: none yet);
  // another configuration (tuning switches changed between launches) rebuilds it
  const long long key = ((long long)variant << 58) | ((long long)a.split << 52) | (delay & ((1ll << 52) - 1));
  const bool queue_loaded = *queue_key == key;
  a.negflag = negflag;
  const char* ep = getenv("APSP_SMALL_EARLYPUB");  // A/B (tuning only)
  a.early_pub = ep ? atoi(ep) : 1;  // measured n = 1024: 0.2377-0.2389 ms vs 0.2419-0.2448
  const char* sp = getenv("APSP_SMALL_SPIN");  // A/B (tuning only)
  a.spin = sp ? atoi(sp) : 0;
  const char* cv = getenv("APSP_SMALL_CLOSE");  // phase-1 variant A/B (tuning only)
  a.close_v = cv ? atoi(cv) : 1;
  // the queue lives in the work buffer: built and uploaded with the first launch on it
  int4* dq = reinterpret_cast<int4*>(fb + small_flag_bytes(nb));
  a.queue = dq;
  if (!queue_loaded) {
    std::vector<int4> q;
    a.total = small_queue(nb, delay, &q);
    if ((e = cudaMemcpyAsync(dq, q.data(), q.size() * sizeof(int4), cudaMemcpyHostToDevice, s)) != cudaSuccess)
      return e;
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;  // q is a local
    *queue_key = -1;  // set once the flags are zeroed too, below
  } else {
    a.total = small_queue(nb, delay, nullptr);
  }
  // zero flags: the previous launch's last CTA left them so (fw_small_kernel's epilogue); a new work
  // buffer is zeroed here, with its queue upload
  if (!queue_loaded) {
    if ((e = cudaMemsetAsync(a.counter, 0, small_flag_bytes(nb), s)) != cudaSuccess) return e;
    *queue_key = key;
  }
  // persistent grid: every CTA must be resident (tasks wait on each other)
  // (queried once: the event window of a small launch is ~0.3 ms, host work inside it shows)
  static int occ = 0;
  if (!occ && (e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fw_small_kernel<T>, SNT, 0)) != cudaSuccess)
    return e;
  if (occ < 1) return cudaErrorInvalidConfiguration;
  const int per_sm = ctas_per_sm < 1 ? 1 : (ctas_per_sm > occ ? occ : ctas_per_sm);
  long long grid = (long long)sms * per_sm;
  if (grid > a.total) grid = a.total;
  // APSP_SMALL_PROFILE=1 (tuning only): per-CTA cycle counters, summarised on stderr
  const bool prof = getenv("APSP_SMALL_PROFILE") != nullptr;
  if (prof && (e = cudaMalloc(&a.prof, grid * 16 * sizeof(unsigned long long))) != cudaSuccess) return e;
  if (prof && (e = cudaMemsetAsync(a.prof, 0, grid * 16 * sizeof(unsigned long long), s)) != cudaSuccess) return e;
  fw_small_kernel<T><<<(unsigned)grid, SNT, 0, s>>>(a);
  if ((e = cudaGetLastError()) != cudaSuccess || !prof) return e;
  std::vector<unsigned long long> hp(grid * 16);
  cudaStreamSynchronize(s);
  cudaMemcpy(hp.data(), a.prof, hp.size() * 8, cudaMemcpyDeviceToHost);
  cudaFree(a.prof);
  double t[12] = {0};
  for (long long b = 0; b < grid; ++b)
    for (int x = 0; x < 12; ++x) t[x] += (double)hp[b * 16 + x];
  const double all = t[0] + t[1] + t[2] + t[3] + t[4] + t[5] + t[11];
  fprintf(stderr, "[small] CTAs %lld: wait %.1f%% sig %.1f%% | per task (cycles): P1 %.0f P2R %.0f P2C %.0f P3 %.0f F %.0f"
                  " | counts %.0f %.0f %.0f %.0f %.0f | kernel cycles/CTA %.0f\n",
          grid, 100 * t[0] / all, 100 * t[11] / all, t[1] / std::max(1.0, t[6]), t[2] / std::max(1.0, t[7]),
          t[3] / std::max(1.0, t[8]), t[4] / std::max(1.0, t[9]), t[5] / std::max(1.0, t[10]), t[6], t[7], t[8], t[9],
          t[10], all / grid);
  return cudaSuccess;
}

template cudaError_t launch_fw_small<int>(int*, long long, int, void*, int*, long long, long long*, int, cudaStream_t);
template cudaError_t launch_fw_small<float>(float*, long long, int, void*, int*, long long, long long*, int, cudaStream_t);

}  // namespace apsp
