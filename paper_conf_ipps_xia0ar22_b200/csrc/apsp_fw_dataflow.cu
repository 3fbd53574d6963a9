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
#include <cstdint>

namespace apsp {
namespace {

#ifndef DF_GROUPS
#define DF_GROUPS 1
#endif
constexpr int BM = 128, BN = 128, BK = 32, GNT = 256, GROUPS = DF_GROUPS, STAGES = 3;
constexpr int CTAS_PER_SM = 2 / GROUPS;  // two groups per SM either way
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

template <typename T>
struct DFArgs {
  T* D;            // n_pad x n_pad, row-major, ld
  long long ld;
  int nb;
  T* pbuf;         // 2 x (2nb+1) tiles of 128x128: [p][0] diagonal, [p][1+j] row panel, [p][1+nb+i] column panel
  int* ver;        // nb*nb
  int* diagready;  // [2]
  int* rowready;   // [2][nb]
  int* colready;   // [2][nb]
  int* done2;      // [nb]
  int* done3;      // [nb]
  unsigned long long* counter;
  int* negflag;
  long long total;   // nb^3 tasks
  long long delay;   // G3R tasks placed before G2 in a segment
  long long stagger; // clock cycles group 1 waits before its first task
  unsigned long long* prof;  // optional [CTAs x GROUPS x 8] cycle counters (thread 0 of each group)
};


// panel copies of round k (parity k % 2), 128x128 tiles with ld 128:
//   D = A(k,k) closed, D^T, row panel A(k,j), column panel A(i,k) transposed
template <typename T>
__device__ __forceinline__ T* pb_diag(const DFArgs<T>& a, int k) {
  return a.pbuf + (long long)(k & 1) * (2 * a.nb + 2) * TILE_ELEMS;
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
__device__ __forceinline__ T* pb_colT(const DFArgs<T>& a, int k, int i) {
  return pb_diag(a, k) + (long long)(2 + a.nb + i) * TILE_ELEMS;
}


// Phase 1 inside a group: in-place FW closure of one 128x128 tile (the same
// register blocking as phase1_kernel in apsp_kernels.cu); result also to out2.
template <typename T>
__device__ __noinline__ void group_phase1(T* tile, long long ld, T* out2, T* out2t, int* negflag, T* scratch, int g,
                                         int gtid) {
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
};


// A group's task slot (shared memory, double-buffered by iteration parity):
// the task index, its decoded form, the operands of a min-plus task and
// whether its dependencies were already seen met. Thread 0 fills the slot of
// the next iteration while the current task runs.
template <typename T>
struct Slot {
  long long t;
  Task tk;
  GDesc<T> d;
  int ready;
};

template <typename T>
__device__ void fill_desc(const DFArgs<T>& a, const Task& tk, GDesc<T>& d) {
  const int k = tk.k;
  T* const tile = a.D + (long long)tk.i * BM * a.ld + (long long)tk.j * BN;
  d.Cin = tile; d.Cout = tile; d.ldc = (int)a.ld;
  d.a_rows = 0; d.c2t = 0; d.bulk = 0;
  if (tk.type == T_P2R) {         // A(k,j) = D (x) A(k,j)
    d.A = pb_diagT(a, k); d.lda = BM; d.B = tile; d.ldb = (int)a.ld; d.Cout2 = pb_row(a, k, tk.j);
  } else if (tk.type == T_P2C) {  // A(i,k) = A(i,k) (x) D; the copy goes to the transposed column panel
    d.A = tile; d.lda = (int)a.ld; d.a_rows = 1; d.B = pb_diag(a, k); d.ldb = BN;
    d.Cout2 = pb_colT(a, k, tk.i); d.c2t = 1;
  } else {                        // A(i,j) = min(A(i,j), A(i,k) (x) A(k,j)) from the panel copies
    d.A = pb_colT(a, k, tk.i); d.lda = BM; d.B = pb_row(a, k, tk.j); d.ldb = BN; d.Cout2 = nullptr;
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
#ifdef DF_INLINE
#define DF_MP_INLINE __forceinline__
#else
#define DF_MP_INLINE __noinline__
#endif
template <typename T>
__device__ DF_MP_INLINE void group_minplus(const GDesc<T>* d, T* stage0, unsigned full0, unsigned empty0, unsigned c0,
                                           int gtid, int g, const DFArgs<T>* args, long long nxt,
                                           Slot<T>* ns) {
  using V4 = typename DV<T>::V4;
  constexpr int NK = BM / BK;  // 4 chunks of depth 32
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
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        const unsigned bytes = BK * BM * (unsigned)sizeof(T);
        mb_expect_tx(full0 + 8 * stage, 2 * bytes);
        bulk_g2s(saddr(st), d->A + (long long)c * BK * BM, bytes, full0 + 8 * stage);
        bulk_g2s(saddr(st + BK * ALD), d->B + (long long)c * BK * BN, bytes, full0 + 8 * stage);
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
  load_chunk((int)(c0 % STAGES), 0, -1);  // (the previous task ended with a barrier)
  load_chunk((int)((c0 + 1) % STAGES), 1, -1);

  T acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = DV<T>::inf();
  const int s_lo = (int)((c0 + 1) % STAGES), s_hi = (int)((c0 + 2) % STAGES);

#pragma unroll 1
  for (int c = 0; c < NK; ++c) {
    const unsigned G = c0 + c;
    const int s = (int)(G % STAGES);
    if (c == NK - 1) {
      // C goes to the stages of chunks c0+1 and c0+2 once every warp released them
      mb_wait(empty0 + 8 * s_lo, ((c0 + 1) / STAGES) & 1);
      mb_wait(empty0 + 8 * s_hi, ((c0 + 2) / STAGES) & 1);
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
    if (c == 1 && gtid == SCH) {  // the next task's slot
      ns->t = nxt;
      if (nxt < args->total) {
        const Task tn = decode(nxt, args->nb, args->delay);
        ns->tk = tn;
        if (tn.type != T_P1) fill_desc(*args, tn, ns->d);
        ns->ready = deps_met(*args, tn) ? 1 : 0;
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
#pragma unroll
          for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int jp = 0; jp < 4; ++jp) {
              const float2 s0 = __fadd2_rn(make_float2(x0[i], x0[i]), p0[jp]);
              const float2 s1 = __fadd2_rn(make_float2(x1[i], x1[i]), p1[jp]);
              float& c0 = acc[4 * h + i][2 * jp];
              float& c1 = acc[4 * h + i][2 * jp + 1];
              c0 = fminf(fminf(c0, s0.x), s1.x);
              c1 = fminf(fminf(c1, s0.y), s1.y);
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
      const T* crow = (i < 4 ? cs_lo : cs_hi) + (ty * 4 + (i & 3)) * CLD;
      const V4 x0 = *reinterpret_cast<const V4*>(crow + tx * 4);
      const V4 x1 = *reinterpret_cast<const V4*>(crow + 64 + tx * 4);
      acc[i][0] = DV<T>::vmin(acc[i][0], x0.x); acc[i][1] = DV<T>::vmin(acc[i][1], x0.y);
      acc[i][2] = DV<T>::vmin(acc[i][2], x0.z); acc[i][3] = DV<T>::vmin(acc[i][3], x0.w);
      acc[i][4] = DV<T>::vmin(acc[i][4], x1.x); acc[i][5] = DV<T>::vmin(acc[i][5], x1.y);
      acc[i][6] = DV<T>::vmin(acc[i][6], x1.z); acc[i][7] = DV<T>::vmin(acc[i][7], x1.w);
      V4 v0, v1;
      v0.x = acc[i][0]; v0.y = acc[i][1]; v0.z = acc[i][2]; v0.w = acc[i][3];
      v1.x = acc[i][4]; v1.y = acc[i][5]; v1.z = acc[i][6]; v1.w = acc[i][7];
      *reinterpret_cast<V4*>(Cout + (long long)r * ldc + tx * 4) = v0;
      *reinterpret_cast<V4*>(Cout + (long long)r * ldc + 64 + tx * 4) = v1;
      if (Cout2 && !d->c2t) {
        *reinterpret_cast<V4*>(Cout2 + r * BN + tx * 4) = v0;
        *reinterpret_cast<V4*>(Cout2 + r * BN + 64 + tx * 4) = v1;
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

template <typename T>
__global__ void __launch_bounds__(GNT * GROUPS, CTAS_PER_SM) fw_dataflow_kernel(const __grid_constant__ DFArgs<T> a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ __align__(8) unsigned long long bars[GROUPS][2 * STAGES];
  __shared__ Slot<T> slots[GROUPS][2];
  const int g = threadIdx.x / GNT, gtid = threadIdx.x % GNT;
  T* const stage0 = reinterpret_cast<T*>(smem_raw) + g * STAGES * STAGE_ELEMS;
  const unsigned full0 = saddr(&bars[g][0]), empty0 = full0 + 8 * STAGES;
  if (gtid == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mb_init(full0 + 8 * s, 1);  // one arrival per chunk (+ transaction bytes of bulk copies)
      mb_init(empty0 + 8 * s, GNT / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (gtid == SCH) {
    if ((GROUPS > 1 ? g > 0 : blockIdx.x >= gridDim.x / 2) && a.stagger > 0) {  // half the groups start later
      const long long t0 = clock64();
      while (clock64() - t0 < a.stagger) __nanosleep(256);
    }
    Slot<T>& s0 = slots[g][0];
    s0.t = (long long)atomicAdd(a.counter, 1ull);
    s0.ready = 0;
    if (s0.t < a.total) {
      s0.tk = decode(s0.t, a.nb, a.delay);
      if (s0.tk.type != T_P1) fill_desc(a, s0.tk, s0.d);
    }
  }
  gbar(g);
  unsigned chunk = 0;
  unsigned long long pr[6] = {0, 0, 0, 0, 0, 0};  // wait, body, tail, tasks, p1 cycles, waits that blocked
  long long tc0 = clock64();
  for (int it = 0;; ++it) {
    Slot<T>& S = slots[g][it & 1];
    Slot<T>* N = &slots[g][(it + 1) & 1];
    const long long t = S.t;
    if (t >= a.total) break;
    const Task tk = S.tk;
    if (!S.ready) {  // uniform: the slot was published by the last barrier
      if (gtid == SCH && !deps_met(a, tk)) {
        while (!deps_met(a, tk)) __nanosleep(64);
        pr[5]++;
      }
      gbar(g);
    }
    long long nxt = 0;
    if (gtid == SCH) nxt = (long long)atomicAdd(a.counter, 1ull);  // the result is needed in chunk 1
    const long long tc1 = clock64();
    pr[0] += tc1 - tc0;
    if (tk.type == T_P1) {
      T* const tile = a.D + (long long)tk.i * BM * a.ld + (long long)tk.j * BN;
      group_phase1<T>(tile, a.ld, pb_diag(a, tk.k), pb_diagT(a, tk.k), a.negflag, stage0, g, gtid);
      if (gtid == SCH) {
        N->t = nxt;
        if (nxt < a.total) {
          N->tk = decode(nxt, a.nb, a.delay);
          N->ready = 0;
          if (N->tk.type != T_P1) fill_desc(a, N->tk, N->d);
        }
      }
    } else {
      group_minplus<T>(&S.d, stage0, full0, empty0, chunk, gtid, g, &a, nxt, N);
      chunk += BM / BK;
    }
    const long long tc2 = clock64();
    pr[1] += tc2 - tc1;
    if (tk.type == T_P1) pr[4] += tc2 - tc1;
    pr[3]++;
    gbar(g);  // every thread's stores of this task are issued; the next slot is published
    // published right away by the SIG thread (its warp absorbs the fence; measured
    // better than deferring it under the next task's first loads)
    if (gtid == SIG) signal_done(a, tk);
    tc0 = clock64();
    pr[2] += tc0 - tc2;
  }
  if (a.prof && gtid == SCH) {
    unsigned long long* o = a.prof + ((long long)blockIdx.x * GROUPS + g) * 8;
    for (int i = 0; i < 6; ++i) o[i] = pr[i];
  }
}

}  // namespace

template <typename T>
cudaError_t launch_fw_dataflow(T* D, long long ld, int nb, void* work, int* negflag, long long delay,
                               long long stagger, cudaStream_t s, unsigned long long* prof) {
  if (nb <= 0) return cudaSuccess;
  const int smem = GROUPS * STAGES * STAGE_ELEMS * (int)sizeof(T);
  cudaError_t e = cudaFuncSetAttribute(fw_dataflow_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  DFArgs<T> a;
  a.D = D; a.ld = ld; a.nb = nb;
  a.pbuf = static_cast<T*>(work);
  int* f = reinterpret_cast<int*>(static_cast<char*>(work) + fw_dataflow_pbuf_bytes(nb, sizeof(T)));
  a.counter = reinterpret_cast<unsigned long long*>(f); f += 2;  // first: 8-byte aligned
  a.ver = f; f += (long long)nb * nb;
  a.diagready = f; f += 2;
  a.rowready = f; f += 2 * nb;
  a.colready = f; f += 2 * nb;
  a.done2 = f; f += nb;
  a.done3 = f; f += nb;
  a.negflag = negflag;
  a.total = (long long)nb * nb * nb;
  a.delay = delay;
  a.stagger = stagger;
  a.prof = prof;
  e = cudaMemsetAsync(a.counter, 0, fw_dataflow_flag_bytes(nb), s);
  if (e != cudaSuccess) return e;
  long long grid = (long long)sms * CTAS_PER_SM;
  if (grid > a.total) grid = a.total;
  fw_dataflow_kernel<T><<<(unsigned)grid, GNT * GROUPS, smem, s>>>(a);
  return cudaGetLastError();
}

long long fw_dataflow_pbuf_bytes(int nb, size_t elem) {
  return 2ll * (2 * nb + 2) * TILE_ELEMS * (long long)elem;  // (kept a multiple of 8 bytes)
}
long long fw_dataflow_flag_bytes(int nb) { return ((long long)nb * nb + 6ll * nb + 4) * 4; }
long long fw_dataflow_work_bytes(int nb, size_t elem) {
  return fw_dataflow_pbuf_bytes(nb, elem) + fw_dataflow_flag_bytes(nb);
}

template cudaError_t launch_fw_dataflow<int>(int*, long long, int, void*, int*, long long, long long, cudaStream_t,
                                             unsigned long long*);
template cudaError_t launch_fw_dataflow<float>(float*, long long, int, void*, int*, long long, long long,
                                               cudaStream_t, unsigned long long*);

}  // namespace apsp
