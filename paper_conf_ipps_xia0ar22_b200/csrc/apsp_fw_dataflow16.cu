// apsp_fw_dataflow16.cu — the packed int16 blocked Floyd–Warshall (DESIGN.md
// reading R16) as ONE persistent dataflow launch: the schedule, task queue and
// flag protocol of apsp_fw_dataflow.cu (apsp_df_common.cuh), with the tile
// engine of the packed path (apsp_kernels16.cu): every 32-bit register holds
// two adjacent int16 columns and one VIADDMNMX.S16x2 (__viaddmin_s16x2)
// performs c = min(c, a + b) on both halves — 2 relaxations per instruction.
//
// Tasks (PAPER.md:62 steps 1-3; Alg. 1 l.3, l.7, l.11, l.17) and their panel
// copies, double-buffered by round parity p = k % 2:
//   P1(k)       closure of A(k,k) in int32 registers (as phase1_16_kernel);
//               writes D (int16, row-major) and D^T "dup" (32-bit words
//               [kk][r] holding D[r][kk] in both halves)
//   P2(k; k,j)  A(k,j) = D (x) A(k,j):  A operand D^T dup, B = the tile;
//               copy to the row panel (int16, row-major)
//   P2(k; i,k)  A(i,k) = A(i,k) (x) D:  A = the tile (transposed + duplicated
//               on load), B = D; copy to the column panel as dup words [c][r]
//   P3(k; i,j)  A(i,j) = min(A(i,j), colT(i) (x) row(j)): both operand chunks
//               are contiguous blocks of the panel copies (16 KB of dup words +
//               8 KB of int16), fetched by one thread with two cp.async.bulk
// The A operand is kept duplicated in the panel copy (64 KB per tile instead of
// 32 KB) so phase 3 stages it with a bulk copy instead of a register PRMT pass.
#include "apsp_kernels.cuh"
#include "apsp_df_common.cuh"

#include <cuda_runtime.h>
#include <climits>
#include <cstdint>
#include <cstdlib>

namespace apsp {
namespace {

#ifndef DF16_CTAS
#define DF16_CTAS 2
#endif
constexpr int BM = 128, BN = 128, BK = 32, GNT = 256, STAGES = 3, CTAS_PER_SM = DF16_CTAS;
constexpr int A_WORDS = BK * BM;                             // As[kk][r], 32-bit dup words
constexpr int B_HALVES = BK * BN;                            // Bs[kk][c], int16
constexpr int STAGE_BYTES = A_WORDS * 4 + B_HALVES * 2;      // 24 KB
constexpr long long T16 = (long long)BM * BN * 2;            // int16 tile
constexpr long long T32 = (long long)BM * BN * 4;            // dup-word tile
// the two-round (pair) queue by default: n = 16384 3.248e13 vs 3.193e13 one-round, n = 65536
// 3.346e13 vs 3.217e13 (the int16 tasks are twice as fast as int32 ones, so the
// per-task cost the pairs halve weighs twice as much)
constexpr bool kPair16Default = true;
// ... from nb = 128 on: below, the pair queue's longer chain per round costs more than the halved
// per-task overhead saves (n = 4096: 3.30 vs 2.64-2.71 ms; n = 8192: 18.2 vs 17.5 ms)
constexpr int kPair16MinNb = 128;
constexpr int SIG = 32, SCH = 64;
static_assert(64 * BN * 2 <= STAGE_BYTES, "half an int16 C tile must fit one stage");

__device__ __forceinline__ void gbar(int g) { asm volatile("bar.sync %0, %1;" ::"r"(g + 1), "r"(GNT) : "memory"); }
__device__ __forceinline__ unsigned dup_lo(unsigned w) { return __byte_perm(w, 0, 0x1010); }
__device__ __forceinline__ unsigned dup_hi(unsigned w) { return __byte_perm(w, 0, 0x3232); }
__device__ __forceinline__ unsigned dup16(int x) { return ((unsigned)x & 0xFFFFu) | ((unsigned)x << 16); }

struct DFArgs16 {
  short* D;  // n_pad x n_pad int16, row-major, ld
  long long ld;
  int nb;
  unsigned char* pbuf;  // 2 parities x [diag16 | diagT dup | nb row16 | nb colT dup]
  int* ver;
  int* diagready;
  int* rowready;
  int* colready;
  int* done2;
  int* done3;
  unsigned long long* counter;
  long long total;
  long long delay;
  unsigned long long* prof;
  int npar;   // panel-copy parities: 2, or 4 with the pair queue (round k's copies live until round k+4)
  int pairq;  // 1 = the two-round queue (decode2, T_PAIR: rounds k, k+1 of one tile in one depth-256 task)
};

__device__ __forceinline__ unsigned char* pb_base(const DFArgs16& a, int k) {
  return a.pbuf + (long long)(k & (a.npar - 1)) * (T16 + T32 + (long long)a.nb * (T16 + T32));
}
__device__ __forceinline__ short* pb_diag16(const DFArgs16& a, int k) { return reinterpret_cast<short*>(pb_base(a, k)); }
__device__ __forceinline__ unsigned* pb_diagTd(const DFArgs16& a, int k) {
  return reinterpret_cast<unsigned*>(pb_base(a, k) + T16);
}
__device__ __forceinline__ short* pb_row16(const DFArgs16& a, int k, int j) {
  return reinterpret_cast<short*>(pb_base(a, k) + T16 + T32 + (long long)j * T16);
}
__device__ __forceinline__ unsigned* pb_colTd(const DFArgs16& a, int k, int i) {
  return reinterpret_cast<unsigned*>(pb_base(a, k) + T16 + T32 + (long long)a.nb * T16 + (long long)i * T32);
}

// P1: closure of one int16 tile in int32 registers (weights >= 0 on this path:
// no negative-cycle check). Same ownership and row/column publication as
// group_phase1 in apsp_fw_dataflow.cu. Values never exceed INF16 (min with C).
__device__ __noinline__ void group_phase1_16(short* tile, long long ld, short* d16, unsigned* dTd, int* scratch, int g,
                                            int gtid) {
  int* rowbuf = scratch;            // [2][128]
  int* colbuf = scratch + 2 * 128;  // [2][128]
  const int tx = gtid & 15, ty = gtid >> 4;
  int acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    const short4 v0 = __ldcg(reinterpret_cast<const short4*>(tile + r * ld + tx * 4));
    const short4 v1 = __ldcg(reinterpret_cast<const short4*>(tile + r * ld + 64 + tx * 4));
    acc[i][0] = v0.x; acc[i][1] = v0.y; acc[i][2] = v0.z; acc[i][3] = v0.w;
    acc[i][4] = v1.x; acc[i][5] = v1.y; acc[i][6] = v1.z; acc[i][7] = v1.w;
  }
#pragma unroll
  for (int half = 0; half < 2; ++half) {
    for (int q = 0; q < 16; ++q) {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int p = u & 1;
        const int io = half * 4 + u;
        if (ty == q) {
          *reinterpret_cast<int4*>(&rowbuf[p * 128 + tx * 4]) = make_int4(acc[io][0], acc[io][1], acc[io][2], acc[io][3]);
          *reinterpret_cast<int4*>(&rowbuf[p * 128 + 64 + tx * 4]) =
              make_int4(acc[io][4], acc[io][5], acc[io][6], acc[io][7]);
        }
        if (tx == q) {
          *reinterpret_cast<int4*>(&colbuf[p * 128 + ty * 4]) = make_int4(acc[0][io], acc[1][io], acc[2][io], acc[3][io]);
          *reinterpret_cast<int4*>(&colbuf[p * 128 + 64 + ty * 4]) =
              make_int4(acc[4][io], acc[5][io], acc[6][io], acc[7][io]);
        }
        gbar(g);
        const int4 a0 = *reinterpret_cast<const int4*>(&colbuf[p * 128 + ty * 4]);
        const int4 a1 = *reinterpret_cast<const int4*>(&colbuf[p * 128 + 64 + ty * 4]);
        const int4 b0 = *reinterpret_cast<const int4*>(&rowbuf[p * 128 + tx * 4]);
        const int4 b1 = *reinterpret_cast<const int4*>(&rowbuf[p * 128 + 64 + tx * 4]);
        const int av[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const int bv[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[i][j] = __viaddmin_s32(av[i], bv[j], acc[i][j]);
      }
    }
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    const short4 v0 = make_short4((short)acc[i][0], (short)acc[i][1], (short)acc[i][2], (short)acc[i][3]);
    const short4 v1 = make_short4((short)acc[i][4], (short)acc[i][5], (short)acc[i][6], (short)acc[i][7]);
    *reinterpret_cast<short4*>(tile + r * ld + tx * 4) = v0;
    *reinterpret_cast<short4*>(tile + r * ld + 64 + tx * 4) = v1;
    *reinterpret_cast<short4*>(d16 + r * BN + tx * 4) = v0;
    *reinterpret_cast<short4*>(d16 + r * BN + 64 + tx * 4) = v1;
  }
#pragma unroll
  for (int j = 0; j < 8; ++j) {  // D^T dup: word [c][r] = D[r][c] in both halves
    const int c = (j < 4) ? (tx * 4 + j) : (64 + tx * 4 + j - 4);
    *reinterpret_cast<uint4*>(dTd + c * BM + ty * 4) =
        make_uint4(dup16(acc[0][j]), dup16(acc[1][j]), dup16(acc[2][j]), dup16(acc[3][j]));
    *reinterpret_cast<uint4*>(dTd + c * BM + 64 + ty * 4) =
        make_uint4(dup16(acc[4][j]), dup16(acc[5][j]), dup16(acc[6][j]), dup16(acc[7][j]));
  }
}

struct GDesc16 {
  const void* A;  // a_rows = 0: dup words [kk][r] (ld 128 words); 1: int16 tile rows r (ld lda), dup'ed on load
  const short* B; // int16 rows kk of 128 columns (ld ldb)
  const void* A2; // pair task: round k+1's panel copies (chunks 4..7), same layout as A / B
  const short* B2;
  int nk;         // chunks of depth 32: 4 (one round), 8 (pair task)
  const short* Cin;
  short* Cout;
  void* Cout2;    // c2 = 1: int16 copy (ld 128); c2 = 2: dup words transposed [c][r]; 0: none
  int lda, ldb, ldc;
  int a_rows, c2;
  int bulk;       // 1: A and B chunks are contiguous blocks of the panel copies
};

struct Slot16 {
  long long t;
  Task tk;
  GDesc16 d;
  int ready;
};

__device__ void fill_desc16(const DFArgs16& a, const Task& tk, GDesc16& d) {
  const int k = tk.k;
  short* const tile = a.D + (long long)tk.i * BM * a.ld + (long long)tk.j * BN;
  d.Cin = tile; d.Cout = tile; d.ldc = (int)a.ld;
  d.a_rows = 0; d.bulk = 0; d.nk = BM / BK; d.A2 = nullptr; d.B2 = nullptr;
  if (tk.type == T_P2R) {         // A(k,j) = D (x) A(k,j)
    d.A = pb_diagTd(a, k); d.lda = BM; d.B = tile; d.ldb = (int)a.ld;
    d.Cout2 = pb_row16(a, k, tk.j); d.c2 = 1;
  } else if (tk.type == T_P2C) {  // A(i,k) = A(i,k) (x) D
    d.A = tile; d.lda = (int)a.ld; d.a_rows = 1; d.B = pb_diag16(a, k); d.ldb = BN;
    d.Cout2 = pb_colTd(a, k, tk.i); d.c2 = 2;
  } else {                        // phase 3 from the panel copies
    d.A = pb_colTd(a, k, tk.i); d.lda = BM; d.B = pb_row16(a, k, tk.j); d.ldb = BN;
    d.Cout2 = nullptr; d.c2 = 0; d.bulk = 1;
    if (tk.type == T_PAIR) {      // then round k+1: min(., A(i,k+1) (x) A(k+1,j)) (min is order-free)
      d.A2 = pb_colTd(a, k + 1, tk.i); d.B2 = pb_row16(a, k + 1, tk.j); d.nk = 2 * (BM / BK);
    }
  }
}

// One 128x128 int16 min-plus tile update of depth 128 by a group (see
// group_minplus in apsp_fw_dataflow.cu for the chunk / barrier bookkeeping).
// Thread (ty, tx) owns rows {4ty..4ty+3, 64+4ty..64+4ty+3} x columns
// 8tx..8tx+7 (4 packed registers per row): per depth step 3 LDS.128 (two of
// dup'ed A, one of 8 int16 B) feed 32 VIADDMNMX.S16x2 = 64 relaxations.
__device__ __forceinline__ void group_minplus16(const GDesc16* d, unsigned char* stage0, unsigned full0, unsigned empty0,
                                            unsigned c0, int gtid, int g, const DFArgs16* args, long long nxt,
                                            Slot16* ns) {
  const int NK = d->nk;  // 4 chunks of depth 32 (8 for a pair task)
  const int lane = gtid & 31;
  const int tx = gtid & 15, ty = gtid >> 4;
  const bool bulk = d->bulk;
  auto load_chunk = [&](int stage, int c, long long wait_G) {
    unsigned char* st = stage0 + stage * STAGE_BYTES;
    unsigned* sa = reinterpret_cast<unsigned*>(st);
    short* sb = reinterpret_cast<short*>(st + A_WORDS * 4);
    if (bulk) {
      if (gtid == 0) {
        if (wait_G >= 0) mb_wait(empty0 + 8 * stage, ((unsigned)wait_G / STAGES) & 1);
        // generic -> async proxy: stage (shared::cta) and, once per task, the panel copies other
        // CTAs wrote with generic stores and this CTA acquired before the task (global)
        if (c == 0 || c == 4) asm volatile("fence.proxy.async.global;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mb_expect_tx(full0 + 8 * stage, A_WORDS * 4 + B_HALVES * 2);
        const int cr = c & 3;  // chunk within its round (pair tasks: chunks 4..7 from round k+1)
        const unsigned* const Ar = static_cast<const unsigned*>(c < 4 ? d->A : d->A2);
        const short* const Br = c < 4 ? d->B : d->B2;
        bulk_g2s(saddr(sa), Ar + (long long)cr * A_WORDS, A_WORDS * 4, full0 + 8 * stage);
        bulk_g2s(saddr(sb), Br + (long long)cr * B_HALVES, B_HALVES * 2, full0 + 8 * stage);
      }
      return;
    }
    if (wait_G >= 0) mb_wait(empty0 + 8 * stage, ((unsigned)wait_G / STAGES) & 1);
    const int ldb = d->ldb;
    const int brow = gtid >> 4, bpart = gtid & 15;  // B: 32 rows x 16 x 16 B
    if (!d->a_rows) {  // P2R: A = D^T dup (32 rows x 32 x 16 B), B = tile rows, both by cp.async
      const unsigned* ag = static_cast<const unsigned*>(d->A) + ((gtid >> 5) + c * BK) * BM + (gtid & 31) * 4;
      unsigned* const adst = sa + (gtid >> 5) * BM + (gtid & 31) * 4;
#pragma unroll
      for (int q = 0; q < 4; ++q) cp16(adst + q * 8 * BM, ag + q * 8 * BM);
#pragma unroll
      for (int q = 0; q < 2; ++q)
        cp16(sb + (brow + 16 * q) * BN + bpart * 8, d->B + (long long)(brow + 16 * q + c * BK) * ldb + bpart * 8);
      mb_cp_arrive_inc(full0 + 8 * stage);
    } else {  // P2C: A = tile rows, transposed and duplicated through registers; B = D
      const int r = gtid & (BM - 1), h = gtid >> 7;
      const short* ag = static_cast<const short*>(d->A) + (long long)r * d->lda + c * BK + h * 16;
      const uint4 v0 = __ldcg(reinterpret_cast<const uint4*>(ag));
      const uint4 v1 = __ldcg(reinterpret_cast<const uint4*>(ag + 8));
      uint4 w[2];
#pragma unroll
      for (int q = 0; q < 2; ++q) w[q] = __ldcg(reinterpret_cast<const uint4*>(d->B + (long long)(brow + 16 * q + c * BK) * ldb + bpart * 8));
      const unsigned x[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
#pragma unroll
      for (int m = 0; m < 8; ++m) {
        sa[(h * 16 + 2 * m) * BM + r] = dup_lo(x[m]);
        sa[(h * 16 + 2 * m + 1) * BM + r] = dup_hi(x[m]);
      }
#pragma unroll
      for (int q = 0; q < 2; ++q) *reinterpret_cast<uint4*>(sb + (brow + 16 * q) * BN + bpart * 8) = w[q];
    }
    gbar(g);
    if (gtid == 0) mb_arrive(full0 + 8 * stage);
  };
  load_chunk((int)(c0 % STAGES), 0, -1);
  load_chunk((int)((c0 + 1) % STAGES), 1, -1);

  unsigned acc[8][4];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int p = 0; p < 4; ++p) acc[i][p] = 0x7FFF7FFFu;
  // the C tile goes to the stages of chunks c0+NK-3 and c0+NK-2 (free during the last chunk)
  const unsigned g_lo = c0 + NK - 3, g_hi = c0 + NK - 2;
  const int s_lo = (int)(g_lo % STAGES), s_hi = (int)(g_hi % STAGES);

#pragma unroll 1
  for (int c = 0; c < NK; ++c) {
    const unsigned G = c0 + c;
    const int s = (int)(G % STAGES);
    if (c == NK - 1) {  // C (int16 128 x 256 B) into the two stages free during the last chunk
      mb_wait(empty0 + 8 * s_lo, (g_lo / STAGES) & 1);
      mb_wait(empty0 + 8 * s_hi, (g_hi / STAGES) & 1);
      const int ldc = d->ldc;
      short* const cs_lo = reinterpret_cast<short*>(stage0 + s_lo * STAGE_BYTES);
      short* const cs_hi = reinterpret_cast<short*>(stage0 + s_hi * STAGE_BYTES);
      const int cr = gtid >> 4, cc = (gtid & 15) * 8;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        cp16(cs_lo + (cr + 16 * q) * BN + cc, d->Cin + (long long)(cr + 16 * q) * ldc + cc);
        cp16(cs_hi + (cr + 16 * q) * BN + cc, d->Cin + (long long)(64 + cr + 16 * q) * ldc + cc);
      }
      cp_commit();
    }
    if (c == 1 && gtid == SCH) {
      ns->t = nxt;
      if (nxt < args->total) {
        const Task tn = args->pairq ? decode2(nxt, args->nb, args->delay) : decode(nxt, args->nb, args->delay);
        ns->tk = tn;
        if (tn.type != T_P1) fill_desc16(*args, tn, ns->d);
        ns->ready = deps_np(*args, tn) ? 1 : 0;
      }
    }
    mb_wait(full0 + 8 * s, (G / STAGES) & 1);
    const unsigned* as = reinterpret_cast<const unsigned*>(stage0 + s * STAGE_BYTES);
    const unsigned short* bs = reinterpret_cast<const unsigned short*>(stage0 + s * STAGE_BYTES + A_WORDS * 4);
#ifdef DF16_PIPE
    // operands of step kk+1 loaded into separate registers before step kk's
    // 32 DPX instructions (explicit register double-buffering)
    uint4 a0 = *reinterpret_cast<const uint4*>(as + ty * 4);
    uint4 a1 = *reinterpret_cast<const uint4*>(as + 64 + ty * 4);
    uint4 bv = *reinterpret_cast<const uint4*>(bs + tx * 8);
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      uint4 na0, na1, nbv;
      if (kk + 1 < BK) {
        na0 = *reinterpret_cast<const uint4*>(as + (kk + 1) * BM + ty * 4);
        na1 = *reinterpret_cast<const uint4*>(as + (kk + 1) * BM + 64 + ty * 4);
        nbv = *reinterpret_cast<const uint4*>(bs + (kk + 1) * BN + tx * 8);
      }
      const unsigned av[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
      const unsigned b[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int p = 0; p < 4; ++p) acc[i][p] = __viaddmin_s16x2(av[i], b[p], acc[i][p]);
      if (kk + 1 < BK) { a0 = na0; a1 = na1; bv = nbv; }
    }
#else
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      const uint4 a0 = *reinterpret_cast<const uint4*>(as + kk * BM + ty * 4);
      const uint4 a1 = *reinterpret_cast<const uint4*>(as + kk * BM + 64 + ty * 4);
      const uint4 bv = *reinterpret_cast<const uint4*>(bs + kk * BN + tx * 8);
      const unsigned av[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
      const unsigned b[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int p = 0; p < 4; ++p) acc[i][p] = __viaddmin_s16x2(av[i], b[p], acc[i][p]);
    }
#endif
    __syncwarp();
    if (lane == 0) mb_arrive(empty0 + 8 * s);
    if (c + 2 < NK) {
      const unsigned Gn = G + 2;
      load_chunk((int)(Gn % STAGES), c + 2, Gn >= STAGES ? (long long)(Gn - STAGES) : -1ll);
    }
  }
  cp_wait_all();
  gbar(g);
  {
    short* const Cout = d->Cout;
    const int ldc = d->ldc;
    const short* const cs_lo = reinterpret_cast<const short*>(stage0 + s_lo * STAGE_BYTES);
    const short* const cs_hi = reinterpret_cast<const short*>(stage0 + s_hi * STAGE_BYTES);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
      const uint4 cv = *reinterpret_cast<const uint4*>((i < 4 ? cs_lo : cs_hi) + (ty * 4 + (i & 3)) * BN + tx * 8);
      acc[i][0] = __vmins2(acc[i][0], cv.x);
      acc[i][1] = __vmins2(acc[i][1], cv.y);
      acc[i][2] = __vmins2(acc[i][2], cv.z);
      acc[i][3] = __vmins2(acc[i][3], cv.w);
      const uint4 o = make_uint4(acc[i][0], acc[i][1], acc[i][2], acc[i][3]);
      *reinterpret_cast<uint4*>(Cout + (long long)r * ldc + tx * 8) = o;
      if (d->c2 == 1) *reinterpret_cast<uint4*>(static_cast<short*>(d->Cout2) + r * BN + tx * 8) = o;
    }
    if (d->c2 == 2) {  // column panel copy, dup words transposed: [c][r], c = 8tx + j
      unsigned* const o2 = static_cast<unsigned*>(d->Cout2);
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const int c = tx * 8 + j;
        const int p = j >> 1;
        unsigned w[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) w[i] = (j & 1) ? dup_hi(acc[i][p]) : dup_lo(acc[i][p]);
        *reinterpret_cast<uint4*>(o2 + c * BM + ty * 4) = make_uint4(w[0], w[1], w[2], w[3]);
        *reinterpret_cast<uint4*>(o2 + c * BM + 64 + ty * 4) = make_uint4(w[4], w[5], w[6], w[7]);
      }
    }
  }
}

__global__ void __launch_bounds__(GNT, CTAS_PER_SM) fw_dataflow16_kernel(const __grid_constant__ DFArgs16 a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ __align__(8) unsigned long long bars[2 * STAGES];
  __shared__ Slot16 slots[2];
  const int gtid = threadIdx.x, g = 0;
  unsigned char* const stage0 = smem_raw;
  const unsigned full0 = saddr(&bars[0]), empty0 = full0 + 8 * STAGES;
  if (gtid == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mb_init(full0 + 8 * s, 1);
      mb_init(empty0 + 8 * s, GNT / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (gtid == SCH) {
    Slot16& s0 = slots[0];
    s0.t = (long long)atomicAdd(a.counter, 1ull);
    s0.ready = 0;
    if (s0.t < a.total) {
      s0.tk = a.pairq ? decode2(s0.t, a.nb, a.delay) : decode(s0.t, a.nb, a.delay);
      if (s0.tk.type != T_P1) fill_desc16(a, s0.tk, s0.d);
    }
  }
  gbar(g);
  unsigned chunk = 0;
  unsigned long long pr[6] = {0, 0, 0, 0, 0, 0};
  long long tc0 = clock64();
  for (int it = 0;; ++it) {
    Slot16& S = slots[it & 1];
    Slot16* N = &slots[(it + 1) & 1];
    const long long t = S.t;
    if (t >= a.total) break;
    const Task tk = S.tk;
    if (!S.ready) {
      if (gtid == SCH && !deps_np(a, tk)) {
        while (!deps_np(a, tk)) __nanosleep(64);
        pr[5]++;
      }
      gbar(g);
    }
    long long nxt = 0;
    if (gtid == SCH) nxt = (long long)atomicAdd(a.counter, 1ull);
    const long long tc1 = clock64();
    pr[0] += tc1 - tc0;
    if (tk.type == T_P1) {
      short* const tile = a.D + (long long)tk.i * BM * a.ld + (long long)tk.j * BN;
      group_phase1_16(tile, a.ld, pb_diag16(a, tk.k), pb_diagTd(a, tk.k), reinterpret_cast<int*>(stage0), g, gtid);
      if (gtid == SCH) {
        N->t = nxt;
        if (nxt < a.total) {
          N->tk = a.pairq ? decode2(nxt, a.nb, a.delay) : decode(nxt, a.nb, a.delay);
          N->ready = 0;
          if (N->tk.type != T_P1) fill_desc16(a, N->tk, N->d);
        }
      }
    } else {
      group_minplus16(&S.d, stage0, full0, empty0, chunk, gtid, g, &a, nxt, N);
      chunk += S.d.nk;
    }
    const long long tc2 = clock64();
    pr[1] += tc2 - tc1;
    if (tk.type == T_P1) pr[4] += tc2 - tc1;
    pr[3]++;
    gbar(g);
    if (gtid == SIG) signal_np(a, tk);
    tc0 = clock64();
    pr[2] += tc0 - tc2;
  }
  if (a.prof && gtid == SCH) {
    unsigned long long* o = a.prof + (long long)blockIdx.x * 8;
    for (int i = 0; i < 6; ++i) o[i] = pr[i];
  }
}

}  // namespace

long long fw_dataflow16_pbuf_bytes(int nb) { return 4ll * (T16 + T32 + (long long)nb * (T16 + T32)); }  // 4 parities
long long fw_dataflow16_work_bytes(int nb) { return fw_dataflow16_pbuf_bytes(nb) + fw_dataflow_flag_bytes(nb); }
int fw_dataflow16_ctas_per_sm() { return CTAS_PER_SM; }

cudaError_t launch_fw_dataflow16(short* D, long long ld, int nb, void* work, long long delay, cudaStream_t s,
                                 unsigned long long* prof) {
  if (nb <= 0) return cudaSuccess;
  const int smem = STAGES * STAGE_BYTES;
  cudaError_t e = cudaFuncSetAttribute(fw_dataflow16_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  DFArgs16 a;
  a.D = D; a.ld = ld; a.nb = nb;
  a.pbuf = static_cast<unsigned char*>(work);
  int* f = reinterpret_cast<int*>(static_cast<char*>(work) + fw_dataflow16_pbuf_bytes(nb));
  a.counter = reinterpret_cast<unsigned long long*>(f); f += 2;
  a.ver = f; f += (long long)nb * nb;
  a.diagready = f; f += 4;  // (the flag block is sized for 4 parities: fw_dataflow_flag_bytes)
  a.rowready = f; f += 4 * nb;
  a.colready = f; f += 4 * nb;
  a.done2 = f; f += nb;
  a.done3 = f; f += nb;
  // the two-round (pair) queue: APSP_DF16_PAIR=0/1 overrides the default (A/B)
  int pairq = kPair16Default && nb >= kPair16MinNb;
  if (const char* ev = getenv("APSP_DF16_PAIR")) pairq = atoi(ev) != 0 && nb >= 2;
  a.pairq = pairq;
  a.npar = pairq ? 4 : 2;
  a.total = pairq ? pair_total(nb) : (long long)nb * nb * nb;
  a.delay = delay;
  a.prof = prof;
  e = cudaMemsetAsync(a.counter, 0, fw_dataflow_flag_bytes(nb), s);
  if (e != cudaSuccess) return e;
  long long grid = (long long)sms * CTAS_PER_SM;
  if (grid > a.total) grid = a.total;
  fw_dataflow16_kernel<<<(unsigned)grid, GNT, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace apsp
