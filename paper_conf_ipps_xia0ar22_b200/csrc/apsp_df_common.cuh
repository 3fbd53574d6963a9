// apsp_df_common.cuh — pieces shared by the persistent dataflow kernels
// (apsp_fw_dataflow.cu: int32 / fp32; apsp_fw_dataflow16.cu: packed int16):
// PTX wrappers (cp.async, cp.async.bulk, mbarriers, relaxed flag accesses),
// the task decoding of the dependency-ordered queue and the per-tile flag
// protocol. See apsp_fw_dataflow.cu for the schedule. Internal (not the C ABI).
#pragma once
#include <cuda_runtime.h>
#include <climits>
#include <cstdint>

namespace apsp {
namespace {

__device__ __forceinline__ unsigned saddr(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void cp16(void* smem, const void* gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(saddr(smem)), "l"(gmem));
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;\n" ::); }
__device__ __forceinline__ void cp_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::); }
__device__ __forceinline__ void mb_init(unsigned bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mb_arrive(unsigned bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mb_wait(unsigned bar, unsigned parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "DFW_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra DFW_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void mb_expect_tx(unsigned bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(unsigned dst, const void* src, unsigned bytes, unsigned bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ void mb_cp_arrive_inc(unsigned bar) {  // counts +1 then -1: no net arrival
  asm volatile("cp.async.mbarrier.arrive.shared::cta.b64 [%0];" ::"r"(bar) : "memory");
}

__device__ __forceinline__ int ld_relaxed(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(int* p, int v) {
  asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_relaxed_add(int* p, int v) {
  asm volatile("red.relaxed.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// system scope (flags written or read by a peer GPU over NVLink, sharded kernel)
__device__ __forceinline__ int ld_relaxed_sys(const int* p) {
  int v;
  asm volatile("ld.relaxed.sys.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_sys(int* p, int v) {
  asm volatile("st.relaxed.sys.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_relaxed_sys_add(int* p, int v) {
  asm volatile("red.relaxed.sys.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

enum { T_P1 = 0, T_P2R = 1, T_P2C = 2, T_P3 = 3 };
struct Task {
  int type, k, i, j;
};

// i-th value of [0, nb) without the excluded values s0 < s1 < s2 (-1 = none)
__host__ __device__ __forceinline__ int skip3(int x, int s0, int s1, int s2) {
  if (s0 >= 0 && x >= s0) ++x;
  if (s1 >= 0 && x >= s1) ++x;
  if (s2 >= 0 && x >= s2) ++x;
  return x;
}

__host__ __device__ __forceinline__ Task p2_task(int nb, int k, long long x) {
  Task t;
  t.k = k;
  if (x < nb - 1) {
    t.type = T_P2R; t.i = k; t.j = skip3((int)x, k, -1, -1);
  } else {
    t.type = T_P2C; t.i = skip3((int)(x - (nb - 1)), k, -1, -1); t.j = k;
  }
  return t;
}
// G3L(k): (k+1,k+1), row k+1 (j not in {k,k+1}), column k+1 (i not in {k,k+1})
__host__ __device__ __forceinline__ Task g3l_task(int nb, int k, long long x) {
  Task t;
  t.type = T_P3; t.k = k;
  if (x == 0) { t.i = k + 1; t.j = k + 1; return t; }
  x -= 1;
  if (x < nb - 2) { t.i = k + 1; t.j = skip3((int)x, k, k + 1, -1); return t; }
  x -= nb - 2;
  t.i = skip3((int)x, k, k + 1, -1); t.j = k + 1;
  return t;
}
// The bulk of a round's phase 3 (an R x W block of tiles) in column bands of
// BAND tiles: all rows of band 0, then band 1, ... Consecutive tasks share the
// band's row-panel tiles (BAND x 64 KB, L2-resident) and one column-panel tile
// per row, so the round's panels never need to fit in L2 at once (at nb = 1024
// the two panels are 128 MB > the 126 MB L2; row-major order re-read the whole
// row panel from HBM for every tile row).
#ifndef DF_BAND
#define DF_BAND 64
#endif
constexpr int BAND = DF_BAND;
__host__ __device__ __forceinline__ void banded(long long x, int R, int W, int& r, int& c) {
  const int nfull = W / BAND;
  const long long per = (long long)R * BAND;
  if (x < nfull * per) {
    const int b = (int)(x / per);
    const long long y = x - b * per;
    r = (int)(y / BAND);
    c = b * BAND + (int)(y % BAND);
  } else {
    const long long y = x - nfull * per;
    const int wl = W - nfull * BAND;
    r = (int)(y / wl);
    c = nfull * BAND + (int)(y % wl);
  }
}

// G3R(k), k <= nb-2: tiles with i,j not in {k,k+1}; row k+2, column k+2 first
__host__ __device__ __forceinline__ Task g3r_task(int nb, int k, long long x) {
  Task t;
  t.type = T_P3; t.k = k;
  int r, c;
  if (k + 2 < nb) {
    if (x < nb - 2) { t.i = k + 2; t.j = skip3((int)x, k, k + 1, -1); return t; }
    x -= nb - 2;
    if (x < nb - 3) { t.i = skip3((int)x, k, k + 1, k + 2); t.j = k + 2; return t; }
    x -= nb - 3;
    banded(x, nb - 3, nb - 3, r, c);
    t.i = skip3(r, k, k + 1, k + 2);
    t.j = skip3(c, k, k + 1, k + 2);
    return t;
  }
  banded(x, nb - 2, nb - 2, r, c);
  t.i = skip3(r, k, k + 1, -1);
  t.j = skip3(c, k, k + 1, -1);
  return t;
}

__host__ __device__ Task decode(long long g, int nb, long long delay) {
  Task t;
  if (g == 0) { t.type = T_P1; t.k = 0; t.i = t.j = 0; return t; }
  g -= 1;
  const long long n1 = nb - 1, n2 = nb - 2;
  const long long s0 = 4 * n1;  // seg(0) = G2(0) + G3L(0) + P1(1)
  if (g < s0) {
    if (g < 2 * n1) return p2_task(nb, 0, g);
    g -= 2 * n1;
    if (g == 0) return g3l_task(nb, 0, 0);
    if (g == 1) { t.type = T_P1; t.k = 1; t.i = t.j = 1; return t; }
    return g3l_task(nb, 0, g - 1);
  }
  g -= s0;
  int k;
  long long r3;  // segment k: G3R(k-1) size r3
  const long long mid = (long long)(nb - 2) * nb * nb;  // segments 1..nb-2 are nb^2 tasks each
  if (g < mid) {
    k = 1 + (int)(g / ((long long)nb * nb));
    g -= (long long)(k - 1) * nb * nb;
    r3 = n2 * n2;

  } else {
    g -= mid;
    const long long last = n2 * n2 + 2 * n1;  // seg(nb-1) = G3R(nb-2) + G2(nb-1)
    if (g >= last) {                           // tail: G3R(nb-1), all (i,j) != nb-1
      g -= last;
      t.type = T_P3; t.k = nb - 1;
      int r, c;
      banded(g, (int)n1, (int)n1, r, c);
      t.i = r; t.j = c;
      return t;
    }
    k = nb - 1;
    r3 = n2 * n2;

  }
  const long long d = delay < r3 ? delay : r3;
  if (g < d) return g3r_task(nb, k - 1, g);
  g -= d;
  if (g < 2 * n1) return p2_task(nb, k, g);
  g -= 2 * n1;
  if (g < r3 - d) return g3r_task(nb, k - 1, d + g);
  g -= r3 - d;

  if (g == 0) return g3l_task(nb, k, 0);
  if (g == 1) { t.type = T_P1; t.k = k + 1; t.i = t.j = k + 1; return t; }
  return g3l_task(nb, k, g - 1);
}

// ---- two-round ("pair") schedule of the single-GPU int32 / fp32 kernel ---------------------
// Rounds are paired (k, k+1), k even. Every tile (i, j) with i, j not in {k, k+1} gets BOTH
// rounds' phase-3 updates in ONE task (T_PAIR: depth 256, the C tile read and written once per
// two rounds); the tiles on rows / columns k and k+1 stay single-round tasks. Panel copies are
// kept for four rounds (parity k % 4), so round k+2's and k+3's panels can be computed while
// the pairs of (k, k+1) still read theirs. Queue, segment p (k = 2p):
//   PRL(k-2)  pairs of (k-2, k-1) on rows / columns k and k+1: (k,k) first, then P1(k)
//   PRB(k-2)  the other pairs of (k-2, k-1) (banded), the first `delay` of them here
//   G2(k), G3L(k)[(k+1,k+1)], P1(k+1), G3L(k)[rest], G2(k+1), G3K(k+1), PRB(k-2)[delay:]
// where G3L(k) = round k on row / column k+1 and G3K(k+1) = round k+1 on row / column k.
// Segment 0 has no PRL / PRB; after the last pair, the tail is its PR (even nb) or, for odd
// nb, a last single round k = nb-1 (segment [PRL(k-2) with P1(k), PRB, G2(k)] + its phase 3).
// Every dependency of an entry lies earlier in the queue (tests/test_schedule.py).
enum { T_PAIR = 5 };

// x-th value of [0, nb) without the (distinct, any order, -1 = none) values e[0..3]
__host__ __device__ __forceinline__ int skip4(int x, int e0, int e1, int e2, int e3) {
  int e[4] = {e0, e1, e2, e3};
  for (int a = 0; a < 4; ++a)  // sort ascending, -1 last
    for (int b = a + 1; b < 4; ++b) {
      const bool swap = (e[b] >= 0 && (e[a] < 0 || e[b] < e[a]));
      if (swap) { const int t = e[a]; e[a] = e[b]; e[b] = t; }
    }
  for (int a = 0; a < 4; ++a)
    if (e[a] >= 0 && x >= e[a]) ++x;
  return x;
}

// G3K(k1): round k1 = k+1 on row / column k = k1-1 (tiles (k, j), j != k1; (i, k), i not in {k, k1})
__host__ __device__ __forceinline__ Task g3k_task(int nb, int k1, long long x) {
  Task t;
  t.type = T_P3; t.k = k1;
  const int k = k1 - 1;
  if (x < nb - 1) { t.i = k; t.j = skip3((int)x, k1, -1, -1); return t; }
  x -= nb - 1;
  t.i = skip3((int)x, k, k1, -1); t.j = k;
  return t;
}

// PRL(kp): pairs of (kp, kp+1) on rows / columns L = {k, k+1} < nb (k = kp+2), P1(k) second
__host__ __device__ __forceinline__ Task prl_task(int nb, int kp, long long x) {
  Task t;
  const int k = kp + 2, k1 = k + 1;
  t.type = T_PAIR; t.k = kp;
  if (x == 0) { t.i = k; t.j = k; return t; }
  if (x == 1) { t.type = T_P1; t.k = k; t.i = t.j = k; return t; }
  x -= 2;
  const int m = nb - 2;  // indices not in {kp, kp+1}
  if (x < m - 1) { t.i = k; t.j = skip4((int)x, kp, kp + 1, k, -1); return t; }      // row k
  x -= m - 1;
  if (x < m - 1) { t.i = skip4((int)x, kp, kp + 1, k, -1); t.j = k; return t; }      // column k
  x -= m - 1;
  if (x < m - 1) { t.i = k1; t.j = skip4((int)x, kp, kp + 1, k, -1); return t; }     // row k+1
  x -= m - 1;
  t.i = skip4((int)x, kp, kp + 1, k, k1); t.j = k1;                                  // column k+1
  return t;
}

__host__ __device__ __forceinline__ long long pair_prl_size(int nb, int k) {  // PRL(k-2), incl. P1(k)
  const long long m = nb - 2;
  return (k + 1 < nb) ? 4 * m - 3 : 2 * m;
}
__host__ __device__ __forceinline__ long long pair_singles_size(int nb) { return 8ll * nb - 9; }
__host__ __device__ __forceinline__ long long pair_seg_size(int nb, int k) {  // segment of pair k/2, k >= 2
  const long long m = nb - 2, c = (k + 1 < nb) ? 2 : 1;
  return pair_prl_size(nb, k) + (m - c) * (m - c) + ((k + 1 < nb) ? pair_singles_size(nb) : 2ll * nb - 2);
}
__host__ __device__ __forceinline__ long long pair_total(int nb) {
  if (nb == 1) return 1;
  const int np = nb / 2;  // pairs; odd nb: + the last single round k = nb - 1
  long long t = 8ll * nb - 8;  // segment 0: P1(0) + the singles of rounds 0, 1
  for (int p = 1; p < np; ++p) t += pair_seg_size(nb, 2 * p);
  if (nb & 1) t += pair_seg_size(nb, nb - 1) + (long long)(nb - 1) * (nb - 1);
  else t += (long long)(nb - 2) * (nb - 2);
  return t;
}

// the singles of pair (k, k+1), k + 1 < nb: G2(k), G3L(k)[0], P1(k+1), G3L(k)[1:], G2(k+1), G3K(k+1)
__host__ __device__ __forceinline__ Task pair_single(int nb, int k, long long x) {
  const long long n2 = 2ll * (nb - 1), n3 = 2ll * nb - 3;
  if (x < n2) return p2_task(nb, k, x);
  x -= n2;
  if (x == 0) return g3l_task(nb, k, 0);
  if (x == 1) { Task t; t.type = T_P1; t.k = k + 1; t.i = t.j = k + 1; return t; }
  x -= 2;
  if (x < n3 - 1) return g3l_task(nb, k, x + 1);
  x -= n3 - 1;
  if (x < n2) return p2_task(nb, k + 1, x);
  x -= n2;
  return g3k_task(nb, k + 1, x);
}

// PRB(kp): pairs of (kp, kp+1) on tiles with i, j not in {kp, kp+1, kp+2, kp+3 (< nb)}, banded
__host__ __device__ __forceinline__ Task prb_task(int nb, int kp, long long x) {
  const int e3 = kp + 3 < nb ? kp + 3 : -1, e2 = kp + 2 < nb ? kp + 2 : -1;
  const int w = nb - 2 - (e2 >= 0) - (e3 >= 0);
  int r, c;
  banded(x, w, w, r, c);
  Task t;
  t.type = T_PAIR; t.k = kp;
  t.i = skip4(r, kp, kp + 1, e2, e3);
  t.j = skip4(c, kp, kp + 1, e2, e3);
  return t;
}

__host__ __device__ Task decode2(long long g, int nb, long long delay) {
  Task t;
  if (g == 0) { t.type = T_P1; t.k = 0; t.i = t.j = 0; return t; }
  if (nb == 1) return t;
  g -= 1;
  const long long single = pair_singles_size(nb);
  if (g < single) return pair_single(nb, 0, g);
  g -= single;
  const int np = nb / 2;
  // middle segments p = 1 .. np-1 (k + 1 < nb) all have the same size
  const long long sm = np >= 2 ? pair_seg_size(nb, 2) : 0;
  const bool odd_tail = (nb & 1) != 0;
  int k;
  long long off;
  if (np >= 2 && g < (long long)(np - 1) * sm) {
    const int p = 1 + (int)(g / sm);
    k = 2 * p;
    off = g % sm;
  } else {
    g -= (long long)(np - 1) * sm;
    if (!odd_tail) {  // tail: the pairs of (nb-2, nb-1) on the tiles not in {nb-2, nb-1}
      const int kp = nb - 2, w = nb - 2;
      int r, c;
      banded(g, w, w, r, c);
      t.type = T_PAIR; t.k = kp; t.i = r; t.j = c;  // i, j < nb - 2: no skip needed
      return t;
    }
    k = nb - 1;  // odd nb: the last single round
    const long long sl = pair_seg_size(nb, k);
    if (g >= sl) {  // its phase 3, all (i, j) != k
      g -= sl;
      int r, c;
      banded(g, nb - 1, nb - 1, r, c);
      t.type = T_P3; t.k = k; t.i = r; t.j = c;  // k = nb - 1: no skip needed
      return t;
    }
    off = g;
  }
  // segment of round k (k = 2p, or the odd last single round): PRL(k-2), PRB(k-2)[0:d], singles, PRB[d:]
  const long long prl = pair_prl_size(nb, k);
  if (off < prl) return prl_task(nb, k - 2, off);
  off -= prl;
  const long long m = nb - 2, c = (k + 1 < nb) ? 2 : 1, prb = (m - c) * (m - c);
  const long long d = delay < prb ? delay : prb;
  if (off < d) return prb_task(nb, k - 2, off);
  off -= d;
  const long long sing = (k + 1 < nb) ? single : 2ll * nb - 2;
  if (off < sing) return (k + 1 < nb) ? pair_single(nb, k, off) : p2_task(nb, k, off);
  off -= sing;
  return prb_task(nb, k - 2, d + off);
}

// Dependency test and publication below work on any argument block with the
// flag fields of DFArgs (nb, ver, diagready, rowready, colready, done2, done3).
// Dependency test of task t (one thread): up to three flags, read with
// independent relaxed loads (one round trip), then an acquire fence once met.
template <class Args>
__device__ bool deps_met(const Args& a, const Task& t) {
  const int nb = a.nb, k = t.k, p = k & 1;
  const int* f0 = a.ver + (long long)t.i * nb + t.j;
  const int* f1;
  const int* f2;
  int v1, v2;
  const int v0 = k;
  if (t.type == T_P1) {
    f1 = a.done2 + (k >= 2 ? k - 2 : 0); v1 = k >= 2 ? 2 * (nb - 1) : INT_MIN;
    f2 = f1; v2 = v1;
  } else if (t.type == T_P3) {
    f1 = a.rowready + p * nb + t.j; v1 = k + 1;
    f2 = a.colready + p * nb + t.i; v2 = k + 1;
  } else {
    f1 = a.diagready + p; v1 = k + 1;
    f2 = a.done3 + (k >= 2 ? k - 2 : 0); v2 = k >= 2 ? (nb - 1) * (nb - 1) : INT_MIN;
  }
  const int x0 = ld_relaxed(f0), x1 = ld_relaxed(f1), x2 = ld_relaxed(f2);
  if (x0 >= v0 && x1 >= v1 && x2 >= v2) {
    // acquire: later reads (after the CTA learns of this) see the producers' data.
    // fence.acquire (an L1 invalidation here) instead of fence.acq_rel, which would
    // also wait for this thread's own outstanding copies
    asm volatile("fence.acquire.gpu;" ::: "memory");
    return true;
  }
  return false;
}

// Publish task t (one thread, after a group barrier that follows every
// thread's stores of t): one release fence, then the flags.
template <class Args>
__device__ void signal_done(const Args& a, const Task& t) {
  const int nb = a.nb, k = t.k, p = k & 1;
  asm volatile("fence.release.gpu;" ::: "memory");
  st_relaxed(a.ver + (long long)t.i * nb + t.j, k + 1);
  switch (t.type) {
    case T_P1: st_relaxed(a.diagready + p, k + 1); break;
    case T_P2R: st_relaxed(a.rowready + p * nb + t.j, k + 1); red_relaxed_add(a.done2 + k, 1); break;
    case T_P2C: st_relaxed(a.colready + p * nb + t.i, k + 1); red_relaxed_add(a.done2 + k, 1); break;
    default: red_relaxed_add(a.done3 + k, 1); break;
  }
}

// Dependencies / publication with a.npar panel-copy parities (the copies of round k are
// rewritten by round k + npar) and the pair task T_PAIR (rounds k, k+1 of one tile): any argument
// block with DFArgs' flag fields plus npar (the packed16 kernel; the int32 kernel keeps its own
// copies, deps_single / signal_single, whose code layout it was measured with).
template <class Args>
__device__ bool deps_np(const Args& a, const Task& t) {
  const int nb = a.nb, k = t.k, np = a.npar, p = k & (np - 1);
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
template <class Args>
__device__ void signal_np(const Args& a, const Task& t) {
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

}  // namespace
}  // namespace apsp
