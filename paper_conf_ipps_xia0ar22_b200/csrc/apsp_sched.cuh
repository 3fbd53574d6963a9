// apsp_sched.cuh — building blocks shared by the in-core and out-of-core
// schedulers: min-plus tile-family descriptors and the blocked-FW closure of
// a square sub-matrix, which is both the whole in-core
// single-GPU algorithm and stage 1 of the out-of-core Algorithm 1
// ("apply the blocked version ... recursively").
#pragma once
#include "apsp_internal.h"

namespace apsp {

template <typename T>
inline MinPlusDesc<T> mkdesc(T* Cout, const T* Cin, const T* A, const T* B, long long ldc, long long lda,
                             long long ldb, int tiles_i, int tiles_j, int skip_i, int skip_j) {
  MinPlusDesc<T> d;
  d.Cout = Cout; d.Cin = Cin; d.A = A; d.B = B;
  d.ldc_out = ldc; d.ldc_in = ldc; d.lda = lda; d.ldb = ldb;
  d.tiles_i = tiles_i; d.tiles_j = tiles_j; d.skip_i = skip_i; d.skip_j = skip_j;
  return d;
}

template <typename T>
inline double desc_relax(const MinPlusDesc<T>& d, int K) {
  return (double)d.tiles_i * d.tiles_j * kTile * kTile * (double)K;
}

// Phases 1 and 2 of round k on the m x m sub-matrix at base (stream s).
template <typename T>
apsp_status fw_pivot(Handle* h, T* base, long long ld, long long m, long long k, cudaStream_t s) {
  const long long b = kTile, nb = m / b;
  apsp_status st;
  T* band = base + k * b * ld;
  h->ev_begin(0, s);
  if ((st = h->cuda(launch_phase1<T>(band + k * b, ld, h->d_flag, s), "phase1"))) return st;
  h->ev_end((double)b * b * b, s);
  if (nb == 1) return APSP_OK;
  MinPlusDesc<T> d[2];
  d[0] = mkdesc<T>(band, band, band + k * b, band, ld, ld, ld, 1, (int)(nb - 1), -1, (int)k);
  d[1] = mkdesc<T>(base + k * b, base + k * b, base + k * b, band + k * b, ld, ld, ld, (int)(nb - 1), 1, (int)k, -1);
  h->ev_begin(1, s);
  if ((st = h->cuda(launch_minplus<T>(d, 2, (int)b, s), "phase2"))) return st;
  h->ev_end(desc_relax(d[0], (int)b) + desc_relax(d[1], (int)b), s);
  return APSP_OK;
}

// Blocked FW closure of the m x m sub-matrix at `base` (row stride ld),
// rounds [k0, k1) of m/b. m is a multiple of b = kTile.
// Round k: phase 1 on A(k,k); phase 2 on row + column panels (one launch);
// phase 3 on all A(i,j), i != k, j != k.
//
// Lookahead (when h->side is set): phase 3 of round k is split into
//   3A  the tiles of row k+1 and column k+1 (the next round's panels), then
//   3B  every other tile (i, j not in {k, k+1}).
// Phases 1+2 of round k+1 only touch row/column k+1 and only need 3A, so they
// run on the high-priority side stream while 3B runs on s; round k+1's phase
// 3 waits for both. Phases 1 and 2 (a single CTA for ~20 us, then one wave)
// leave the critical path.
template <typename T>
apsp_status fw_closure(Handle* h, T* base, long long ld, long long m, long long k0, long long k1,
                       cudaStream_t s) {
  const long long b = kTile, nb = m / b;
  apsp_status st;
  const bool la = h->side != nullptr && nb > 2;
  if (k0 < k1 && (st = fw_pivot<T>(h, base, ld, m, k0, s))) return st;
  for (long long k = k0; k < k1; ++k) {
    T* band = base + k * b * ld;
    if (nb == 1) break;
    if (!la || k + 1 >= nb) {
      MinPlusDesc<T> p3 = mkdesc<T>(base, base, base + k * b, band, ld, ld, ld, (int)(nb - 1), (int)(nb - 1), (int)k,
                                    (int)k);
      h->ev_begin(2, s);
      if ((st = h->cuda(launch_minplus<T>(&p3, 1, (int)b, s), "phase3"))) return st;
      h->ev_end(desc_relax(p3, (int)b), s);
      if (k + 1 < k1 && (st = fw_pivot<T>(h, base, ld, m, k + 1, s))) return st;
      continue;
    }
    const long long k2 = k + 1;
    // 3A: row k+1 (all j != k) and column k+1 (i not in {k, k+1})
    MinPlusDesc<T> a[2];
    T* rowk2 = base + k2 * b * ld;
    a[0] = mkdesc<T>(rowk2, rowk2, rowk2 + k * b, band, ld, ld, ld, 1, (int)(nb - 1), -1, (int)k);
    a[1] = mkdesc<T>(base + k2 * b, base + k2 * b, base + k * b, band + k2 * b, ld, ld, ld, (int)(nb - 2), 1,
                     (int)k, -1);
    a[1].skip_i2 = (int)k2;
    h->ev_begin(2, s);
    if ((st = h->cuda(launch_minplus<T>(a, 2, (int)b, s), "phase3a"))) return st;
    h->ev_end(desc_relax(a[0], (int)b) + desc_relax(a[1], (int)b), s);
    if (k2 < k1) {
      if ((st = h->cuda(cudaEventRecord(h->ev_la[0], s), "event"))) return st;
      if ((st = h->cuda(cudaStreamWaitEvent(h->side, h->ev_la[0], 0), "wait"))) return st;
      if ((st = fw_pivot<T>(h, base, ld, m, k2, h->side))) return st;
      if ((st = h->cuda(cudaEventRecord(h->ev_la[1], h->side), "event"))) return st;
    }
    // 3B: the rest
    MinPlusDesc<T> p3 = mkdesc<T>(base, base, base + k * b, band, ld, ld, ld, (int)(nb - 2), (int)(nb - 2), (int)k,
                                  (int)k);
    p3.skip_i2 = (int)k2;
    p3.skip_j2 = (int)k2;
    h->ev_begin(2, s);
    if ((st = h->cuda(launch_minplus<T>(&p3, 1, (int)b, s), "phase3b"))) return st;
    h->ev_end(desc_relax(p3, (int)b), s);
    if (k2 < k1 && (st = h->cuda(cudaStreamWaitEvent(s, h->ev_la[1], 0), "wait"))) return st;
  }
  return APSP_OK;
}

}  // namespace apsp
