// apsp_api.cu — the C ABI (include/apsp.h) and the round schedulers.
//
//   in-core, 1 GPU        rounds k = 0 .. n_pad/b - 1 of the blocked FW
//                         (PAPER.md:62): phase1 -> phase2 (row+col, one
//                         launch) -> phase3, all on one stream.
//   in-core, P ranks      1-D block-row shard (build extension; the paper is
//                         single-GPU). Round k: the owner of row
//                         band k runs phase 1 and the row panel, the band is
//                         broadcast (NCCL over NVLink, or a device copy in
//                         virtual-rank mode), then every rank updates its
//                         column-panel tiles and its phase-3 tiles.
//   out-of-core, 1 GPU    Algorithm 1 with super-blocks of
//                         B rows streamed from pinned host memory
//                         (apsp_ooc.cu).
#include "apsp_internal.h"

#include <cstdlib>
#include <nccl.h>
#include "apsp_sched.cuh"

#include <cstdio>
#include <cstring>
#include <cmath>
#include <cstdarg>
#include <string>
#include <vector>
#include <algorithm>

using namespace apsp;

static thread_local std::string g_last_error = "";

static apsp_status fail_global(apsp_status st, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return st;
}

namespace apsp {

apsp_status global_fail(apsp_status st, const char* msg) { return fail_global(st, "%s", msg); }

apsp_status Handle::fail(apsp_status st, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  err = buf;
  g_last_error = buf;
  if (st == APSP_ECUDA || st == APSP_ENCCL) poisoned = true;
  return st;
}

apsp_status Handle::cuda(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return APSP_OK;
  return fail(e == cudaErrorMemoryAllocation ? APSP_ENOMEM : APSP_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

void Handle::ev_begin(int cls, cudaStream_t s) {
  if (!timing) return;
  TimedEvent te;
  te.cls = cls;
  cudaEventCreate(&te.a);
  cudaEventCreate(&te.b);
  cudaEventRecord(te.a, s);
  events.push_back(te);
}

void Handle::ev_end(double relax, cudaStream_t s) {
  if (!timing || events.empty()) return;
  cudaEventRecord(events.back().b, s);
  events.back().relax = relax;
}

void Handle::collect_events() {
  for (auto& te : events) {
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, te.a, te.b) == cudaSuccess) {
      stats.ms[te.cls] += ms;
      stats.launches[te.cls] += 1;
      stats.relax[te.cls] += te.relax;
    }
    cudaEventDestroy(te.a);
    cudaEventDestroy(te.b);
  }
  events.clear();
}

// One round k of the in-core blocked FW over this handle's shards.
template <typename T>
static apsp_status incore_round(Handle* h, long long k) {
  const long long b = h->b, ld = h->ld, nb = h->n_pad / b;
  const long long R = h->rows_per_rank;
  const int owner = (int)((k * b) / R);
  cudaStream_t s = h->stream;
  apsp_status st;

  // ---- owner: phase 1 (+ row panel) on its band -------------------------
  Shard* own = nullptr;
  for (auto& sh : h->shards)
    if (sh.rank == owner) own = &sh;
  T* band = nullptr;
  if (own) {
    band = static_cast<T*>(own->D) + (k * b - own->row_begin) * ld;
    h->ev_begin(0);
    if ((st = h->cuda(launch_phase1<T>(band + k * b, ld, h->d_flag, s), "phase1"))) return st;
    h->ev_end((double)b * b * b);
    MinPlusDesc<T> dr = mkdesc<T>(band, band, band + k * b, band, ld, ld, ld, 1, (int)(nb - 1), -1, (int)k);
    h->ev_begin(1);
    if ((st = h->cuda(launch_minplus<T>(&dr, 1, (int)b, s), "phase2-row"))) return st;
    h->ev_end(desc_relax(dr, (int)b));
  }

  // ---- pivot band to every shard ------------------------------------------
  const T* panel = nullptr;
  const size_t band_elems = (size_t)b * (size_t)h->n_pad;
  h->ev_begin(3);
  if (h->virt) {
    if ((st = h->cuda(cudaMemcpyAsync(h->panel, band, band_elems * sizeof(T), cudaMemcpyDeviceToDevice, s),
                      "panel copy")))
      return st;
    panel = static_cast<const T*>(h->panel);
  } else {
    if ((st = h->bcast(own ? (void*)band : h->panel, band_elems * sizeof(T), owner, s))) return st;
    panel = own ? band : static_cast<const T*>(h->panel);
  }
  h->ev_end(0);

  // ---- every shard: column panel, then phase 3 ----------------------------
  for (auto& sh : h->shards) {
    T* D = static_cast<T*>(sh.D);
    const int local_tiles = (int)(R / b);
    const int skip_i = (sh.rank == owner) ? (int)((k * b - sh.row_begin) / b) : -1;
    const int tiles_i = local_tiles - (skip_i >= 0 ? 1 : 0);
    MinPlusDesc<T> dc = mkdesc<T>(D + k * b, D + k * b, D + k * b, panel + k * b, ld, ld, ld, tiles_i, 1, skip_i, -1);
    h->ev_begin(1);
    if ((st = h->cuda(launch_minplus<T>(&dc, 1, (int)b, s), "phase2-col"))) return st;
    h->ev_end(desc_relax(dc, (int)b));
    MinPlusDesc<T> p3 = mkdesc<T>(D, D, D + k * b, panel, ld, ld, ld, tiles_i, (int)(nb - 1), skip_i, (int)k);
    h->ev_begin(2);
    if ((st = h->cuda(launch_minplus<T>(&p3, 1, (int)b, s), "phase3"))) return st;
    h->ev_end(desc_relax(p3, (int)b));
  }
  return APSP_OK;
}

// All rounds of the sharded (1-D block-row) schedule with lookahead:
//   side stream X: pivot(k) = owner's phase 1 + row panel of band k, then the
//                  band broadcast (NCCL) / device copy into panel[k & 1];
//   main stream S: round k = every shard's column-panel tiles, then phase 3.
// During round k the owner of band k+1 first updates its band-(k+1) tiles, so
// pivot(k+1) — including its broadcast over NVLink — runs on X while S does the
// rest of round k's phase 3. A panel buffer is rewritten only after the phase 3
// that read it (two rounds earlier) has finished. All ranks issue the
// broadcasts in the same order (k = 0, 1, ...) on X.
template <typename T>
static apsp_status sharded_lookahead(Handle* h) {
  const long long b = h->b, ld = h->ld, nb = h->n_pad / b;
  const long long R = h->rows_per_rank;
  const int local_tiles = (int)(R / b);
  cudaStream_t S = h->stream, X = h->side;
  const size_t band_elems = (size_t)b * (size_t)h->n_pad;
  T* panels[2] = {static_cast<T*>(h->panel), static_cast<T*>(h->panel) + band_elems};
  apsp_status st;
  for (auto& e : h->ev_sh)
    if (!e && (st = h->cuda(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event"))) return st;
  cudaEvent_t ev_bcast = h->ev_sh[0], ev_band = h->ev_sh[1], ev_p3 = h->ev_sh[2];

  auto owner_of = [&](long long k) { return (int)((k * b) / R); };
  auto shard_of = [&](int rank) -> Shard* {
    for (auto& sh : h->shards)
      if (sh.rank == rank) return &sh;
    return nullptr;
  };
  auto local_tile = [&](const Shard* sh, long long k) { return (int)((k * b - sh->row_begin) / b); };
  auto Dp = [&](const Shard* sh) { return static_cast<T*>(sh->D); };

  // pivot(k) on X; returns the panel round k reads
  auto pivot = [&](long long k, const T*& panel_k) -> apsp_status {
    Shard* own = shard_of(owner_of(k));
    T* band = own ? Dp(own) + (long long)local_tile(own, k) * b * ld : nullptr;
    if (own) {
      h->ev_begin(0, X);
      if ((st = h->cuda(launch_phase1<T>(band + k * b, ld, h->d_flag, X), "phase1"))) return st;
      h->ev_end((double)b * b * b, X);
      MinPlusDesc<T> dr = mkdesc<T>(band, band, band + k * b, band, ld, ld, ld, 1, (int)(nb - 1), -1, (int)k);
      h->ev_begin(1, X);
      if ((st = h->cuda(launch_minplus<T>(&dr, 1, (int)b, X), "phase2-row"))) return st;
      h->ev_end(desc_relax(dr, (int)b), X);
    }
    // panel[k & 1] was last read by round k-2, whose end is ev_p3's latest record
    if (k >= 2 && (st = h->cuda(cudaStreamWaitEvent(X, ev_p3, 0), "wait"))) return st;
    T* dst = panels[k & 1];
    h->ev_begin(3, X);
    if (h->virt) {
      if ((st = h->cuda(cudaMemcpyAsync(dst, band, band_elems * sizeof(T), cudaMemcpyDeviceToDevice, X), "panel")))
        return st;
      panel_k = dst;
    } else {
      if ((st = h->bcast(own ? (void*)band : (void*)dst, band_elems * sizeof(T), owner_of(k), X))) return st;
      panel_k = own ? band : dst;
    }
    h->ev_end(0, X);
    return h->cuda(cudaEventRecord(ev_bcast, X), "event");
  };

  const T* next_panel = nullptr;
  if ((st = h->cuda(cudaEventRecord(ev_p3, S), "event"))) return st;  // X must not run ahead of prior S work
  if ((st = h->cuda(cudaStreamWaitEvent(X, ev_p3, 0), "wait"))) return st;
  if ((st = pivot(0, next_panel))) return st;
  for (long long k = 0; k < nb; ++k) {
    const T* panel = next_panel;
    if ((st = h->cuda(cudaStreamWaitEvent(S, ev_bcast, 0), "wait"))) return st;
    // column-panel tiles of every shard
    for (auto& sh : h->shards) {
      const int skip = sh.rank == owner_of(k) ? local_tile(&sh, k) : -1;
      T* D = Dp(&sh);
      MinPlusDesc<T> dc = mkdesc<T>(D + k * b, D + k * b, D + k * b, panel + k * b, ld, ld, ld,
                                    local_tiles - (skip >= 0), 1, skip, -1);
      h->ev_begin(1, S);
      if ((st = h->cuda(launch_minplus<T>(&dc, 1, (int)b, S), "phase2-col"))) return st;
      h->ev_end(desc_relax(dc, (int)b), S);
    }
    const long long k1 = k + 1;
    Shard* own1 = k1 < nb ? shard_of(owner_of(k1)) : nullptr;
    if (own1) {  // band k+1 first, then its pivot can start on X
      T* D = Dp(own1);
      T* row = D + (long long)local_tile(own1, k1) * b * ld;
      MinPlusDesc<T> pa = mkdesc<T>(row, row, row + k * b, panel, ld, ld, ld, 1, (int)(nb - 1), -1, (int)k);
      h->ev_begin(2, S);
      if ((st = h->cuda(launch_minplus<T>(&pa, 1, (int)b, S), "phase3a"))) return st;
      h->ev_end(desc_relax(pa, (int)b), S);
      if ((st = h->cuda(cudaEventRecord(ev_band, S), "event"))) return st;
      if ((st = h->cuda(cudaStreamWaitEvent(X, ev_band, 0), "wait"))) return st;
    }
    if (k1 < nb && (st = pivot(k1, next_panel))) return st;
    // the rest of phase 3
    for (auto& sh : h->shards) {
      int s0 = sh.rank == owner_of(k) ? local_tile(&sh, k) : -1;
      int s1 = (own1 == &sh) ? local_tile(&sh, k1) : -1;
      if (s0 < 0) std::swap(s0, s1);
      const int tiles_i = local_tiles - (s0 >= 0) - (s1 >= 0);
      if (tiles_i <= 0) continue;
      T* D = Dp(&sh);
      MinPlusDesc<T> p3 = mkdesc<T>(D, D, D + k * b, panel, ld, ld, ld, tiles_i, (int)(nb - 1), s0, (int)k);
      p3.skip_i2 = s1;
      h->ev_begin(2, S);
      if ((st = h->cuda(launch_minplus<T>(&p3, 1, (int)b, S), "phase3"))) return st;
      h->ev_end(desc_relax(p3, (int)b), S);
    }
    if ((st = h->cuda(cudaEventRecord(ev_p3, S), "event"))) return st;
  }
  return APSP_OK;
}

// All rounds of a single-GPU in-core closure in one persistent dataflow launch
// (apsp_fw_dataflow.cu). The phases are not separable in time, so the launch
// is timed as one event of class 2 carrying all n_pad^3 relaxations.
// Small n (apsp_fw_small.cu): the same schedule with 64x64 tiles, all rounds in one launch.
template <typename T>
static apsp_status run_small(Handle* h) {
  const int nb = (int)(h->n_pad / 64);
  apsp_status st;
  const long long wb = fw_small_work_bytes(nb, sizeof(T));
  if (!h->df_work) {
    if ((st = h->cuda(cudaMallocAsync(&h->df_work, wb, h->stream), "cudaMalloc dataflow (small)"))) return st;
    h->device_bytes += wb;
  }
  // CTAs per SM and queue delay measured per size: one CTA per SM up to
  // n_pad = 1024 (the critical path dominates), two above (more tasks per round in flight)
  int ctas = h->n_pad <= 1024 ? 1 : 2;
  if (const char* e = getenv("APSP_SMALL_CTAS")) ctas = atoi(e);  // tuning experiments only
  const long long delay = h->df_delay > 0 ? h->df_delay : kSmallDelay;
  h->kernel = APSP_KERNEL_SMALL;
  h->ev_begin(2);
  if ((st = h->cuda(launch_fw_small<T>(static_cast<T*>(h->shards[0].D), h->ld, nb, h->df_work, h->d_flag, delay,
                                       &h->small_queue_key, ctas, h->stream),
                    "fw_small")))
    return st;
  h->ev_end((double)h->n_pad * h->n_pad * h->n_pad);
  return APSP_OK;
}

template <typename T>
static apsp_status run_dataflow(Handle* h, bool timed = true) {
  if (h->small) return run_small<T>(h);
  const int nb = (int)(h->n_pad / h->b);
  apsp_status st;
  if (!h->df_work) {
    long long wb = fw_dataflow_work_bytes(nb, sizeof(T));
    if (getenv("APSP_DF_WORK2")) wb = fw_dataflow_work_bytes(nb, nb, sizeof(T));  // A/B: 2-parity size
    if ((st = h->cuda(cudaMallocAsync(&h->df_work, wb, h->stream), "cudaMalloc dataflow"))) return st;
    h->device_bytes += wb;
  }
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const long long delay = h->df_delay > 0 ? h->df_delay : 8ll * sms;
  long long stagger = 0;
  if (const char* e = getenv("APSP_DF_STAGGER")) stagger = atoll(e);  // tuning experiments only
  // APSP_DF_PROFILE=1: per-group cycle counters printed to stderr (tuning experiments only)
  unsigned long long* prof = nullptr;
  const bool want_prof = getenv("APSP_DF_PROFILE") != nullptr;
  const size_t prof_bytes = (size_t)sms * 2 * 8 * sizeof(unsigned long long);  // 2 groups per SM
  if (want_prof && (st = h->cuda(cudaMalloc(&prof, prof_bytes), "cudaMalloc prof"))) return st;
  if (timed) h->ev_begin(2);
  int used_pair = 0;
  if ((st = h->cuda(launch_fw_dataflow<T>(static_cast<T*>(h->shards[0].D), h->ld, nb, h->df_work, h->d_flag, delay,
                                          stagger, h->stream, prof, &used_pair),
                    "fw_dataflow")))
    return st;
  h->kernel = used_pair ? APSP_KERNEL_DATAFLOW_PAIR : APSP_KERNEL_DATAFLOW;
  if (timed) h->ev_end((double)h->n_pad * h->n_pad * h->n_pad);
  if (want_prof) {
    std::vector<unsigned long long> hp(prof_bytes / 8);
    cudaStreamSynchronize(h->stream);
    cudaMemcpy(hp.data(), prof, prof_bytes, cudaMemcpyDeviceToHost);
    cudaFree(prof);
    double tot[6] = {0, 0, 0, 0, 0, 0};
    for (int i = 0; i < sms * 2; ++i)
      for (int j = 0; j < 6; ++j) tot[j] += (double)hp[(size_t)i * 8 + j];
    const double all = tot[0] + tot[1] + tot[2];
    fprintf(stderr, "[df] groups %d: wait %.2f%% body %.2f%% tail %.2f%% | tasks %.0f blocked %.0f p1 %.2f%% | "
            "body/task %.0f cyc\n", sms * 2, 100 * tot[0] / all, 100 * tot[1] / all, 100 * tot[2] / all, tot[3],
            tot[5], 100 * tot[4] / all, (tot[1] - tot[4]) / (tot[3] - nb));
  }
  return APSP_OK;
}

// All rounds over a 1-D block-row shard in one persistent launch per GPU
// (launch_fw_dataflow_sharded): the owner of each round stores the pivot panels
// into every rank's panel buffer itself (peer stores over NVLink between GPUs,
// plain stores between virtual ranks), so no collective runs between rounds.
// NCCL ranks exchange CUDA IPC handles of their work buffers once (ncclAllGather)
// and pass a barrier after zeroing their flags, before any peer may store into them.
template <typename T>
static apsp_status run_dataflow_sharded(Handle* h) {
  const int nb = (int)(h->n_pad / h->b), P = h->world, nl = nb / P;
  const long long wb = fw_dataflow_work_bytes(nb, nl, sizeof(T));
  const long long pbb = fw_dataflow_pbuf_bytes(nb, nl, sizeof(T), 2), fbb = fw_dataflow_flag_bytes(nb, nl);
  apsp_status st;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const long long delay = h->df_delay > 0 ? h->df_delay : 8ll * sms / (h->virt ? P : 1);
  std::vector<DFShard> ranks;
  if (h->virt) {
    if (h->sh_work.empty()) {
      for (int r = 0; r < P; ++r) {
        void* w = nullptr;
        if ((st = h->cuda(cudaMallocAsync(&w, wb, h->stream), "cudaMalloc dataflow shard"))) return st;
        h->sh_work.push_back(w);
        h->device_bytes += wb;
      }
    }
    for (int r = 0; r < P; ++r) {
      DFShard d;
      memset(&d, 0, sizeof(d));
      d.rank = r;
      d.D = h->shards[r].D;
      d.work = h->sh_work[r];
      for (int e = 0; e < P; ++e) d.peer_work[e] = h->sh_work[e];
      ranks.push_back(d);
      if ((st = h->cuda(cudaMemsetAsync(static_cast<char*>(h->sh_work[r]) + pbb, 0, fbb, h->stream), "memset flags")))
        return st;
    }
  } else {
    // (work buffer and peer mappings: prepare_sharded_peers, called by run_incore_rounds)
    DFShard d;
    memset(&d, 0, sizeof(d));
    d.rank = h->rank;
    d.D = h->shards[0].D;
    d.work = h->sh_work[0];
    for (int e = 0; e < P; ++e) d.peer_work[e] = h->sh_peer[e];
    ranks.push_back(d);
    if ((st = h->cuda(cudaMemsetAsync(static_cast<char*>(h->sh_work[0]) + pbb, 0, fbb, h->stream), "memset flags")))
      return st;
    if (P > 1) {  // every rank's flags are zero before any rank's kernel may store into them
      ncclResult_t r = ncclAllReduce(h->d_flag, h->d_flag, 1, ncclInt32, ncclMax, static_cast<ncclComm_t>(h->comm),
                                     h->stream);
      if (r != ncclSuccess) return h->fail(APSP_ENCCL, "ncclAllReduce(barrier): %s", ncclGetErrorString(r));
    }
  }
  h->ev_begin(2);
  if ((st = h->cuda(launch_fw_dataflow_sharded<T>(ranks.data(), (int)ranks.size(), P, nb, h->ld, h->d_flag, delay,
                                                  h->stream),
                    "fw_dataflow_sharded")))
    return st;
  h->ev_end((double)h->n_pad * h->n_pad * h->n_pad / (h->virt ? 1 : P));
  return APSP_OK;
}

// NCCL ranks: this rank's shard work buffer (plain cudaMalloc, exportable through CUDA
// IPC) and every peer's, mapped once per handle: the 64-B IPC handles are all-gathered
// over the communicator, then every rank reports whether it could open all of them
// (all-reduce min). If any rank could not (no P2P path between the GPUs), every rank
// keeps the launch-per-phase schedule with NCCL broadcasts (h->sh_disabled).
template <typename T>
static apsp_status prepare_sharded_peers(Handle* h) {
  if (h->sh_ipc_open || h->sh_disabled) return APSP_OK;
  const int nb = (int)(h->n_pad / h->b), P = h->world, nl = nb / P;
  const long long wb = fw_dataflow_work_bytes(nb, nl, sizeof(T));
  apsp_status st;
  if (h->sh_work.empty()) {
    void* w = nullptr;
    if ((st = h->cuda(cudaMalloc(&w, wb), "cudaMalloc dataflow shard"))) return st;
    h->sh_work.push_back(w);
    h->device_bytes += wb;
  }
  h->sh_peer[h->rank] = h->sh_work[0];
  if (P == 1) {
    h->sh_ipc_open = true;
    return APSP_OK;
  }
  struct Msg {
    cudaIpcMemHandle_t hd;
    int ok;
    int pad[15];
  };
  Msg mine;
  memset(&mine, 0, sizeof(mine));
  mine.ok = cudaIpcGetMemHandle(&mine.hd, h->sh_work[0]) == cudaSuccess;
  cudaGetLastError();
  char* dbuf = nullptr;
  if ((st = h->cuda(cudaMalloc(&dbuf, (size_t)(P + 1) * sizeof(Msg)), "cudaMalloc ipc"))) return st;
  std::vector<Msg> all(P);
  ncclComm_t comm = static_cast<ncclComm_t>(h->comm);
  Msg* dmsg = reinterpret_cast<Msg*>(dbuf);
  int* dok = reinterpret_cast<int*>(dbuf + (size_t)P * sizeof(Msg));
  cudaError_t ce = cudaMemcpyAsync(dmsg + h->rank, &mine, sizeof(mine), cudaMemcpyHostToDevice, h->stream);
  ncclResult_t r = ncclSuccess;
  if (ce == cudaSuccess) r = ncclAllGather(dmsg + h->rank, dmsg, sizeof(Msg), ncclUint8, comm, h->stream);
  if (ce == cudaSuccess && r == ncclSuccess)
    ce = cudaMemcpyAsync(all.data(), dmsg, (size_t)P * sizeof(Msg), cudaMemcpyDeviceToHost, h->stream);
  if (ce == cudaSuccess) ce = cudaStreamSynchronize(h->stream);
  int ok = 1;
  if (ce == cudaSuccess && r == ncclSuccess) {
    for (int e = 0; e < P; ++e) ok &= all[e].ok;
    for (int e = 0; e < P && ok; ++e) {
      if (e == h->rank) continue;
      if (cudaIpcOpenMemHandle(&h->sh_peer[e], all[e].hd, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        h->sh_peer[e] = nullptr;
        ok = 0;
      }
    }
    ce = cudaMemcpyAsync(dok, &ok, sizeof(int), cudaMemcpyHostToDevice, h->stream);
    if (ce == cudaSuccess) r = ncclAllReduce(dok, dok, 1, ncclInt32, ncclMin, comm, h->stream);
    if (ce == cudaSuccess && r == ncclSuccess) ce = cudaMemcpyAsync(&ok, dok, sizeof(int), cudaMemcpyDeviceToHost, h->stream);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(h->stream);
  }
  cudaFree(dbuf);
  if (r != ncclSuccess) return h->fail(APSP_ENCCL, "IPC handle exchange: %s", ncclGetErrorString(r));
  if ((st = h->cuda(ce, "IPC handle exchange"))) return st;
  if (!ok) {
    for (int e = 0; e < P; ++e)
      if (e != h->rank && h->sh_peer[e]) cudaIpcCloseMemHandle(h->sh_peer[e]);
    for (auto& p : h->sh_peer) p = nullptr;
    h->sh_disabled = true;
    return APSP_OK;
  }
  h->sh_ipc_open = true;
  return APSP_OK;
}

// R25 (apsp_config.exact_f32): an int32 matrix whose every candidate sum is an integer of
// magnitude <= 2^24 (checked at init: weights in [0, W], 2 (n - 1) W <= 2^24) is closed by the
// fp32 engine: converted to fp32 in place (APSP_INF_I32 -> +inf), one fp32 dataflow launch,
// converted back. Each fp32 add then returns the exact integer sum and min is exact, so the
// result is the int32 APSP bit for bit. The two conversions are inside the closure's event.
static apsp_status run_dataflow_f32x(Handle* h) {
  const long long count = h->rows_per_rank * h->ld;
  int* const D = static_cast<int*>(h->shards[0].D);
  apsp_status st;
  h->ev_begin(2);
  if ((st = h->cuda(launch_i32_to_f32(D, count, h->stream), "i32 -> f32"))) return st;
  if ((st = run_dataflow<float>(h, false))) return st;
  if ((st = h->cuda(launch_f32_to_i32(reinterpret_cast<float*>(D), count, h->stream), "f32 -> i32"))) return st;
  h->ev_end((double)h->n_pad * h->n_pad * h->n_pad);
  h->arith = APSP_ARITH_F32_EXACT;
  return APSP_OK;
}

apsp_status run_incore_rounds(Handle* h, long long k0, long long k1) {
  h->kernel = APSP_KERNEL_PER_PHASE;  // (the dataflow / sharded paths below set their own)
  if (h->world == 1 && !h->use_comm && !h->virt && h->dataflow && k0 == 0 && k1 == h->n_pad / h->b) {
    if (h->modef32x && !h->small) return run_dataflow_f32x(h);
    return h->dtype == APSP_I32 ? run_dataflow<int>(h) : run_dataflow<float>(h);
  }
  if ((h->virt || h->use_comm) && h->dataflow && h->world <= 8 && k0 == 0 && k1 == h->n_pad / h->b) {
    apsp_status st;
    if (!h->virt &&
        (st = h->dtype == APSP_I32 ? prepare_sharded_peers<int>(h) : prepare_sharded_peers<float>(h)))
      return st;
    if (!h->sh_disabled) {
      h->kernel = APSP_KERNEL_SHARDED;
      return h->dtype == APSP_I32 ? run_dataflow_sharded<int>(h) : run_dataflow_sharded<float>(h);
    }
  }
  if (h->world == 1 && !h->use_comm) {  // single GPU: the whole closure, with lookahead
    return h->dtype == APSP_I32
               ? fw_closure<int>(h, static_cast<int*>(h->shards[0].D), h->ld, h->n_pad, k0, k1, h->stream)
               : fw_closure<float>(h, static_cast<float*>(h->shards[0].D), h->ld, h->n_pad, k0, k1, h->stream);
  }
  if (h->side && k0 == 0 && k1 == h->n_pad / h->b)
    return h->dtype == APSP_I32 ? sharded_lookahead<int>(h) : sharded_lookahead<float>(h);
  for (long long k = k0; k < k1; ++k) {
    apsp_status st = (h->dtype == APSP_I32) ? incore_round<int>(h, k) : incore_round<float>(h, k);
    if (st) return st;
  }
  return APSP_OK;
}

}  // namespace apsp

// ======================================================================
//                                C ABI
// ======================================================================

extern "C" {

void apsp_config_default(apsp_config* cfg) {
  if (!cfg) return;
  memset(cfg, 0, sizeof(*cfg));
  cfg->struct_size = (int32_t)sizeof(apsp_config);
  cfg->device = -1;
  cfg->world_size = 1;
  cfg->rank = 0;
}

const char* apsp_version(void) { return "apsp-b200 0.1 sm_100a"; }

const char* apsp_last_error(const apsp_handle* h) {
  if (h) return reinterpret_cast<const Handle*>(h)->err.c_str();
  return g_last_error.c_str();
}

apsp_status apsp_partition(int64_t n, int32_t tile, int32_t world_size, int32_t rank, int64_t* n_pad,
                           int64_t* row_begin, int64_t* row_count) {
  if (n < 0 || world_size < 1 || rank < 0 || rank >= world_size || !n_pad || !row_begin || !row_count)
    return fail_global(APSP_EINVAL, "apsp_partition: bad arguments");
  if (tile == 0) tile = kTile;
  if (tile != kTile) return fail_global(APSP_EINVAL, "apsp_partition: tile must be %d", kTile);
  const int64_t unit = (int64_t)tile * world_size;
  int64_t np = ((n + unit - 1) / unit) * unit;
  if (np == 0) np = unit;
  const int64_t R = np / world_size;
  const int64_t rb = (int64_t)rank * R;
  *n_pad = np;
  *row_begin = rb;
  *row_count = std::max<int64_t>(0, std::min<int64_t>(rb + R, n) - rb);
  return APSP_OK;
}

apsp_status apsp_dist_device_bytes(int64_t n, int32_t tile, int32_t world_size, int32_t virtual_ranks,
                                   int64_t* bytes) {
  if (!bytes) return fail_global(APSP_EINVAL, "apsp_dist_device_bytes: NULL");
  int64_t np = 0, rb = 0, rc = 0;
  if (apsp_status st = apsp_partition(n, tile, world_size, 0, &np, &rb, &rc)) return st;
  const int64_t per_rank = (np / world_size) * np * (int64_t)sizeof(int32_t);
  *bytes = (virtual_ranks && world_size > 1) ? per_rank * world_size : per_rank;
  return APSP_OK;
}

apsp_status apsp_nccl_unique_id(void* out128) {
  if (!out128) return fail_global(APSP_EINVAL, "apsp_nccl_unique_id: NULL");
  return nccl_unique_id(out128) ? APSP_OK : fail_global(APSP_ENCCL, "ncclGetUniqueId failed");
}

// Host validation of a CSR graph (O(n + m)) and the int32 range rule (R5).
static apsp_status validate_csr(int64_t n, const int64_t* row_ptr, const int32_t* col_idx, const void* weights,
                                apsp_dtype dtype, bool* has_neg_out, int64_t* maxabs_out) {
  if (row_ptr[0] != 0) return fail_global(APSP_EINVAL, "row_ptr[0] != 0");
  for (int64_t i = 0; i < n; ++i)
    if (row_ptr[i + 1] < row_ptr[i]) return fail_global(APSP_EINVAL, "row_ptr not monotone at %lld", (long long)i);
  const int64_t m = row_ptr[n];
  if (m > 0 && (!col_idx || !weights)) return fail_global(APSP_EINVAL, "col_idx/weights NULL with m > 0");
  for (int64_t e = 0; e < m; ++e)
    if (col_idx[e] < 0 || col_idx[e] >= n) return fail_global(APSP_EINVAL, "col_idx[%lld] out of range", (long long)e);
  bool has_neg = false;
  int64_t maxabs = 0;
  if (dtype == APSP_I32) {
    const int32_t* w = static_cast<const int32_t*>(weights);
    for (int64_t e = 0; e < m; ++e) {
      int64_t v = w[e];
      if (v < 0) has_neg = true;
      maxabs = std::max<int64_t>(maxabs, v < 0 ? -v : v);
    }
    const int64_t bound = has_neg ? ((int64_t)1 << 28) : (int64_t)APSP_INF_I32;
    if (n > 1 && (__int128)(n - 1) * maxabs >= bound)
      return fail_global(APSP_ERANGE, "(n-1)*max|w| = %lld >= %lld: int32 distances could reach infinity",
                         (long long)((n - 1) * maxabs), (long long)bound);
  } else {
    const float* w = static_cast<const float*>(weights);
    for (int64_t e = 0; e < m; ++e) {
      if (!std::isfinite(w[e])) return fail_global(APSP_EINVAL, "weight %lld is not finite", (long long)e);
      if (w[e] < 0) has_neg = true;
    }
  }
  *has_neg_out = has_neg;
  *maxabs_out = maxabs;
  return APSP_OK;
}

// Copy the caller's config (NULL = defaults) and check the fields every entry point shares.
static apsp_status load_config(const apsp_config* cfg_in, apsp_config* cfg) {
  apsp_config_default(cfg);
  if (!cfg_in) return APSP_OK;
  if (cfg_in->struct_size != 0 && cfg_in->struct_size != (int32_t)sizeof(apsp_config))
    return fail_global(APSP_EINVAL, "apsp_config.struct_size %d != %d", cfg_in->struct_size, (int)sizeof(apsp_config));
  *cfg = *cfg_in;
  for (int32_t r : cfg->reserved)
    if (r != 0) return fail_global(APSP_EINVAL, "apsp_config.reserved must be 0");
  if (cfg->schedule < APSP_SCHED_AUTO || cfg->schedule > APSP_SCHED_SMALL)
    return fail_global(APSP_EINVAL, "apsp_config.schedule %d is not an APSP_SCHED_* value", cfg->schedule);
  if (cfg->minplus_variant < 0 || cfg->minplus_variant > 2)
    return fail_global(APSP_EINVAL, "apsp_config.minplus_variant must be 0, 1 or 2");
  if (cfg->dataflow_delay < 0) return fail_global(APSP_EINVAL, "apsp_config.dataflow_delay < 0");
  if (cfg->exact_f32 != 0 && cfg->exact_f32 != 1) return fail_global(APSP_EINVAL, "apsp_config.exact_f32 must be 0 or 1");
  if (cfg->dist_device_bytes < 0) return fail_global(APSP_EINVAL, "apsp_config.dist_device_bytes < 0");
  return APSP_OK;
}

// Handles other than the in-core blocked FW cannot take a caller-owned matrix.
static apsp_status no_dist_device(const apsp_config& cfg, const char* what) {
  if (cfg.dist_device) return fail_global(APSP_EINVAL, "%s: apsp_config.dist_device is for apsp_init_from_csr only", what);
  return APSP_OK;
}

apsp_status apsp_init_from_csr(apsp_handle** out, int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                               const void* weights, apsp_dtype dtype, const apsp_config* cfg_in) {
  NvtxRange nvtx_("apsp_init_from_csr");
  if (!out) return fail_global(APSP_EINVAL, "apsp_init_from_csr: out is NULL");
  *out = nullptr;
  apsp_config cfg;
  if (apsp_status cst = load_config(cfg_in, &cfg)) return cst;
  if (n < 0) return fail_global(APSP_EINVAL, "n < 0");
  if (n > (int64_t)INT32_MAX) return fail_global(APSP_EINVAL, "n exceeds int32 vertex ids");
  if (!row_ptr) return fail_global(APSP_EINVAL, "row_ptr is NULL");
  if (dtype != APSP_I32 && dtype != APSP_F32) return fail_global(APSP_EINVAL, "bad dtype");
  if (cfg.tile == 0) cfg.tile = kTile;
  if (cfg.tile != kTile) return fail_global(APSP_EINVAL, "tile must be %d in this build", kTile);
  if (cfg.world_size < 1 || cfg.rank < 0 || cfg.rank >= cfg.world_size)
    return fail_global(APSP_EINVAL, "bad world_size/rank");
  if (cfg.world_size > 1 && !cfg.virtual_ranks && !cfg.nccl_unique_id)
    return fail_global(APSP_EINVAL, "world_size > 1 needs nccl_unique_id (or virtual_ranks)");
  if (cfg.dist_device) {
    int64_t need = 0;
    if (apsp_dist_device_bytes(n, cfg.tile, cfg.world_size, cfg.virtual_ranks, &need) != APSP_OK)
      return fail_global(APSP_EINVAL, "apsp_dist_device_bytes failed");
    if (cfg.dist_device_bytes < need)
      return fail_global(APSP_EINVAL, "apsp_config.dist_device_bytes %lld < %lld needed", (long long)cfg.dist_device_bytes,
                         (long long)need);
    if (reinterpret_cast<uintptr_t>(cfg.dist_device) % 256 != 0)
      return fail_global(APSP_EINVAL, "apsp_config.dist_device must be 256-byte aligned");
    if (cfg.force_out_of_core) return fail_global(APSP_EINVAL, "dist_device and force_out_of_core exclude each other");
  }

  bool has_neg = false;
  int64_t maxabs = 0;
  apsp_status vst = validate_csr(n, row_ptr, col_idx, weights, dtype, &has_neg, &maxabs);
  if (vst != APSP_OK) return vst;

  Handle* h = new Handle();
  h->n = n;
  h->b = cfg.tile;
  h->dtype = dtype;
  h->world = cfg.world_size;
  h->rank = cfg.virtual_ranks ? 0 : cfg.rank;
  h->virt = cfg.virtual_ranks && cfg.world_size > 1;
  h->timing = cfg.timing != 0;
  h->has_neg = has_neg;
  h->max_abs_w = maxabs;
  h->arith = dtype == APSP_F32 ? APSP_ARITH_F32 : APSP_ARITH_I32;
  h->elem = sizeof(int32_t);

  apsp_status st = init_handle(h, cfg, row_ptr, col_idx, weights);
  if (st != APSP_OK) {
    g_last_error = h->err;
    delete_handle(h);
    return st;
  }
  *out = reinterpret_cast<apsp_handle*>(h);
  return APSP_OK;
}

apsp_status apsp_init_boundary(apsp_handle** out, int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                               const void* weights, apsp_dtype dtype, const int32_t* comp, int32_t k,
                               const apsp_config* cfg_in) {
  NvtxRange nvtx_("apsp_init_boundary");
  if (!out) return fail_global(APSP_EINVAL, "apsp_init_boundary: out is NULL");
  *out = nullptr;
  apsp_config cfg;
  if (apsp_status cst = load_config(cfg_in, &cfg)) return cst;
  if (n < 1 || n > (int64_t)INT32_MAX) return fail_global(APSP_EINVAL, "bad n");
  if (!row_ptr || !comp) return fail_global(APSP_EINVAL, "row_ptr / comp is NULL");
  if (dtype != APSP_I32 && dtype != APSP_F32) return fail_global(APSP_EINVAL, "bad dtype");
  if (k < 1) return fail_global(APSP_EINVAL, "k < 1");
  if (cfg.world_size != 1) return fail_global(APSP_EINVAL, "the boundary algorithm runs on one GPU");
  if (apsp_status dst = no_dist_device(cfg, "apsp_init_boundary")) return dst;
  for (int64_t v = 0; v < n; ++v)
    if (comp[v] < 0 || comp[v] >= k) return fail_global(APSP_EINVAL, "comp[%lld] out of [0, k)", (long long)v);
  bool has_neg = false;
  int64_t maxabs = 0;
  apsp_status vst = validate_csr(n, row_ptr, col_idx, weights, dtype, &has_neg, &maxabs);
  if (vst != APSP_OK) return vst;

  Handle* h = new Handle();
  h->n = n;
  h->dtype = dtype;
  h->timing = cfg.timing != 0;
  h->has_neg = has_neg;
  h->max_abs_w = maxabs;
  h->arith = dtype == APSP_F32 ? APSP_ARITH_F32 : APSP_ARITH_I32;
  h->elem = 4;
  h->mode = APSP_MODE_BOUNDARY;
  apsp_status st = setup_device(h, cfg);
  if (!st) st = bnd_setup(h, cfg, row_ptr, col_idx, weights, comp, k);
  if (st != APSP_OK) {
    g_last_error = h->err;
    delete_handle(h);
    return st;
  }
  *out = reinterpret_cast<apsp_handle*>(h);
  return APSP_OK;
}

apsp_status apsp_init_johnson(apsp_handle** out, int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                              const void* weights, apsp_dtype dtype, double delta, int64_t batch,
                              const apsp_config* cfg_in) {
  NvtxRange nvtx_("apsp_init_johnson");
  if (!out) return fail_global(APSP_EINVAL, "apsp_init_johnson: out is NULL");
  *out = nullptr;
  apsp_config cfg;
  if (apsp_status cst = load_config(cfg_in, &cfg)) return cst;
  if (n < 1 || n > (int64_t)INT32_MAX) return fail_global(APSP_EINVAL, "bad n");
  if (!row_ptr) return fail_global(APSP_EINVAL, "row_ptr is NULL");
  if (dtype != APSP_I32 && dtype != APSP_F32) return fail_global(APSP_EINVAL, "bad dtype");
  if (cfg.world_size < 1 || cfg.rank < 0 || cfg.rank >= cfg.world_size)
    return fail_global(APSP_EINVAL, "bad world_size/rank");
  if (!(delta >= 0) || !std::isfinite(delta)) return fail_global(APSP_EINVAL, "delta must be finite and >= 0");
  if (apsp_status dst = no_dist_device(cfg, "apsp_init_johnson")) return dst;
  bool has_neg = false;
  int64_t maxabs = 0;
  apsp_status vst = validate_csr(n, row_ptr, col_idx, weights, dtype, &has_neg, &maxabs);
  if (vst != APSP_OK) return vst;

  Handle* h = new Handle();
  h->n = n;
  h->dtype = dtype;
  h->timing = cfg.timing != 0;
  h->has_neg = has_neg;
  h->max_abs_w = maxabs;
  h->arith = dtype == APSP_F32 ? APSP_ARITH_F32 : APSP_ARITH_I32;
  h->elem = 4;
  h->mode = APSP_MODE_JOHNSON;
  h->world = cfg.world_size;  // sources are split by rank; no communicator is needed
  h->rank = cfg.rank;
  apsp_status st = setup_device(h, cfg);
  if (!st) st = jn_setup(h, cfg, row_ptr, col_idx, weights, delta, batch);
  if (st != APSP_OK) {
    g_last_error = h->err;
    delete_handle(h);
    return st;
  }
  *out = reinterpret_cast<apsp_handle*>(h);
  return APSP_OK;
}

apsp_status apsp_select(int64_t n, const int64_t* row_ptr, const int32_t* col_idx, const void* weights,
                        apsp_dtype dtype, const int32_t* comp, int32_t k, const apsp_config* cfg_in,
                        apsp_selection* out) {
  NvtxRange nvtx_("apsp_select");
  if (!out) return fail_global(APSP_EINVAL, "apsp_select: out is NULL");
  memset(out, 0, sizeof(*out));
  for (double& e : out->est_seconds) e = -1.0;
  apsp_config cfg;
  if (apsp_status cst = load_config(cfg_in, &cfg)) return cst;
  if (n < 1 || n > (int64_t)INT32_MAX || !row_ptr) return fail_global(APSP_EINVAL, "bad n / row_ptr");
  if (dtype != APSP_I32 && dtype != APSP_F32) return fail_global(APSP_EINVAL, "bad dtype");
  if (comp && k < 1) return fail_global(APSP_EINVAL, "k < 1");
  bool has_neg = false;
  int64_t maxabs = 0;
  apsp_status st = validate_csr(n, row_ptr, col_idx, weights, dtype, &has_neg, &maxabs);
  if (st) return st;
  const double dn = (double)n, m = (double)row_ptr[n];
  out->density = m / (dn * dn);
  // §IV-C density filter
  int cand;
  if (out->density > 0.01) cand = (1 << APSP_MODE_INCORE) | (1 << APSP_MODE_JOHNSON);
  else if (out->density < 1e-4) cand = (1 << APSP_MODE_JOHNSON) | (1 << APSP_MODE_BOUNDARY);
  else cand = 1 << APSP_MODE_JOHNSON;
  if (!comp) cand &= ~(1 << APSP_MODE_BOUNDARY);  // no partition given (the paper uses METIS)
  if (!cand) cand = 1 << APSP_MODE_JOHNSON;
  if (dtype == APSP_F32 && has_neg) cand = 1 << APSP_MODE_INCORE;  // Johnson takes fp32 w >= 0 (R19)
  int64_t nb_nodes = 0;
  if (comp) {
    for (int64_t v = 0; v < n; ++v)
      if (comp[v] < 0 || comp[v] >= k) return fail_global(APSP_EINVAL, "comp[%lld] out of [0, k)", (long long)v);
    std::vector<char> isb(n, 0);
    for (int64_t u = 0; u < n; ++u)
      for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e)
        if (comp[col_idx[e]] != comp[u]) isb[u] = isb[col_idx[e]] = 1;
    for (int64_t v = 0; v < n; ++v) nb_nodes += isb[v];
    out->boundary_nodes = nb_nodes;
  }
  out->candidates = cand;
  // cost models (§IV-B), calibrated on this device
  std::string err;
  int dev = cfg.device;
  if (dev < 0 && cudaGetDevice(&dev) != cudaSuccess) return fail_global(APSP_ECUDA, "no CUDA device");
  if (cudaSetDevice(dev) != cudaSuccess) return fail_global(APSP_ECUDA, "no CUDA device (the library has no CPU path)");
  const long long avail = device_free_bytes(dev, (long long)n * n * 4);
  if (avail < 0) return fail_global(APSP_ECUDA, "no CUDA device (the library has no CPU path)");
  const double budget = cfg.device_budget_bytes > 0 ? (double)cfg.device_budget_bytes : (double)avail - (1 << 30);
  const double W = 4.0, mat = dn * dn * W;
  const bool ooc = mat > budget;
  double c_unit = 0, TH = 0;
  const bool need_fw = (cand >> APSP_MODE_INCORE & 1) || (cand >> APSP_MODE_BOUNDARY & 1);
  if (need_fw && (st = fw_seconds_per_relax(cfg, std::min<int64_t>(8192, std::max<int64_t>(1024, n)), &c_unit, &err)))
    return fail_global(st, "apsp_select: FW calibration: %s", err.c_str());
  if (ooc && (st = hostlink_rate(dev, &TH, &err))) return fail_global(st, "apsp_select: host link: %s", err.c_str());
  if (cand >> APSP_MODE_INCORE & 1) {
    double t = c_unit * dn * dn * dn;
    if (ooc) {
      const double b = 4096, nd = std::ceil(dn / b);
      t = std::max(t, nd * W * (3 * b * b + dn * dn) / TH);
    }
    out->est_seconds[APSP_MODE_INCORE] = t;
  }
  if (cand >> APSP_MODE_JOHNSON & 1) {
    double t = 0;
    if ((st = johnson_seconds(cfg, n, row_ptr, col_idx, weights, dtype, has_neg, 5, &t, &err)))
      return fail_global(st, "apsp_select: Johnson sampling: %s", err.c_str());
    if (ooc) t = std::max(t, W * dn * dn / TH);
    out->est_seconds[APSP_MODE_JOHNSON] = t;
  }
  if (cand >> APSP_MODE_BOUNDARY & 1) {
    const double kk = (double)k, B = (double)nb_nodes / kk;
    const double nop = dn * dn * dn / (kk * kk) + std::pow(kk * B, 3) + dn * kk * B * B + dn * dn * B;
    out->est_seconds[APSP_MODE_BOUNDARY] = nop * c_unit;
  }
  out->method = -1;
  for (int mth : {APSP_MODE_INCORE, APSP_MODE_JOHNSON, APSP_MODE_BOUNDARY})
    if ((out->candidates >> mth & 1) && out->est_seconds[mth] >= 0 &&
        (out->method < 0 || out->est_seconds[mth] < out->est_seconds[out->method]))
      out->method = mth;
  if (out->method < 0) out->method = APSP_MODE_JOHNSON;
  return APSP_OK;
}

apsp_status apsp_solve(apsp_handle* hh) {
  NvtxRange nvtx_("apsp_solve");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->mode != APSP_MODE_BOUNDARY && h->mode != APSP_MODE_JOHNSON) return apsp_fw_blocked(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (apsp_status pst = settle(h)) return pst;  // pending asynchronous work first
  if (h->fw_done) return h->fail(APSP_ESTATE, "apsp_solve already ran (apsp_reinit first)");
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  memset(&h->stats, 0, sizeof(h->stats));
  if (h->mode == APSP_MODE_JOHNSON) {
    if ((st = jn_run(h))) return st;
    if (h->timing) h->collect_events();
    h->stats.relax[2] = (double)jn_edges(h);
    h->fw_done = true;
    h->canonical = true;
    return APSP_OK;
  }
  if ((st = bnd_run(h))) return st;
  return finish_fw(h, true);
}

apsp_status apsp_fw_rounds(apsp_handle* hh, int64_t k_begin, int64_t k_end) {
  NvtxRange nvtx_("apsp_fw_rounds");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (apsp_status pst = settle(h)) return pst;  // pending asynchronous work first
  if (h->mode != APSP_MODE_INCORE && h->mode != APSP_MODE_OUT_OF_CORE)
    return h->fail(APSP_ESTATE, "apsp_fw_rounds: blocked-FW handles only");
  if (h->mode16) return h->fail(APSP_ESTATE, "apsp_fw_rounds: not available with packed16");
  const long long nb = h->n_pad / h->b;
  if (k_begin != h->next_round || k_end < k_begin || k_end > nb)
    return h->fail(APSP_ESTATE, "rounds must run in order: next is %lld of %lld", h->next_round, nb);
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  if (h->mode == APSP_MODE_OUT_OF_CORE) {
    // out of core the unit is a super-round of B/b rounds (Algorithm 1)
    const long long kb = h->ooc_B / h->b;
    if (k_begin % kb || (k_end % kb && k_end != nb))
      return h->fail(APSP_EINVAL, "out of core, rounds run in super-rounds of %lld", kb);
    memset(&h->stats, 0, sizeof(h->stats));
    h->kernel = APSP_KERNEL_OUT_OF_CORE;
    if ((st = run_out_of_core_range(h, k_begin / kb, (k_end + kb - 1) / kb))) return st;
    h->next_round = k_end;
    return finish_fw(h, k_end == nb);
  }
  if ((st = run_incore_rounds(h, k_begin, k_end))) return st;
  h->next_round = k_end;
  return finish_fw(h, k_end == nb);
}

apsp_status apsp_fw_blocked(apsp_handle* hh) {
  NvtxRange nvtx_("apsp_fw_blocked");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (apsp_status pst = settle(h)) return pst;  // pending asynchronous work first
  if (h->fw_done) return h->fail(APSP_ESTATE, "apsp_fw_blocked already ran");
  if (h->mode == APSP_MODE_BOUNDARY || h->mode == APSP_MODE_JOHNSON)
    return h->fail(APSP_ESTATE, "boundary / Johnson handle: use apsp_solve");
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  memset(&h->stats, 0, sizeof(h->stats));
  const long long nb = h->n_pad / h->b;
  // the remaining rounds: all of them, or those after apsp_fw_rounds / apsp_restore
  if (h->mode == APSP_MODE_OUT_OF_CORE) {
    const long long kb = h->ooc_B / h->b;
    if (h->next_round % kb) return h->fail(APSP_ESTATE, "out of core, rounds run in super-rounds of %lld", kb);
    h->kernel = APSP_KERNEL_OUT_OF_CORE;
    if ((st = run_out_of_core_range(h, h->next_round / kb, nb / kb))) return st;
    h->next_round = nb;
    return finish_fw(h, true);
  }
  if (h->mode16) {
    if (h->next_round != 0) return h->fail(APSP_ESTATE, "packed16: no partial runs");
    if ((st = run_fw16(h))) return st;
    h->next_round = nb;
    return finish_fw(h, true);
  }
  if ((st = run_incore_rounds(h, h->next_round, nb))) return st;
  h->next_round = nb;
  return finish_fw(h, true);
}

apsp_status apsp_fw_blocked_async(apsp_handle* hh) {
  NvtxRange nvtx_("apsp_fw_blocked_async");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (apsp_status pst = settle(h)) return pst;
  if (h->mode != APSP_MODE_INCORE) return apsp_fw_blocked(hh);  // synchronous placements
  if (h->fw_done) return h->fail(APSP_ESTATE, "apsp_fw_blocked already ran");
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  memset(&h->stats, 0, sizeof(h->stats));
  const long long nb = h->n_pad / h->b;
  if (h->mode16) {  // packed16: the exactness check is read by apsp_synchronize
    if (h->next_round != 0) return h->fail(APSP_ESTATE, "packed16: no partial runs");
    if ((st = enqueue_fw16(h))) return st;
  } else if ((st = run_incore_rounds(h, h->next_round, nb))) {
    return st;
  }
  h->next_round = nb;
  return finish_fw_async(h);
}

apsp_status apsp_get_dist_async(apsp_handle* hh, int64_t row_begin, int64_t row_count, void* out, int64_t ld_out) {
  NvtxRange nvtx_("apsp_get_dist_async");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (row_count < 0 || row_begin < 0 || row_begin + row_count > h->n || ld_out < h->n || (row_count > 0 && !out))
    return h->fail(APSP_EINVAL, "get_dist: bad row range / ld_out / out");
  if (row_count == 0) return APSP_OK;
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  if (h->mode != APSP_MODE_INCORE) {  // synchronous placements: settle first
    if ((st = settle(h))) return st;
    return get_rows(h, row_begin, row_count, out, ld_out);
  }
  return get_rows_async(h, row_begin, row_count, out, ld_out);  // (packed16 int16 result: widened on the device)
}

apsp_status apsp_load_csr(apsp_handle* hh, const int64_t* row_ptr, const int32_t* col_idx, const void* weights) {
  NvtxRange nvtx_("apsp_load_csr");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (apsp_status pst = settle(h)) return pst;
  if (h->mode != APSP_MODE_INCORE || h->virt)
    return h->fail(APSP_ESTATE, "apsp_load_csr: in-core handles without virtual ranks only");
  if (!row_ptr) return h->fail(APSP_EINVAL, "row_ptr is NULL");
  bool has_neg = false;
  int64_t maxabs = 0;
  if (apsp_status vst = validate_csr(h->n, row_ptr, col_idx, weights, h->dtype, &has_neg, &maxabs)) {
    h->err = g_last_error;
    return vst;
  }
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  h->has_neg = has_neg;
  h->max_abs_w = maxabs;
  // packed16 handle (R16): int16 again if this graph is eligible, else straight to int32
  if (h->mode16) h->fell_back16 = has_neg || maxabs > 8191;
  h->modef32x = f32x_eligible(h);  // R25: decided per graph
  if (h->dtype == APSP_I32 && !h->mode16) h->arith = h->modef32x ? APSP_ARITH_F32_EXACT : APSP_ARITH_I32;
  return load_csr(h, row_ptr, col_idx, weights);
}

apsp_status apsp_synchronize(apsp_handle* hh) {
  NvtxRange nvtx_("apsp_synchronize");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  return settle(h);
}

apsp_status apsp_reinit(apsp_handle* hh) {
  NvtxRange nvtx_("apsp_reinit");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (apsp_status pst = settle(h)) return pst;  // pending asynchronous work first
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  if (h->mode == APSP_MODE_OUT_OF_CORE) return ooc_reinit(h);
  if (h->mode == APSP_MODE_BOUNDARY) return bnd_reinit(h);
  if (h->mode == APSP_MODE_JOHNSON) return jn_reinit(h);
  return run_init(h);
}

apsp_status apsp_get_dist(apsp_handle* hh, int64_t row_begin, int64_t row_count, void* out, int64_t ld_out) {
  NvtxRange nvtx_("apsp_get_dist");
  if (!hh) return fail_global(APSP_EINVAL, "NULL handle");
  Handle* h = reinterpret_cast<Handle*>(hh);
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (apsp_status pst = settle(h)) return pst;  // pending asynchronous work first
  if (row_count < 0 || row_begin < 0 || row_begin + row_count > h->n || ld_out < h->n || (row_count > 0 && !out))
    return h->fail(APSP_EINVAL, "get_dist: bad row range / ld_out / out");
  if (row_count == 0) return APSP_OK;
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  return get_rows(h, row_begin, row_count, out, ld_out);
}

apsp_status apsp_local_rows(const apsp_handle* hh, int64_t* row_begin, int64_t* row_count) {
  if (!hh || !row_begin || !row_count) return fail_global(APSP_EINVAL, "NULL argument");
  const Handle* h = reinterpret_cast<const Handle*>(hh);
  if (h->mode == APSP_MODE_JOHNSON) {
    long long r0, rc;
    jn_local_rows(h, &r0, &rc);
    *row_begin = r0;
    *row_count = rc;
    return APSP_OK;
  }
  if (h->virt || h->world == 1) {
    *row_begin = 0;
    *row_count = h->n;
    return APSP_OK;
  }
  if (h->mode == APSP_MODE_OUT_OF_CORE) {  // rank r: bands [r nd/P, (r+1) nd/P) (apsp_ooc.cu)
    const int64_t rb = (int64_t)h->rank * h->rows_per_rank;
    *row_begin = rb;
    *row_count = std::max<int64_t>(0, std::min<int64_t>(rb + h->rows_per_rank, h->n) - rb);
    return APSP_OK;
  }
  int64_t np;
  return apsp_partition(h->n, h->b, h->world, h->rank, &np, row_begin, row_count);
}

apsp_status apsp_get_info(const apsp_handle* hh, apsp_info* info) {
  if (!hh || !info) return fail_global(APSP_EINVAL, "NULL argument");
  const Handle* h = reinterpret_cast<const Handle*>(hh);
  memset(info, 0, sizeof(*info));
  info->n = h->n;
  info->n_pad = h->n_pad;
  info->tile = h->b;
  info->dtype = h->dtype;
  info->world_size = h->world;
  info->rank = h->rank;
  info->mode = h->mode;
  info->ooc_block = h->mode == APSP_MODE_OUT_OF_CORE ? (int32_t)h->ooc_B
                   : h->mode == APSP_MODE_BOUNDARY ? (int32_t)bnd_ooc_rows(h) : 0;
  info->rounds = h->n_pad / h->b;
  info->device_bytes = h->device_bytes;
  info->host_bytes = h->host_bytes;
  info->dist_device = h->shards.empty() ? nullptr : h->shards[0].D;
  info->ld = h->ld;
  info->arith = h->arith;
  info->packed16_eligible = h->mode16 ? 1 : 0;
  if (h->result16) info->dist_device = h->d16;
  info->boundary_nodes = bnd_boundary_nodes(h);
  info->edges_scanned = jn_edges(h);
  info->kernel = h->kernel;
  info->exact_f32_eligible = h->modef32x ? 1 : 0;
  return APSP_OK;
}

apsp_status apsp_get_phase_stats(const apsp_handle* hh, apsp_phase_stats* out) {
  if (!hh || !out) return fail_global(APSP_EINVAL, "NULL argument");
  *out = reinterpret_cast<const Handle*>(hh)->stats;
  return APSP_OK;
}

void apsp_destroy(apsp_handle* hh) {
  if (!hh) return;
  delete_handle(reinterpret_cast<Handle*>(hh));
}

apsp_status apsp_trim_memory(int32_t device) {
  int dev = device;
  if (dev < 0 && cudaGetDevice(&dev) != cudaSuccess) return fail_global(APSP_ECUDA, "no CUDA device");
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) != cudaSuccess) return fail_global(APSP_ECUDA, "no memory pool");
  if (cudaDeviceSynchronize() != cudaSuccess || cudaMemPoolTrimTo(pool, 0) != cudaSuccess)
    return fail_global(APSP_ECUDA, "cudaMemPoolTrimTo failed");
  return APSP_OK;
}

}  // extern "C"
