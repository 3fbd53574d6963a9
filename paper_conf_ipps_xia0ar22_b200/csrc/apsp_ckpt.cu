// apsp_ckpt.cu — checkpoint / resume of a blocked-FW run.
//
// The blocked FW has a consistent state after every round k: dist[i][j] is the
// shortest i -> j path with intermediates in {0 .. k*b - 1} (the FW invariant,
// PAPER.md:60). Out of core (Algorithm 1) the state after a
// super-round is the pinned host bands plus the bands resident in HBM. A
// checkpoint writes that state (this rank's padded rows) and the next round to a
// file; a restore loads it into a handle created for the same graph and
// configuration, and apsp_fw_rounds / apsp_fw_blocked continue from there.
//
// File: a fixed 128-byte little-endian header (CkptHeader) followed by the
// rank's rows_per_rank x n_pad elements (row-major, padded rows included).
#include "apsp_internal.h"

#include <cstdio>
#include <cstring>
#include <vector>

namespace apsp {
namespace {

struct CkptHeader {
  char magic[8];        // "APSPCKP1"
  int32_t version;      // 1
  int32_t dtype;        // apsp_dtype
  int64_t n, n_pad, rows;  // rows = padded rows stored (this rank)
  int32_t mode;         // APSP_MODE_INCORE / APSP_MODE_OUT_OF_CORE
  int32_t ooc_block;    // B out of core, else 0
  int32_t world, rank;
  int64_t row_begin;    // first padded row stored
  int64_t next_round;   // rounds 0 .. next_round-1 applied
  int32_t has_neg;      // negative arc weights present (affects canonicalisation)
  int32_t neg_cycle;    // this rank's negative-cycle flag (d_flag) after rounds 0 .. next_round-1:
                        // phase 1 flags a cycle only in the round of its largest vertex (R6),
                        // so a resumed run must inherit it
  int64_t reserved[6];
};
static_assert(sizeof(CkptHeader) == 128, "checkpoint header is 128 bytes");

const char kMagic[8] = {'A', 'P', 'S', 'P', 'C', 'K', 'P', '1'};

void fill_header(const Handle* h, CkptHeader* hd) {
  memset(hd, 0, sizeof(*hd));
  memcpy(hd->magic, kMagic, 8);
  hd->version = 1;
  hd->dtype = h->dtype;
  hd->n = h->n;
  hd->n_pad = h->n_pad;
  hd->rows = h->rows_per_rank;
  hd->mode = h->mode;
  hd->ooc_block = h->mode == APSP_MODE_OUT_OF_CORE ? (int32_t)h->ooc_B : 0;
  hd->world = h->world;
  hd->rank = h->rank;
  hd->row_begin = h->mode == APSP_MODE_OUT_OF_CORE ? ooc_row_begin(h) : h->shards[0].row_begin;
  hd->next_round = h->next_round;
  hd->has_neg = h->has_neg ? 1 : 0;
  hd->neg_cycle = 0;
}

apsp_status check_handle(Handle* h) {
  if (h->poisoned) return h->fail(APSP_ESTATE, "handle poisoned by an earlier CUDA/NCCL error");
  if (apsp_status pst = settle(h)) return pst;  // pending asynchronous work first
  if (h->mode != APSP_MODE_INCORE && h->mode != APSP_MODE_OUT_OF_CORE)
    return h->fail(APSP_ESTATE, "checkpoint: blocked-FW handles only");
  if (h->mode16) return h->fail(APSP_ESTATE, "checkpoint: not available with packed16");
  if (h->virt) return h->fail(APSP_ESTATE, "checkpoint: not available with virtual ranks");
  return h->cuda(cudaSetDevice(h->device), "cudaSetDevice");
}

// in core: rows [0, rows) of shard 0 through a pinned staging buffer
apsp_status incore_io(Handle* h, FILE* f, bool save) {
  apsp_status st;
  const size_t row_bytes = (size_t)h->ld * h->elem;
  const long long blk = std::max<long long>(1, (long long)((64ull << 20) / row_bytes));
  void* stage = nullptr;
  if ((st = h->cuda(cudaHostAlloc(&stage, blk * row_bytes, cudaHostAllocDefault), "cudaHostAlloc stage"))) return st;
  char* D = static_cast<char*>(h->shards[0].D);
  for (long long r = 0; r < h->rows_per_rank && !st; r += blk) {
    const long long rr = std::min(blk, h->rows_per_rank - r);
    if (save) {
      st = h->cuda(cudaMemcpyAsync(stage, D + r * row_bytes, rr * row_bytes, cudaMemcpyDeviceToHost, h->stream), "D2H");
      if (!st) st = h->cuda(cudaStreamSynchronize(h->stream), "sync");
      if (!st && fwrite(stage, row_bytes, rr, f) != (size_t)rr) st = h->fail(APSP_EINVAL, "checkpoint: write failed");
    } else {
      if (fread(stage, row_bytes, rr, f) != (size_t)rr) st = h->fail(APSP_EINVAL, "restore: file too short");
      if (!st) st = h->cuda(cudaMemcpyAsync(D + r * row_bytes, stage, rr * row_bytes, cudaMemcpyHostToDevice, h->stream), "H2D");
      if (!st) st = h->cuda(cudaStreamSynchronize(h->stream), "sync");
    }
  }
  cudaFreeHost(stage);
  return st;
}

// out of core: band by band (resident bands through a host buffer)
apsp_status ooc_io(Handle* h, FILE* f, bool save) {
  apsp_status st = APSP_OK;
  const size_t bb = (size_t)h->ooc_B * h->n_pad * h->elem;
  void* buf = nullptr;
  if ((st = h->cuda(cudaHostAlloc(&buf, bb, cudaHostAllocDefault), "cudaHostAlloc band"))) return st;
  for (long long I = 0; I < ooc_bands(h) && !st; ++I) {
    if (save) {
      st = ooc_band_copy(h, I, buf, false);
      if (!st && fwrite(buf, 1, bb, f) != bb) st = h->fail(APSP_EINVAL, "checkpoint: write failed");
    } else {
      if (fread(buf, 1, bb, f) != bb) st = h->fail(APSP_EINVAL, "restore: file too short");
      if (!st) st = ooc_band_copy(h, I, buf, true);
    }
  }
  cudaFreeHost(buf);
  return st;
}

}  // namespace
}  // namespace apsp

using namespace apsp;

extern "C" {

apsp_status apsp_checkpoint(apsp_handle* hh, const char* path) {
  if (!hh || !path) return global_fail(APSP_EINVAL, "apsp_checkpoint: NULL argument");
  Handle* h = reinterpret_cast<Handle*>(hh);
  apsp_status st;
  if ((st = check_handle(h))) return st;
  if ((st = h->cuda(cudaStreamSynchronize(h->stream), "sync"))) return st;
  FILE* f = fopen(path, "wb");
  if (!f) return h->fail(APSP_EINVAL, "apsp_checkpoint: cannot open %s", path);
  CkptHeader hd;
  fill_header(h, &hd);
  int flag = 0;
  if ((st = h->cuda(cudaMemcpy(&flag, h->d_flag, sizeof(int), cudaMemcpyDeviceToHost), "D2H flag"))) {
    fclose(f);
    return st;
  }
  hd.neg_cycle = flag ? 1 : 0;
  if (fwrite(&hd, sizeof(hd), 1, f) != 1) st = h->fail(APSP_EINVAL, "checkpoint: write failed");
  if (!st) st = h->mode == APSP_MODE_OUT_OF_CORE ? ooc_io(h, f, true) : incore_io(h, f, true);
  if (fclose(f) != 0 && !st) st = h->fail(APSP_EINVAL, "checkpoint: close failed");
  return st;
}

apsp_status apsp_restore(apsp_handle* hh, const char* path) {
  if (!hh || !path) return global_fail(APSP_EINVAL, "apsp_restore: NULL argument");
  Handle* h = reinterpret_cast<Handle*>(hh);
  apsp_status st;
  if ((st = check_handle(h))) return st;
  FILE* f = fopen(path, "rb");
  if (!f) return h->fail(APSP_EINVAL, "apsp_restore: cannot open %s", path);
  CkptHeader hd, want;
  fill_header(h, &want);
  if (fread(&hd, sizeof(hd), 1, f) != 1 || memcmp(hd.magic, kMagic, 8) || hd.version != 1) {
    fclose(f);
    return h->fail(APSP_EINVAL, "apsp_restore: %s is not a checkpoint", path);
  }
  if (hd.dtype != want.dtype || hd.n != want.n || hd.n_pad != want.n_pad || hd.rows != want.rows ||
      hd.mode != want.mode || hd.ooc_block != want.ooc_block || hd.world != want.world || hd.rank != want.rank ||
      hd.row_begin != want.row_begin || hd.has_neg != want.has_neg || hd.next_round < 0 ||
      hd.next_round > h->n_pad / h->b) {
    fclose(f);
    return h->fail(APSP_EINVAL, "apsp_restore: checkpoint does not match this handle (n, dtype, placement, B)");
  }
  st = h->mode == APSP_MODE_OUT_OF_CORE ? ooc_io(h, f, false) : incore_io(h, f, false);
  fclose(f);
  if (st) return st;
  const int flag = hd.neg_cycle ? 1 : 0;
  if ((st = h->cuda(cudaMemcpy(h->d_flag, &flag, sizeof(int), cudaMemcpyHostToDevice), "H2D flag"))) return st;
  h->next_round = hd.next_round;
  h->fw_done = hd.next_round == h->n_pad / h->b;
  h->canonical = false;
  return APSP_OK;
}

}  // extern "C"
