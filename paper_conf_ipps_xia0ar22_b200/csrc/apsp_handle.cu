// apsp_handle.cu — handle lifetime: device selection, 1-D block-row
// partition, allocation, NCCL communicator, CSR upload + init kernel
// (PAPER.md:60), negative-cycle status, and result read-back (get_dist).
#include "apsp_internal.h"
#include "apsp_sched.cuh"

#include <nccl.h>

#include <algorithm>
#include <cstring>

namespace apsp {

bool nccl_unique_id(void* out128) {
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return false;
  memcpy(out128, &id, sizeof(id));
  return true;
}

apsp_status Handle::bcast(void* buf, size_t bytes, int root, cudaStream_t s) {
  ncclResult_t r = ncclBroadcast(buf, buf, bytes, ncclUint8, root, static_cast<ncclComm_t>(comm), s);
  if (r != ncclSuccess) return fail(APSP_ENCCL, "ncclBroadcast: %s", ncclGetErrorString(r));
  return APSP_OK;
}

template <typename T>
static apsp_status upload_csr(Handle* h, const int64_t* row_ptr, const int32_t* col, const void* w) {
  apsp_status st;
  for (auto& sh : h->shards) {
    const long long R = h->rows_per_rank;
    const long long real = std::max<long long>(0, std::min<long long>(R, h->n - sh.row_begin));
    sh.real_rows = real;
    if (real <= 0) continue;
    const long long e0 = row_ptr[sh.row_begin];
    const long long me = row_ptr[sh.row_begin + real] - e0;
    sh.e0 = e0;
    if ((st = h->cuda(cudaMalloc(&sh.d_rp, (real + 1) * sizeof(long long)), "cudaMalloc csr"))) return st;
    if ((st = h->cuda(cudaMemcpyAsync(sh.d_rp, row_ptr + sh.row_begin, (real + 1) * sizeof(long long),
                                      cudaMemcpyHostToDevice, h->stream), "H2D row_ptr")))
      return st;
    h->device_bytes += (real + 1) * sizeof(long long);
    if (me > 0) {
      if ((st = h->cuda(cudaMalloc(&sh.d_col, me * sizeof(int)), "cudaMalloc csr"))) return st;
      if ((st = h->cuda(cudaMalloc(&sh.d_w, me * sizeof(T)), "cudaMalloc csr"))) return st;
      sh.cap_arcs = me;
      if ((st = h->cuda(cudaMemcpyAsync(sh.d_col, col + e0, me * sizeof(int), cudaMemcpyHostToDevice, h->stream),
                        "H2D col")))
        return st;
      if ((st = h->cuda(cudaMemcpyAsync(sh.d_w, static_cast<const T*>(w) + e0, me * sizeof(T),
                                        cudaMemcpyHostToDevice, h->stream), "H2D w")))
        return st;
      h->device_bytes += me * (sizeof(int) + sizeof(T));
    }
  }
  return APSP_OK;
}

// A new graph with the same n and dtype into an in-core handle (serving loops):
// the CSR slices are copied into the handle's device arrays (grown only if the
// arc count exceeds their capacity; the copy completes before return, so the
// caller may reuse its arrays) and the CSR -> dense init is enqueued.
apsp_status load_csr(Handle* h, const int64_t* row_ptr, const int32_t* col, const void* w) {
  apsp_status st;
  const size_t we = sizeof(int32_t);  // int32 and fp32 weights
  for (auto& sh : h->shards) {
    const long long real = sh.real_rows;
    if (real <= 0) continue;
    const long long e0 = row_ptr[sh.row_begin];
    const long long me = row_ptr[sh.row_begin + real] - e0;
    sh.e0 = e0;
    if (me > sh.cap_arcs) {
      cudaFree(sh.d_col);
      cudaFree(sh.d_w);
      sh.d_col = nullptr;
      sh.d_w = nullptr;
      if ((st = h->cuda(cudaMalloc(&sh.d_col, me * sizeof(int)), "cudaMalloc csr"))) return st;
      if ((st = h->cuda(cudaMalloc(&sh.d_w, me * we), "cudaMalloc csr"))) return st;
      h->device_bytes += (me - sh.cap_arcs) * (sizeof(int) + we);
      sh.cap_arcs = me;
    }
    if ((st = h->cuda(cudaMemcpyAsync(sh.d_rp, row_ptr + sh.row_begin, (real + 1) * sizeof(long long),
                                      cudaMemcpyHostToDevice, h->stream), "H2D row_ptr")))
      return st;
    if (me > 0) {
      if ((st = h->cuda(cudaMemcpyAsync(sh.d_col, col + e0, me * sizeof(int), cudaMemcpyHostToDevice, h->stream),
                        "H2D col")))
        return st;
      if ((st = h->cuda(cudaMemcpyAsync(sh.d_w, static_cast<const char*>(w) + e0 * we, me * we,
                                        cudaMemcpyHostToDevice, h->stream), "H2D w")))
        return st;
    }
  }
  // the host arrays are read before return (the stream was idle: settled by the caller)
  if ((st = h->cuda(cudaStreamSynchronize(h->stream), "H2D csr sync"))) return st;
  h->fw_done = false;
  h->next_round = 0;
  return run_init(h);
}

// R25: every candidate sum a + b of the blocked FW is a sum of two restricted shortest-path
// lengths (phase 3: panel entries final for the round; phases 1-2: FW within a tile),
// each of at most n - 1 arcs of weight in [0, W], so |a + b| <= 2 (n - 1) W. With that <= 2^24
// every sum is an integer fp32 represents exactly, one RN add returns it, and min is exact: the
// fp32 closure equals the int32 one. Non-negative weights (no negative cycles, no drift below 0),
// single-GPU in-core 128-tile dataflow schedule (the path run_dataflow_f32x takes).
bool f32x_eligible(const Handle* h) {
  if (!h->want_f32x || h->dtype != APSP_I32 || h->has_neg || h->mode16) return false;
  if (h->mode != APSP_MODE_INCORE || h->world != 1 || h->virt || h->use_comm || !h->dataflow || h->small)
    return false;
  const double bound = 2.0 * (double)(h->n > 0 ? h->n - 1 : 0) * (double)h->max_abs_w;
  return bound <= 16777216.0;
}

// a1: CSR -> dense for every local shard, from the device CSR.
apsp_status run_init(Handle* h) {
  apsp_status st;
  h->result16 = false;
  if (h->mode16 && !h->fell_back16) {
    const Shard& sh = h->shards[0];
    if ((st = h->cuda(launch_init16(h->d16, h->ld, h->n_pad, h->n_pad, h->n, sh.d_rp, sh.d_col,
                                    static_cast<const int*>(sh.d_w), h->stream),
                      "init16")))
      return st;
    h->arith = APSP_ARITH_S16X2;
  }
  for (auto& sh : h->shards) {
    if (!sh.D) continue;
    cudaError_t e;
    if (h->dtype == APSP_I32)
      e = launch_init_rows<int>(static_cast<int*>(sh.D), h->ld, h->n_pad, sh.row_begin, h->rows_per_rank, h->n,
                                sh.d_rp, sh.e0, sh.d_col, static_cast<const int*>(sh.d_w), h->stream);
    else
      e = launch_init_rows<float>(static_cast<float*>(sh.D), h->ld, h->n_pad, sh.row_begin, h->rows_per_rank, h->n,
                                  sh.d_rp, sh.e0, sh.d_col, static_cast<const float*>(sh.d_w), h->stream);
    if ((st = h->cuda(e, "init_rows"))) return st;
  }
  if ((st = h->cuda(cudaMemsetAsync(h->d_flag, 0, sizeof(int), h->stream), "memset flag"))) return st;
  h->next_round = 0;
  h->fw_done = false;
  h->canonical = false;
  return APSP_OK;
}

static apsp_status init_placement(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col,
                                  const void* w);

apsp_status init_handle(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col,
                        const void* w) {
  apsp_status st;
  if ((st = setup_device(h, cfg))) return st;

  int64_t np, rb, rc;
  if (apsp_partition(h->n, h->b, h->world, h->virt ? 0 : h->rank, &np, &rb, &rc) != APSP_OK)
    return h->fail(APSP_EINVAL, "partition failed");
  h->n_pad = np;
  h->rows_per_rank = np / h->world;
  h->ld = np;
  // small n on one GPU: the 64-tile dataflow kernel (its per-round critical path is ~8x
  // shorter; measured crossover in DESIGN.md §5); APSP_SCHED_SMALL forces it at any n
  const bool one_gpu = h->world == 1 && !h->virt && cfg.force_nccl != 1;
  h->small = h->dataflow && one_gpu &&
             (cfg.schedule == APSP_SCHED_SMALL || (cfg.schedule == APSP_SCHED_AUTO && np <= kSmallAutoMaxN));

  // ---- in-core or out-of-core? ---------------------------------------------
  return init_placement(h, cfg, row_ptr, col, w);
}

// Device selection, kernel attributes, pool policy, streams, status flag.
apsp_status setup_device(Handle* h, const apsp_config& cfg) {
  apsp_status st;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
    return h->fail(APSP_ECUDA, "no CUDA device visible (the library has no CPU path)");
  if (cfg.device >= 0) {
    if (cfg.device >= ndev) return h->fail(APSP_EINVAL, "device %d >= device count %d", cfg.device, ndev);
    h->device = cfg.device;
  } else if ((st = h->cuda(cudaGetDevice(&h->device), "cudaGetDevice"))) {
    return st;
  }
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  cudaDeviceProp prop;
  if ((st = h->cuda(cudaGetDeviceProperties(&prop, h->device), "cudaGetDeviceProperties"))) return st;
  if (prop.major < 10) return h->fail(APSP_ECUDA, "device %s is sm_%d%d; this library is built for sm_100a", prop.name,
                                      prop.major, prop.minor);
  if ((st = h->cuda(configure_kernels(), "configure_kernels"))) return st;
  {
    // keep freed pool memory cached (apsp_trim_memory releases it)
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, h->device) == cudaSuccess) {
      unsigned long long thr = ~0ull;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  g_minplus_variant = cfg.minplus_variant;  // launch-per-phase min-plus kernel (apsp_kernels.cuh)
  // schedule: APSP_SCHED_AUTO = the persistent dataflow kernel on one GPU (int32 and fp32);
  // sharded placements (world > 1, virtual ranks, NCCL at world 1) default to the
  // launch-per-phase schedule with NCCL broadcasts; APSP_SCHED_DATAFLOW selects the sharded
  // dataflow kernel there (peer stores of the pivot panels).
  const bool sharded = h->world > 1 || cfg.force_nccl == 1;
  h->dataflow = cfg.schedule == APSP_SCHED_DATAFLOW || cfg.schedule == APSP_SCHED_SMALL ||
                (cfg.schedule == APSP_SCHED_AUTO && !sharded);
  h->df_delay = cfg.dataflow_delay;
  if (cfg.stream) {
    h->stream = static_cast<cudaStream_t>(cfg.stream);
  } else {
    if ((st = h->cuda(cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking), "cudaStreamCreate"))) return st;
    h->own_stream = true;
  }
  if (!cfg.no_lookahead) {  // the launch-per-phase lookahead's side stream (off: tests / A-B timing)
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    if ((st = h->cuda(cudaStreamCreateWithPriority(&h->side, cudaStreamNonBlocking, hi), "side stream"))) return st;
    for (auto& e : h->ev_la)
      if ((st = h->cuda(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event"))) return st;
  }
  if ((st = h->cuda(cudaMalloc(&h->d_flag, sizeof(int)), "cudaMalloc flag"))) return st;
  return h->cuda(cudaMemsetAsync(h->d_flag, 0, sizeof(int), h->stream), "memset flag");
}

// Device memory a new handle may use. apsp_destroy returns its big buffers to the device's
// stream-ordered pool, which keeps them cached (no driver round trip for the next handle); but
// cudaMemGetInfo does not count that cached memory as free, and plain cudaMalloc cannot use it.
// So when the driver's free memory is short of `want` (the caller's in-core working set) the
// pool's unused memory is returned to the driver first: without this a handle created after a
// large one was destroyed would see almost nothing free and fall back to the out-of-core path.
long long device_free_bytes(int device, long long want) {
  size_t free_b = 0, total_b = 0;
  if (cudaMemGetInfo(&free_b, &total_b) != cudaSuccess) return -1;
  if (want > (long long)free_b - (1ll << 30)) {
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess && cudaMemPoolTrimTo(pool, 0) == cudaSuccess &&
        cudaMemGetInfo(&free_b, &total_b) != cudaSuccess)
      return -1;
  }
  return (long long)free_b;
}

// The NCCL communicator of a sharded placement (one per handle).
static apsp_status create_comm(Handle* h, const apsp_config& cfg) {
  ncclUniqueId id;
  if (cfg.nccl_unique_id) {
    memcpy(&id, cfg.nccl_unique_id, sizeof(id));
  } else if (h->world == 1) {
    if (ncclGetUniqueId(&id) != ncclSuccess) return h->fail(APSP_ENCCL, "ncclGetUniqueId failed");
  } else {
    return h->fail(APSP_EINVAL, "nccl_unique_id is NULL");
  }
  ncclComm_t comm;
  ncclResult_t r = ncclCommInitRank(&comm, h->world, id, h->rank);
  if (r != ncclSuccess) return h->fail(APSP_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
  h->comm = comm;
  return APSP_OK;
}

// In-core (1-D block-row shards, packed int16) or out-of-core placement + init.
static apsp_status init_placement(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col,
                                  const void* w) {
  apsp_status st;
  const int nshards = h->virt ? h->world : 1;
  const long long mat_bytes = (long long)nshards * h->rows_per_rank * h->ld * (long long)h->elem;
  // force_nccl: run the sharded schedule with a 1-rank NCCL communicator even at
  // world_size 1, so a single GPU exercises the broadcast / all-reduce path
  h->use_comm = (h->world > 1 && !h->virt) || (h->world == 1 && cfg.force_nccl == 1);
  // two pivot-band panels (double-buffered by round parity)
  const long long panel_bytes =
      (h->world > 1 || h->use_comm) ? 2 * (long long)h->b * h->ld * (long long)h->elem : 0;
  const long long avail = device_free_bytes(h->device, mat_bytes + panel_bytes);
  if (avail < 0) return h->fail(APSP_ECUDA, "cudaMemGetInfo failed");
  long long budget = cfg.device_budget_bytes > 0 ? cfg.device_budget_bytes
                                                 : avail - (1ll << 30);  // keep 1 GiB headroom
  // a caller-owned matrix (cfg.dist_device, checked against mat_bytes by apsp_init_from_csr)
  // keeps the handle in core; only the library's own buffers count against the budget
  const bool need_ooc =
      cfg.force_out_of_core || ((cfg.dist_device ? 0 : mat_bytes) + panel_bytes > budget);
  if (need_ooc) {
    // out of core, on one GPU or replicated over the P ranks' band subsets (apsp_ooc.cu);
    // the ranks exchange only the finished pivot band of every super-round (NCCL broadcast)
    h->mode = APSP_MODE_OUT_OF_CORE;
    if (h->use_comm && (st = create_comm(h, cfg))) return st;
    return ooc_setup(h, cfg, budget, row_ptr, col, w);
  }

  // packed int16 (R16): single GPU, in core, int32 weights in [0, 8191]
  h->mode16 = cfg.packed16 == 1 && h->dtype == APSP_I32 && !h->has_neg && h->max_abs_w <= 8191 &&
              h->world == 1 && !h->virt && cfg.force_nccl != 1;
  if (h->mode16) {
    const long long b16 = h->n_pad * h->n_pad * 2;
    if (cfg.dist_device) {  // int16 working matrix in the first half; the int32 redo reuses the whole buffer
      h->dist_external = true;
      h->d16 = static_cast<short*>(cfg.dist_device);
    } else if ((st = h->cuda(cudaMallocAsync(reinterpret_cast<void**>(&h->d16), b16, h->stream),
                             "cudaMalloc dist16"))) {
      return st;
    }
    if ((st = h->cuda(cudaMalloc(&h->d_max16, sizeof(int)), "cudaMalloc"))) return st;
    h->device_bytes = h->dist_external ? 0 : b16;
    Shard sh;  // the int32 matrix is allocated only if the int16 result must be redone
    h->shards.push_back(sh);
    if ((st = upload_csr<int>(h, row_ptr, col, w))) return st;
    if ((st = run_init(h))) return st;
    return h->cuda(cudaStreamSynchronize(h->stream), "init sync");
  }

  // R25 exact fp32 closure (apsp_config.exact_f32): decided per graph (f32x_eligible)
  h->want_f32x = cfg.exact_f32 == 1;
  h->modef32x = f32x_eligible(h);
  if (h->modef32x) h->arith = APSP_ARITH_F32_EXACT;

  if (cfg.dist_device) {
    h->dist_external = true;
    h->d_base = cfg.dist_device;
  } else {
    if ((st = h->cuda(cudaMallocAsync(&h->d_base, mat_bytes, h->stream), "cudaMalloc dist"))) return st;
    h->device_bytes = mat_bytes;
  }
  if (panel_bytes) {
    if ((st = h->cuda(cudaMallocAsync(&h->panel, panel_bytes, h->stream), "cudaMalloc panel"))) return st;
    h->device_bytes += panel_bytes;
  }
  for (int s = 0; s < nshards; ++s) {
    Shard sh;
    sh.rank = h->virt ? s : h->rank;
    sh.row_begin = (long long)sh.rank * h->rows_per_rank;
    sh.D = static_cast<char*>(h->d_base) + (size_t)s * h->rows_per_rank * h->ld * h->elem;
    h->shards.push_back(sh);
  }

  if (h->use_comm && (st = create_comm(h, cfg))) return st;

  if ((st = h->dtype == APSP_I32 ? upload_csr<int>(h, row_ptr, col, w) : upload_csr<float>(h, row_ptr, col, w)))
    return st;
  if ((st = run_init(h))) return st;
  return h->cuda(cudaStreamSynchronize(h->stream), "init sync");
}

// The packed int16 closure as one persistent dataflow launch, timed as one
// event of class 2 carrying all n_pad^3 relaxations (as run_dataflow in apsp_api.cu).
static apsp_status run_dataflow16(Handle* h) {
  const int nb = (int)(h->n_pad / h->b);
  apsp_status st;
  if (!h->df_work) {
    if ((st = h->cuda(cudaMallocAsync(&h->df_work, fw_dataflow16_work_bytes(nb), h->stream), "cudaMalloc dataflow16")))
      return st;
    h->device_bytes += fw_dataflow16_work_bytes(nb);
  }
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const long long delay = h->df_delay > 0 ? h->df_delay : 4ll * fw_dataflow16_ctas_per_sm() * sms;
  h->kernel = APSP_KERNEL_DATAFLOW16;
  h->ev_begin(2);
  if ((st = h->cuda(launch_fw_dataflow16(h->d16, h->ld, nb, h->df_work, delay, h->stream), "fw_dataflow16")))
    return st;
  h->ev_end((double)h->n_pad * h->n_pad * h->n_pad);
  return APSP_OK;
}

// Packed int16 closure (VIADDMNMX.S16x2) with exactness check; int32 redo if the
// largest finite distance reaches 8192 (R16).
static apsp_status run_fw16_int32(Handle* h);

// Enqueue the int16 closure and its exactness check (the max finite entry to pinned
// h_max16); the result is provisionally int16 (result16) until check_fw16 reads it.
// A graph already known to need int32 (fell_back16) is enqueued in int32 directly.
apsp_status enqueue_fw16(Handle* h) {
  apsp_status st;
  const long long nb = h->n_pad / h->b;
  if (h->fell_back16) return run_fw16_int32(h);
  if (h->dataflow) {  // default: every round in one persistent launch (apsp_fw_dataflow16.cu)
    if ((st = run_dataflow16(h))) return st;
  } else {
    h->kernel = APSP_KERNEL_PER_PHASE;
    if ((st = fw_closure<short>(h, h->d16, h->ld, h->n_pad, 0, nb, h->stream))) return st;
  }
  if (!h->h_max16 && (st = h->cuda(cudaHostAlloc(&h->h_max16, sizeof(int), cudaHostAllocDefault), "cudaHostAlloc")))
    return st;
  if ((st = h->cuda(launch_max_finite16(h->d16, h->ld, h->n_pad, h->n_pad, h->d_max16, h->stream), "max16")))
    return st;
  if ((st = h->cuda(cudaMemcpyAsync(h->h_max16, h->d_max16, sizeof(int), cudaMemcpyDeviceToHost, h->stream),
                    "D2H max")))
    return st;
  h->result16 = true;
  h->arith = APSP_ARITH_S16X2;
  h->pending16 = true;
  return APSP_OK;
}

// After the stream is synchronized: keep the int16 result if it is provably exact, else
// redo in int32 (and from now on run this graph in int32), synchronously.
static apsp_status check_fw16(Handle* h) {
  if (!h->pending16) return APSP_OK;
  h->pending16 = false;
  if (*h->h_max16 < 8192) return APSP_OK;
  h->fell_back16 = true;  // distances too long for int16
  h->result16 = false;
  apsp_status st;
  if ((st = run_fw16_int32(h))) return st;
  return h->cuda(cudaStreamSynchronize(h->stream), "fw16 int32 redo");
}

apsp_status run_fw16(Handle* h) {
  apsp_status st;
  if ((st = enqueue_fw16(h))) return st;
  if ((st = h->cuda(cudaStreamSynchronize(h->stream), "fw16 sync"))) return st;
  return check_fw16(h);
}

static apsp_status run_fw16_int32(Handle* h) {
  apsp_status st;
  const long long nb = h->n_pad / h->b;
  Shard& sh = h->shards[0];
  if (!sh.D) {
    const long long mat_bytes = h->n_pad * h->ld * 4;
    if (h->dist_external) {  // the caller's buffer (it held the int16 working matrix)
      h->d_base = h->d16;
    } else {
      if ((st = h->cuda(cudaMallocAsync(&h->d_base, mat_bytes, h->stream), "cudaMalloc dist (int32 fallback)")))
        return st;
      h->device_bytes += mat_bytes;
    }
    sh.D = h->d_base;
  }
  if ((st = h->cuda(launch_init_rows<int>(static_cast<int*>(sh.D), h->ld, h->n_pad, 0, h->n_pad, h->n, sh.d_rp,
                                          sh.e0, sh.d_col, static_cast<const int*>(sh.d_w), h->stream),
                    "init_rows")))
    return st;
  h->result16 = false;
  h->arith = APSP_ARITH_I32;
  h->kernel = APSP_KERNEL_PER_PHASE;
  return fw_closure<int>(h, static_cast<int*>(sh.D), h->ld, h->n_pad, 0, nb, h->stream);
}

void delete_handle(Handle* h) {
  if (!h) return;
  cudaSetDevice(h->device);
  if (h->side) cudaStreamSynchronize(h->side);
  if (h->copy_stream) cudaStreamSynchronize(h->copy_stream);
  if (h->stream) {
    // large buffers come from the device's stream-ordered pool (cudaMallocAsync); the
    // pool keeps them for the next handle instead of returning them to the driver
    if (!h->dist_external) {  // a caller-owned apsp_config.dist_device is never freed here
      if (h->d_base) cudaFreeAsync(h->d_base, h->stream);
      if (h->d16) cudaFreeAsync(h->d16, h->stream);
    }
    if (h->panel) cudaFreeAsync(h->panel, h->stream);
    if (h->df_work) cudaFreeAsync(h->df_work, h->stream);
    if (h->virt)
      for (void* w : h->sh_work) cudaFreeAsync(w, h->stream);
    h->d_base = h->panel = h->df_work = nullptr;
    h->d16 = nullptr;
    cudaStreamSynchronize(h->stream);
  }
  for (auto& te : h->events) {
    cudaEventDestroy(te.a);
    cudaEventDestroy(te.b);
  }
  if (!h->virt) {  // NCCL-rank shard buffer and the peers' buffers opened through CUDA IPC
    for (int e = 0; e < 8; ++e)
      if (h->sh_peer[e] && e != h->rank) cudaIpcCloseMemHandle(h->sh_peer[e]);
    for (void* w : h->sh_work) cudaFree(w);
  }
  if (h->comm) ncclCommDestroy(static_cast<ncclComm_t>(h->comm));
  ooc_free(h);
  bnd_free(h);
  jn_free(h);
  for (auto& sh : h->shards) {
    cudaFree(sh.d_rp);
    cudaFree(sh.d_col);
    cudaFree(sh.d_w);
  }
  cudaFree(h->d_max16);
  if (h->copy_stream) {
    cudaStreamSynchronize(h->copy_stream);
    cudaStreamDestroy(h->copy_stream);
  }
  for (auto& e : h->copy_ev)
    if (e) cudaEventDestroy(e);
  cudaFree(h->d_widen);
  cudaFree(h->d_flag);
  if (h->h_flag) cudaFreeHost(h->h_flag);
  if (h->h_max16) cudaFreeHost(h->h_max16);
  cudaFree(h->d_widen_async);
  if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
  if (h->side) {
    cudaStreamSynchronize(h->side);
    cudaStreamDestroy(h->side);
  }
  for (auto& e : h->ev_la)
    if (e) cudaEventDestroy(e);
  for (auto& e : h->ev_sh)
    if (e) cudaEventDestroy(e);
  delete h;
}

apsp_status settle(Handle* h) {
  if (!h->pending) return APSP_OK;
  const bool fw = h->pending_fw;
  h->pending = h->pending_fw = false;
  apsp_status st;
  if ((st = h->cuda(cudaSetDevice(h->device), "cudaSetDevice"))) return st;
  if ((st = h->cuda(cudaStreamSynchronize(h->stream), "async sync"))) return st;
  if (h->copy_stream && (st = h->cuda(cudaStreamSynchronize(h->copy_stream), "async sync"))) return st;
  if (h->pending16) {
    const bool redo = *h->h_max16 >= 8192;
    std::vector<Handle::CopyReq> reqs;
    reqs.swap(h->pending_copies);
    if ((st = check_fw16(h))) return st;
    if (redo)  // the copies enqueued from the provisional int16 result: again from the int32 redo
      for (const auto& q : reqs)
        if ((st = get_rows(h, q.r0, q.cnt, q.out, q.ld))) return st;
  }
  h->pending_copies.clear();
  if (fw) {
    if (h->timing) h->collect_events();
    if (*h->h_flag) return h->fail(APSP_ENEGCYCLE, "negative cycle detected: distances are unspecified");
  }
  return APSP_OK;
}

// The end of an asynchronous closure: the flag's D2H is enqueued, settle() reads it.
apsp_status finish_fw_async(Handle* h) {
  apsp_status st;
  if (h->use_comm) {
    ncclResult_t r = ncclAllReduce(h->d_flag, h->d_flag, 1, ncclInt32, ncclMax, static_cast<ncclComm_t>(h->comm),
                                   h->stream);
    if (r != ncclSuccess) return h->fail(APSP_ENCCL, "ncclAllReduce(flag): %s", ncclGetErrorString(r));
  }
  if (!h->h_flag && (st = h->cuda(cudaHostAlloc(&h->h_flag, sizeof(int), cudaHostAllocDefault), "cudaHostAlloc flag")))
    return st;
  if ((st = h->cuda(cudaMemcpyAsync(h->h_flag, h->d_flag, sizeof(int), cudaMemcpyDeviceToHost, h->stream),
                    "D2H flag")))
    return st;
  h->canonical = false;
  h->fw_done = true;
  h->pending = h->pending_fw = true;
  return APSP_OK;
}

// Enqueue the D2H of rows [r0, r0+cnt) on the handle's stream (in core, not
// packed16); other placements copy synchronously through get_rows.
apsp_status get_rows_async(Handle* h, long long r0, long long cnt, void* out, long long ld_out) {
  if (h->mode != APSP_MODE_INCORE || h->result16) return get_rows(h, r0, cnt, out, ld_out);  // (int16: async while pending16)
  if (h->mode16 && !h->shards[0].D) return h->fail(APSP_ESTATE, "no int32 matrix yet");
  apsp_status st;
  const char* base;
  if (h->world > 1 && !h->virt) {
    const long long rb = h->shards[0].row_begin;
    if (r0 < rb || r0 + cnt > rb + h->rows_per_rank)
      return h->fail(APSP_EINVAL, "rows [%lld, %lld) are not local to rank %d", r0, r0 + cnt, h->rank);
    base = static_cast<const char*>(h->shards[0].D) + (size_t)(r0 - rb) * h->ld * h->elem;
  } else {
    base = static_cast<const char*>(h->d_base) + (size_t)r0 * h->ld * h->elem;
  }
  if (h->dtype == APSP_I32 && h->has_neg && !h->canonical) {
    for (auto& sh : h->shards)
      if ((st = h->cuda(launch_canonicalize_i32(static_cast<int*>(sh.D), h->ld, h->rows_per_rank, h->n_pad, h->stream),
                        "canonicalize")))
        return st;
    h->canonical = true;
  }
  if ((st = h->cuda(cudaMemcpy2DAsync(out, (size_t)ld_out * h->elem, base, (size_t)h->ld * h->elem,
                                      (size_t)h->n * h->elem, (size_t)cnt, cudaMemcpyDeviceToHost, h->stream),
                    "D2H dist")))
    return st;
  h->pending = true;
  return APSP_OK;
}

apsp_status finish_fw(Handle* h, bool all_rounds) {
  apsp_status st;
  int flag = 0;
  if (h->use_comm) {
    ncclResult_t r = ncclAllReduce(h->d_flag, h->d_flag, 1, ncclInt32, ncclMax, static_cast<ncclComm_t>(h->comm),
                                   h->stream);
    if (r != ncclSuccess) return h->fail(APSP_ENCCL, "ncclAllReduce(flag): %s", ncclGetErrorString(r));
  }
  if ((st = h->cuda(cudaMemcpyAsync(&flag, h->d_flag, sizeof(int), cudaMemcpyDeviceToHost, h->stream), "D2H flag")))
    return st;
  if ((st = h->cuda(cudaStreamSynchronize(h->stream), "fw sync"))) return st;
  if (h->use_comm) {  // a peer's failure surfaces here instead of as a later hang
    ncclResult_t ar = ncclSuccess;
    if (ncclCommGetAsyncError(static_cast<ncclComm_t>(h->comm), &ar) != ncclSuccess || ar != ncclSuccess) {
      h->poisoned = true;
      return h->fail(APSP_ENCCL, "NCCL asynchronous error: %s", ncclGetErrorString(ar));
    }
  }
  if (h->timing) h->collect_events();
  h->canonical = false;
  if (all_rounds) h->fw_done = true;
  if (flag) return h->fail(APSP_ENEGCYCLE, "negative cycle detected: distances are unspecified");
  return APSP_OK;
}

apsp_status get_rows(Handle* h, long long r0, long long cnt, void* out, long long ld_out) {
  if (h->mode == APSP_MODE_OUT_OF_CORE) return ooc_get_rows(h, r0, cnt, out, ld_out);
  if (h->mode == APSP_MODE_BOUNDARY) return bnd_get_rows(h, r0, cnt, out, ld_out);
  if (h->mode == APSP_MODE_JOHNSON) return jn_get_rows(h, r0, cnt, out, ld_out);
  apsp_status st;
  if (h->mode16 && !h->shards[0].D && !h->result16)
    return h->fail(APSP_ESTATE, "no int32 matrix yet");
  if (h->result16) {
    // widen int16 rows to int32 on the device (INF16 -> APSP_INF_I32) into two
    // alternating staging blocks; the D2H of one block overlaps the widening of the next
    const long long ldw = (h->n + 7) / 8 * 8;
    const long long blk = std::max<long long>(1, std::min<long long>(cnt, (64ll << 20) / (ldw * 4)));
    if (h->widen_rows < blk) {
      cudaFree(h->d_widen);
      h->d_widen = nullptr;
      if ((st = h->cuda(cudaMalloc(&h->d_widen, 2 * blk * ldw * 4), "cudaMalloc widen"))) return st;
      h->widen_rows = blk;
    }
    if (!h->copy_stream) {
      if ((st = h->cuda(cudaStreamCreateWithFlags(&h->copy_stream, cudaStreamNonBlocking), "stream"))) return st;
      for (auto& e : h->copy_ev)
        if ((st = h->cuda(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event"))) return st;
    }
    if (h->pending16) {
      // asynchronous copy: the whole request is widened in ONE kernel right behind the
      // closure (in submission order it precedes the next graph's persistent kernel, which
      // would otherwise hold every SM while later staging blocks wait), then one D2H on the
      // copy stream overlaps whatever runs next. settle() waits (and replays if the int16
      // result is rejected).
      const long long need = cnt * ldw;
      if (h->widen_async_elems < need) {
        cudaFree(h->d_widen_async);
        h->d_widen_async = nullptr;
        if ((st = h->cuda(cudaMalloc(&h->d_widen_async, need * 4), "cudaMalloc widen"))) return st;
        h->widen_async_elems = need;
      }
      if ((st = h->cuda(cudaStreamWaitEvent(h->stream, h->copy_ev[2], 0), "wait"))) return st;  // previous async D2H
      if ((st = h->cuda(launch_widen16(h->d16 + r0 * h->ld, h->ld, h->d_widen_async, ldw, cnt, h->n, h->stream),
                        "widen16")))
        return st;
      if ((st = h->cuda(cudaEventRecord(h->copy_ev[0], h->stream), "event"))) return st;
      if ((st = h->cuda(cudaStreamWaitEvent(h->copy_stream, h->copy_ev[0], 0), "wait"))) return st;
      if ((st = h->cuda(cudaMemcpy2DAsync(out, (size_t)ld_out * 4, h->d_widen_async, (size_t)ldw * 4,
                                          (size_t)h->n * 4, (size_t)cnt, cudaMemcpyDeviceToHost, h->copy_stream),
                        "D2H dist")))
        return st;
      if ((st = h->cuda(cudaEventRecord(h->copy_ev[2], h->copy_stream), "event"))) return st;
      h->pending_copies.push_back({r0, cnt, out, ld_out});
      h->pending = true;
      return APSP_OK;
    }
    int b = 0;
    for (long long r = r0; r < r0 + cnt; r += blk, b ^= 1) {
      const long long rr = std::min(blk, r0 + cnt - r);
      int* stage = h->d_widen + (size_t)b * h->widen_rows * ldw;
      // the D2H that last read this staging block must be done before it is rewritten
      if ((st = h->cuda(cudaStreamWaitEvent(h->stream, h->copy_ev[2 + b], 0), "wait"))) return st;
      if ((st = h->cuda(launch_widen16(h->d16 + r * h->ld, h->ld, stage, ldw, rr, h->n, h->stream), "widen16")))
        return st;
      if ((st = h->cuda(cudaEventRecord(h->copy_ev[b], h->stream), "event"))) return st;
      if ((st = h->cuda(cudaStreamWaitEvent(h->copy_stream, h->copy_ev[b], 0), "wait"))) return st;
      if ((st = h->cuda(cudaMemcpy2DAsync(static_cast<int*>(out) + (r - r0) * ld_out, (size_t)ld_out * 4, stage,
                                          (size_t)ldw * 4, (size_t)h->n * 4, (size_t)rr, cudaMemcpyDeviceToHost,
                                          h->copy_stream),
                        "D2H dist")))
        return st;
      if ((st = h->cuda(cudaEventRecord(h->copy_ev[2 + b], h->copy_stream), "event"))) return st;
    }
    return h->cuda(cudaStreamSynchronize(h->copy_stream), "get_dist sync");
  }
  const bool was_pending = h->pending;
  if ((st = get_rows_async(h, r0, cnt, out, ld_out))) return st;
  h->pending = was_pending;
  return h->cuda(cudaStreamSynchronize(h->stream), "get_dist sync");
}

}  // namespace apsp
