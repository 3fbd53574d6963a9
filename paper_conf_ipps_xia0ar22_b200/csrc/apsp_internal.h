// apsp_internal.h — handle state shared by the C ABI and the schedulers.
#pragma once
#include "../../include/apsp.h"
#include "apsp_kernels.cuh"

#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>
#include <string>
#include <vector>

namespace apsp {

// n_pad up to which APSP_SCHED_AUTO picks the 64-tile small-n kernel (apsp_fw_small.cu)
constexpr long long kSmallAutoMaxN = 2048;
// its default queue delay (dataflow_delay = 0): G3R(k-1) tasks queued before round k's panels
constexpr long long kSmallDelay = 0;

// NVTX range for the duration of a scope (C-ABI entry points, out-of-core
// super-rounds): shows up in Nsight timelines and `ncu --nvtx` filters; a
// no-op when no tool is attached (NVTX3 is header-only).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
};

// A block of rows of the (padded) distance matrix resident on the device.
struct Shard {
  int rank = 0;              // owner rank of these rows
  long long row_begin = 0;   // first padded row
  void* D = nullptr;         // rows_per_rank x ld elements, row-major
  // device copy of this shard's CSR slice, kept for apsp_reinit
  long long* d_rp = nullptr;
  int* d_col = nullptr;
  void* d_w = nullptr;
  long long real_rows = 0, e0 = 0;
  long long cap_arcs = 0;    // arcs d_col / d_w can hold (apsp_load_csr reuses them)
};

struct TimedEvent {
  int cls = 0;
  cudaEvent_t a = nullptr, b = nullptr;
  double relax = 0;
};

struct Handle {
  // problem
  long long n = 0, n_pad = 0;
  int b = kTile;
  apsp_dtype dtype = APSP_I32;
  size_t elem = 4;
  bool has_neg = false;
  long long max_abs_w = 0;
  // packed int16 path (apsp_kernels16.cu)
  bool mode16 = false;      // requested and eligible: try int16 first
  bool result16 = false;    // the current result lives in d16
  bool fell_back16 = false; // this graph needed int32: later runs go straight to int32
  short* d16 = nullptr;     // n_pad x n_pad int16 matrix (single GPU, in core)
  int* d_max16 = nullptr;
  int* d_widen = nullptr;   // 2 staging blocks for get_dist of an int16 result
  long long widen_rows = 0;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t copy_ev[4] = {nullptr, nullptr, nullptr, nullptr};  // widened[2], copied[2]
  int arith = APSP_ARITH_I32;
  // R25 exact-fp32 closure of an int32 matrix (apsp_config.exact_f32 and the bound holds)
  bool modef32x = false;
  bool want_f32x = false;   // apsp_config.exact_f32 (re-checked against each graph loaded)
  // placement
  int device = 0;
  int world = 1, rank = 0;
  bool virt = false;
  bool use_comm = false;    // NCCL communicator present (world > 1, or forced at world 1)
  long long rows_per_rank = 0, ld = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  cudaStream_t side = nullptr;        // high-priority stream for lookahead phases 1+2
  cudaEvent_t ev_la[2] = {nullptr, nullptr};
  std::vector<Shard> shards;
  void* d_base = nullptr;   // allocation behind the shards (in-core)
  bool dist_external = false;  // d_base / d16 is the caller's apsp_config.dist_device (not freed)
  void* panel = nullptr;    // b x ld pivot band received from the owner
  int* d_flag = nullptr;    // negative-cycle flag (device)
  void* comm = nullptr;     // ncclComm_t
  // out-of-core
  int mode = APSP_MODE_INCORE;
  long long ooc_B = 0;
  void* ooc_dev = nullptr;  // out-of-core state (apsp_ooc.cu): per-rank band buffers, pinned host bands
  void* ooc_streams[3] = {nullptr, nullptr, nullptr};
  // boundary algorithm (apsp_boundary.cu)
  void* bnd = nullptr;
  // Johnson's algorithm, batched Near-Far (apsp_johnson.cu)
  void* jn = nullptr;
  // single-GPU in-core dataflow kernel (apsp_fw_dataflow.cu)
  bool dataflow = true;     // apsp_config.schedule (APSP_SCHED_PER_PHASE: launch per phase)
  bool small = false;       // dataflow with 64x64 tiles (apsp_fw_small.cu): small n, APSP_SCHED_SMALL
  long long small_queue_key = -1;   // configuration of the task queue in df_work (-1: none)
  int kernel = 0;           // APSP_KERNEL_* of the last blocked-FW closure (apsp_info.kernel)
  long long df_delay = 0;   // apsp_config.dataflow_delay (0 = auto)
  void* df_work = nullptr;
  // sharded dataflow kernel (multi-GPU / virtual ranks): per-rank work buffers
  std::vector<void*> sh_work;          // virtual ranks: one per shard (pool); NCCL ranks: this rank's (cudaMalloc, IPC)
  void* sh_peer[8] = {};               // NCCL ranks: every rank's work buffer opened through CUDA IPC
  bool sh_ipc_open = false;
  bool sh_disabled = false;            // peer mapping failed on some rank: launch-per-phase + NCCL broadcasts
  // bookkeeping
  long long device_bytes = 0, host_bytes = 0;
  long long next_round = 0;
  bool fw_done = false, canonical = false, poisoned = false;
  bool pending = false;     // asynchronous work enqueued (apsp_*_async); settle() waits for it
  bool pending_fw = false;  // ... including a closure whose negative-cycle flag is still unread
  int* h_flag = nullptr;    // pinned host copy of d_flag for the asynchronous closure
  // packed16 asynchronous closure: the exactness check (max finite entry < 8192) is read
  // by settle(); copies enqueued meanwhile are replayed from the int32 redo if it fails
  int* h_max16 = nullptr;   // pinned
  int* d_widen_async = nullptr;      // one staging block for a whole asynchronous int16 -> int32 copy
  long long widen_async_elems = 0;
  bool pending16 = false;
  struct CopyReq {
    long long r0, cnt;
    void* out;
    long long ld;
  };
  std::vector<CopyReq> pending_copies;
  bool timing = false;
  std::vector<TimedEvent> events;
  apsp_phase_stats stats{};
  std::string err;

  apsp_status fail(apsp_status st, const char* fmt, ...);
  apsp_status cuda(cudaError_t e, const char* what);
  apsp_status bcast(void* buf, size_t bytes, int root, cudaStream_t s);
  cudaEvent_t ev_sh[3] = {nullptr, nullptr, nullptr};  // sharded lookahead: bcast, band, p3
  // class: 0 phase1, 1 phase2, 2 phase3, 3 comm / host transfer
  void ev_begin(int cls, cudaStream_t s);
  void ev_end(double relax, cudaStream_t s);
  void ev_begin(int cls) { ev_begin(cls, stream); }
  void ev_end(double relax) { ev_end(relax, stream); }
  void collect_events();
};

apsp_status init_handle(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col,
                        const void* w);
// R25: may this handle's current graph be closed by the fp32 engine exactly? (apsp_handle.cu)
bool f32x_eligible(const Handle* h);
void delete_handle(Handle* h);
apsp_status run_init(Handle* h);
apsp_status run_fw16(Handle* h);  // packed int16 closure, verify, int32 fallback
apsp_status enqueue_fw16(Handle* h);  // the same without waiting: settle() checks (h->pending16)
apsp_status run_incore_rounds(Handle* h, long long k0, long long k1);
apsp_status finish_fw(Handle* h, bool all_rounds);
// wait for pending asynchronous work (apsp_fw_blocked_async / apsp_get_dist_async)
apsp_status settle(Handle* h);
// apsp_load_csr: a new CSR (same n, dtype) into an in-core handle, init enqueued
apsp_status load_csr(Handle* h, const int64_t* row_ptr, const int32_t* col, const void* w);
apsp_status finish_fw_async(Handle* h);
apsp_status get_rows_async(Handle* h, long long r0, long long cnt, void* out, long long ld_out);
apsp_status get_rows(Handle* h, long long r0, long long cnt, void* out, long long ld_out);
bool nccl_unique_id(void* out128);

// out-of-core (apsp_ooc.cu)
apsp_status ooc_setup(Handle* h, const apsp_config& cfg, long long budget, const int64_t* row_ptr,
                      const int32_t* col, const void* w);
apsp_status run_out_of_core(Handle* h);
apsp_status run_out_of_core_range(Handle* h, long long K0, long long K1);
long long ooc_bands(const Handle* h);      // this process's bands
long long ooc_row_begin(const Handle* h);  // first padded row of this process's bands
apsp_status ooc_band_copy(Handle* h, long long I, void* buf, bool to_handle);
apsp_status ooc_get_rows(Handle* h, long long r0, long long cnt, void* out, long long ld_out);
void ooc_free(Handle* h);
apsp_status ooc_reinit(Handle* h);

// boundary algorithm (apsp_boundary.cu)
apsp_status bnd_setup(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col, const void* w,
                      const int32_t* comp, int k);
long long bnd_ooc_rows(const Handle* h);  // out of core: rows per output buffer, else 0
apsp_status bnd_reinit(Handle* h);
apsp_status bnd_run(Handle* h);
apsp_status bnd_get_rows(Handle* h, long long r0, long long cnt, void* out, long long ld_out);
long long bnd_boundary_nodes(const Handle* h);
void bnd_free(Handle* h);
// Johnson's algorithm with batched Near-Far SSSP (apsp_johnson.cu)
apsp_status jn_setup(Handle* h, const apsp_config& cfg, const int64_t* row_ptr, const int32_t* col, const void* w,
                     double delta, long long batch, bool sample = false);
apsp_status jn_sample_seconds(Handle* h, int k, unsigned long long seed, double* seconds);
apsp_status jn_reinit(Handle* h);
apsp_status jn_run(Handle* h);
apsp_status jn_get_rows(Handle* h, long long r0, long long cnt, void* out, long long ld_out);
long long jn_edges(const Handle* h);
void jn_local_rows(const Handle* h, long long* r0, long long* rc);
void jn_free(Handle* h);
// method selection (apsp_select.cu)
apsp_status fw_seconds_per_relax(const apsp_config& cfg, long long n0, double* out, std::string* err);
apsp_status hostlink_rate(int device, double* out, std::string* err);
apsp_status johnson_seconds(const apsp_config& cfg, long long n, const int64_t* row_ptr, const int32_t* col,
                            const void* w, apsp_dtype dtype, bool has_neg, int k, double* out, std::string* err);
// checkpoint / resume helpers
apsp_status global_fail(apsp_status st, const char* msg);
// common device / stream setup of a handle (apsp_handle.cu)
apsp_status setup_device(Handle* h, const apsp_config& cfg);
// free device memory, the memory pool trimmed first when it is short of `want` (apsp_handle.cu); -1 on error
long long device_free_bytes(int device, long long want);

}  // namespace apsp
