// apsp_kernels.cuh — internal interface between the schedulers (apsp_api.cu)
// and the sm_100a kernels (apsp_kernels.cu). Not part of the C ABI.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include <vector>

namespace apsp {

constexpr int kTile = 128;  // b: tile edge = round depth ("b x b" blocks)

// One rectangular family of output tiles for the min-plus kernel:
//   Cout(ti,tj) = min(Cin(ti,tj), A(ti, 0:K) (x) B(0:K, tj))
// where tile (ti, tj) has its top-left element at
//   Cin  + ti*128*ldc_in  + tj*128      (same for Cout with ldc_out)
//   A    + ti*128*lda                    (128 rows x K, row-major, A already at column 0 of the depth)
//   B    + tj*128                        (K rows x 128, row-major)
// ti runs over tiles_i values skipping skip_i (>= 0) and tj over tiles_j
// values skipping skip_j (>= 0): tiles_i / tiles_j count the tiles AFTER the
// skip, so ti in [0, tiles_i + (skip_i>=0)).
template <typename T>
struct MinPlusDesc {
  T* Cout;
  const T* Cin;
  const T* A;
  const T* B;
  long long ldc_out, ldc_in, lda, ldb;
  int tiles_i, tiles_j, skip_i, skip_j;
  int skip_i2 = -1, skip_j2 = -1;  // optional second skipped index, > skip_i / skip_j
  int K = 0;                       // depth, used by launch_minplus_batched only
};

// Many tile families in one launch: descs / prefix are DEVICE arrays of nf
// descriptors (each with its own K, a multiple of 32) and nf+1 CTA offsets
// (prefix[0] = 0, prefix[nf] = total tiles).
template <typename T>
cudaError_t launch_minplus_batched(const MinPlusDesc<T>* descs, const long long* prefix, int nf, long long total,
                                   cudaStream_t s);

// phase 1 on `count` tiles (device array of tile pointers, same ld), one CTA each
template <typename T>
cudaError_t launch_phase1_batched(T* const* tiles, int count, long long ld, int* negflag, cudaStream_t s);

// small helpers (boundary algorithm)
template <typename T>
cudaError_t launch_fill(T* p, long long count, T value, cudaStream_t s);
// dst = min(dst, src) on a rows x cols block
template <typename T>
cudaError_t launch_min_into(T* dst, long long ldd, const T* src, long long lds, long long rows, long long cols,
                            cudaStream_t s);
// out[r][c] = D[rowmap[r]][colmap[c]] for r < cnt, c < ncols (int32: values >= INF/2 -> INF)
template <typename T>
cudaError_t launch_gather(const T* D, long long ld, const int* rowmap, const int* colmap, T* out, long long ldo,
                          long long cnt, long long ncols, cudaStream_t s);

// Phase 2 / phase 3 / out-of-core products: up to two tile families in one
// launch (grid = total tiles). K must be a positive multiple of 32.
template <typename T>
cudaError_t launch_minplus(const MinPlusDesc<T>* d, int ndesc, int K, cudaStream_t s);

// Phase 1: in-place FW closure of one 128x128 tile (ld elements per row).
// Sets *negflag = 1 if a diagonal element is negative when its step starts.
template <typename T>
cudaError_t launch_phase1(T* tile, long long ld, int* negflag, cudaStream_t s);

// CSR -> dense init of `rows` rows starting at global row row_begin into D
// (ld elements per row, n_pad columns). row_ptr is the LOCAL slice
// (rows+1 entries, absolute arc offsets minus row_ptr_base).
template <typename T>
cudaError_t launch_init_rows(T* D, long long ld, long long n_pad, long long row_begin, long long rows,
                             long long n, const long long* row_ptr, long long row_ptr_base,
                             const int* col, const T* w, cudaStream_t s);

// int32 only: values >= INF/2 become INF (drifted infinities under negative
// weights, reading R5). rows x cols block at ld.
cudaError_t launch_canonicalize_i32(int* D, long long ld, long long rows, long long cols, cudaStream_t s);

// R25 (apsp_config.exact_f32): count int32 entries to fp32 in place (APSP_INF_I32 -> +inf) and
// back (+inf -> APSP_INF_I32); count % 4 == 0, 16-byte aligned.
cudaError_t launch_i32_to_f32(int* D, long long count, cudaStream_t s);
cudaError_t launch_f32_to_i32(float* D, long long count, cudaStream_t s);

// Per-device kernel attributes (dynamic shared memory opt-in). Call once per
// device before the first launch.
cudaError_t configure_kernels();

// ---- packed int16 path (apsp_kernels16.cu): VIADDMNMX.S16x2, 2 relax/instr ----
template <>
cudaError_t launch_minplus<short>(const MinPlusDesc<short>* d, int ndesc, int K, cudaStream_t s);
template <>
cudaError_t launch_phase1<short>(short* tile, long long ld, int* negflag, cudaStream_t s);
// rows 0..rows-1 (global = local, single GPU) of the int16 matrix from a CSR
// with absolute offsets; INF16 = 16383; weights must lie in [0, 8191]
cudaError_t launch_init16(short* D, long long ld, long long n_pad, long long rows, long long n,
                          const long long* row_ptr, const int* col, const int* w, cudaStream_t s);
// *out = max entry < INF16 (or -1)
cudaError_t launch_max_finite16(const short* D, long long ld, long long rows, long long cols, int* out,
                                cudaStream_t s);
// int16 rows -> int32 rows, INF16 -> APSP_INF_I32
cudaError_t launch_widen16(const short* S, long long lds, int* D, long long ldd, long long rows, long long cols,
                           cudaStream_t s);
cudaError_t configure_kernels16();

// The TMA + mbarrier persistent variant of launch_minplus (apsp_minplus_tma.cu).
// g_minplus_variant (set from apsp_config.minplus_variant): 0 = cp.async +
// mbarrier pipeline (default), 1 = cp.async + one CTA barrier per chunk,
// 2 = TMA persistent kernel (measured slower in round 1: its persistent grid
// also blocks the lookahead phases 1+2).
template <typename T>
cudaError_t launch_minplus_tma(const MinPlusDesc<T>* d, int ndesc, int K, cudaStream_t s);
cudaError_t configure_tma_kernels();
extern int g_minplus_variant;

// The whole single-GPU blocked FW (all nb rounds, phases 1-3) as one
// persistent dataflow kernel (apsp_fw_dataflow.cu). `work` is a device buffer
// of fw_dataflow_work_bytes(nb, sizeof(T)) bytes (panel copies + flags; the
// flags are zeroed by the launch). delay: phase-3 tasks queued between a
// round's phase-1 task and its phase-2 tasks; stagger: cycles the second
// group of every CTA waits before its first task.
template <typename T>
cudaError_t launch_fw_dataflow(T* D, long long ld, int nb, void* work, int* negflag, long long delay,
                               long long stagger, cudaStream_t s, unsigned long long* prof = nullptr,
                               int* used_pair = nullptr);
long long fw_dataflow_pbuf_bytes(int nb, size_t elem);
long long fw_dataflow_flag_bytes(int nb);
long long fw_dataflow_work_bytes(int nb, size_t elem);
long long fw_dataflow_pbuf_bytes(int nb, int nl, size_t elem, int npar);
long long fw_dataflow_flag_bytes(int nb, int nl);

// The same kernel over a 1-D block-row shard (rank q of P owns tile rows
// [q*nl, (q+1)*nl), nl = nb/P): the owner of round k stores the closed diagonal
// block and the row panel straight into every rank's panel buffer (peer stores:
// NVLink for other GPUs, plain stores for virtual ranks on one GPU) and raises
// their flags, so no collective runs between rounds. `work` of each rank holds
// fw_dataflow_work_bytes(nb, nl, elem) bytes at the same layout on every rank;
// peer_work[r] is rank r's `work` as seen from this process. One launch runs the
// nv ranks listed (nv = P: virtual ranks on one GPU; nv = 1: this process's rank).
struct DFShard {
  int rank;
  void* D;                 // this rank's rows (rows_per_rank x ld)
  void* work;              // == peer_work[rank]
  void* peer_work[8];
};
long long fw_dataflow_work_bytes(int nb, int nl, size_t elem);
template <typename T>
cudaError_t launch_fw_dataflow_sharded(const DFShard* ranks, int nv, int P, int nb, long long ld, int* negflag,
                                       long long delay, cudaStream_t s);

// The whole single-GPU blocked FW for small n with 64x64 tiles (apsp_fw_small.cu): the
// dataflow schedule above at b = 64 (nb = n_pad / 64 rounds), one 256-thread CTA per task.
// `work` holds fw_small_work_bytes(nb, elem) bytes (panel copies + flags + the task queue). *queue_key
// (-1 for a new work buffer) names the queue configuration already in `work`; on a mismatch the
// queue is rebuilt and uploaded and the flags zeroed (afterwards each launch's last CTA re-zeroes them).
template <typename T>
cudaError_t launch_fw_small(T* D, long long ld, int nb, void* work, int* negflag, long long delay, long long* queue_key,
                            int ctas_per_sm, cudaStream_t s);
long long fw_small_work_bytes(int nb, size_t elem);
// its task queue (host-built, critical path first; type 4 = fused P3(k; k+1,k+1) + P1(k+1))
long long small_queue(int nb, long long delay, std::vector<int4>* q);

// The packed int16 closure (R16) as one persistent dataflow launch
// (apsp_fw_dataflow16.cu); `work` holds fw_dataflow16_work_bytes(nb) bytes.
cudaError_t launch_fw_dataflow16(short* D, long long ld, int nb, void* work, long long delay, cudaStream_t s,
                                 unsigned long long* prof = nullptr);
long long fw_dataflow16_work_bytes(int nb);
int fw_dataflow16_ctas_per_sm();

}  // namespace apsp
