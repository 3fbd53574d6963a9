/*
 * apsp.h — C ABI of the B200 (sm_100a) blocked Floyd–Warshall APSP library
 * (libapsp.so, built from paper_conf_ipps_xia0ar22_b200/csrc/).
 *
 * Problem (§II): G = (V, E), n = |V|, m = |E|, w[i][j] the weight
 * of the arc from v_i to v_j; compute the n x n matrix dist where dist[i][j]
 * is the shortest distance from v_i to v_j. The graph arrives as CSR (the
 * paper's inputs are sparse adjacency matrices); the
 * distance element type is int32 (the paper's `int`), with an
 * fp32 instantiation for real weights (BASELINE.json config 4).
 *
 * Method (§II-A, and Algorithm 1, §III-A):
 * blocked Floyd–Warshall. dist is split into b x b tiles A(i,j); round k runs
 *   phase 1  A(k,k) := FW closure of A(k,k)
 *   phase 2  A(k,j) := min(A(k,j), A(k,k) (x) A(k,j)),  A(i,k) := min(A(i,k), A(i,k) (x) A(k,k))
 *   phase 3  A(i,j) := min(A(i,j), A(i,k) (x) A(k,j))   for i != k, j != k
 * where (x) is the min-plus product (MinPlus Multiply). When
 * n*n does not fit in device memory the library streams row bands from
 * pinned host memory (out-of-core, Algorithm 1 and PAPER.md:197).
 *
 * Conventions for every call:
 *  - Plain C; no exception crosses the boundary; every call returns
 *    apsp_status and never aborts the process.
 *  - Pointers are HOST pointers unless named *_device.
 *  - Error behaviour: on a non-OK status apsp_last_error(h) (or
 *    apsp_last_error(NULL) for failures before a handle exists) returns a
 *    one-line message. After APSP_ECUDA or APSP_ENCCL the handle is
 *    poisoned: only apsp_destroy is valid.
 *  - A handle is not thread-safe; different handles may be used from
 *    different threads on different devices.
 *  - Multi-GPU (world_size > 1, one process per GPU): every rank makes the
 *    same sequence of calls (init -> fw -> destroy), like an MPI collective.
 */
#ifndef APSP_H_
#define APSP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct apsp_handle apsp_handle; /* opaque, library-owned */

typedef enum { APSP_I32 = 0, APSP_F32 = 1 } apsp_dtype;

typedef enum {
  APSP_OK = 0,
  APSP_EINVAL = 1,     /* bad argument: NULL pointer, n < 0, row_ptr not monotone,
                          col out of [0, n), non-finite fp32 weight, bad config */
  APSP_ERANGE = 2,     /* int32 distances could reach APSP_INF_I32 (see init) */
  APSP_ENOMEM = 3,     /* device or pinned host allocation failed */
  APSP_ECUDA = 4,      /* CUDA runtime error (no device, launch failure ...) */
  APSP_ENCCL = 5,      /* NCCL error (multi-GPU only) */
  APSP_ENEGCYCLE = 6,  /* the graph holds a negative cycle; distances unspecified */
  APSP_ESTATE = 7      /* call out of order (e.g. get_dist before fw_blocked) */
} apsp_status;

/* int32 "no path" value in the output (and the internal infinity):
 * 2^30 - 1, so INF + INF still fits in int32 and the branch-free min-plus
 * update (PAPER.md:60's infinity) never overflows. fp32 uses +INFINITY. */
#define APSP_INF_I32 0x3FFFFFFF

#define APSP_MODE_INCORE 0
#define APSP_MODE_OUT_OF_CORE 1
#define APSP_MODE_BOUNDARY 2
#define APSP_MODE_JOHNSON 3

/* apsp_config.schedule: how the in-core blocked FW is scheduled. */
#define APSP_SCHED_AUTO 0       /* single GPU: the persistent dataflow kernel (all rounds and
                                   phases in one launch; 64x64 tiles for n_pad <= 2048, 128x128
                                   above); sharded placements: launch-per-phase
                                   rounds with NCCL pivot-band broadcasts */
#define APSP_SCHED_PER_PHASE 1  /* one launch per phase and round (phase 1, phase 2, phase 3) */
#define APSP_SCHED_DATAFLOW 2   /* the dataflow kernel; on sharded placements its sharded form,
                                   whose round owners store the pivot panels into every rank's
                                   panel buffer over NVLink (peer stores) */
#define APSP_SCHED_SMALL 3      /* single GPU: the dataflow schedule with 64x64 tiles (b = 64),
                                   built for small n, where the 128-tile rounds' critical path
                                   (phase 1 -> panel tile -> next diagonal tile) dominates; AUTO
                                   selects it for n_pad <= 2048. Sharded placements: as DATAFLOW */

typedef struct {
  int32_t struct_size;          /* = sizeof(apsp_config) (ABI versioning); 0 = defaults */
  int32_t device;               /* CUDA ordinal; -1 = current device */
  int32_t world_size;           /* number of ranks (1 = single GPU) */
  int32_t rank;                 /* this process's rank, 0 <= rank < world_size */
  const void* nccl_unique_id;   /* 128-byte ncclUniqueId from apsp_nccl_unique_id on
                                   rank 0, broadcast by the caller (e.g. with
                                   torch.distributed); NULL when world_size == 1 */
  int32_t virtual_ranks;        /* 1 = run all world_size shards in THIS process on
                                   one device, panel broadcast = device copy (tests the
                                   sharded schedule on one GPU); rank is ignored */
  int32_t tile;                 /* round depth b (tile edge); 0 = auto (128). Must be 128
                                   in this build (the kernels' tile edge) */
  void* stream;                 /* cudaStream_t to enqueue on; NULL = library stream */
  void* dist_device;            /* optional CALLER-OWNED device buffer (e.g. a torch tensor's
                                   data_ptr on cfg.device) that holds this process's rows of
                                   dist: row-major, ld = n_pad elements (apsp_dist_device_bytes
                                   gives the size; 256-byte aligned). The library never frees
                                   it; it must outlive the handle and not be touched while the
                                   handle's work is in flight. In-core blocked FW only
                                   (apsp_init_from_csr); APSP_EINVAL if it is too small, with
                                   force_out_of_core, or for boundary / Johnson handles. The
                                   matrix then does not count against device_budget_bytes (the
                                   handle never goes out of core). With packed16 the int16
                                   working matrix occupies the first half of the buffer.
                                   NULL = the library allocates */
  int64_t dist_device_bytes;    /* size of dist_device in bytes (>= apsp_dist_device_bytes) */
  int64_t device_budget_bytes;  /* 0 = use free device memory; smaller forces the
                                   out-of-core path (tests) */
  int32_t ooc_block;            /* out-of-core super-block (band height) B; 0 = auto;
                                   multiple of the tile */
  int32_t timing;               /* 1 = record CUDA events around every launch and
                                   accumulate per-phase device times (apsp_phase_stats) */
  int32_t force_out_of_core;    /* 1 = use the out-of-core path even if n*n fits */
  int32_t packed16;             /* 1 = int32 inputs whose weights lie in [0, 8191]
                                   are solved in packed int16 pairs (VIADDMNMX.S16x2,
                                   two relaxations per DPX instruction). The result is
                                   checked (max finite entry < 8192 proves it exact,
                                   DESIGN.md R16) and recomputed in int32 otherwise, so
                                   the output is always the exact int32 APSP. Single-GPU
                                   in-core only; ignored elsewhere. apsp_info.arith
                                   reports which arithmetic produced the result */
  int32_t schedule;             /* APSP_SCHED_* (0 = auto) */
  int32_t no_lookahead;         /* launch-per-phase schedule: 1 = no lookahead (phases 1-2
                                   of round k+1 are not overlapped with round k's phase 3) */
  int32_t ooc_stream_all;       /* out of core: 1 = keep no band resident in HBM (every
                                   band streamed from pinned host memory each super-round,
                                   the paper's setting) */
  int32_t force_nccl;           /* 1 = run the sharded schedule with a real 1-rank NCCL
                                   communicator at world_size 1 (exercises the broadcast /
                                   all-reduce path on one GPU) */
  int32_t minplus_variant;      /* launch-per-phase min-plus kernel: 0 = cp.async + mbarrier
                                   pipeline (default), 1 = cp.async + CTA barrier per chunk,
                                   2 = TMA persistent (an A/B experiment, measured slower) */
  int32_t dataflow_delay;       /* dataflow kernel queue delay (phase-3 tasks of round k-1
                                   queued before round k's panels); 0 = auto */
  int32_t exact_f32;            /* 1 = int32 inputs with weights in [0, W] and
                                   2 (n - 1) W <= 2^24 are closed by the fp32 engine
                                   (FADD2 + FMNMX3 instead of VIADDMNMX): every candidate
                                   sum of the blocked FW is an integer of magnitude <= 2^24,
                                   so each fp32 add is exact and the int32 output is
                                   bit-exact (R25, a proof before the run, no
                                   check after it). Single-GPU in-core 128-tile dataflow
                                   schedule only (n_pad > 2048); ignored elsewhere and for
                                   graphs outside the bound. apsp_info.arith reports
                                   APSP_ARITH_F32_EXACT when it applies */
  int32_t reserved[3];          /* must be 0 (APSP_EINVAL otherwise) */
} apsp_config;

/* Fill *cfg with defaults (struct_size set, device -1, world 1, rank 0). */
void apsp_config_default(apsp_config* cfg);

/*
 * apsp_init_from_csr — copy the graph to the device and build the initial
 * distance matrix ("initializes the matrix dist with the input
 * weights for the edges (which will be infinity when there are no edges)").
 *
 *   n         number of vertices, 0 <= n; vertices are 0..n-1
 *   row_ptr   host int64[n+1], row_ptr[0] = 0, non-decreasing; arcs of source u
 *             are e in [row_ptr[u], row_ptr[u+1])
 *   col_idx   host int32[m], m = row_ptr[n]; destination of arc e, in [0, n)
 *   weights   host int32[m] (APSP_I32) or float[m] (APSP_F32), finite
 *   dtype     element type of weights and of the distance matrix
 *   cfg       may be NULL (defaults)
 *
 * Semantics: dist[i][i] = 0; dist[u][v] = min over arcs u->v of w (duplicates
 * keep the minimum; a self-loop gives min(0, w)); all other entries infinity.
 * Ownership: the CSR arrays are read during the call only (copied).
 * Errors: APSP_EINVAL (see enum), APSP_ERANGE for int32 when
 * (n-1)*max|w| >= 2^28 with negative weights present or >= APSP_INF_I32 with
 * all weights >= 0; APSP_ENOMEM; APSP_ECUDA; APSP_ENCCL.
 * On success *out is a new handle (to be released with apsp_destroy).
 * With world_size > 1 each rank initialises only its own block of rows.
 */
apsp_status apsp_init_from_csr(apsp_handle** out, int64_t n, const int64_t* row_ptr,
                               const int32_t* col_idx, const void* weights, apsp_dtype dtype,
                               const apsp_config* cfg);

/*
 * apsp_init_boundary — set up the boundary algorithm (Djidjev et al.,
 * PAPER.md:139-150, eq. (1); Algorithm 3) for a graph with a
 * small separator. Same CSR arguments and semantics as apsp_init_from_csr,
 * plus a partition of the vertices (the paper uses METIS; the caller
 * provides it here):
 *   comp      host int32[n], component of each vertex, in [0, k)
 *   k         number of components, >= 1
 * A vertex with an arc to another component is a boundary node. Work
 * is O(k s^3 + NB^3 + n * NB * s) for components of size s and NB boundary
 * nodes instead of n^3. Single GPU. When the n x n result does not fit the
 * device budget (cfg->device_budget_bytes, else free memory) or
 * cfg->force_out_of_core = 1, the out-of-core form of Algorithm 3 runs: the
 * diagonal blocks (S_dia) and the boundary matrix (S_bound) stay in HBM, the
 * remaining memory S_rem holds two buffers of N_row whole block rows that two
 * streams fill and copy to a pinned host matrix alternately (Alg. 3
 * l.20); block rows that still fit stay resident in HBM (R21; none
 * when forced or with cfg->ooc_stream_all). The transfers are part of
 * apsp_solve. Run with apsp_solve; apsp_get_dist as usual.
 * Errors: as apsp_init_from_csr; APSP_EINVAL for a bad comp / k; APSP_ENOMEM
 * when not even S_dia + S_bound + two one-block-row buffers fit, or pinned
 * host memory for the streamed rows cannot be allocated.
 */
apsp_status apsp_init_boundary(apsp_handle** out, int64_t n, const int64_t* row_ptr,
                               const int32_t* col_idx, const void* weights, apsp_dtype dtype,
                               const int32_t* comp, int32_t k, const apsp_config* cfg);

/*
 * apsp_init_johnson — set up Johnson's algorithm (§II-B): one
 * single-source shortest-path run per source vertex, each by the Near-Far
 * method in ONE thread block, a persistent grid of blocks walking the
 * sources (Algorithm 2). Same CSR arguments, semantics and errors
 * as apsp_init_from_csr, plus:
 *   delta     the Near-Far bucket width Delta in weight units; 0 = auto
 *             (4 x the mean |weight|). Any delta > 0 gives the same distances
 *   batch     sources per batch when the result does not fit in device
 *             memory (Algorithm 2's `bat`; rows of a finished batch go
 *             to a pinned host matrix while the next batch runs); 0 = auto
 * Work is O(n * m * (re-expansions)) instead of n^3, so it wins on sparse
 * graphs (the paper's selection finding). The n x n result stays
 * in device memory when it fits the budget (cfg->device_budget_bytes, else
 * free memory), otherwise in pinned host memory (cfg->force_out_of_core = 1
 * forces this). Negative int32 weights are reweighted (Johnson: Bellman–Ford
 * potentials); a negative cycle makes apsp_solve return
 * APSP_ENEGCYCLE. fp32 weights must be >= 0 (else APSP_EINVAL). With
 * cfg->world_size = P > 1 (one handle per GPU / rank, cfg->rank set) rank r
 * computes the rows of sources [r*ceil(n/P), (r+1)*ceil(n/P)) (apsp_local_rows):
 * the SSSP instances are independent, so no communicator is used and
 * nccl_unique_id may be NULL. Run with apsp_solve; apsp_get_dist as usual (own
 * rows only); apsp_info.edges_scanned reports the arcs the last run relaxed.
 */
apsp_status apsp_init_johnson(apsp_handle** out, int64_t n, const int64_t* row_ptr,
                              const int32_t* col_idx, const void* weights, apsp_dtype dtype,
                              double delta, int64_t batch, const apsp_config* cfg);

/*
 * apsp_select — choose the method for a graph as the paper does (§IV,
 * PAPER.md:199-323). EXPERIMENTAL: the density filter is the selector SURVEY §8(f)
 * NEXT-4 names; the calibrated cost models behind it are outside the hot-path scope
 * and are kept as an aid, not a tuned component.
 * Density filter (§IV-C), density = m / n^2:
 *   > 1 %       blocked FW or Johnson
 *   < 0.01 %    Johnson or the boundary algorithm (only if a partition comp/k is
 *               given; the paper computes one with METIS)
 *   otherwise   Johnson
 * then the smallest cost-model estimate among the kept methods (§IV-B),
 * calibrated on this device at call time: blocked FW T0*(n/n0)^3 from a timed
 * random graph of n0 <= 8192 vertices; Johnson (n_b/k)*T from k = 5
 * randomly chosen batches actually run; boundary N_op * c_unit
 * with c_unit = the FW kernels' per-relaxation cost; plus the data
 * transfer models when the n x n result exceeds device memory.
 * Arguments as apsp_init_from_csr; comp/k as apsp_init_boundary or NULL/0.
 * Runs kernels on cfg->device (about 0.1-1 s); the graph is not retained.
 */
typedef struct {
  int32_t method;          /* APSP_MODE_INCORE (blocked FW; out of core when too big),
                              APSP_MODE_JOHNSON or APSP_MODE_BOUNDARY */
  int32_t candidates;      /* bit (1 << mode) per method the density filter kept */
  double density;          /* m / n^2 */
  double est_seconds[4];   /* estimate per mode index ([0] FW, [2] boundary,
                              [3] Johnson); -1 = not estimated */
  int64_t boundary_nodes;  /* boundary nodes of the given partition, else 0 */
} apsp_selection;

apsp_status apsp_select(int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                        const void* weights, apsp_dtype dtype, const int32_t* comp, int32_t k,
                        const apsp_config* cfg, apsp_selection* out);

/*
 * apsp_solve — run the method the handle was created for: the blocked
 * Floyd–Warshall (apsp_init_from_csr, same as apsp_fw_blocked), the boundary
 * algorithm (apsp_init_boundary) or Johnson's algorithm (apsp_init_johnson).
 * Blocks until done; APSP_ENEGCYCLE as apsp_fw_blocked.
 */
apsp_status apsp_solve(apsp_handle* h);

/*
 * apsp_fw_blocked — run the whole blocked Floyd–Warshall (all n/b rounds,
 * PAPER.md:62; out-of-core: Algorithm 1). Blocks until the
 * device work is done. Returns APSP_ENEGCYCLE if a negative cycle exists
 * (detected as a negative diagonal entry at the start of a phase-1 step; the
 * distances are then unspecified), APSP_ESTATE if already run.
 */
apsp_status apsp_fw_blocked(apsp_handle* h);

/*
 * apsp_reinit — rebuild the initial distance matrix (same semantics as
 * apsp_init_from_csr) from the device-resident copy of the CSR the handle
 * keeps, so that apsp_fw_blocked can run again on the same graph without a
 * host round trip (benchmark steps with inputs resident in HBM). Asynchronous
 * on the handle's stream.
 */
apsp_status apsp_reinit(apsp_handle* h);

/*
 * apsp_fw_rounds — run rounds [k_begin, k_end) only. After rounds 0..K-1,
 * dist[i][j] is the shortest path whose intermediates all lie in
 * {0 .. K*b - 1}, i.e. the plain FW state after K*b outer iterations
 * (PAPER.md:60). Used for per-round parity and checkpointing. Rounds must be
 * run in order; out of core they run in whole super-rounds (k_begin and k_end
 * multiples of ooc_block/tile, or k_end = the last round). apsp_fw_blocked
 * afterwards runs the remaining rounds.
 */
apsp_status apsp_fw_rounds(apsp_handle* h, int64_t k_begin, int64_t k_end);

/*
 * apsp_checkpoint / apsp_restore — save and resume a blocked-FW run (in core or
 * out of core; not packed16, virtual ranks, boundary or Johnson handles). After
 * rounds 0 .. k-1 the matrix is the FW state "intermediates in {0 .. k*b-1}"
 * (PAPER.md:60); out of core it is the pinned host bands plus the HBM-resident
 * bands after a super-round (Algorithm 1). apsp_checkpoint
 * writes this rank's padded rows and the next round to `path` (a 128-byte
 * header + rows x n_pad elements); apsp_restore loads such a file into a handle
 * created by apsp_init_from_csr for the same graph, dtype and placement (n,
 * n_pad, world/rank, out-of-core band height), after which apsp_fw_rounds or
 * apsp_fw_blocked continue with the remaining rounds. Synchronous.
 * Errors: APSP_EINVAL (cannot open / short file / mismatching checkpoint),
 * APSP_ESTATE (unsupported handle), APSP_ECUDA, APSP_ENOMEM.
 */
apsp_status apsp_checkpoint(apsp_handle* h, const char* path);
apsp_status apsp_restore(apsp_handle* h, const char* path);

/*
 * apsp_get_dist — copy rows [row_begin, row_begin+row_count), columns [0, n),
 * of dist into the caller's host buffer out (row_count x ld_out elements of
 * dtype, ld_out >= n; pinned memory is faster). Unreachable pairs read
 * APSP_INF_I32 (int32) or +INFINITY (fp32). With world_size > 1 (NCCL mode)
 * the rows must lie in this rank's block (apsp_local_rows). Valid after
 * apsp_init_from_csr (returns the initial matrix) and after apsp_fw_blocked.
 */
apsp_status apsp_get_dist(apsp_handle* h, int64_t row_begin, int64_t row_count, void* out,
                          int64_t ld_out);

/*
 * Asynchronous variants for serving loops (several graphs in flight: the D2H of
 * one result overlaps the closure of the next graph on another handle).
 *
 * apsp_fw_blocked_async — enqueue the whole blocked Floyd–Warshall
 *   on the handle's stream and return without waiting (in core; out of core it
 *   runs synchronously like apsp_fw_blocked, same statuses). The negative-cycle
 *   status is delivered by apsp_synchronize; with packed16 the int16 exactness
 *   check too (if it fails, apsp_synchronize redoes the closure in int32 and
 *   replays the copies already enqueued, so `out` buffers end exact).
 * apsp_get_dist_async — enqueue the D2H of rows [row_begin, row_begin+row_count)
 *   (same arguments and row rules as apsp_get_dist) behind the closure on the
 *   handle's stream; `out` must stay valid until apsp_synchronize returns and
 *   should be pinned (pageable memory makes the copy synchronous). Out-of-core,
 *   boundary and Johnson handles copy synchronously.
 * apsp_synchronize — wait for everything enqueued on the handle; returns
 *   APSP_ENEGCYCLE if the asynchronous closure found a negative cycle (the
 *   distances, including those already copied, are then unspecified),
 *   APSP_ECUDA on a device error, APSP_OK otherwise. Every other call on a
 *   handle with pending asynchronous work synchronizes it first (and returns
 *   its error, if any).
 */
apsp_status apsp_fw_blocked_async(apsp_handle* h);
/*
 * apsp_load_csr — put the next graph (same n and dtype, any arc count) into an
 *   existing in-core handle (not out of core / virtual ranks: APSP_ESTATE; a
 *   packed16 handle solves it in int16 if its weights qualify, else in int32) instead
 *   of creating a new one: validated and range-checked as in apsp_init_from_csr
 *   (same errors), copied to the handle's device CSR arrays (grown if needed)
 *   before return — the caller may reuse its arrays — and the CSR -> dense init
 *    enqueued on the handle's stream. Then apsp_fw_blocked[_async].
 *   With world_size > 1 every rank passes the whole CSR (each uploads its rows).
 */
apsp_status apsp_load_csr(apsp_handle* h, const int64_t* row_ptr, const int32_t* col_idx,
                          const void* weights);
apsp_status apsp_get_dist_async(apsp_handle* h, int64_t row_begin, int64_t row_count, void* out,
                                int64_t ld_out);
apsp_status apsp_synchronize(apsp_handle* h);

/*
 * apsp_debug_queue — diagnostics for tests: the persistent dataflow kernel's task queue,
 * computed on the host by the same decoder the kernel runs. P = 0: the single-GPU queue;
 * P >= 1: rank q's queue of the sharded kernel (nb % P == 0); P = -1: the small-n kernel's
 * queue (64-wide tiles, APSP_SCHED_SMALL). Writes up to `cap` tasks as (type, k, i, j) int32
 * quadruples (type 0 = phase 1 of round k, 1 = row-panel tile (k, j), 2 = column-panel tile
 * (i, k), 3 = phase-3 tile (i, j), 4 = phase-3 tile (k+1, k+1) of round k fused with phase 1
 * of round k+1; i, j global tile indices) and returns the queue length (-1 on bad
 * arguments). No device is touched.
 */
int64_t apsp_debug_queue(int32_t nb, int32_t P, int32_t q, int64_t delay, int32_t* out, int64_t cap);

/* Rows [*row_begin, *row_begin + *row_count) of dist held by this rank. */
apsp_status apsp_local_rows(const apsp_handle* h, int64_t* row_begin, int64_t* row_count);

/*
 * apsp_partition — the 1-D block-row partition used for world_size ranks
 * (host-only arithmetic, no device needed): n is padded to n_pad, a multiple
 * of tile*world_size; rank r owns padded rows [r*n_pad/world, (r+1)*n_pad/world)
 * and, of those, the real rows [*row_begin, *row_begin + *row_count).
 * owner of round k = (k*tile) / (n_pad/world).
 */
apsp_status apsp_partition(int64_t n, int32_t tile, int32_t world_size, int32_t rank,
                           int64_t* n_pad, int64_t* row_begin, int64_t* row_count);

/*
 * apsp_dist_device_bytes — bytes a caller-owned apsp_config.dist_device buffer needs for
 * apsp_init_from_csr(n, ..., dtype, cfg) (host-only arithmetic, no device needed):
 * (n_pad / world_size) * n_pad * 4 per rank (int32 and fp32 elements; n_pad from
 * apsp_partition), times world_size with virtual_ranks (all shards in one buffer).
 */
apsp_status apsp_dist_device_bytes(int64_t n, int32_t tile, int32_t world_size, int32_t virtual_ranks,
                                   int64_t* bytes);

typedef struct {
  int64_t n, n_pad;
  int32_t tile, dtype, world_size, rank, mode; /* mode: APSP_MODE_* */
  int32_t ooc_block;                           /* B when out-of-core, else 0 */
  int64_t rounds;                              /* n_pad / tile */
  int64_t device_bytes;                        /* device memory the handle holds */
  int64_t host_bytes;                          /* pinned host memory (out-of-core) */
  void* dist_device;                           /* in-core: device base of this rank's
                                                  rows (row-major, ld = ld elements,
                                                  int16 when arith == APSP_ARITH_S16X2);
                                                  NULL out-of-core */
  int64_t ld;
  int32_t arith;                               /* APSP_ARITH_*: arithmetic of the current
                                                  result (or of the next run) */
  int32_t packed16_eligible;                   /* packed16 requested and the input allows it */
  int64_t boundary_nodes;                      /* boundary algorithm: boundary nodes, else 0 */
  int64_t edges_scanned;                       /* Johnson: arcs relaxed by the last run, else 0 */
  int32_t kernel;                              /* APSP_KERNEL_*: what ran the last blocked-FW
                                                  closure (0 = none yet / other methods) */
  int32_t exact_f32_eligible;                  /* exact_f32 requested and the input allows it */
} apsp_info;

#define APSP_KERNEL_PER_PHASE 1      /* launch-per-phase rounds (phase1 / min-plus kernels) */
#define APSP_KERNEL_DATAFLOW 2       /* fw_dataflow_kernel, one round per task */
#define APSP_KERNEL_DATAFLOW_PAIR 3  /* fw_dataflow_kernel, two rounds per bulk task (decode2) */
#define APSP_KERNEL_SMALL 4          /* fw_small_kernel, 64x64 tiles */
#define APSP_KERNEL_DATAFLOW16 5     /* fw_dataflow16_kernel, packed int16 */
#define APSP_KERNEL_SHARDED 6        /* fw_dataflow_kernel<sharded> */
#define APSP_KERNEL_OUT_OF_CORE 7    /* the out-of-core band scheduler (min-plus kernels) */

#define APSP_ARITH_I32 0   /* VIADDMNMX (int32 DPX), 1 relaxation / instruction */
#define APSP_ARITH_S16X2 1 /* VIADDMNMX.S16x2, 2 relaxations / instruction, verified exact */
#define APSP_ARITH_F32 2   /* fp32: FADD2 (one A value against a column pair) + FMNMX3
                              (two depth steps folded into one accumulator update) */
#define APSP_ARITH_F32_EXACT 3 /* int32 distances closed by the fp32 engine (apsp_config.exact_f32,
                                  R25): the matrix converted to fp32 in place before the
                                  closure and back after it; bit-exact by the a priori bound */

apsp_status apsp_get_info(const apsp_handle* h, apsp_info* info);

typedef struct {
  double ms[4];          /* accumulated device time: [0] phase 1, [1] phase 2,
                            [2] phase 3, [3] comm / host transfers */
  int64_t launches[4];   /* kernel launches (or transfers) per class */
  double relax[4];       /* relaxations performed per class */
} apsp_phase_stats;

/* Per-phase device times of the last apsp_fw_blocked (needs cfg.timing = 1). */
apsp_status apsp_get_phase_stats(const apsp_handle* h, apsp_phase_stats* out);

/* Rank-0 helper: write a fresh 128-byte ncclUniqueId into out128. */
apsp_status apsp_nccl_unique_id(void* out128);

/* Release everything the handle owns. NULL is allowed. The large device
 * buffers come from the device's stream-ordered memory pool (cudaMallocAsync),
 * which keeps freed memory cached for the next handle (no driver round trip). */
void apsp_destroy(apsp_handle* h);

/* Return the cached pool memory of `device` (-1 = current) to the driver. */
apsp_status apsp_trim_memory(int32_t device);

/* Last error message of h (thread-local message when h is NULL). Never NULL. */
const char* apsp_last_error(const apsp_handle* h);

/* Library version string, e.g. "apsp-b200 0.1 sm_100a". */
const char* apsp_version(void);

#ifdef __cplusplus
}
#endif

#endif /* APSP_H_ */
