// apsp_kernels.cu — sm_100a kernels of the blocked Floyd–Warshall hot path.
//
//   init_rows      CSR -> dense distance rows
//   phase1         FW closure of the pivot tile A(k,k) (PAPER.md:62 step 1;
//                  Algorithm 1 line 3)
//   minplus        C = min(C, A (x) B) on 128x128 output tiles — phase 2
//                  (pivot row/column panels, PAPER.md:62 step 2, Alg. 1 l.7/11)
//                  and phase 3 (all other tiles, PAPER.md:62 step 3, Alg. 1
//                  l.17), and the depth-B products of the out-of-core path.
//
// The relaxation c = min(c, a + b) is one DPX instruction on
// Blackwell: __viaddmin_s32 -> SASS VIADDMNMX (int32). fp32 uses FADD + FMNMX.
// Tensor cores are not used: min-plus is not a multiply-add contraction.
#include "apsp_kernels.cuh"

#include <cuda_runtime.h>
#include <cstdint>
#include <cfloat>

namespace apsp {

// ----------------------------------------------------------------- values --

template <typename T> struct Val;
template <> struct Val<int> {
  static __device__ __forceinline__ int inf() { return 0x3FFFFFFF; }  // = APSP_INF_I32
  // min(c, a + b): VIADDMNMX on sm_90+/sm_100a
  static __device__ __forceinline__ int relax(int a, int b, int c) { return __viaddmin_s32(a, b, c); }
  static __device__ __forceinline__ int vmin(int a, int b) { return min(a, b); }
};
template <> struct Val<float> {
  static __device__ __forceinline__ float inf() { return __int_as_float(0x7f800000); }
  static __device__ __forceinline__ float relax(float a, float b, float c) { return fminf(c, __fadd_rn(a, b)); }
  static __device__ __forceinline__ float vmin(float a, float b) { return fminf(a, b); }
};

template <typename T> struct Vec4;
template <> struct Vec4<int> { using type = int4; };
template <> struct Vec4<float> { using type = float4; };

// ------------------------------------------------------------- cp.async --

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

// ------------------------------------------------------------- min-plus --
//
// CTA: 256 threads, one 128x128 output tile, register-blocked 8x8 per thread
// (two 4-row groups x two 4-col groups, 64 rows apart, so that every LDS is
// a 16-byte vector and B reads of a warp are contiguous). The depth K is
// streamed in chunks of 32 through a 3-stage cp.async pipeline:
//   As[s][128 rows][32+4]  (A chunk, row-major as in HBM; +4 pad breaks the
//                           bank aliasing of rows 4 apart)
//   Bs[s][32][128]         (B chunk, row-major)
// The accumulator starts as the C tile; C is written only after the whole
// depth has been read, so phase 2 (where A or B aliases C) is out-of-place
// per tile.

constexpr int MP_BM = 128, MP_BN = 128, MP_BK = 32, MP_NT = 256, MP_STAGES = 3;
constexpr int MP_ALD = MP_BK + 4;
constexpr int MP_BLD = MP_BN;
constexpr int MP_STAGE_ELEMS = MP_BM * MP_ALD + MP_BK * MP_BLD;  // 8704 words = 34 KB
constexpr int MP_CLD = MP_BN + 4;  // C tile rows staged in smem (64 rows per stage)
static_assert(64 * MP_CLD <= MP_STAGE_ELEMS, "half a C tile must fit one stage");

template <typename T>
struct MinPlusArgs {
  MinPlusDesc<T> d0, d1;
  long long n0;  // tiles in d0 (blockIdx.x < n0 -> d0)
  int K;
};

template <typename T>
constexpr int minplus_smem_bytes() {
  return MP_STAGES * MP_STAGE_ELEMS * (int)sizeof(T);
}

// Two depth steps kk, kk+1 of the 8x8 register block: acc[i][j] = min(acc[i][j],
// a[i][u] + b_u[j]) for u = 0, 1 (b_u = row kk+u of the B stage at column tx*4 and
// 64+tx*4). int32: one VIADDMNMX per relaxation. fp32: FADD2 (scalar a broadcast
// against a column pair) + FMNMX3 folding both steps = 1 instruction per relaxation
// instead of FADD + FMNMX; each candidate is still one RN add and min is exact, so
// the result is bit-identical to the one-step update.
template <typename T>
__device__ __forceinline__ void relax_two_steps(T (&acc)[8][8], const T (&a)[8][2], const T* brow0, const T* brow1,
                                                int tx) {
  using V4 = typename Vec4<T>::type;
  if constexpr (sizeof(T) == 4 && T(0.5) != T(0)) {
    const V4 b00 = *reinterpret_cast<const V4*>(brow0 + tx * 4);
    const V4 b01 = *reinterpret_cast<const V4*>(brow0 + 64 + tx * 4);
    const V4 b10 = *reinterpret_cast<const V4*>(brow1 + tx * 4);
    const V4 b11 = *reinterpret_cast<const V4*>(brow1 + 64 + tx * 4);
    const float2 p0[4] = {make_float2(b00.x, b00.y), make_float2(b00.z, b00.w), make_float2(b01.x, b01.y),
                          make_float2(b01.z, b01.w)};
    const float2 p1[4] = {make_float2(b10.x, b10.y), make_float2(b10.z, b10.w), make_float2(b11.x, b11.y),
                          make_float2(b11.z, b11.w)};
    // column pair outer, the four sums of each depth step grouped: the pair operand of
    // back-to-back FADD2s comes from the operand reuse cache (as in apsp_fw_dataflow.cu)
#pragma unroll
    for (int jp = 0; jp < 4; ++jp)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        float2 s0[4], s1[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) s0[i] = __fadd2_rn(make_float2(a[4 * h + i][0], a[4 * h + i][0]), p0[jp]);
#pragma unroll
        for (int i = 0; i < 4; ++i) s1[i] = __fadd2_rn(make_float2(a[4 * h + i][1], a[4 * h + i][1]), p1[jp]);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          acc[4 * h + i][2 * jp] = fminf(fminf(acc[4 * h + i][2 * jp], s0[i].x), s1[i].x);
          acc[4 * h + i][2 * jp + 1] = fminf(fminf(acc[4 * h + i][2 * jp + 1], s0[i].y), s1[i].y);
        }
      }
  } else {
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const T* brow = u ? brow1 : brow0;
      const V4 b0 = *reinterpret_cast<const V4*>(brow + tx * 4);
      const V4 b1 = *reinterpret_cast<const V4*>(brow + 64 + tx * 4);
      const T b[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = Val<T>::relax(a[i][u], b[j], acc[i][j]);
    }
  }
}

template <typename T>
__global__ void __launch_bounds__(MP_NT, 2) minplus_kernel(const __grid_constant__ MinPlusArgs<T> args) {
  using V4 = typename Vec4<T>::type;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  // stage s = [A chunk 128 x 36][B chunk 32 x 128], contiguous
  T* const stage0 = reinterpret_cast<T*>(smem_raw);

  long long t = blockIdx.x;
  const bool second = t >= args.n0;
  const MinPlusDesc<T>& d = second ? args.d1 : args.d0;
  if (second) t -= args.n0;
  int ti = (int)(t / d.tiles_j);
  int tj = (int)(t - (long long)ti * d.tiles_j);
  if (d.skip_i >= 0 && ti >= d.skip_i) ++ti;
  if (d.skip_i2 >= 0 && ti >= d.skip_i2) ++ti;
  if (d.skip_j >= 0 && tj >= d.skip_j) ++tj;
  if (d.skip_j2 >= 0 && tj >= d.skip_j2) ++tj;

  const T* __restrict__ Cin = d.Cin + (long long)ti * MP_BM * d.ldc_in + (long long)tj * MP_BN;
  T* __restrict__ Cout = d.Cout + (long long)ti * MP_BM * d.ldc_out + (long long)tj * MP_BN;
  const T* __restrict__ A = d.A + (long long)ti * MP_BM * d.lda;
  const T* __restrict__ B = d.B + (long long)tj * MP_BN;
  const long long lda = d.lda, ldb = d.ldb, ldc_in = d.ldc_in, ldc_out = d.ldc_out;

  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;

  // per-thread copy coordinates: A chunk = 128 rows x 8 x 16B (rows tid/8 + 32q),
  // B chunk = 32 rows x 32 x 16B (rows tid/32 + 8q)
  const T* const a_src = A + (tid >> 3) * lda + (tid & 7) * 4;
  const T* const b_src = B + (tid >> 5) * ldb + (tid & 31) * 4;
  const int a_dst = (tid >> 3) * MP_ALD + (tid & 7) * 4;
  const int b_dst = MP_BM * MP_ALD + (tid >> 5) * MP_BLD + (tid & 31) * 4;
  auto load_chunk = [&](int stage, int chunk) {
    T* st = stage0 + stage * MP_STAGE_ELEMS;
    const T* ag = a_src + chunk * MP_BK;
    const T* bg = b_src + (long long)chunk * MP_BK * ldb;
#pragma unroll
    for (int q = 0; q < 4; ++q) cp_async16(st + a_dst + q * 32 * MP_ALD, ag + q * 32 * lda);
#pragma unroll
    for (int q = 0; q < 4; ++q) cp_async16(st + b_dst + q * 8 * MP_BLD, bg + q * 8 * ldb);
  };

  const int nk = args.K / MP_BK;
#pragma unroll
  for (int s = 0; s < MP_STAGES - 1; ++s) {
    if (s < nk) load_chunk(s, s);
    cp_async_commit();
  }

  // The accumulators start at +infinity and C is folded in at the end:
  // min is exact, so min(C, min_kk(a + b)) equals the in-order update. C is
  // fetched by cp.async into the two stages that are free during the last
  // chunk, so its HBM latency hides behind that chunk's relaxations.
  T acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = Val<T>::inf();
  T* const cs_lo = stage0 + (nk % MP_STAGES) * MP_STAGE_ELEMS;        // C rows 0..63
  T* const cs_hi = stage0 + ((nk + 1) % MP_STAGES) * MP_STAGE_ELEMS;  // C rows 64..127

  for (int c = 0; c < nk; ++c) {
    cp_async_wait<MP_STAGES - 2>();
    __syncthreads();
    {
      int cn = c + MP_STAGES - 1;
      if (cn < nk) load_chunk(cn % MP_STAGES, cn);
      if (c == nk - 1) {  // C tile: 128 rows x 32 x 16B, rows tid/32 + 8q
        const T* cg = Cin + (tid >> 5) * ldc_in + (tid & 31) * 4;
        const int cd = (tid >> 5) * MP_CLD + (tid & 31) * 4;
#pragma unroll
        for (int q = 0; q < 8; ++q) cp_async16(cs_lo + cd + q * 8 * MP_CLD, cg + q * 8 * ldc_in);
#pragma unroll
        for (int q = 0; q < 8; ++q) cp_async16(cs_hi + cd + q * 8 * MP_CLD, cg + (64 + q * 8) * ldc_in);
      }
      cp_async_commit();
    }
    const T* as = stage0 + (c % MP_STAGES) * MP_STAGE_ELEMS;
    const T* bs = as + MP_BM * MP_ALD;
#pragma unroll
    for (int k2 = 0; k2 < MP_BK / 2; ++k2) {
      T a[8][2];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
        const T* ap = as + r * MP_ALD + k2 * 2;
        a[i][0] = ap[0]; a[i][1] = ap[1];
      }
      relax_two_steps<T>(acc, a, bs + (k2 * 2) * MP_BLD, bs + (k2 * 2 + 1) * MP_BLD, tx);
    }
  }
  cp_async_wait<0>();
  __syncthreads();

#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    const T* crow = (i < 4 ? cs_lo : cs_hi) + (ty * 4 + (i & 3)) * MP_CLD;
    V4 c0 = *reinterpret_cast<const V4*>(crow + tx * 4);
    V4 c1 = *reinterpret_cast<const V4*>(crow + 64 + tx * 4);
    V4 v0, v1;
    v0.x = Val<T>::vmin(acc[i][0], c0.x); v0.y = Val<T>::vmin(acc[i][1], c0.y);
    v0.z = Val<T>::vmin(acc[i][2], c0.z); v0.w = Val<T>::vmin(acc[i][3], c0.w);
    v1.x = Val<T>::vmin(acc[i][4], c1.x); v1.y = Val<T>::vmin(acc[i][5], c1.y);
    v1.z = Val<T>::vmin(acc[i][6], c1.z); v1.w = Val<T>::vmin(acc[i][7], c1.w);
    *reinterpret_cast<V4*>(Cout + r * ldc_out + tx * 4) = v0;
    *reinterpret_cast<V4*>(Cout + r * ldc_out + 64 + tx * 4) = v1;
  }
}

// ------------------------------------------------ min-plus, mbarrier pipeline --
//
// Same tiling and shared layout as minplus_kernel, but the 3-stage pipeline is
// synchronised with mbarriers instead of a CTA barrier per chunk:
//   full[s]  (256 arrivals): each thread's cp.async.mbarrier.arrive.noinc fires
//            when ITS copies into stage s have landed, so the stage becomes
//            readable without any thread having to reach a sync point;
//   empty[s] (8 arrivals): each warp arrives after its last read of stage s.
// A warp refills the stage of chunk c-1 with its share of chunk c+2 after it
// finished chunk c and the stage's empty barrier shows every warp is past c-1,
// so warps may drift by about a chunk without stalling each other. The C tile
// is fetched into the two stages that are free during the last chunk after one
// CTA barrier (the only one per tile besides the epilogue's).

__device__ __forceinline__ unsigned smem_addr(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(unsigned bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mb_arrive(unsigned bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mb_cp_arrive(unsigned bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mb_wait(unsigned bar, unsigned parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "MBW_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra MBW_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}

template <typename T>
__device__ __forceinline__ void tile_of(const MinPlusDesc<T>& d, long long t, int& ti, int& tj) {
  ti = (int)(t / d.tiles_j);
  tj = (int)(t - (long long)ti * d.tiles_j);
  if (d.skip_i >= 0 && ti >= d.skip_i) ++ti;
  if (d.skip_i2 >= 0 && ti >= d.skip_i2) ++ti;
  if (d.skip_j >= 0 && tj >= d.skip_j) ++tj;
  if (d.skip_j2 >= 0 && tj >= d.skip_j2) ++tj;
}

template <typename T>
__device__ __forceinline__ void minplus_mbar_tile(const MinPlusDesc<T>& d, int ti, int tj, int K,
                                                  unsigned char* smem_raw, unsigned long long* bars);

template <typename T>
__global__ void __launch_bounds__(MP_NT, 2) minplus_mbar_kernel(const __grid_constant__ MinPlusArgs<T> args) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ __align__(8) unsigned long long bars[2 * MP_STAGES];
  long long t = blockIdx.x;
  const bool second = t >= args.n0;
  const MinPlusDesc<T>& d = second ? args.d1 : args.d0;
  if (second) t -= args.n0;
  int ti, tj;
  tile_of(d, t, ti, tj);
  minplus_mbar_tile<T>(d, ti, tj, args.K, smem_raw, bars);
}

// Many tile families in one launch (the boundary algorithm's products, one
// family per component pair): descs[f] in device memory, prefix[f] = first
// CTA of family f (prefix[nf] = grid), depth per family in desc.K.
template <typename T>
__global__ void __launch_bounds__(MP_NT, 2) minplus_batched_kernel(const MinPlusDesc<T>* __restrict__ descs,
                                                                   const long long* __restrict__ prefix, int nf) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ __align__(8) unsigned long long bars[2 * MP_STAGES];
  __shared__ MinPlusDesc<T> sd;
  __shared__ long long st0;
  if (threadIdx.x == 0) {
    const long long t = blockIdx.x;
    int lo = 0, hi = nf - 1;  // last f with prefix[f] <= t
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (prefix[mid] <= t) lo = mid; else hi = mid - 1;
    }
    sd = descs[lo];
    st0 = prefix[lo];
  }
  __syncthreads();
  const MinPlusDesc<T> d = sd;
  int ti, tj;
  tile_of(d, (long long)blockIdx.x - st0, ti, tj);
  minplus_mbar_tile<T>(d, ti, tj, d.K, smem_raw, bars);
}

template <typename T>
__device__ __forceinline__ void minplus_mbar_tile(const MinPlusDesc<T>& d, int ti, int tj, int K,
                                                  unsigned char* smem_raw, unsigned long long* bars) {
  using V4 = typename Vec4<T>::type;
  T* const stage0 = reinterpret_cast<T*>(smem_raw);
  const unsigned full0 = smem_addr(bars), empty0 = full0 + 8 * MP_STAGES;

  const T* __restrict__ Cin = d.Cin + (long long)ti * MP_BM * d.ldc_in + (long long)tj * MP_BN;
  T* __restrict__ Cout = d.Cout + (long long)ti * MP_BM * d.ldc_out + (long long)tj * MP_BN;
  const T* __restrict__ A = d.A + (long long)ti * MP_BM * d.lda;
  const T* __restrict__ B = d.B + (long long)tj * MP_BN;
  const long long lda = d.lda, ldb = d.ldb, ldc_in = d.ldc_in, ldc_out = d.ldc_out;

  const int tid = threadIdx.x;
  const int lane = tid & 31;
  const int tx = tid & 15, ty = tid >> 4;
  if (tid == 0) {
    for (int s = 0; s < MP_STAGES; ++s) {
      mb_init(full0 + 8 * s, MP_NT);
      mb_init(empty0 + 8 * s, MP_NT / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  const T* const a_src = A + (tid >> 3) * lda + (tid & 7) * 4;
  const T* const b_src = B + (tid >> 5) * ldb + (tid & 31) * 4;
  const int a_dst = (tid >> 3) * MP_ALD + (tid & 7) * 4;
  const int b_dst = MP_BM * MP_ALD + (tid >> 5) * MP_BLD + (tid & 31) * 4;
  auto load_chunk = [&](int stage, int chunk) {
    T* st = stage0 + stage * MP_STAGE_ELEMS;
    const T* ag = a_src + chunk * MP_BK;
    const T* bg = b_src + (long long)chunk * MP_BK * ldb;
#pragma unroll
    for (int q = 0; q < 4; ++q) cp_async16(st + a_dst + q * 32 * MP_ALD, ag + q * 32 * lda);
#pragma unroll
    for (int q = 0; q < 4; ++q) cp_async16(st + b_dst + q * 8 * MP_BLD, bg + q * 8 * ldb);
    mb_cp_arrive(full0 + 8 * stage);
  };

  const int nk = K / MP_BK;
  for (int s = 0; s < MP_STAGES - 1 && s < nk; ++s) load_chunk(s, s);

  T acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = Val<T>::inf();
  T* const cs_lo = stage0 + (nk % MP_STAGES) * MP_STAGE_ELEMS;
  T* const cs_hi = stage0 + ((nk + 1) % MP_STAGES) * MP_STAGE_ELEMS;

  int s = 0, ph = 0;  // stage of chunk c and its use parity
  for (int c = 0; c < nk; ++c) {
    if (c == nk - 1) {
      // every warp is past chunk nk-2: the two other stages are free for C
      __syncthreads();
      const T* cg = Cin + (tid >> 5) * ldc_in + (tid & 31) * 4;
      const int cd = (tid >> 5) * MP_CLD + (tid & 31) * 4;
#pragma unroll
      for (int q = 0; q < 8; ++q) cp_async16(cs_lo + cd + q * 8 * MP_CLD, cg + q * 8 * ldc_in);
#pragma unroll
      for (int q = 0; q < 8; ++q) cp_async16(cs_hi + cd + q * 8 * MP_CLD, cg + (64 + q * 8) * ldc_in);
      cp_async_commit();
    }
    mb_wait(full0 + 8 * s, (unsigned)ph);
    const T* as = stage0 + s * MP_STAGE_ELEMS;
    const T* bs = as + MP_BM * MP_ALD;
#pragma unroll
    for (int k2 = 0; k2 < MP_BK / 2; ++k2) {
      T a[8][2];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
        const T* ap = as + r * MP_ALD + k2 * 2;
        a[i][0] = ap[0]; a[i][1] = ap[1];
      }
      relax_two_steps<T>(acc, a, bs + (k2 * 2) * MP_BLD, bs + (k2 * 2 + 1) * MP_BLD, tx);
    }
    __syncwarp();
    if (lane == 0) mb_arrive(empty0 + 8 * s);
    // refill the stage of chunk c-1 with this thread's share of chunk c+2
    const int cn = c + MP_STAGES - 1;
    if (cn < nk) {
      const int sn = cn % MP_STAGES;  // == (c - 1) % 3
      if (c >= 1) mb_wait(empty0 + 8 * sn, (unsigned)(((c - 1) / MP_STAGES) & 1));
      load_chunk(sn, cn);
    }
    if (++s == MP_STAGES) {
      s = 0;
      ph ^= 1;
    }
  }
  cp_async_wait<0>();
  __syncthreads();

#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    const T* crow = (i < 4 ? cs_lo : cs_hi) + (ty * 4 + (i & 3)) * MP_CLD;
    V4 c0 = *reinterpret_cast<const V4*>(crow + tx * 4);
    V4 c1 = *reinterpret_cast<const V4*>(crow + 64 + tx * 4);
    V4 v0, v1;
    v0.x = Val<T>::vmin(acc[i][0], c0.x); v0.y = Val<T>::vmin(acc[i][1], c0.y);
    v0.z = Val<T>::vmin(acc[i][2], c0.z); v0.w = Val<T>::vmin(acc[i][3], c0.w);
    v1.x = Val<T>::vmin(acc[i][4], c1.x); v1.y = Val<T>::vmin(acc[i][5], c1.y);
    v1.z = Val<T>::vmin(acc[i][6], c1.z); v1.w = Val<T>::vmin(acc[i][7], c1.w);
    *reinterpret_cast<V4*>(Cout + r * ldc_out + tx * 4) = v0;
    *reinterpret_cast<V4*>(Cout + r * ldc_out + 64 + tx * 4) = v1;
  }
}

template <typename T>
static long long desc_tiles(const MinPlusDesc<T>& d) {
  return (long long)d.tiles_i * (long long)d.tiles_j;
}

int g_minplus_variant = 0;

template <typename T>
cudaError_t launch_minplus(const MinPlusDesc<T>* d, int ndesc, int K, cudaStream_t s) {
  if (g_minplus_variant == 2) return launch_minplus_tma<T>(d, ndesc, K, s);
  if (K <= 0 || K % MP_BK) return cudaErrorInvalidValue;
  MinPlusArgs<T> a;
  a.d0 = d[0];
  a.d1 = ndesc > 1 ? d[1] : d[0];
  a.n0 = desc_tiles(d[0]);
  a.K = K;
  long long total = a.n0 + (ndesc > 1 ? desc_tiles(d[1]) : 0);
  if (total <= 0) return cudaSuccess;
  if (ndesc > 1 && a.n0 == 0) { a.d0 = a.d1; a.n0 = total; }
  constexpr int smem = minplus_smem_bytes<T>();
  if (g_minplus_variant == 1)
    minplus_kernel<T><<<(unsigned)total, MP_NT, smem, s>>>(a);
  else
    minplus_mbar_kernel<T><<<(unsigned)total, MP_NT, smem, s>>>(a);
  return cudaGetLastError();
}

// --------------------------------------------------------------- phase 1 --
//
// One CTA of 256 threads closes a 128x128 tile in place with the plain FW
// recurrence (PAPER.md:60 restricted to the tile). Thread (ty, tx) keeps the
// same 8x8 register block as the min-plus kernel: rows {4ty..4ty+3,
// 64+4ty..64+4ty+3} x columns {4tx..4tx+3, 64+4tx..64+4tx+3}. Step kk needs
// column kk and row kk; their owners publish them (two 16-byte stores each)
// to a double-buffered shared copy, then one barrier, then every thread does
// 64 relaxations. In place is exact because row kk and column kk do not change
// in step kk when A[kk][kk] = 0; A[kk][kk] < 0 at the start of step kk is a
// negative cycle (flagged; the result is then unspecified).

template <typename T>
__device__ __forceinline__ void phase1_body(T* tile, long long ld, int* negflag);

template <typename T>
__global__ void __launch_bounds__(256) phase1_kernel(T* tile, long long ld, int* negflag) {
  phase1_body<T>(tile, ld, negflag);
}

// one pivot tile per CTA (the boundary algorithm closes all components' tiles of a round at once)
template <typename T>
__global__ void __launch_bounds__(256) phase1_batched_kernel(T* const* tiles, long long ld, int* negflag) {
  phase1_body<T>(tiles[blockIdx.x], ld, negflag);
}

template <typename T>
__device__ __forceinline__ void phase1_body(T* tile, long long ld, int* negflag) {
  using V4 = typename Vec4<T>::type;
  __shared__ __align__(16) T rowbuf[2][kTile];
  __shared__ __align__(16) T colbuf[2][kTile];
  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
  T acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    V4 v0 = *reinterpret_cast<const V4*>(tile + r * ld + tx * 4);
    V4 v1 = *reinterpret_cast<const V4*>(tile + r * ld + 64 + tx * 4);
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
        const int p = u & 1;  // kk & 1
        const int io = half * 4 + u;  // register row / column of kk for its owners
        if (ty == q) {  // row kk lives in this thread's rows: publish my 8 columns of it
          V4 x0, x1;
          x0.x = acc[io][0]; x0.y = acc[io][1]; x0.z = acc[io][2]; x0.w = acc[io][3];
          x1.x = acc[io][4]; x1.y = acc[io][5]; x1.z = acc[io][6]; x1.w = acc[io][7];
          *reinterpret_cast<V4*>(&rowbuf[p][tx * 4]) = x0;
          *reinterpret_cast<V4*>(&rowbuf[p][64 + tx * 4]) = x1;
        }
        if (tx == q) {  // column kk: publish my 8 rows of it
          V4 y0, y1;
          y0.x = acc[0][io]; y0.y = acc[1][io]; y0.z = acc[2][io]; y0.w = acc[3][io];
          y1.x = acc[4][io]; y1.y = acc[5][io]; y1.z = acc[6][io]; y1.w = acc[7][io];
          *reinterpret_cast<V4*>(&colbuf[p][ty * 4]) = y0;
          *reinterpret_cast<V4*>(&colbuf[p][64 + ty * 4]) = y1;
        }
        __syncthreads();
        if (tid == 0 && rowbuf[p][kk] < T(0)) neg = true;
        const V4 a0 = *reinterpret_cast<const V4*>(&colbuf[p][ty * 4]);
        const V4 a1 = *reinterpret_cast<const V4*>(&colbuf[p][64 + ty * 4]);
        const V4 b0 = *reinterpret_cast<const V4*>(&rowbuf[p][tx * 4]);
        const V4 b1 = *reinterpret_cast<const V4*>(&rowbuf[p][64 + tx * 4]);
        const T a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const T bb[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[i][j] = Val<T>::relax(a[i], bb[j], acc[i][j]);
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
  }
}

template <typename T>
cudaError_t launch_phase1(T* tile, long long ld, int* negflag, cudaStream_t s) {
  phase1_kernel<T><<<1, 256, 0, s>>>(tile, ld, negflag);
  return cudaGetLastError();
}

template <typename T>
cudaError_t launch_phase1_batched(T* const* tiles, int count, long long ld, int* negflag, cudaStream_t s) {
  if (count <= 0) return cudaSuccess;
  phase1_batched_kernel<T><<<count, 256, 0, s>>>(tiles, ld, negflag);
  return cudaGetLastError();
}
template cudaError_t launch_phase1_batched<int>(int* const*, int, long long, int*, cudaStream_t);
template cudaError_t launch_phase1_batched<float>(float* const*, int, long long, int*, cudaStream_t);

// ------------------------------------------------------------------ init --
//
// One CTA per row: fill the row with infinity (16-byte stores, 0 on the
// diagonal), barrier, then scatter-min the row's arcs (duplicate arcs keep
// the minimum; a self-loop gives min(0, w)).

__device__ __forceinline__ void atomic_min_t(int* p, int v) { atomicMin(p, v); }
__device__ __forceinline__ void atomic_min_t(float* p, float v) {
  int* ip = reinterpret_cast<int*>(p);
  int old = *ip;
  while (v < __int_as_float(old)) {
    int prev = atomicCAS(ip, old, __float_as_int(v));
    if (prev == old) break;
    old = prev;
  }
}

template <typename T>
__global__ void __launch_bounds__(256) init_rows_kernel(T* D, long long ld, long long n_pad, long long row_begin,
                                                        long long n, const long long* __restrict__ row_ptr,
                                                        long long row_ptr_base, const int* __restrict__ col,
                                                        const T* __restrict__ w) {
  using V4 = typename Vec4<T>::type;
  const long long lr = blockIdx.x;
  const long long r = row_begin + lr;
  T* row = D + lr * ld;
  const T INF = Val<T>::inf();
  const long long q4 = n_pad >> 2;
  for (long long q = threadIdx.x; q < q4; q += blockDim.x) {
    V4 x;
    x.x = INF; x.y = INF; x.z = INF; x.w = INF;
    const long long c = q * 4;
    if (r >= c && r < c + 4) {
      const int o = (int)(r - c);
      if (o == 0) x.x = T(0); else if (o == 1) x.y = T(0); else if (o == 2) x.z = T(0); else x.w = T(0);
    }
    reinterpret_cast<V4*>(row)[q] = x;
  }
  __syncthreads();
  if (r < n) {
    const long long e0 = row_ptr[lr] - row_ptr_base, e1 = row_ptr[lr + 1] - row_ptr_base;
    for (long long e = e0 + threadIdx.x; e < e1; e += blockDim.x) atomic_min_t(row + col[e], w[e]);
  }
}

template <typename T>
cudaError_t launch_init_rows(T* D, long long ld, long long n_pad, long long row_begin, long long rows, long long n,
                             const long long* row_ptr, long long row_ptr_base, const int* col, const T* w,
                             cudaStream_t s) {
  if (rows <= 0) return cudaSuccess;
  init_rows_kernel<T><<<(unsigned)rows, 256, 0, s>>>(D, ld, n_pad, row_begin, n, row_ptr, row_ptr_base, col, w);
  return cudaGetLastError();
}

// ---------------------------------------------------------- canonicalize --

__global__ void canonicalize_kernel(int* D, long long ld, long long rows, long long cols) {
  const int INF = 0x3FFFFFFF;
  const long long total = rows * cols;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    long long r = i / cols, c = i - r * cols;
    int* p = D + r * ld + c;
    if (*p >= INF / 2) *p = INF;
  }
}

cudaError_t launch_canonicalize_i32(int* D, long long ld, long long rows, long long cols, cudaStream_t s) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  canonicalize_kernel<<<148 * 8, 256, 0, s>>>(D, ld, rows, cols);
  return cudaGetLastError();
}

// R25 (apsp_config.exact_f32): an int32 matrix to fp32 and back, in place, 16 B per thread and
// step (count is a multiple of 4: n_pad is a multiple of 128). APSP_INF_I32 <-> +inf; every
// other value is an integer of magnitude <= 2^24, exact in fp32 both ways.
__global__ void i32_to_f32_kernel(int4* D, long long count4) {
  const int INF = 0x3FFFFFFF;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < count4;
       i += (long long)gridDim.x * blockDim.x) {
    const int4 v = D[i];
    float4 f;
    f.x = v.x == INF ? __int_as_float(0x7f800000) : (float)v.x;
    f.y = v.y == INF ? __int_as_float(0x7f800000) : (float)v.y;
    f.z = v.z == INF ? __int_as_float(0x7f800000) : (float)v.z;
    f.w = v.w == INF ? __int_as_float(0x7f800000) : (float)v.w;
    reinterpret_cast<float4*>(D)[i] = f;
  }
}
__global__ void f32_to_i32_kernel(float4* D, long long count4) {
  const int INF = 0x3FFFFFFF;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < count4;
       i += (long long)gridDim.x * blockDim.x) {
    const float4 f = D[i];
    int4 v;
    v.x = isinf(f.x) ? INF : __float2int_rn(f.x);
    v.y = isinf(f.y) ? INF : __float2int_rn(f.y);
    v.z = isinf(f.z) ? INF : __float2int_rn(f.z);
    v.w = isinf(f.w) ? INF : __float2int_rn(f.w);
    reinterpret_cast<int4*>(D)[i] = v;
  }
}
cudaError_t launch_i32_to_f32(int* D, long long count, cudaStream_t s) {
  if (count <= 0) return cudaSuccess;
  i32_to_f32_kernel<<<148 * 8, 256, 0, s>>>(reinterpret_cast<int4*>(D), count / 4);
  return cudaGetLastError();
}
cudaError_t launch_f32_to_i32(float* D, long long count, cudaStream_t s) {
  if (count <= 0) return cudaSuccess;
  f32_to_i32_kernel<<<148 * 8, 256, 0, s>>>(reinterpret_cast<float4*>(D), count / 4);
  return cudaGetLastError();
}

// ------------------------------------------------------ batched min-plus --

template <typename T>
cudaError_t launch_minplus_batched(const MinPlusDesc<T>* descs, const long long* prefix, int nf, long long total,
                                   cudaStream_t s) {
  if (nf <= 0 || total <= 0) return cudaSuccess;
  minplus_batched_kernel<T><<<(unsigned)total, MP_NT, minplus_smem_bytes<T>(), s>>>(descs, prefix, nf);
  return cudaGetLastError();
}

// --------------------------------------------------------------- helpers --

template <typename T>
__global__ void fill_kernel(T* p, long long count, T v) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < count;
       i += (long long)gridDim.x * blockDim.x)
    p[i] = v;
}

template <typename T>
cudaError_t launch_fill(T* p, long long count, T value, cudaStream_t s) {
  if (count <= 0) return cudaSuccess;
  fill_kernel<T><<<148 * 4, 256, 0, s>>>(p, count, value);
  return cudaGetLastError();
}

template <typename T>
__global__ void min_into_kernel(T* dst, long long ldd, const T* src, long long lds, long long cols) {
  T* d = dst + blockIdx.x * ldd;
  const T* q = src + blockIdx.x * lds;
  for (long long c = threadIdx.x; c < cols; c += blockDim.x) d[c] = Val<T>::vmin(d[c], q[c]);
}

template <typename T>
cudaError_t launch_min_into(T* dst, long long ldd, const T* src, long long lds, long long rows, long long cols,
                            cudaStream_t s) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  min_into_kernel<T><<<(unsigned)rows, 256, 0, s>>>(dst, ldd, src, lds, cols);
  return cudaGetLastError();
}

template <typename T>
__device__ __forceinline__ T canon_inf(T v) { return v; }
template <>
__device__ __forceinline__ int canon_inf<int>(int v) { return v >= 0x3FFFFFFF / 2 ? 0x3FFFFFFF : v; }

template <typename T>
__global__ void gather_kernel(const T* D, long long ld, const int* rowmap, const int* colmap, T* out, long long ldo,
                              long long ncols) {
  const T* src = D + (long long)rowmap[blockIdx.x] * ld;
  T* dst = out + blockIdx.x * ldo;
  for (long long c = threadIdx.x; c < ncols; c += blockDim.x) dst[c] = canon_inf<T>(src[colmap[c]]);
}

template <typename T>
cudaError_t launch_gather(const T* D, long long ld, const int* rowmap, const int* colmap, T* out, long long ldo,
                          long long cnt, long long ncols, cudaStream_t s) {
  if (cnt <= 0 || ncols <= 0) return cudaSuccess;
  gather_kernel<T><<<(unsigned)cnt, 256, 0, s>>>(D, ld, rowmap, colmap, out, ldo, ncols);
  return cudaGetLastError();
}

template cudaError_t launch_minplus_batched<int>(const MinPlusDesc<int>*, const long long*, int, long long,
                                                 cudaStream_t);
template cudaError_t launch_minplus_batched<float>(const MinPlusDesc<float>*, const long long*, int, long long,
                                                   cudaStream_t);
template cudaError_t launch_fill<int>(int*, long long, int, cudaStream_t);
template cudaError_t launch_fill<float>(float*, long long, float, cudaStream_t);
template cudaError_t launch_min_into<int>(int*, long long, const int*, long long, long long, long long, cudaStream_t);
template cudaError_t launch_min_into<float>(float*, long long, const float*, long long, long long, long long,
                                            cudaStream_t);
template cudaError_t launch_gather<int>(const int*, long long, const int*, const int*, int*, long long, long long,
                                        long long, cudaStream_t);
template cudaError_t launch_gather<float>(const float*, long long, const int*, const int*, float*, long long,
                                          long long, long long, cudaStream_t);

// --------------------------------------------------------- instantiations --

cudaError_t configure_kernels() {
  cudaError_t e = cudaFuncSetAttribute(minplus_mbar_kernel<int>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       minplus_smem_bytes<int>());
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(minplus_mbar_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           minplus_smem_bytes<float>());
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(minplus_batched_kernel<int>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           minplus_smem_bytes<int>());
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(minplus_batched_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           minplus_smem_bytes<float>());
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(minplus_kernel<int>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       minplus_smem_bytes<int>());
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(minplus_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           minplus_smem_bytes<float>());
  if (e != cudaSuccess) return e;
  if ((e = configure_kernels16()) != cudaSuccess) return e;
  return configure_tma_kernels();
}

template cudaError_t launch_minplus<int>(const MinPlusDesc<int>*, int, int, cudaStream_t);
template cudaError_t launch_minplus<float>(const MinPlusDesc<float>*, int, int, cudaStream_t);
template cudaError_t launch_phase1<int>(int*, long long, int*, cudaStream_t);
template cudaError_t launch_phase1<float>(float*, long long, int*, cudaStream_t);
template cudaError_t launch_init_rows<int>(int*, long long, long long, long long, long long, long long,
                                           const long long*, long long, const int*, const int*, cudaStream_t);
template cudaError_t launch_init_rows<float>(float*, long long, long long, long long, long long, long long,
                                             const long long*, long long, const int*, const float*, cudaStream_t);

}  // namespace apsp
