// apsp_minplus_tma.cu — the phase-2 / phase-3 min-plus tile kernel, TMA +
// mbarrier pipeline, persistent CTAs (sm_100a).
//
// Computes, for every 128x128 output tile of up to two tile families,
//   Cout(ti,tj) = min(Cin(ti,tj), A(ti, 0:K) (x) B(0:K, tj))
// which is phase 2 (PAPER.md:62 step 2; Alg. 1 l.7/11) and phase 3 (P:62
// step 3; Alg. 1 l.17) of the blocked Floyd–Warshall, and the depth-B
// products of the out-of-core path.
//
// Structure (B200-first; differs from the paper's shared-memory MinPlus):
//  * 2 CTAs/SM, 256 threads each, persistent: CTA c takes tiles c, c+G, ...
//  * the depth is streamed in 32-deep chunks through S=3 shared stages; each
//    chunk = one TMA box of A (128 rows x 32, 128B-swizzled so the 8-byte
//    row reads of a warp hit distinct banks) + one TMA box of B (32 x 128),
//    signalled on a "full" mbarrier with expect_tx;
//  * one elected thread (warp 0, lane 0) is the producer: before reusing a
//    stage it waits on that stage's "empty" mbarrier, which the 8 consumer
//    warps arrive on after their last read — there is no CTA-wide barrier in
//    the main loop, so warps drift freely inside the 3-stage window and the
//    producer prefetches across tile boundaries (no per-tile pipeline ramp);
//  * 8x8 outputs per thread in registers, accumulators start at the
//    min-identity and C is folded in at the end (min is exact), read with
//    LDG after a TMA L2 prefetch issued when the tile starts;
//  * int32: one VIADDMNMX (DPX) per relaxation; fp32: FADD + FMNMX.
#include "apsp_kernels.cuh"

#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdint>
#include <cstring>
#include <type_traits>

namespace apsp {

namespace {

constexpr int TM_NT = 256;
constexpr int TM_S = 3;            // pipeline stages
constexpr int TM_BK = 32;          // depth per chunk
constexpr int TM_A_BYTES = 128 * TM_BK * 4;   // 16 KB
constexpr int TM_B_BYTES = TM_BK * 128 * 4;   // 16 KB
constexpr int TM_STAGE_BYTES = TM_A_BYTES + TM_B_BYTES;
constexpr int TM_SMEM = TM_S * TM_STAGE_BYTES + 1024 /*align*/ + 16 * TM_S /*barriers*/;

template <typename T> struct V;
template <> struct V<int> {
  static __device__ __forceinline__ int ident() { return 0x7FFFFFFF; }
  static __device__ __forceinline__ int relax(int a, int b, int c) { return __viaddmin_s32(a, b, c); }
  static __device__ __forceinline__ int vmin(int a, int b) { return min(a, b); }
  using v4 = int4;
  using v2 = int2;
};
template <> struct V<float> {
  static __device__ __forceinline__ float ident() { return __int_as_float(0x7f800000); }
  static __device__ __forceinline__ float relax(float a, float b, float c) { return fminf(c, __fadd_rn(a, b)); }
  static __device__ __forceinline__ float vmin(float a, float b) { return fminf(a, b); }
  using v4 = float4;
  using v2 = float2;
};

struct TmaFamily {
  CUtensorMap mapA;   // box {32, 128} over A (cols = depth), 128B swizzle
  CUtensorMap mapB;   // box {128, 32} over B
  CUtensorMap mapC;   // box {128, 128} over Cin (L2 prefetch only)
  long long ldc_in, ldc_out;
  const void* Cin;
  void* Cout;
  int tiles_i, tiles_j, skip_i, skip_i2, skip_j, skip_j2;
};

struct TmaArgs {
  TmaFamily f[2];
  long long n0, total;  // tiles in family 0, all tiles
  int nk;               // chunks per tile (K / 32)
};

// ---------------------------------------------------------------- PTX ------

__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(unsigned bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(unsigned bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned bar, unsigned parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(unsigned dst, const CUtensorMap* map, int x, int y, unsigned bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          dst),
      "l"(map), "r"(x), "r"(y), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void tma_prefetch_2d(const CUtensorMap* map, int x, int y) {
  asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global [%0, {%1, %2}];" ::"l"(map), "r"(x), "r"(y) : "memory");
}

__device__ __forceinline__ void tile_coords(const TmaArgs& a, long long t, int& fam, int& ti, int& tj) {
  fam = t >= a.n0 ? 1 : 0;
  if (fam) t -= a.n0;
  const TmaFamily& f = a.f[fam];
  ti = (int)(t / f.tiles_j);
  tj = (int)(t - (long long)ti * f.tiles_j);
  if (f.skip_i >= 0 && ti >= f.skip_i) ++ti;
  if (f.skip_i2 >= 0 && ti >= f.skip_i2) ++ti;
  if (f.skip_j >= 0 && tj >= f.skip_j) ++tj;
  if (f.skip_j2 >= 0 && tj >= f.skip_j2) ++tj;
}

// Producer: issue the TMA loads of this CTA's chunks [st->next, limit) (one
// elected thread). Chunk q goes to stage q % S; before reusing a stage the
// producer waits until all 8 consumer warps released its previous use.
struct ProducerState {
  int next;       // next chunk to issue
  int total;      // chunks of this CTA
  unsigned full0, empty0, stage_base;
};

__device__ __noinline__ void produce(const TmaArgs& args, ProducerState* st, int limit) {
  const int nk = args.nk;
  const long long G = gridDim.x;
  while (st->next < limit && st->next < st->total) {
    const int q = st->next;
    const int s = q % TM_S;
    const int u = q / TM_S;
    if (u > 0) mbar_wait(st->empty0 + 8 * s, (unsigned)((u - 1) & 1));
    const int lt = q / nk;
    const int c = q - lt * nk;
    int fam, ti, tj;
    tile_coords(args, blockIdx.x + lt * G, fam, ti, tj);
    const TmaFamily& f = args.f[fam];
    const unsigned dst = st->stage_base + s * TM_STAGE_BYTES;
    const unsigned bar = st->full0 + 8 * s;
    mbar_expect_tx(bar, TM_STAGE_BYTES);
    tma_load_2d(dst, &f.mapA, c * TM_BK, ti * 128, bar);
    tma_load_2d(dst + TM_A_BYTES, &f.mapB, tj * 128, c * TM_BK, bar);
    if (c == 0) tma_prefetch_2d(&f.mapC, tj * 128, ti * 128);
    st->next = q + 1;
  }
}

template <typename T>
__global__ void __launch_bounds__(TM_NT, 2) minplus_tma_kernel(const __grid_constant__ TmaArgs args) {
  using v4 = typename V<T>::v4;
  using v2 = typename V<T>::v2;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  // 1024-byte aligned stage area (128B swizzle atoms), barriers after it
  unsigned char* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const unsigned stage_base = smem_u32(smem);
  const unsigned full0 = stage_base + TM_S * TM_STAGE_BYTES, empty0 = full0 + 8 * TM_S;

  const int tid = threadIdx.x;
  const int lane = tid & 31;
  const int tx = tid & 15, ty = tid >> 4;
  const int G = gridDim.x;
  const int my_tiles = args.total > (long long)blockIdx.x ? (int)((args.total - 1 - blockIdx.x) / G + 1) : 0;

  __shared__ ProducerState pst;
  if (tid == 0) {
    for (int s = 0; s < TM_S; ++s) {
      mbar_init(full0 + 8 * s, 1);
      mbar_init(empty0 + 8 * s, TM_NT / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    pst.next = 0;
    pst.total = my_tiles * args.nk;
    pst.full0 = full0;
    pst.empty0 = empty0;
    pst.stage_base = stage_base;
    produce(args, &pst, TM_S - 1);
  }
  __syncthreads();

  int s = 0, phase = 0, q = 0;  // consumer: stage, its parity, chunk counter
  for (int lt = 0; lt < my_tiles; ++lt) {
    T acc[8][8];
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[i][j] = V<T>::ident();

    for (int c = 0; c < args.nk; ++c, ++q) {
      if (tid == 0) produce(args, &pst, q + TM_S);
      mbar_wait(full0 + 8 * s, (unsigned)phase);
      const unsigned char* As = smem + s * TM_STAGE_BYTES;
      const T* Bs = reinterpret_cast<const T*>(As + TM_A_BYTES);
#pragma unroll
      for (int k2 = 0; k2 < TM_BK / 2; ++k2) {
        // A row r, depth 2*k2..2*k2+1: 16B chunk k2/2 of the 128B row, swizzled by r%8
        T a[8][2];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
          const int chunk = (k2 >> 1) ^ (r & 7);
          const v2 x = *reinterpret_cast<const v2*>(As + r * 128 + chunk * 16 + (k2 & 1) * 8);
          a[i][0] = x.x;
          a[i][1] = x.y;
        }
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const T* brow = Bs + (k2 * 2 + u) * 128;
          const v4 b0 = *reinterpret_cast<const v4*>(brow + tx * 4);
          const v4 b1 = *reinterpret_cast<const v4*>(brow + 64 + tx * 4);
          const T b[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
          for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int j = 0; j < 8; ++j) acc[i][j] = V<T>::relax(a[i][u], b[j], acc[i][j]);
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(empty0 + 8 * s);
      if (++s == TM_S) {
        s = 0;
        phase ^= 1;
      }
    }

    // epilogue: Cout = min(Cin, acc)
    int fam, ti, tj;
    tile_coords(args, blockIdx.x + (long long)lt * G, fam, ti, tj);
    const TmaFamily& f = args.f[fam];
    const T* Cin = static_cast<const T*>(f.Cin) + (long long)(ti * 128 + ty * 4) * f.ldc_in + tj * 128 + tx * 4;
    T* Cout = static_cast<T*>(f.Cout) + (long long)(ti * 128 + ty * 4) * f.ldc_out + tj * 128 + tx * 4;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const long long ri = (i < 4) ? i : (64 + i - 4);
      const v4 c0 = *reinterpret_cast<const v4*>(Cin + ri * f.ldc_in);
      const v4 c1 = *reinterpret_cast<const v4*>(Cin + ri * f.ldc_in + 64);
      v4 o0, o1;
      o0.x = V<T>::vmin(acc[i][0], c0.x); o0.y = V<T>::vmin(acc[i][1], c0.y);
      o0.z = V<T>::vmin(acc[i][2], c0.z); o0.w = V<T>::vmin(acc[i][3], c0.w);
      o1.x = V<T>::vmin(acc[i][4], c1.x); o1.y = V<T>::vmin(acc[i][5], c1.y);
      o1.z = V<T>::vmin(acc[i][6], c1.z); o1.w = V<T>::vmin(acc[i][7], c1.w);
      *reinterpret_cast<v4*>(Cout + ri * f.ldc_out) = o0;
      *reinterpret_cast<v4*>(Cout + ri * f.ldc_out + 64) = o1;
    }
  }
}

// ------------------------------------------------------------- host side ---

PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

template <typename T>
bool encode(CUtensorMap* m, const void* base, unsigned long long cols, unsigned long long rows, long long ld,
            unsigned box_c, unsigned box_r, bool swz) {
  auto fn = get_encode();
  if (!fn) return false;
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {(cuuint64_t)ld * sizeof(T)};
  cuuint32_t box[2] = {box_c, box_r};
  cuuint32_t es[2] = {1, 1};
  const CUtensorMapDataType dt =
      std::is_same<T, int>::value ? CU_TENSOR_MAP_DATA_TYPE_INT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32;
  CUresult r = fn(m, dt, 2,
                  const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  swz ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

template <typename T>
bool make_family(TmaFamily& f, const MinPlusDesc<T>& d, int K) {
  const int ti_span = d.tiles_i + (d.skip_i >= 0) + (d.skip_i2 >= 0);
  const int tj_span = d.tiles_j + (d.skip_j >= 0) + (d.skip_j2 >= 0);
  const unsigned long long rows = (unsigned long long)ti_span * 128, cols = (unsigned long long)tj_span * 128;
  if (!encode<T>(&f.mapA, d.A, (unsigned long long)K, rows, d.lda, TM_BK, 128, true)) return false;
  if (!encode<T>(&f.mapB, d.B, cols, (unsigned long long)K, d.ldb, 128, TM_BK, false)) return false;
  if (!encode<T>(&f.mapC, d.Cin, cols, rows, d.ldc_in, 128, 128, false)) return false;
  f.ldc_in = d.ldc_in;
  f.ldc_out = d.ldc_out;
  f.Cin = d.Cin;
  f.Cout = d.Cout;
  f.tiles_i = d.tiles_i;
  f.tiles_j = d.tiles_j;
  f.skip_i = d.skip_i;
  f.skip_i2 = d.skip_i2;
  f.skip_j = d.skip_j;
  f.skip_j2 = d.skip_j2;
  return true;
}

int g_num_sms = 0;

}  // namespace

cudaError_t configure_tma_kernels() {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  if ((e = cudaFuncSetAttribute(minplus_tma_kernel<int>, cudaFuncAttributeMaxDynamicSharedMemorySize, TM_SMEM)))
    return e;
  if ((e = cudaFuncSetAttribute(minplus_tma_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, TM_SMEM)))
    return e;
  if (!get_encode()) return cudaErrorNotSupported;
  return cudaSuccess;
}

template <typename T>
cudaError_t launch_minplus_tma(const MinPlusDesc<T>* d, int ndesc, int K, cudaStream_t s) {
  if (K <= 0 || K % TM_BK) return cudaErrorInvalidValue;
  TmaArgs a;
  memset(&a, 0, sizeof(a));
  const long long t0 = (long long)d[0].tiles_i * d[0].tiles_j;
  const long long t1 = ndesc > 1 ? (long long)d[1].tiles_i * d[1].tiles_j : 0;
  if (t0 + t1 <= 0) return cudaSuccess;
  int k = 0;
  if (t0 > 0) {
    if (!make_family<T>(a.f[k++], d[0], K)) return cudaErrorInvalidValue;
  }
  if (t1 > 0) {
    if (!make_family<T>(a.f[k++], d[1], K)) return cudaErrorInvalidValue;
  }
  a.n0 = t0 > 0 ? t0 : t1;
  a.total = t0 + t1;
  a.nk = K / TM_BK;
  const int sms = g_num_sms > 0 ? g_num_sms : 148;
  const long long grid = a.total < 2LL * sms ? a.total : 2LL * sms;
  minplus_tma_kernel<T><<<(unsigned)grid, TM_NT, TM_SMEM, s>>>(a);
  return cudaGetLastError();
}

template cudaError_t launch_minplus_tma<int>(const MinPlusDesc<int>*, int, int, cudaStream_t);
template cudaError_t launch_minplus_tma<float>(const MinPlusDesc<float>*, int, int, cudaStream_t);

}  // namespace apsp
