// apsp_kernels16.cu — packed int16 path: two relaxations per DPX instruction.
//
// Same method as apsp_kernels.cu (init, phase 1, min-plus
// phases 2/3), on a distance matrix of int16 where each 32-bit register
// holds two adjacent columns and one VIADDMNMX.S16x2 (__viaddmin_s16x2)
// performs c = min(c, a + b) on both halves. Measured peak 3.70e13 relax/s
// vs 1.85e13 for int32 (MEASURED_DPX.json).
//
// Exactness (reading R16): the 16-bit "infinity" is INF16 = 16383,
// so INF16 + INF16 = 32766 never wraps. With non-negative weights <= 8191, a
// finished matrix whose finite entries are all < T = 8192 is the exact APSP:
// every finite entry is the length of a real walk (sums through INF16 are
// >= INF16 and never win), entries whose true distance is < 16383 are exact,
// and if some reachable pair had a true distance >= T its shortest path would
// pass a vertex v at true distance in [T, T + 8191] — an exact entry >= T.
// apsp_fw_blocked checks the maximum finite entry (verify16) and, if it is
// >= T, recomputes in int32.
#include "apsp_kernels.cuh"

#include <cuda_runtime.h>
#include <cstdint>

namespace apsp {

namespace {

constexpr short INF16 = 0x3FFF;

// ------------------------------------------------------------- min-plus --
// CTA 256 threads, one 128x128 int16 output tile; thread (ty, tx) owns rows
// {4ty..4ty+3, 64+4ty..64+4ty+3} x columns 8tx..8tx+7 (4 packed registers
// per row). Depth in chunks of 32 through 3 stages:
//   As[s][128][32+4] 32-bit words, each the A value duplicated in both halves
//                    (staged through registers: LDG.128 of 8 int16, PRMT-dup,
//                    STS.128 x2 — one chunk ahead of its use)
//   Bs[s][32][128]   int16, cp.async
constexpr int S_BK = 32, S_NT = 256, S_ST = 3;
constexpr int S_ALD = S_BK + 4;
constexpr int S_A_WORDS = 128 * S_ALD;
constexpr int S_B_HALVES = S_BK * 128;
constexpr int S_STAGE_BYTES = S_A_WORDS * 4 + S_B_HALVES * 2;
constexpr int S_SMEM = S_ST * S_STAGE_BYTES;

struct Args16 {
  MinPlusDesc<short> d0, d1;
  long long n0;
  int K;
};

__device__ __forceinline__ void cp_async16b(void* smem, const void* gmem) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem));
}
__device__ __forceinline__ void commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void wait_group() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

__global__ void __launch_bounds__(S_NT, 2) minplus16_kernel(const __grid_constant__ Args16 args) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  long long t = blockIdx.x;
  const bool second = t >= args.n0;
  const MinPlusDesc<short>& d = second ? args.d1 : args.d0;
  if (second) t -= args.n0;
  int ti = (int)(t / d.tiles_j);
  int tj = (int)(t - (long long)ti * d.tiles_j);
  if (d.skip_i >= 0 && ti >= d.skip_i) ++ti;
  if (d.skip_i2 >= 0 && ti >= d.skip_i2) ++ti;
  if (d.skip_j >= 0 && tj >= d.skip_j) ++tj;
  if (d.skip_j2 >= 0 && tj >= d.skip_j2) ++tj;
  const short* __restrict__ Cin = d.Cin + (long long)ti * 128 * d.ldc_in + (long long)tj * 128;
  short* __restrict__ Cout = d.Cout + (long long)ti * 128 * d.ldc_out + (long long)tj * 128;
  const short* __restrict__ A = d.A + (long long)ti * 128 * d.lda;
  const short* __restrict__ B = d.B + (long long)tj * 128;
  const long long lda = d.lda, ldb = d.ldb;

  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
  // A chunk: 128 rows x 32 int16 = 4 x 16B per row; thread loads rows tid/4 and tid/4+64, part tid%4
  const int a_row = tid >> 2, a_part = tid & 3;
  const short* a_src = A + a_row * lda + a_part * 8;
  // B chunk: 32 rows x 256 B = 16 x 16B per row; thread copies rows tid/16 and tid/16+16, part tid%16
  const int b_row = tid >> 4, b_part = tid & 15;
  const short* b_src = B + b_row * ldb + b_part * 8;

  auto stageA = [&](int s) { return reinterpret_cast<unsigned*>(smem_raw + s * S_STAGE_BYTES); };
  auto stageB = [&](int s) {
    return reinterpret_cast<unsigned short*>(smem_raw + s * S_STAGE_BYTES + S_A_WORDS * 4);
  };
  auto load_b = [&](int s, int chunk) {
    unsigned short* bs = stageB(s);
    const short* g = b_src + (long long)chunk * S_BK * ldb;
    cp_async16b(bs + b_row * 128 + b_part * 8, g);
    cp_async16b(bs + (b_row + 16) * 128 + b_part * 8, g + 16 * ldb);
  };
  auto load_a_regs = [&](int chunk, uint4& r0, uint4& r1) {
    const short* g = a_src + chunk * S_BK;
    r0 = *reinterpret_cast<const uint4*>(g);
    r1 = *reinterpret_cast<const uint4*>(g + 64 * lda);
  };
  auto store_a = [&](int s, const uint4& r0, const uint4& r1) {
    unsigned* as = stageA(s);
    const unsigned w0[4] = {r0.x, r0.y, r0.z, r0.w};
    const unsigned w1[4] = {r1.x, r1.y, r1.z, r1.w};
    unsigned d0[8], d1[8];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      d0[2 * q] = __byte_perm(w0[q], 0, 0x1010);
      d0[2 * q + 1] = __byte_perm(w0[q], 0, 0x3232);
      d1[2 * q] = __byte_perm(w1[q], 0, 0x1010);
      d1[2 * q + 1] = __byte_perm(w1[q], 0, 0x3232);
    }
    unsigned* p0 = as + a_row * S_ALD + a_part * 8;
    unsigned* p1 = as + (a_row + 64) * S_ALD + a_part * 8;
    *reinterpret_cast<uint4*>(p0) = make_uint4(d0[0], d0[1], d0[2], d0[3]);
    *reinterpret_cast<uint4*>(p0 + 4) = make_uint4(d0[4], d0[5], d0[6], d0[7]);
    *reinterpret_cast<uint4*>(p1) = make_uint4(d1[0], d1[1], d1[2], d1[3]);
    *reinterpret_cast<uint4*>(p1 + 4) = make_uint4(d1[4], d1[5], d1[6], d1[7]);
  };

  const int nk = args.K / S_BK;
  // prologue: chunks 0 and 1
#pragma unroll
  for (int s = 0; s < S_ST - 1; ++s) {
    if (s < nk) {
      load_b(s, s);
      uint4 r0, r1;
      load_a_regs(s, r0, r1);
      store_a(s, r0, r1);
    }
    commit();
  }

  unsigned acc[8][4];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int p = 0; p < 4; ++p) acc[i][p] = 0x7FFF7FFFu;
  // C (128 rows x 256 B) is fetched during the last chunk into the two stages
  // that are then free: rows 0..63 -> stage nk%3, rows 64..127 -> stage (nk+1)%3
  unsigned short* const c_lo = reinterpret_cast<unsigned short*>(smem_raw + (nk % S_ST) * S_STAGE_BYTES);
  unsigned short* const c_hi = reinterpret_cast<unsigned short*>(smem_raw + ((nk + 1) % S_ST) * S_STAGE_BYTES);

  for (int c = 0; c < nk; ++c) {
    wait_group<S_ST - 2>();
    __syncthreads();
    const int cn = c + S_ST - 1;
    uint4 ra0, ra1;
    if (cn < nk) {
      load_b(cn % S_ST, cn);
      load_a_regs(cn, ra0, ra1);
    }
    if (c == nk - 1) {
      const int cr = tid >> 4, cc = (tid & 15) * 8;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        cp_async16b(c_lo + (cr + 16 * q) * 128 + cc, Cin + (cr + 16 * q) * d.ldc_in + cc);
        cp_async16b(c_hi + (cr + 16 * q) * 128 + cc, Cin + (64 + cr + 16 * q) * d.ldc_in + cc);
      }
    }
    commit();
    const unsigned* as = stageA(c % S_ST);
    const unsigned short* bs = stageB(c % S_ST);
#pragma unroll
    for (int k4 = 0; k4 < S_BK / 4; ++k4) {
      unsigned a[8][4];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
        const uint4 v = *reinterpret_cast<const uint4*>(as + r * S_ALD + k4 * 4);
        a[i][0] = v.x; a[i][1] = v.y; a[i][2] = v.z; a[i][3] = v.w;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint4 bv = *reinterpret_cast<const uint4*>(bs + (k4 * 4 + u) * 128 + tx * 8);
        const unsigned b[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int p = 0; p < 4; ++p) acc[i][p] = __viaddmin_s16x2(a[i][u], b[p], acc[i][p]);
      }
    }
    // stage cn was last read in chunk c-1; every thread passed this chunk's barrier
    if (cn < nk) store_a(cn % S_ST, ra0, ra1);
  }
  wait_group<0>();
  __syncthreads();

#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    const uint4 cv = *reinterpret_cast<const uint4*>((i < 4 ? c_lo : c_hi) + (ty * 4 + (i & 3)) * 128 + tx * 8);
    uint4 o;
    o.x = __vmins2(acc[i][0], cv.x);
    o.y = __vmins2(acc[i][1], cv.y);
    o.z = __vmins2(acc[i][2], cv.z);
    o.w = __vmins2(acc[i][3], cv.w);
    *reinterpret_cast<uint4*>(Cout + r * d.ldc_out + tx * 8) = o;
  }
}

// --------------------------------------------------------------- phase 1 --
// 128x128 int16 tile closed in place, computed in int32 registers with the
// same 8x8 ownership and double-buffered row/column publication as the int32
// phase-1 kernel (one barrier per step).
__global__ void __launch_bounds__(256) phase1_16_kernel(short* tile, long long ld) {
  __shared__ __align__(16) int rowbuf[2][128];
  __shared__ __align__(16) int colbuf[2][128];
  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
  int acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    const short4 v0 = *reinterpret_cast<const short4*>(tile + r * ld + tx * 4);
    const short4 v1 = *reinterpret_cast<const short4*>(tile + r * ld + 64 + tx * 4);
    acc[i][0] = v0.x; acc[i][1] = v0.y; acc[i][2] = v0.z; acc[i][3] = v0.w;
    acc[i][4] = v1.x; acc[i][5] = v1.y; acc[i][6] = v1.z; acc[i][7] = v1.w;
  }
#pragma unroll
  for (int half = 0; half < 2; ++half) {
    for (int q = 0; q < 16; ++q) {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int p = u & 1;
        const int io = half * 4 + u;
        if (ty == q) {
          *reinterpret_cast<int4*>(&rowbuf[p][tx * 4]) = make_int4(acc[io][0], acc[io][1], acc[io][2], acc[io][3]);
          *reinterpret_cast<int4*>(&rowbuf[p][64 + tx * 4]) =
              make_int4(acc[io][4], acc[io][5], acc[io][6], acc[io][7]);
        }
        if (tx == q) {
          *reinterpret_cast<int4*>(&colbuf[p][ty * 4]) = make_int4(acc[0][io], acc[1][io], acc[2][io], acc[3][io]);
          *reinterpret_cast<int4*>(&colbuf[p][64 + ty * 4]) =
              make_int4(acc[4][io], acc[5][io], acc[6][io], acc[7][io]);
        }
        __syncthreads();
        const int4 a0 = *reinterpret_cast<const int4*>(&colbuf[p][ty * 4]);
        const int4 a1 = *reinterpret_cast<const int4*>(&colbuf[p][64 + ty * 4]);
        const int4 b0 = *reinterpret_cast<const int4*>(&rowbuf[p][tx * 4]);
        const int4 b1 = *reinterpret_cast<const int4*>(&rowbuf[p][64 + tx * 4]);
        const int a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const int b[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[i][j] = __viaddmin_s32(a[i], b[j], acc[i][j]);
      }
    }
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = (i < 4) ? (ty * 4 + i) : (64 + ty * 4 + i - 4);
    *reinterpret_cast<short4*>(tile + r * ld + tx * 4) =
        make_short4((short)acc[i][0], (short)acc[i][1], (short)acc[i][2], (short)acc[i][3]);
    *reinterpret_cast<short4*>(tile + r * ld + 64 + tx * 4) =
        make_short4((short)acc[i][4], (short)acc[i][5], (short)acc[i][6], (short)acc[i][7]);
  }
}

// ------------------------------------------------------------------ init --
__device__ __forceinline__ void atomic_min16(short* p, short v) {
  unsigned* w = reinterpret_cast<unsigned*>(reinterpret_cast<uintptr_t>(p) & ~(uintptr_t)3);
  const int sh = (reinterpret_cast<uintptr_t>(p) & 2) ? 16 : 0;
  unsigned old = *w;
  for (;;) {
    const short cur = (short)((old >> sh) & 0xFFFF);
    if (cur <= v) return;
    const unsigned nw = (old & ~(0xFFFFu << sh)) | ((unsigned)(unsigned short)v << sh);
    const unsigned prev = atomicCAS(w, old, nw);
    if (prev == old) return;
    old = prev;
  }
}

__global__ void __launch_bounds__(256) init16_kernel(short* D, long long ld, long long n_pad, long long n,
                                                     const long long* __restrict__ row_ptr, long long base,
                                                     const int* __restrict__ col, const int* __restrict__ w) {
  const long long r = blockIdx.x;
  short* row = D + r * ld;
  const long long q8 = n_pad >> 3;  // 16-byte groups
  for (long long q = threadIdx.x; q < q8; q += blockDim.x) {
    short v[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) v[e] = (q * 8 + e == r) ? (short)0 : INF16;
    *reinterpret_cast<uint4*>(row + q * 8) = *reinterpret_cast<const uint4*>(v);
  }
  __syncthreads();
  if (r < n) {
    const long long e0 = row_ptr[r] - base, e1 = row_ptr[r + 1] - base;
    for (long long e = e0 + threadIdx.x; e < e1; e += blockDim.x) atomic_min16(row + col[e], (short)w[e]);
  }
}

// max finite (< INF16) entry of rows x cols at ld -> atomicMax(*out)
__global__ void max_finite16_kernel(const short* D, long long ld, long long rows, long long cols, int* out) {
  int m = -1;
  const long long c8 = cols >> 3;
  const long long total = rows * c8;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const long long r = i / c8, q = i - r * c8;
    const uint4 v = *reinterpret_cast<const uint4*>(D + r * ld + q * 8);
    const unsigned w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int lo = (short)(w[k] & 0xFFFF), hi = (short)(w[k] >> 16);
      if (lo < INF16) m = max(m, lo);
      if (hi < INF16) m = max(m, hi);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
  if ((threadIdx.x & 31) == 0) atomicMax(out, m);
}

// int16 rows -> int32 rows (INF16 -> APSP_INF_I32); one CTA per row, 8 values per step
__global__ void widen16_kernel(const short* S, long long lds, int* D, long long ldd, long long cols) {
  const short* src = S + blockIdx.x * lds;
  int* dst = D + blockIdx.x * ldd;
  const long long c8 = cols >> 3;
  for (long long q = threadIdx.x; q < c8; q += blockDim.x) {
    const uint4 v = *reinterpret_cast<const uint4*>(src + q * 8);
    const unsigned w[4] = {v.x, v.y, v.z, v.w};
    int o[8];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const short lo = (short)(w[k] & 0xFFFF), hi = (short)(w[k] >> 16);
      o[2 * k] = lo >= INF16 ? 0x3FFFFFFF : (int)lo;
      o[2 * k + 1] = hi >= INF16 ? 0x3FFFFFFF : (int)hi;
    }
    *reinterpret_cast<int4*>(dst + q * 8) = make_int4(o[0], o[1], o[2], o[3]);
    *reinterpret_cast<int4*>(dst + q * 8 + 4) = make_int4(o[4], o[5], o[6], o[7]);
  }
  for (long long c = c8 * 8 + threadIdx.x; c < cols; c += blockDim.x) {
    const short v = src[c];
    dst[c] = v >= INF16 ? 0x3FFFFFFF : (int)v;
  }
}

}  // namespace

template <>
cudaError_t launch_minplus<short>(const MinPlusDesc<short>* d, int ndesc, int K, cudaStream_t s) {
  if (K <= 0 || K % S_BK) return cudaErrorInvalidValue;
  Args16 a;
  a.d0 = d[0];
  a.d1 = ndesc > 1 ? d[1] : d[0];
  a.n0 = (long long)d[0].tiles_i * d[0].tiles_j;
  a.K = K;
  const long long total = a.n0 + (ndesc > 1 ? (long long)d[1].tiles_i * d[1].tiles_j : 0);
  if (total <= 0) return cudaSuccess;
  if (ndesc > 1 && a.n0 == 0) {
    a.d0 = a.d1;
    a.n0 = total;
  }
  minplus16_kernel<<<(unsigned)total, S_NT, S_SMEM, s>>>(a);
  return cudaGetLastError();
}

template <>
cudaError_t launch_phase1<short>(short* tile, long long ld, int* /*negflag: weights >= 0*/, cudaStream_t s) {
  phase1_16_kernel<<<1, 256, 0, s>>>(tile, ld);
  return cudaGetLastError();
}

cudaError_t launch_init16(short* D, long long ld, long long n_pad, long long rows, long long n,
                          const long long* row_ptr, const int* col, const int* w, cudaStream_t s) {
  if (rows <= 0) return cudaSuccess;
  init16_kernel<<<(unsigned)rows, 256, 0, s>>>(D, ld, n_pad, n, row_ptr, 0, col, w);
  return cudaGetLastError();
}

cudaError_t launch_max_finite16(const short* D, long long ld, long long rows, long long cols, int* out,
                                cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(out, 0xFF, sizeof(int), s);  // -1
  if (e != cudaSuccess) return e;
  max_finite16_kernel<<<148 * 8, 256, 0, s>>>(D, ld, rows, cols, out);
  return cudaGetLastError();
}

cudaError_t launch_widen16(const short* S, long long lds, int* D, long long ldd, long long rows, long long cols,
                           cudaStream_t s) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  widen16_kernel<<<(unsigned)rows, 256, 0, s>>>(S, lds, D, ldd, cols);
  return cudaGetLastError();
}

cudaError_t configure_kernels16() {
  return cudaFuncSetAttribute(minplus16_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, S_SMEM);
}

}  // namespace apsp
