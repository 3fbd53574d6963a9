// apsp_select.cu — the paper's method selection (§IV): the density
// filter (§IV-C) and, among the methods it keeps, the cost models of §IV-B,
// calibrated on THIS device:
//   blocked FW   T_comp = T0 * (n / n0)^3 for a random graph of n0 vertices timed here
//                (P:247-250); out of core T_tr = n_d * W * (3b^2 + n^2) / TH
//                with b = the band height and TH the measured pinned-copy rate
//   Johnson      run k = 5 randomly chosen batches, T_comp = (n_b / k) * T (P:236-239,
//                footnote P:263); out of core T_tr = W * n^2 / TH
//   boundary     N_op = n^3/k^2 + (k B)^3 + n k B^2 + n^2 B with B the average boundary
//                nodes per component, T_comp = N_op * c_unit, c_unit = the
//                per-relaxation cost T0 / n0^3 of the same min-plus kernels (the paper
//                fits c_unit per NB range on training graphs; reading R20)
// Transfers overlap compute in this build (side streams), so an out-of-core estimate
// is max(T_comp, T_tr) (reading R20).
#include "apsp_internal.h"

#include <algorithm>
#include <chrono>
#include <cmath>
#include <vector>

namespace apsp {

// T0 / n0^3 of the in-core blocked FW on a seeded Erdos-Renyi graph (degree 8,
// int32 weights 1..100); the second of two runs is timed.
apsp_status fw_seconds_per_relax(const apsp_config& cfg, long long n0, double* out, std::string* err) {
  std::vector<int64_t> rp(n0 + 1);
  std::vector<int32_t> col, w;
  const long long deg = 8;
  col.reserve(n0 * deg);
  w.reserve(n0 * deg);
  unsigned long long x = 0x9E3779B97F4A7C15ull;
  for (long long u = 0; u < n0; ++u) {
    rp[u] = (int64_t)col.size();
    for (long long e = 0; e < deg; ++e) {
      x = x * 6364136223846793005ull + 1442695040888963407ull;
      col.push_back((int32_t)((x >> 33) % (unsigned long long)n0));
      w.push_back((int32_t)(1 + ((x >> 13) % 100)));
    }
  }
  rp[n0] = (int64_t)col.size();
  apsp_config c = cfg;
  c.world_size = 1;
  c.rank = 0;
  c.nccl_unique_id = nullptr;
  c.virtual_ranks = 0;
  c.force_out_of_core = 0;
  c.device_budget_bytes = 0;
  c.packed16 = 0;
  c.timing = 0;
  c.dist_device = nullptr;  // the calibration graph gets its own matrix
  c.dist_device_bytes = 0;
  apsp_handle* h = nullptr;
  apsp_status st = apsp_init_from_csr(&h, n0, rp.data(), col.data(), w.data(), APSP_I32, &c);
  if (st) {
    *err = apsp_last_error(nullptr);
    return st;
  }
  double best = 0;
  for (int r = 0; r < 2 && !st; ++r) {
    if (r) st = apsp_reinit(h);
    const auto t0 = std::chrono::steady_clock::now();
    if (!st) st = apsp_fw_blocked(h);
    best = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  }
  if (st) *err = apsp_last_error(h);
  apsp_destroy(h);
  *out = best / ((double)n0 * n0 * n0);
  return st;
}

// pinned host <- device copy rate (bytes/s), 256 MB
apsp_status hostlink_rate(int device, double* out, std::string* err) {
  const size_t bytes = 256ull << 20;
  void* d = nullptr;
  void* hp = nullptr;
  cudaSetDevice(device);
  cudaError_t e = cudaMalloc(&d, bytes);
  if (e == cudaSuccess) e = cudaHostAlloc(&hp, bytes, cudaHostAllocDefault);
  double best = 0;
  for (int r = 0; r < 2 && e == cudaSuccess; ++r) {
    const auto t0 = std::chrono::steady_clock::now();
    e = cudaMemcpy(hp, d, bytes, cudaMemcpyDeviceToHost);
    const double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    best = std::max(best, bytes / s);
  }
  if (d) cudaFree(d);
  if (hp) cudaFreeHost(hp);
  if (e != cudaSuccess) {
    *err = cudaGetErrorString(e);
    return APSP_ECUDA;
  }
  *out = best;
  return APSP_OK;
}

// Johnson's T_comp by batch sampling on a handle without a result matrix
apsp_status johnson_seconds(const apsp_config& cfg, long long n, const int64_t* row_ptr, const int32_t* col,
                            const void* w, apsp_dtype dtype, bool has_neg, int k, double* out, std::string* err) {
  Handle* h = new Handle();
  h->n = n;
  h->dtype = dtype;
  h->has_neg = has_neg;
  h->elem = 4;
  h->mode = APSP_MODE_JOHNSON;
  apsp_config c = cfg;
  c.stream = nullptr;
  apsp_status st = setup_device(h, c);
  if (!st) st = jn_setup(h, c, row_ptr, col, w, 0.0, 0, true);
  if (!st) st = jn_sample_seconds(h, k, 12345, out);
  if (st) *err = h->err;
  delete_handle(h);
  return st;
}

}  // namespace apsp
