// XSBench-shaped macroscopic cross-section lookup: the loop BODY (user code), shared
// verbatim by the runtime-driven kernel and its bare CUDA twin so the comparison measures
// only the runtime ("XSBench ... extracts one of the main kernels in OpenMC";
// SURVEY App. A.0/A.1 for the definition).  Exact arithmetic: integer LCG, IEEE division,
// explicit fma, so results are bit-identical to the CPU oracle.
#pragma once
#include <cstdint>

namespace omprt_kernels {

// Tables passed BY VALUE as a kernel parameter (by-reference structs cost a load
// and registers).  Same layout as omprt_xs_tables.
struct XSTables {
  const double* __restrict__ nuclide_grid;  // [n_iso*n_gp][6]
  const double* __restrict__ unionized;     // [n_union]
  const int32_t* __restrict__ index_grid;   // [n_union][n_iso]
  const int32_t* __restrict__ num_nucs;     // [12]
  const int32_t* __restrict__ mats;         // [12][max_num_nucs]
  const double* __restrict__ concs;         // [12][max_num_nucs]
  int32_t n_isotopes, n_gridpoints, max_num_nucs, pad;
  int64_t n_union;
};

// ---- the proxy apps' LCG (m = 2^63, a = 2806196910506780709, c = 1) ----------------------
constexpr uint64_t kLcgA = 2806196910506780709ull;
constexpr uint64_t kLcgMask = (1ull << 63) - 1;

// (A_k, C_k): the affine map of 2^k LCG steps, s -> A_k s + C_k (mod 2^64; reduced mod 2^63
// at the end, exact because 2^63 | 2^64).  Built at compile time.
struct LcgJumps {
  uint64_t a[64], c[64];
};
__host__ __device__ constexpr LcgJumps make_lcg_jumps() {
  LcgJumps j{};
  uint64_t a = kLcgA, c = 1;
  for (int k = 0; k < 64; ++k) {
    j.a[k] = a;
    j.c[k] = c;
    c = c * (a + 1);
    a = a * a;
  }
  return j;
}
__constant__ LcgJumps kLcgJumpTable = make_lcg_jumps();

// fast_forward_LCG(seed, n): compose the jumps of n's set bits (square-and-multiply).
__device__ __forceinline__ uint64_t lcg_fast_forward(uint64_t seed, uint64_t n) {
  uint64_t a_new = 1, c_new = 0;
  for (int k = 0; n != 0; ++k, n >>= 1) {
    if (n & 1) {
      const uint64_t ak = kLcgJumpTable.a[k];
      a_new *= ak;
      c_new = c_new * ak + kLcgJumpTable.c[k];
    }
  }
  return (a_new * seed + c_new) & kLcgMask;
}

__device__ __forceinline__ double lcg_double(uint64_t& seed) {
  seed = (kLcgA * seed + 1ull) & kLcgMask;
  return __ull2double_rn(seed) * 0x1p-63;  // (double)seed / 2^63, exact scaling
}

// pick_mat: roll against running_i = dist[i] + dist[i-1] + ... + dist[1] (summed in that
// order, as XSBench does); folded at compile time with IEEE round-to-nearest adds.
struct MatRunning {
  double r[12];
};
__host__ __device__ constexpr MatRunning make_mat_running() {
  const double dist[12] = {0.140, 0.052, 0.275, 0.134, 0.154, 0.064,
                           0.066, 0.055, 0.008, 0.015, 0.025, 0.013};
  MatRunning m{};
  for (int i = 0; i < 12; ++i) {
    double running = 0;
    for (int j = i; j > 0; j--) running += dist[j];
    m.r[i] = running;
  }
  return m;
}

__device__ __forceinline__ int pick_mat(uint64_t& seed) {
  constexpr MatRunning run = make_mat_running();
  const double roll = lcg_double(seed);
#pragma unroll
  for (int i = 0; i < 12; ++i)
    if (roll < run.r[i]) return i;
  return 0;
}

// Binary search of the unionized grid: clamp(upper_bound(E) - 1, 0, len - 2).
__device__ __forceinline__ int32_t grid_search(const double* __restrict__ A, int32_t len,
                                               double quarry) {
  int32_t lo = 0, hi = len - 1;
  while (hi - lo > 1) {
    const int32_t mid = lo + ((hi - lo) >> 1);
    if (__ldg(A + mid) > quarry) hi = mid;
    else lo = mid;
  }
  return lo;
}

// One lookup: returns verification = 1 + argmax of the 5 macroscopic cross sections;
// macro_out (nullable) receives them.
template <bool kMacro = false>
__device__ __forceinline__ uint64_t xs_lookup_one(const XSTables& t, uint64_t seed0,
                                                  int64_t i, double* macro_out = nullptr) {
  uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)i);
  const double E = lcg_double(seed);
  const int mat = pick_mat(seed);
  const int32_t idx = grid_search(t.unionized, (int32_t)t.n_union, E);
  const int nn = __ldg(t.num_nucs + mat);
  const int32_t* __restrict__ mrow = t.mats + mat * t.max_num_nucs;
  const double* __restrict__ crow = t.concs + mat * t.max_num_nucs;
  const int32_t* __restrict__ irow = t.index_grid + (int64_t)idx * t.n_isotopes;
  const double2* __restrict__ grid = reinterpret_cast<const double2*>(t.nuclide_grid);
  double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
#pragma unroll 4
  for (int j = 0; j < nn; ++j) {
    const int32_t p = __ldg(mrow + j);
    const double conc = __ldg(crow + j);
    int32_t k = __ldg(irow + p);
    if (k == t.n_gridpoints - 1) --k;
    // gridpoints k and k+1 of nuclide p: 2 x 48 B = 6 x 16 B (16 B aligned)
    const double2* g = grid + ((int64_t)p * t.n_gridpoints + k) * 3;
    const double2 l0 = __ldg(g + 0), l1 = __ldg(g + 1), l2 = __ldg(g + 2);
    const double2 h0 = __ldg(g + 3), h1 = __ldg(g + 4), h2 = __ldg(g + 5);
    const double f = (h0.x - E) / (h0.x - l0.x);
    m0 = fma(fma(-f, h0.y - l0.y, h0.y), conc, m0);  // total
    m1 = fma(fma(-f, h1.x - l1.x, h1.x), conc, m1);  // elastic
    m2 = fma(fma(-f, h1.y - l1.y, h1.y), conc, m2);  // absorption
    m3 = fma(fma(-f, h2.x - l2.x, h2.x), conc, m3);  // fission
    m4 = fma(fma(-f, h2.y - l2.y, h2.y), conc, m4);  // nu-fission
  }
  if constexpr (kMacro) {
    macro_out[0] = m0;
    macro_out[1] = m1;
    macro_out[2] = m2;
    macro_out[3] = m3;
    macro_out[4] = m4;
  }
  // 1 + argmax, strict '>' from max = -1 (the first maximum wins)
  double mx = -1.0;
  uint64_t v = 1;
  if (m0 > mx) { mx = m0; v = 1; }
  if (m1 > mx) { mx = m1; v = 2; }
  if (m2 > mx) { mx = m2; v = 3; }
  if (m3 > mx) { mx = m3; v = 4; }
  if (m4 > mx) { mx = m4; v = 5; }
  return v;
}

}  // namespace omprt_kernels
