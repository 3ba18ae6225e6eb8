// XSBench-shaped macroscopic cross-section lookup: the loop BODY (user code), shared
// verbatim by the runtime-driven kernel and its bare CUDA twin so the comparison measures
// only the runtime ("XSBench ... extracts one of the main kernels in OpenMC";
// SURVEY App. A.0/A.1 for the definition).  Exact arithmetic: integer LCG, IEEE division,
// explicit fma, so results are bit-identical to the CPU oracle.
#pragma once
#include <cstdint>

#include "vec.cuh"

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
  // optional B200 layouts of the same data (omprt_xs_build_accel), all NULL or all set
  const int32_t* __restrict__ bins;         // [2^log2_bins + 1] search brackets per energy bin
  const uint16_t* __restrict__ index_grid16;  // [n_union][n_iso] (n_gp <= 65536)
  const double* __restrict__ brackets;      // [n_iso][n_gp-1][12] (E,t,e,a,f,n) x (k, k+1)
  int32_t log2_bins, pad2;
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

// The affine map (a, c) of n LCG steps: compose the jumps of n's set bits
// (square-and-multiply).
struct LcgMap {
  uint64_t a, c;
};
__device__ __forceinline__ LcgMap lcg_jump(uint64_t n) {
  uint64_t a_new = 1, c_new = 0;
  for (int k = 0; n != 0; ++k, n >>= 1) {
    if (n & 1) {
      const uint64_t ak = kLcgJumpTable.a[k];
      a_new *= ak;
      c_new = c_new * ak + kLcgJumpTable.c[k];
    }
  }
  return {a_new, c_new};
}
__device__ __forceinline__ uint64_t lcg_apply(LcgMap m, uint64_t seed) {
  return (m.a * seed + m.c) & kLcgMask;
}
// The same maps for n = m * 256^b, m in [0, 256), b in [0, 8) (32 KB, compile time): a
// fast-forward composes one per BYTE of n -- 4 for a 26-bit lookup index -- instead of one
// per set bit through a ~24-trip loop.  The maps of one LCG commute, so any composition order
// gives the same (a, c).  (Mattered where a lane starts a lookup alone: RSBench's dynamic
// schedule ran that loop at 1.6 active lanes, 4.4 % of its warp instructions.)
struct LcgByteJumps {
  uint64_t a[8][256], c[8][256];
};
__host__ __device__ constexpr LcgByteJumps make_lcg_byte_jumps() {
  LcgByteJumps t{};
  const LcgJumps j = make_lcg_jumps();
  for (int b = 0; b < 8; ++b)
    for (int m = 0; m < 256; ++m) {
      uint64_t a = 1, c = 0;
      for (int k = 0; k < 8; ++k)
        if ((m >> k) & 1) {
          a *= j.a[8 * b + k];
          c = c * j.a[8 * b + k] + j.c[8 * b + k];
        }
      t.a[b][m] = a;
      t.c[b][m] = c;
    }
  return t;
}
__device__ const LcgByteJumps kLcgByteJumps = make_lcg_byte_jumps();
__device__ __forceinline__ LcgMap lcg_jump_bytes(uint64_t n) {
  uint64_t a_new = 1, c_new = 0;
  for (int b = 0; n != 0; ++b, n >>= 8) {
    const unsigned m = (unsigned)(n & 255u);
    if (m) {
      const uint64_t ak = __ldg(&kLcgByteJumps.a[b][m]);
      a_new *= ak;
      c_new = c_new * ak + __ldg(&kLcgByteJumps.c[b][m]);
    }
  }
  return {a_new, c_new};
}
// fast_forward_LCG(seed, n)
__device__ __forceinline__ uint64_t lcg_fast_forward(uint64_t seed, uint64_t n) {
  return lcg_apply(lcg_jump_bytes(n), seed);
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

// Exact search of the unionized grid accelerated by energy bins: bins[b] = grid_search(b/H)
// is monotone in b, so the answer for E in [b/H, (b+1)/H) lies in [bins[b], bins[b+1]] and
// the same bisection over that bracket (~4 probes instead of ~20) returns the same index.
__device__ __forceinline__ int32_t binned_grid_search(const XSTables& t, double E) {
  const int64_t H = 1ll << t.log2_bins;
  int64_t b = (int64_t)(E * (double)H);  // exact scaling by a power of two
  if (b > H - 1) b = H - 1;
  int32_t lo = __ldg(t.bins + b), hi = __ldg(t.bins + b + 1) + 1;
  if (hi > (int32_t)t.n_union - 1) hi = (int32_t)t.n_union - 1;
  while (hi - lo > 1) {
    const int32_t mid = lo + ((hi - lo) >> 1);
    if (__ldg(t.unionized + mid) > E) hi = mid;
    else lo = mid;
  }
  return lo;
}

// One lookup: returns verification = 1 + argmax of the 5 macroscopic cross sections.
// Accel = false reads the tables exactly as specified (binary search of the unionized grid,
// int32 index grid, 48 B gridpoint records: 6 x 16 B loads per nuclide).  Accel = true reads
// the same values from the B200 layouts (binned search, 16-bit index grid, 96 B bracket
// records loaded by 3 x 256-bit loads) -- identical results, fewer L1 wavefronts.
// Accumulate one nuclide's bracket into the 5 macroscopic cross sections (A.1 "Per nuclide").
__device__ __forceinline__ void xs_accumulate(double E, double conc, double le, double he,
                                              double lt, double ht, double lel, double hel,
                                              double la, double ha, double lf, double hf,
                                              double ln, double hn, double& m0, double& m1,
                                              double& m2, double& m3, double& m4) {
  const double f = (he - E) / (he - le);
  m0 = fma(fma(-f, ht - lt, ht), conc, m0);      // total
  m1 = fma(fma(-f, hel - lel, hel), conc, m1);   // elastic
  m2 = fma(fma(-f, ha - la, ha), conc, m2);      // absorption
  m3 = fma(fma(-f, hf - lf, hf), conc, m3);      // fission
  m4 = fma(fma(-f, hn - ln, hn), conc, m4);      // nu-fission
}

// Test build (Macro): the 5 macroscopic cross sections of a lookup, [total, elastic,
// absorption, fission, nu-fission] -- the values the argmax is taken over, for bitwise parity
// with the oracle.
__device__ __forceinline__ void xs_store_macro(double* __restrict__ mo, double m0, double m1,
                                               double m2, double m3, double m4) {
  mo[0] = m0;
  mo[1] = m1;
  mo[2] = m2;
  mo[3] = m3;
  mo[4] = m4;
}

__device__ __forceinline__ uint64_t xs_argmax5(double m0, double m1, double m2, double m3,
                                               double m4) {
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

// The lookup on the B200 layouts with a software-pipelined nuclide loop: the index entries
// of the next pair of nuclides are requested before the current pair's brackets, so the
// index -> bracket dependency of one pair overlaps the other (measured: x04 in profiles/).
// Same arithmetic in the same order as the plain path.
template <bool Macro = false>
__device__ __forceinline__ uint64_t xs_lookup_accel(const XSTables& t, uint64_t seed0,
                                                    int64_t i, double* __restrict__ mo = nullptr) {
  constexpr int P = 2;
  uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)i);
  const double E = lcg_double(seed);
  const int mat = pick_mat(seed);
  const int32_t idx = binned_grid_search(t, E);
  const int nn = __ldg(t.num_nucs + mat);
  const int32_t* __restrict__ mrow = t.mats + mat * t.max_num_nucs;
  const double* __restrict__ crow = t.concs + mat * t.max_num_nucs;
  const uint16_t* __restrict__ irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
  double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
  int32_t pc[P], kc[P];
#pragma unroll
  for (int u = 0; u < P; ++u) {
    pc[u] = u < nn ? __ldg(mrow + u) : 0;
    kc[u] = u < nn ? (int32_t)__ldg(irow + pc[u]) : 0;
  }
  for (int j = 0; j < nn; j += P) {
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {  // next stage's index entries
      const int jj = j + P + u;
      pn[u] = jj < nn ? __ldg(mrow + jj) : 0;
      kn[u] = jj < nn ? (int32_t)__ldg(irow + pn[u]) : 0;
    }
#pragma unroll
    for (int u = 0; u < P; ++u) {
      if (j + u < nn) {
        int32_t k = kc[u];
        if (k == t.n_gridpoints - 1) --k;
        const double conc = __ldg(crow + j + u);
        // bracket (p, k): E_k E_k1 | t_k t_k1 | e_k e_k1 | a_k a_k1 | f_k f_k1 | n_k n_k1
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
        ld_nc_v4f64(g, le, he, lt, ht);
        ld_nc_v4f64(g + 4, lel, hel, la, ha);
        ld_nc_v4f64(g + 8, lf, hf, ln, hn);
        xs_accumulate(E, conc, le, he, lt, ht, lel, hel, la, ha, lf, hf, ln, hn, m0, m1, m2, m3,
                      m4);
      }
    }
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = pn[u];
      kc[u] = kn[u];
    }
  }
  if constexpr (Macro) xs_store_macro(mo, m0, m1, m2, m3, m4);
  return xs_argmax5(m0, m1, m2, m3, m4);
}

// The lookup as a RESUMABLE body for the runtime's flattened loop
// (omprt::distribute_parallel_for_flat): begin/next sample the lookup and search the grid,
// each step() accumulates P nuclides (the next P index entries prefetched, as
// xs_lookup_accel), end() takes the argmax.  Same values, same order, same fma points as
// xs_lookup_accel, so the verification bits are identical.  A thread's next lookup is
// iv + T*N (Fig. 5): its seed is the current seed advanced by the 2*T*N-step jump, one
// 64-bit multiply-add instead of a fast-forward from the start (exact: the LCG is affine).
// L1 traffic is what bounds this loop (ncu: L1 ~80 % busy), so the bracket records, read
// once, bypass L1 allocation, and with SmemMats the material tables (mats, concs) come
// from a team-shared copy (`mats`/`concs` then point to shared memory).
constexpr int kXSFlatThreads = 256;  // team size of the flattened XS kernels
template <bool Fused, bool SmemMats, bool Macro = false, int P = 2>
struct XSFlatLookup {
  const XSTables& t;
  const uint64_t seed0;
  const int64_t first;
  uint64_t* __restrict__ const ver;
  double* __restrict__ const macro;        // Macro: [count][5] macroscopic xs (test build)
  const int32_t* __restrict__ const mats;  // t.mats, or its team-shared copy
  const double* __restrict__ const concs;  // t.concs, or its team-shared copy
  // Fused: this thread's verification sum lives in a per-thread shared-memory slot
  // (flat_acc_slot), not in a register held across the whole loop (that spilled)
  LcgMap J;
  uint64_t s;
  double E;
  int32_t mat, idx, nn, j;
  double m0, m1, m2, m3, m4;
  int32_t pc[P], kc[P];

  __device__ __forceinline__ XSFlatLookup(const XSTables& tab, uint64_t seed, int64_t first_,
                                          uint64_t* verification, const int32_t* mats_,
                                          const double* concs_, double* macro_ = nullptr)
      : t(tab), seed0(seed), first(first_), ver(verification), macro(macro_), mats(mats_),
        concs(concs_) {}

  __device__ __forceinline__ int32_t mat_at(const int32_t* p) const {
    if constexpr (SmemMats) return *p;
    else return __ldg(p);
  }
  __device__ __forceinline__ double conc_at(const double* p) const {
    if constexpr (SmemMats) return *p;
    else return __ldg(p);
  }

  // this lookup's row of the index grid, and its entry for nuclide q
  __device__ __forceinline__ const uint16_t* index_row() const {
    return t.index_grid16 + (int64_t)idx * t.n_isotopes;
  }
  __device__ __forceinline__ int32_t index_at(const uint16_t* __restrict__ irow,
                                              int32_t q) const {
    return (int32_t)__ldg(irow + q);
  }

  __device__ __forceinline__ void start() {
    uint64_t seed = s;
    E = lcg_double(seed);
    mat = pick_mat(seed);
    idx = binned_grid_search(t, E);
    nn = __ldg(t.num_nucs + mat);
    m0 = m1 = m2 = m3 = m4 = 0.0;
    j = 0;
    const int32_t* __restrict__ mrow = mats + mat * t.max_num_nucs;
    const uint16_t* __restrict__ irow = index_row();
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = u < nn ? mat_at(mrow + u) : 0;
      kc[u] = u < nn ? index_at(irow, pc[u]) : 0;
    }
  }
  template <class Idx>
  __device__ __forceinline__ void begin(Idx iv, Idx stride) {
    J = lcg_jump(2ull * (uint64_t)stride);
    // once per thread here (static schedule): the bit-serial jump, whose constant-bank
    // table costs this 64-register loop no extra registers (the byte table spilled)
    s = lcg_apply(lcg_jump(2ull * (uint64_t)(first + iv)), seed0);
    start();
  }
  template <class Idx>
  __device__ __forceinline__ void next(Idx) {
    s = lcg_apply(J, s);
    start();
  }
  __device__ __forceinline__ bool step() {
    const int32_t* __restrict__ mrow = mats + mat * t.max_num_nucs;
    const double* __restrict__ crow = concs + mat * t.max_num_nucs;
    const uint16_t* __restrict__ irow = index_row();
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {  // next step's index entries
      const int jj = j + P + u;
      pn[u] = jj < nn ? mat_at(mrow + jj) : 0;
      kn[u] = jj < nn ? index_at(irow, pn[u]) : 0;
    }
#pragma unroll
    for (int u = 0; u < P; ++u) {
      if (j + u < nn) {
        int32_t k = kc[u];
        if (k == t.n_gridpoints - 1) --k;
        const double conc = conc_at(crow + j + u);
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
        ld_stream_v4f64(g, le, he, lt, ht);
        ld_stream_v4f64(g + 4, lel, hel, la, ha);
        ld_stream_v4f64(g + 8, lf, hf, ln, hn);
        xs_accumulate(E, conc, le, he, lt, ht, lel, hel, la, ha, lf, hf, ln, hn, m0, m1, m2, m3,
                      m4);
      }
    }
    j += P;
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = pn[u];
      kc[u] = kn[u];
    }
    return j < nn;
  }
  template <class Idx>
  __device__ __forceinline__ void end(Idx iv) {
    const uint64_t v = xs_argmax5(m0, m1, m2, m3, m4);
    if constexpr (Macro) xs_store_macro(macro + (int64_t)iv * 5, m0, m1, m2, m3, m4);
    if constexpr (Fused) *flat_acc_slot() += v;
    else ver[iv] = v;
  }
  // this thread's slot (static shared memory: a constant address, no register)
  // sized for the flattened kernels' 256-thread teams (host-checked): a 1024-slot array
  // took 8 KB of shared memory per team and, through the carve-out, L1 the lookups need
  static __device__ __forceinline__ unsigned long long* flat_acc_slot() {
    __shared__ unsigned long long slots[kXSFlatThreads];
    return slots + threadIdx.x;
  }
};

template <bool Accel, bool Macro = false, int kUnroll = 4>
__device__ __forceinline__ uint64_t xs_lookup_one(const XSTables& t, uint64_t seed0, int64_t i,
                                                  double* __restrict__ mo = nullptr) {
  if constexpr (Accel) return xs_lookup_accel<Macro>(t, seed0, i, mo);
  uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)i);
  const double E = lcg_double(seed);
  const int mat = pick_mat(seed);
  const int32_t idx = Accel ? binned_grid_search(t, E)
                            : grid_search(t.unionized, (int32_t)t.n_union, E);
  const int nn = __ldg(t.num_nucs + mat);
  const int32_t* __restrict__ mrow = t.mats + mat * t.max_num_nucs;
  const double* __restrict__ crow = t.concs + mat * t.max_num_nucs;
  const int64_t row = (int64_t)idx * t.n_isotopes;
  double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
#pragma unroll kUnroll
  for (int j = 0; j < nn; ++j) {
    const int32_t p = __ldg(mrow + j);
    const double conc = __ldg(crow + j);
    int32_t k = Accel ? (int32_t)__ldg(t.index_grid16 + row + p) : __ldg(t.index_grid + row + p);
    if (k == t.n_gridpoints - 1) --k;
    double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
    if constexpr (Accel) {
      // bracket (p, k): E_k E_k1 | t_k t_k1 | e_k e_k1 | a_k a_k1 | f_k f_k1 | n_k n_k1
      const double* g = t.brackets + ((int64_t)p * (t.n_gridpoints - 1) + k) * 12;
      ld_nc_v4f64(g, le, he, lt, ht);
      ld_nc_v4f64(g + 4, lel, hel, la, ha);
      ld_nc_v4f64(g + 8, lf, hf, ln, hn);
    } else {
      // gridpoints k and k+1 of nuclide p: 2 x 48 B = 6 x 16 B (16 B aligned)
      const double2* g = reinterpret_cast<const double2*>(t.nuclide_grid) +
                         ((int64_t)p * t.n_gridpoints + k) * 3;
      const double2 l0 = __ldg(g + 0), l1 = __ldg(g + 1), l2 = __ldg(g + 2);
      const double2 h0 = __ldg(g + 3), h1 = __ldg(g + 4), h2 = __ldg(g + 5);
      le = l0.x; lt = l0.y; lel = l1.x; la = l1.y; lf = l2.x; ln = l2.y;
      he = h0.x; ht = h0.y; hel = h1.x; ha = h1.y; hf = h2.x; hn = h2.y;
    }
    const double f = (he - E) / (he - le);
    m0 = fma(fma(-f, ht - lt, ht), conc, m0);      // total
    m1 = fma(fma(-f, hel - lel, hel), conc, m1);   // elastic
    m2 = fma(fma(-f, ha - la, ha), conc, m2);      // absorption
    m3 = fma(fma(-f, hf - lf, hf), conc, m3);      // fission
    m4 = fma(fma(-f, hn - ln, hn), conc, m4);      // nu-fission
  }
  if constexpr (Macro) xs_store_macro(mo, m0, m1, m2, m3, m4);
  return xs_argmax5(m0, m1, m2, m3, m4);
}

// ---- builders of the accelerated layouts (table preparation, not per lookup) -------------
__global__ void xs_build_bins(const double* __restrict__ U, int32_t len, int32_t log2_bins,
                              int32_t* __restrict__ bins) {
  const int64_t H = 1ll << log2_bins;
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b <= H;
       b += (int64_t)gridDim.x * blockDim.x)
    bins[b] = grid_search(U, len, (double)b / (double)H);
}
__global__ void xs_build_index16(const int32_t* __restrict__ a, uint16_t* __restrict__ b,
                                 int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    b[i] = (uint16_t)a[i];
}
__global__ void xs_build_brackets(const double* __restrict__ g, double* __restrict__ o,
                                  int32_t n_iso, int32_t n_gp) {
  // one bracket record per thread: gridpoints k and k+1 of nuclide p (96 contiguous bytes,
  // 6 x 16 B loads) interleaved into (E,t,e,a,f,n) x (k, k+1) and written as 3 x 32 B
  // stores: o[b*12 + 2c + h] = g[(p*n_gp + k + h)*6 + c]
  const int64_t nb = (int64_t)n_iso * (n_gp - 1);
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nb;
       b += (int64_t)gridDim.x * blockDim.x) {
    const int64_t p = b / (n_gp - 1), k = b - p * (n_gp - 1);
    const double2* src = reinterpret_cast<const double2*>(g + (p * n_gp + k) * 6);
    const double2 l0 = __ldg(src + 0), l1 = __ldg(src + 1), l2 = __ldg(src + 2);
    const double2 h0 = __ldg(src + 3), h1 = __ldg(src + 4), h2 = __ldg(src + 5);
    double* d = o + b * 12;
    st_v4f64(d, l0.x, h0.x, l0.y, h0.y);      // E_k E_k1 t_k t_k1
    st_v4f64(d + 4, l1.x, h1.x, l1.y, h1.y);  // e_k e_k1 a_k a_k1
    st_v4f64(d + 8, l2.x, h2.x, l2.y, h2.y);  // f_k f_k1 n_k n_k1
  }
}

}  // namespace omprt_kernels
