// Exploration harness 7 (NOT part of libomprt.so): the Fig. 5 cyclic loop over lookups
// FLATTENED with the per-lookup nuclide loop.  Under the plain nest a warp runs
// max(num_nucs) nuclide steps per round of 32 lookups (34 when any lane drew the fuel,
// ~99 % of warps) while the mean is ~15.5: half the lanes idle.  Flattened, a lane that
// finishes its lookup stores the result and starts its NEXT Fig. 5 iteration (iv += T*N)
// at once, so lanes stay busy; each thread still runs exactly its own iterations, in order.
// Same arithmetic and order per lookup as the product (bit-identical results).
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/xs_body.cuh"
using namespace omprt_kernels;

struct Setup {
  double E;
  const int32_t* mrow;
  const double* crow;
  const uint16_t* irow;
  int nn;
};

__device__ __forceinline__ Setup setup(const XSTables& t, uint64_t seed0, int64_t i) {
  uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)i);
  Setup s;
  s.E = lcg_double(seed);
  const int mat = pick_mat(seed);
  const int32_t idx = binned_grid_search(t, s.E);
  s.nn = __ldg(t.num_nucs + mat);
  s.mrow = t.mats + mat * t.max_num_nucs;
  s.crow = t.concs + mat * t.max_num_nucs;
  s.irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
  return s;
}

__device__ __forceinline__ void nuc(const XSTables& t, const Setup& s, int j, int32_t p,
                                    int32_t k, double& m0, double& m1, double& m2, double& m3,
                                    double& m4) {
  if (k == t.n_gridpoints - 1) --k;
  const double conc = __ldg(s.crow + j);
  const double* g = t.brackets + ((int64_t)p * (t.n_gridpoints - 1) + k) * 12;
  double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
  ld_nc_v4f64(g, le, he, lt, ht);
  ld_nc_v4f64(g + 4, lel, hel, la, ha);
  ld_nc_v4f64(g + 8, lf, hf, ln, hn);
  xs_accumulate(s.E, conc, le, he, lt, ht, lel, hel, la, ha, lf, hf, ln, hn, m0, m1, m2, m3, m4);
}

// P nuclides per step, the next step's index entries prefetched (as the product)
template <int P>
__device__ __forceinline__ void flat_loop(const XSTables& t, uint64_t seed0, int64_t first,
                                          int32_t n, uint64_t* __restrict__ ver) {
  const int32_t total = gridDim.x * blockDim.x;
  int32_t iv = blockIdx.x * blockDim.x + threadIdx.x;
  if (iv >= n) return;
  Setup s = setup(t, seed0, first + iv);
  double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
  int j = 0;
  int32_t pc[P], kc[P];
#pragma unroll
  for (int u = 0; u < P; ++u) {
    pc[u] = u < s.nn ? __ldg(s.mrow + u) : 0;
    kc[u] = u < s.nn ? (int32_t)__ldg(s.irow + pc[u]) : 0;
  }
  while (true) {
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {
      const int jj = j + P + u;
      pn[u] = jj < s.nn ? __ldg(s.mrow + jj) : 0;
      kn[u] = jj < s.nn ? (int32_t)__ldg(s.irow + pn[u]) : 0;
    }
#pragma unroll
    for (int u = 0; u < P; ++u)
      if (j + u < s.nn) nuc(t, s, j + u, pc[u], kc[u], m0, m1, m2, m3, m4);
    j += P;
    if (j >= s.nn) {
      ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
      iv += total;
      if (iv >= n) break;
      s = setup(t, seed0, first + iv);
      m0 = m1 = m2 = m3 = m4 = 0.0;
      j = 0;
#pragma unroll
      for (int u = 0; u < P; ++u) {
        pc[u] = u < s.nn ? __ldg(s.mrow + u) : 0;
        kc[u] = u < s.nn ? (int32_t)__ldg(s.irow + pc[u]) : 0;
      }
    } else {
#pragma unroll
      for (int u = 0; u < P; ++u) {
        pc[u] = pn[u];
        kc[u] = kn[u];
      }
    }
  }
}


// State-machine form: the binned search also advances one probe per step, so a lane that
// starts a lookup does not hold the warp for the whole search.
template <int P>
__device__ __forceinline__ void flat_sm(const XSTables& t, uint64_t seed0, int64_t first,
                                        int32_t n, uint64_t* __restrict__ ver) {
  const int32_t total = gridDim.x * blockDim.x;
  int32_t iv = blockIdx.x * blockDim.x + threadIdx.x;
  if (iv >= n) return;
  const int64_t H = 1ll << t.log2_bins;
  double E;
  int mat, nn = 0, j = 0, lo, hi;
  bool srch;
  const int32_t *mrow = nullptr;
  const double *crow = nullptr;
  const uint16_t* irow = nullptr;
  double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
  int32_t pc[P], kc[P];
  auto start = [&](int32_t i) {
    uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + i));
    E = lcg_double(seed);
    mat = pick_mat(seed);
    int64_t b = (int64_t)(E * (double)H);
    if (b > H - 1) b = H - 1;
    lo = __ldg(t.bins + b);
    hi = __ldg(t.bins + b + 1) + 1;
    if (hi > (int32_t)t.n_union - 1) hi = (int32_t)t.n_union - 1;
    srch = true;
  };
  start(iv);
  while (true) {
    if (srch) {
      if (hi - lo > 1) {
        const int32_t mid = lo + ((hi - lo) >> 1);
        if (__ldg(t.unionized + mid) > E) hi = mid;
        else lo = mid;
      }
      if (hi - lo <= 1) {
        srch = false;
        nn = __ldg(t.num_nucs + mat);
        mrow = t.mats + mat * t.max_num_nucs;
        crow = t.concs + mat * t.max_num_nucs;
        irow = t.index_grid16 + (int64_t)lo * t.n_isotopes;
        j = 0;
        m0 = m1 = m2 = m3 = m4 = 0.0;
#pragma unroll
        for (int u = 0; u < P; ++u) {
          pc[u] = u < nn ? __ldg(mrow + u) : 0;
          kc[u] = u < nn ? (int32_t)__ldg(irow + pc[u]) : 0;
        }
      }
    } else {
      int32_t pn[P], kn[P];
#pragma unroll
      for (int u = 0; u < P; ++u) {
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
          const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
          double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
          ld_nc_v4f64(g, le, he, lt, ht);
          ld_nc_v4f64(g + 4, lel, hel, la, ha);
          ld_nc_v4f64(g + 8, lf, hf, ln, hn);
          xs_accumulate(E, conc, le, he, lt, ht, lel, hel, la, ha, lf, hf, ln, hn, m0, m1, m2,
                        m3, m4);
        }
      }
      j += P;
#pragma unroll
      for (int u = 0; u < P; ++u) {
        pc[u] = pn[u];
        kc[u] = kn[u];
      }
      if (j >= nn) {
        ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
        iv += total;
        if (iv >= n) break;
        start(iv);
      }
    }
  }
}

// Compact loop-carried state: (iv, E, mat, idx, nn, j, m0..m4, the prefetched (p, k) pairs);
// row pointers are recomputed from (mat, idx) where used.
template <int P>
__device__ __forceinline__ void flat_c(const XSTables& t, uint64_t seed0, int64_t first,
                                       int32_t n, uint64_t* __restrict__ ver) {
  const int32_t total = gridDim.x * blockDim.x;
  int32_t iv = blockIdx.x * blockDim.x + threadIdx.x;
  if (iv >= n) return;
  double E;
  int32_t mat, idx, nn, j;
  double m0, m1, m2, m3, m4;
  int32_t pc[P], kc[P];
  auto start = [&]() {
    uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv));
    E = lcg_double(seed);
    mat = pick_mat(seed);
    idx = binned_grid_search(t, E);
    nn = __ldg(t.num_nucs + mat);
    m0 = m1 = m2 = m3 = m4 = 0.0;
    j = 0;
    const int32_t* mrow = t.mats + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = u < nn ? __ldg(mrow + u) : 0;
      kc[u] = u < nn ? (int32_t)__ldg(irow + pc[u]) : 0;
    }
  };
  start();
  while (true) {
    const int32_t* mrow = t.mats + mat * t.max_num_nucs;
    const double* crow = t.concs + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {
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
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
        ld_nc_v4f64(g, le, he, lt, ht);
        ld_nc_v4f64(g + 4, lel, hel, la, ha);
        ld_nc_v4f64(g + 8, lf, hf, ln, hn);
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
    if (j >= nn) {
      ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
      iv += total;
      if (iv >= n) break;
      start();
    }
  }
}

// Lookup-pipelined flattened loop: while lookup iv's nuclides are processed, the NEXT
// iteration (iv + T*N, Fig. 5) is sampled and its binned search advances one probe per step,
// in straight-line code (the probe load overlaps the step's index/bracket loads).  The next
// lookup's seed comes from the current one by the affine jump of 2*T*N LCG steps (exact).
template <int P>
__device__ __forceinline__ void flat_pipe(const XSTables& t, uint64_t seed0, int64_t first,
                                          int32_t n, uint64_t* __restrict__ ver) {
  const int32_t total = gridDim.x * blockDim.x;
  int32_t iv = blockIdx.x * blockDim.x + threadIdx.x;
  if (iv >= n) return;
  const LcgMap J = lcg_jump(2ull * (uint64_t)total);
  const int64_t H = 1ll << t.log2_bins;
  // next lookup's sampling state
  uint64_t sn = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv));
  double En;
  int32_t matn, lo, hi;
  auto sample = [&]() {  // draws E, mat of the lookup whose seed is sn; starts its search
    uint64_t s = sn;
    En = lcg_double(s);
    matn = pick_mat(s);
    int64_t b = (int64_t)(En * (double)H);
    if (b > H - 1) b = H - 1;
    lo = __ldg(t.bins + b);
    hi = __ldg(t.bins + b + 1) + 1;
    if (hi > (int32_t)t.n_union - 1) hi = (int32_t)t.n_union - 1;
  };
  auto finish_search = [&]() {
    while (hi - lo > 1) {
      const int32_t mid = lo + ((hi - lo) >> 1);
      if (__ldg(t.unionized + mid) > En) hi = mid;
      else lo = mid;
    }
  };
  // current lookup
  double E;
  int32_t mat, idx, nn, j;
  double m0, m1, m2, m3, m4;
  int32_t pc[P], kc[P];
  bool has_next;
  auto promote = [&]() {  // next -> current; sample the one after
    finish_search();
    E = En;
    mat = matn;
    idx = lo;
    nn = __ldg(t.num_nucs + mat);
    m0 = m1 = m2 = m3 = m4 = 0.0;
    j = 0;
    const int32_t* mrow = t.mats + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = u < nn ? __ldg(mrow + u) : 0;
      kc[u] = u < nn ? (int32_t)__ldg(irow + pc[u]) : 0;
    }
    has_next = iv + total < n;
    if (has_next) {
      sn = (J.a * sn + J.c) & kLcgMask;
      sample();
    }
  };
  sample();
  promote();
  while (true) {
    // one probe of the next lookup's search (its load overlaps this step's loads)
    const bool probing = has_next && hi - lo > 1;
    const int32_t mid = lo + ((hi - lo) >> 1);
    const double um = probing ? __ldg(t.unionized + mid) : 0.0;
    const int32_t* mrow = t.mats + mat * t.max_num_nucs;
    const double* crow = t.concs + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {
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
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
        ld_nc_v4f64(g, le, he, lt, ht);
        ld_nc_v4f64(g + 4, lel, hel, la, ha);
        ld_nc_v4f64(g + 8, lf, hf, ln, hn);
        xs_accumulate(E, conc, le, he, lt, ht, lel, hel, la, ha, lf, hf, ln, hn, m0, m1, m2, m3,
                      m4);
      }
    }
    if (probing) {
      if (um > En) hi = mid;
      else lo = mid;
    }
    j += P;
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = pn[u];
      kc[u] = kn[u];
    }
    if (j >= nn) {
      ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
      if (!has_next) break;
      iv += total;
      promote();
    }
  }
}

// F1 with the next lookup's seed from the current one by the affine jump of 2*T*N steps
template <int P>
__device__ __forceinline__ void flat_jump(const XSTables& t, uint64_t seed0, int64_t first,
                                          int32_t n, uint64_t* __restrict__ ver) {
  const int32_t total = gridDim.x * blockDim.x;
  int32_t iv = blockIdx.x * blockDim.x + threadIdx.x;
  if (iv >= n) return;
  const LcgMap J = lcg_jump(2ull * (uint64_t)total);
  uint64_t s0 = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv));
  double E;
  int32_t mat, idx, nn, j;
  double m0, m1, m2, m3, m4;
  int32_t pc[P], kc[P];
  auto start = [&]() {
    uint64_t seed = s0;
    E = lcg_double(seed);
    mat = pick_mat(seed);
    idx = binned_grid_search(t, E);
    nn = __ldg(t.num_nucs + mat);
    m0 = m1 = m2 = m3 = m4 = 0.0;
    j = 0;
    const int32_t* mrow = t.mats + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = u < nn ? __ldg(mrow + u) : 0;
      kc[u] = u < nn ? (int32_t)__ldg(irow + pc[u]) : 0;
    }
  };
  start();
  while (true) {
    const int32_t* mrow = t.mats + mat * t.max_num_nucs;
    const double* crow = t.concs + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {
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
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
        ld_nc_v4f64(g, le, he, lt, ht);
        ld_nc_v4f64(g + 4, lel, hel, la, ha);
        ld_nc_v4f64(g + 8, lf, hf, ln, hn);
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
    if (j >= nn) {
      ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
      iv += total;
      if (iv >= n) break;
      s0 = (J.a * s0 + J.c) & kLcgMask;
      start();
    }
  }
}

template <int P, bool Stream, bool SmemMats>
__device__ __forceinline__ void flat_opt(const XSTables& t, uint64_t seed0, int64_t first,
                                          int32_t n, uint64_t* __restrict__ ver) {
  const int32_t total = gridDim.x * blockDim.x;
  int32_t iv = blockIdx.x * blockDim.x + threadIdx.x;
  if (iv >= n) return;
  const LcgMap J = lcg_jump(2ull * (uint64_t)total);
  uint64_t s0 = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv));
  __shared__ int32_t smats[12 * 34];
  __shared__ double sconcs[12 * 34];
  const int32_t* gm = t.mats;
  const double* gc = t.concs;
  if (SmemMats) {
    for (int k = threadIdx.x; k < 12 * t.max_num_nucs; k += blockDim.x) {
      smats[k] = __ldg(t.mats + k);
      sconcs[k] = __ldg(t.concs + k);
    }
    __syncthreads();
    gm = smats;
    gc = sconcs;
  }
  double E;
  int32_t mat, idx, nn, j;
  double m0, m1, m2, m3, m4;
  int32_t pc[P], kc[P];
  auto start = [&]() {
    uint64_t seed = s0;
    E = lcg_double(seed);
    mat = pick_mat(seed);
    idx = binned_grid_search(t, E);
    nn = __ldg(t.num_nucs + mat);
    m0 = m1 = m2 = m3 = m4 = 0.0;
    j = 0;
    const int32_t* mrow = gm + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = u < nn ? (SmemMats ? mrow[u] : __ldg(mrow + u)) : 0;
      kc[u] = u < nn ? (int32_t)__ldg(irow + pc[u]) : 0;
    }
  };
  start();
  while (true) {
    const int32_t* mrow = gm + mat * t.max_num_nucs;
    const double* crow = gc + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {
      const int jj = j + P + u;
      pn[u] = jj < nn ? (SmemMats ? mrow[jj] : __ldg(mrow + jj)) : 0;
      kn[u] = jj < nn ? (int32_t)__ldg(irow + pn[u]) : 0;
    }
#pragma unroll
    for (int u = 0; u < P; ++u) {
      if (j + u < nn) {
        int32_t k = kc[u];
        if (k == t.n_gridpoints - 1) --k;
        const double conc = SmemMats ? crow[j + u] : __ldg(crow + j + u);
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
        if (Stream) {
          ld_stream_v4f64(g, le, he, lt, ht);
          ld_stream_v4f64(g + 4, lel, hel, la, ha);
          ld_stream_v4f64(g + 8, lf, hf, ln, hn);
        } else {
          ld_nc_v4f64(g, le, he, lt, ht);
          ld_nc_v4f64(g + 4, lel, hel, la, ha);
          ld_nc_v4f64(g + 8, lf, hf, ln, hn);
        }
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
    if (j >= nn) {
      ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
      iv += total;
      if (iv >= n) break;
      s0 = (J.a * s0 + J.c) & kLcgMask;
      start();
    }
  }
}


__device__ __forceinline__ int32_t ld_na_s32(const int32_t* p) {
  int32_t v;
  asm("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ double ld_na_f64(const double* p) {
  double v;
  asm("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
  return v;
}
template <bool S>
__device__ __forceinline__ uint16_t ldidx(const uint16_t* p) {
  if (S) {
    uint16_t v;
    asm("ld.global.nc.L1::no_allocate.u16 %0, [%1];" : "=h"(v) : "l"(p));
    return v;
  }
  return __ldg(p);
}
__device__ __forceinline__ int32_t search_stream(const XSTables& t, double E) {
  const int64_t H = 1ll << t.log2_bins;
  int64_t b = (int64_t)(E * (double)H);
  if (b > H - 1) b = H - 1;
  int32_t lo = ld_na_s32(t.bins + b), hi = ld_na_s32(t.bins + b + 1) + 1;
  if (hi > (int32_t)t.n_union - 1) hi = (int32_t)t.n_union - 1;
  while (hi - lo > 1) {
    const int32_t mid = lo + ((hi - lo) >> 1);
    if (ld_na_f64(t.unionized + mid) > E) hi = mid;
    else lo = mid;
  }
  return lo;
}
template <int P, bool Stream, bool SmemMats, bool SrchStream, bool IdxStream>
__device__ __forceinline__ void flat_opt2(const XSTables& t, uint64_t seed0, int64_t first,
                                          int32_t n, uint64_t* __restrict__ ver) {
  const int32_t total = gridDim.x * blockDim.x;
  int32_t iv = blockIdx.x * blockDim.x + threadIdx.x;
  if (iv >= n) return;
  const LcgMap J = lcg_jump(2ull * (uint64_t)total);
  uint64_t s0 = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv));
  __shared__ int32_t smats[12 * 34];
  __shared__ double sconcs[12 * 34];
  const int32_t* gm = t.mats;
  const double* gc = t.concs;
  if (SmemMats) {
    for (int k = threadIdx.x; k < 12 * t.max_num_nucs; k += blockDim.x) {
      smats[k] = __ldg(t.mats + k);
      sconcs[k] = __ldg(t.concs + k);
    }
    __syncthreads();
    gm = smats;
    gc = sconcs;
  }
  double E;
  int32_t mat, idx, nn, j;
  double m0, m1, m2, m3, m4;
  int32_t pc[P], kc[P];
  auto start = [&]() {
    uint64_t seed = s0;
    E = lcg_double(seed);
    mat = pick_mat(seed);
    idx = SrchStream ? search_stream(t, E) : binned_grid_search(t, E);
    nn = __ldg(t.num_nucs + mat);
    m0 = m1 = m2 = m3 = m4 = 0.0;
    j = 0;
    const int32_t* mrow = gm + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = u < nn ? (SmemMats ? mrow[u] : __ldg(mrow + u)) : 0;
      kc[u] = u < nn ? (int32_t)ldidx<IdxStream>(irow + pc[u]) : 0;
    }
  };
  start();
  while (true) {
    const int32_t* mrow = gm + mat * t.max_num_nucs;
    const double* crow = gc + mat * t.max_num_nucs;
    const uint16_t* irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {
      const int jj = j + P + u;
      pn[u] = jj < nn ? (SmemMats ? mrow[jj] : __ldg(mrow + jj)) : 0;
      kn[u] = jj < nn ? (int32_t)ldidx<IdxStream>(irow + pn[u]) : 0;
    }
#pragma unroll
    for (int u = 0; u < P; ++u) {
      if (j + u < nn) {
        int32_t k = kc[u];
        if (k == t.n_gridpoints - 1) --k;
        const double conc = SmemMats ? crow[j + u] : __ldg(crow + j + u);
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
        if (Stream) {
          ld_stream_v4f64(g, le, he, lt, ht);
          ld_stream_v4f64(g + 4, lel, hel, la, ha);
          ld_stream_v4f64(g + 8, lf, hf, ln, hn);
        } else {
          ld_nc_v4f64(g, le, he, lt, ht);
          ld_nc_v4f64(g + 4, lel, hel, la, ha);
          ld_nc_v4f64(g + 8, lf, hf, ln, hn);
        }
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
    if (j >= nn) {
      ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
      iv += total;
      if (iv >= n) break;
      s0 = (J.a * s0 + J.c) & kLcgMask;
      start();
    }
  }
}

#define KP(NAME, TPB, MINB)                                                                    \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;                                   \
    if (i < n) ver[i] = xs_lookup_one<true>(t, seed, first + i);                               \
  }
#define KS_(NAME, TPB, MINB, P)                                                                \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    flat_sm<P>(t, seed, first, n, ver);                                                        \
  }
#define KC_(NAME, TPB, MINB, P)                                                                \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    flat_c<P>(t, seed, first, n, ver);                                                         \
  }
#define KQ_(NAME, TPB, MINB, P)                                                                \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    flat_pipe<P>(t, seed, first, n, ver);                                                      \
  }
#define KJ_(NAME, TPB, MINB, P)                                                                \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    flat_jump<P>(t, seed, first, n, ver);                                                      \
  }
#define KO_(NAME, TPB, MINB, P, ST, SM)                                                        \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    flat_opt<P, ST, SM>(t, seed, first, n, ver);                                               \
  }
#define KO2_(NAME, TPB, MINB, P, SS, IS)                                                       \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    flat_opt2<P, true, true, SS, IS>(t, seed, first, n, ver);                                  \
  }
#define KF_(NAME, TPB, MINB, P)                                                                \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    flat_loop<P>(t, seed, first, n, ver);                                                      \
  }
KP(e0, 256, 3)
KO_(e1, 256, 4, 2, true, true)
typedef void (*KF)(XSTables, uint64_t, int64_t, int32_t, uint64_t*);
// variants: kernel e1 under L2 access-policy windows (per launch, cudaLaunchKernelEx)
//   0: e0 (product one-lookup-per-thread), 1: e1 no window,
//   2: brackets persisting (hitRatio 1), 3: brackets persisting hitRatio 0.6,
//   4: index16 persisting hitRatio 0.5, 5: unionized+bins? (unionized persisting)
static int g_maxpersist = 0;
extern "C" int xsx_count() { return 6; }
extern "C" int xsx_regs(int v) {
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, (const void*)(v == 0 ? e0 : e1));
  return a.numRegs * 1000 + (int)a.localSizeBytes;
}
extern "C" int xsx_prepare(XSTables) {
  int dev = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&g_maxpersist, cudaDevAttrMaxPersistingL2CacheSize, dev);
  printf("max persisting L2: %d\n", g_maxpersist);
  return (int)cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, g_maxpersist);
}
extern "C" int xsx_run(int v, XSTables t, uint64_t seed, int64_t first, int32_t n,
                       uint64_t* ver, void* stream) {
  if (v == 0) {
    e0<<<(n + 255) / 256, 256, 0, (cudaStream_t)stream>>>(t, seed, first, n, ver);
    return (int)cudaGetLastError();
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(148 * 4);
  cfg.blockDim = dim3(256);
  cfg.stream = (cudaStream_t)stream;
  cudaLaunchAttribute at[1];
  cfg.attrs = at;
  cfg.numAttrs = 0;
  const size_t br = (size_t)t.n_isotopes * (t.n_gridpoints - 1) * 12 * sizeof(double);
  const size_t ix = (size_t)t.n_union * t.n_isotopes * sizeof(uint16_t);
  if (v >= 2) {
    at[0].id = cudaLaunchAttributeAccessPolicyWindow;
    auto& w = at[0].val.accessPolicyWindow;
    w.hitProp = cudaAccessPropertyPersisting;
    w.missProp = cudaAccessPropertyStreaming;
    if (v == 2 || v == 3) {
      w.base_ptr = (void*)t.brackets;
      w.num_bytes = br;
      w.hitRatio = v == 2 ? 1.0f : 0.6f;
    } else if (v == 4) {
      w.base_ptr = (void*)t.index_grid16;
      w.num_bytes = ix;
      w.hitRatio = 0.5f;
    } else {
      w.base_ptr = (void*)t.unionized;
      w.num_bytes = (size_t)t.n_union * 8;
      w.hitRatio = 1.0f;
    }
    cfg.numAttrs = 1;
  }
  cudaLaunchKernelEx(&cfg, e1, t, seed, first, n, ver);
  cudaCtxResetPersistingL2Cache();
  return (int)cudaGetLastError();
}
