// Exploration harness 5 (NOT part of libomprt.so): a coarse index grid.  Only every 2^S-th
// row of the (16-bit) index grid is stored: k0 = index[idx & ~(2^S-1)][p] <= k = index[idx][p],
// and k is reached from k0 by walking the nuclide's brackets while the upper energy of the
// bracket is <= U[idx] (the definition: k = clip(upper_bound(E_p, U[idx]) - 1, 0, n_gp - 2)).
// The walk rarely moves (about (2^S - 1) / 2 / 68 of the nuclides), the index shrinks by 2^S
// and, with the brackets, the hot tables fit the 126 MB L2.  Same arithmetic as the product.
#include <cuda_runtime.h>
#include <cstdint>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/xs_body.cuh"
using namespace omprt_kernels;

static uint16_t* g_ic[6] = {};  // coarse index per S

__global__ void build_coarse(const uint16_t* __restrict__ ig, int64_t n_union, int n_iso, int S,
                             uint16_t* __restrict__ o) {
  const int64_t rows = ((n_union - 1) >> S) + 1;
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < rows * n_iso;
       r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t row = r / n_iso, p = r - row * n_iso;
    o[r] = ig[(row << S) * n_iso + p];
  }
}

template <int S, int P>
__device__ __forceinline__ uint64_t lookup_c(const XSTables& t, const uint16_t* __restrict__ ic,
                                             uint64_t seed0, int64_t i) {
  uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)i);
  const double E = lcg_double(seed);
  const int mat = pick_mat(seed);
  const int32_t idx = binned_grid_search(t, E);
  const double Ue = __ldg(t.unionized + idx);
  const int nn = __ldg(t.num_nucs + mat);
  const int32_t* __restrict__ mrow = t.mats + mat * t.max_num_nucs;
  const double* __restrict__ crow = t.concs + mat * t.max_num_nucs;
  const uint16_t* __restrict__ irow = ic + (int64_t)(idx >> S) * t.n_isotopes;
  const int32_t kmax = t.n_gridpoints - 2;
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
    for (int u = 0; u < P; ++u) {
      const int jj = j + P + u;
      pn[u] = jj < nn ? __ldg(mrow + jj) : 0;
      kn[u] = jj < nn ? (int32_t)__ldg(irow + pn[u]) : 0;
    }
#pragma unroll
    for (int u = 0; u < P; ++u) {
      if (j + u < nn) {
        int32_t k = kc[u];
        const double conc = __ldg(crow + j + u);
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
        ld_nc_v4f64(g, le, he, lt, ht);
        ld_nc_v4f64(g + 4, lel, hel, la, ha);
        ld_nc_v4f64(g + 8, lf, hf, ln, hn);
        while (k < kmax && he <= Ue) {  // walk to the exact bracket (rare)
          ++k;
          g += 12;
          ld_nc_v4f64(g, le, he, lt, ht);
          ld_nc_v4f64(g + 4, lel, hel, la, ha);
          ld_nc_v4f64(g + 8, lf, hf, ln, hn);
        }
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
  return xs_argmax5(m0, m1, m2, m3, m4);
}

#define KP(NAME, TPB, MINB)                                                                    \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;                                   \
    if (i < n) ver[i] = xs_lookup_one<true>(t, seed, first + i);                               \
  }
#define KC(NAME, TPB, MINB, S, P)                                                              \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;                                   \
    if (i < n) ver[i] = lookup_c<S, P>(t, g_icd[S], seed, first + i);                          \
  }
__constant__ const uint16_t* g_icd[6];
KP(c0, 256, 3)
KC(c1, 256, 3, 3, 2)
KC(c2, 256, 3, 4, 2)
KC(c3, 256, 3, 2, 2)
KC(c4, 256, 3, 5, 2)
KC(c5, 256, 4, 3, 2)
KC(c6, 256, 3, 3, 1)
KC(c7, 256, 3, 0, 2)
typedef void (*KF)(XSTables, uint64_t, int64_t, int32_t, uint64_t*);
static KF kf[] = {c0, c1, c2, c3, c4, c5, c6, c7};
extern "C" int xsx_count() { return (int)(sizeof(kf) / sizeof(kf[0])); }
extern "C" int xsx_regs(int v) {
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, (const void*)kf[v]);
  return a.numRegs * 1000 + (int)a.localSizeBytes;
}
extern "C" int xsx_prepare(XSTables t) {
  for (int S = 0; S < 6; ++S) {
    const int64_t rows = ((t.n_union - 1) >> S) + 1;
    if (cudaMalloc(&g_ic[S], rows * t.n_isotopes * sizeof(uint16_t))) return 2;
    build_coarse<<<148 * 8, 256>>>(t.index_grid16, t.n_union, t.n_isotopes, S, g_ic[S]);
  }
  cudaMemcpyToSymbol(g_icd, g_ic, sizeof(g_ic));
  return (int)cudaDeviceSynchronize();
}
extern "C" int xsx_run(int v, XSTables t, uint64_t seed, int64_t first, int32_t n,
                       uint64_t* ver, void* stream) {
  kf[v]<<<(n + 255) / 256, 256, 0, (cudaStream_t)stream>>>(t, seed, first, n, ver);
  return (int)cudaGetLastError();
}
