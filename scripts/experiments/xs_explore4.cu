// Exploration harness 4 (NOT part of libomprt.so): a material-expanded bracket table.
// For every material m and unionized energy e the 96 B brackets of m's nuclides are stored
// contiguously: X_m[e][j] = bracket(mats[m][j], index[e][mats[m][j]]).  A lookup then reads
// one contiguous num_nucs[m] x 96 B segment, with no dependent index load per nuclide.
// Same arithmetic and order as the product (xs_accumulate), so the results are identical.
#include <cuda_runtime.h>
#include <cstdint>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/xs_body.cuh"
using namespace omprt_kernels;

static double* g_x = nullptr;     // all materials' expanded tables
static int64_t* g_off = nullptr;  // [12] offsets (in doubles) of X_m

__global__ void build_expanded(XSTables t, const int64_t* __restrict__ off, int mat, int nn,
                               double* __restrict__ x) {
  const int64_t nrec = t.n_union * nn;
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < nrec;
       r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = r / nn;
    const int j = (int)(r - e * nn);
    const int p = t.mats[mat * t.max_num_nucs + j];
    int k = t.index_grid16[e * t.n_isotopes + p];
    if (k == t.n_gridpoints - 1) --k;
    const double* g = t.brackets + ((int64_t)p * (t.n_gridpoints - 1) + k) * 12;
    double* o = x + off[mat] + r * 12;
#pragma unroll
    for (int c = 0; c < 12; c += 4) {
      double a, b, cc, d;
      ld_nc_v4f64(g + c, a, b, cc, d);
      st_v4f64(o + c, a, b, cc, d);
    }
  }
}

template <int kUnroll, bool Stream>
__device__ __forceinline__ uint64_t lookup_x(const XSTables& t, const double* __restrict__ X,
                                             const int64_t* __restrict__ off, uint64_t seed0,
                                             int64_t i) {
  uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)i);
  const double E = lcg_double(seed);
  const int mat = pick_mat(seed);
  const int32_t idx = binned_grid_search(t, E);
  const int nn = __ldg(t.num_nucs + mat);
  const double* __restrict__ crow = t.concs + mat * t.max_num_nucs;
  const double* __restrict__ seg = X + __ldg(off + mat) + (int64_t)idx * nn * 12;
  double m0 = 0.0, m1 = 0.0, m2 = 0.0, m3 = 0.0, m4 = 0.0;
#pragma unroll kUnroll
  for (int j = 0; j < nn; ++j) {
    const double conc = __ldg(crow + j);
    const double* g = seg + j * 12;
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
    xs_accumulate(E, conc, le, he, lt, ht, lel, hel, la, ha, lf, hf, ln, hn, m0, m1, m2, m3, m4);
  }
  return xs_argmax5(m0, m1, m2, m3, m4);
}

#define KP(NAME, TPB, MINB)                                                                    \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      const double* X, const int64_t* off, uint64_t seed, int64_t first, int32_t n,            \
      uint64_t* ver) {                                                                         \
    const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;                                   \
    if (i < n) ver[i] = xs_lookup_one<true>(t, seed, first + i);                               \
  }
#define KX(NAME, TPB, MINB, U, S)                                                              \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      const double* X, const int64_t* off, uint64_t seed, int64_t first, int32_t n,            \
      uint64_t* ver) {                                                                         \
    const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;                                   \
    if (i < n) ver[i] = lookup_x<U, S>(t, X, off, seed, first + i);                            \
  }
KP(b0, 256, 3)
KX(b1, 256, 3, 2, false)
KX(b2, 256, 3, 4, false)
KX(b3, 256, 3, 2, true)
KX(b4, 256, 3, 4, true)
KX(b5, 256, 4, 2, true)
KX(b6, 128, 8, 2, true)
KX(b7, 256, 2, 4, true)
KX(b8, 256, 4, 4, false)
typedef void (*KF)(XSTables, const double*, const int64_t*, uint64_t, int64_t, int32_t,
                   uint64_t*);
static KF kf[] = {b0, b1, b2, b3, b4, b5, b6, b7, b8};
static int tpb[] = {256, 256, 256, 256, 256, 256, 128, 256, 256};
extern "C" int xsx_count() { return (int)(sizeof(kf) / sizeof(kf[0])); }
extern "C" int xsx_regs(int v) {
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, (const void*)kf[v]);
  return a.numRegs * 1000 + (int)a.localSizeBytes;
}
extern "C" int xsx_prepare(XSTables t) {
  int nn[12];
  if (cudaMemcpy(nn, t.num_nucs, sizeof(nn), cudaMemcpyDeviceToHost)) return 1;
  int64_t off[12], tot = 0;
  for (int m = 0; m < 12; ++m) {
    off[m] = tot;
    tot += (int64_t)nn[m] * t.n_union * 12;
  }
  if (cudaMalloc(&g_x, tot * sizeof(double))) return 2;
  if (cudaMalloc(&g_off, sizeof(off))) return 3;
  cudaMemcpy(g_off, off, sizeof(off), cudaMemcpyHostToDevice);
  for (int m = 0; m < 12; ++m) build_expanded<<<148 * 8, 256>>>(t, g_off, m, nn[m], g_x);
  return (int)cudaDeviceSynchronize();
}
extern "C" int xsx_run(int v, XSTables t, uint64_t seed, int64_t first, int32_t n,
                       uint64_t* ver, void* stream) {
  kf[v]<<<(n + tpb[v] - 1) / tpb[v], tpb[v], 0, (cudaStream_t)stream>>>(t, g_x, g_off, seed,
                                                                         first, n, ver);
  return (int)cudaGetLastError();
}
