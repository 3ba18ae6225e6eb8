// Exploration harness 9 (NOT part of libomprt.so): the flattened XS body with the NEXT
// lookup's grid search advanced one probe per nuclide step.  In the product body a lookup is
// ~12.5 dependent memory round trips: the bins load + ~3.7 bisection probes of the
// unionized grid, then ~7.75 steps of bracket loads (index entries prefetched a step
// ahead).  Here, while lookup k walks its nuclides, lookup k+1 (Fig. 5: iv + T*N, whose
// seed is one LCG jump away) has its bins loaded and its bisection probes issued one per
// step, each probe's value consumed a step later, so the search latency hides under the
// bracket loads.  Same arithmetic per lookup (bit-identical verification); static schedule
// only (the next iteration of a thread must be known).
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/xs_body.cuh"
using namespace omprt_kernels;

constexpr int kThreads = 256;
constexpr int kMatSmem = 12 * 48;

template <int P = 2, bool Early = false>
struct XSPrefetchLookup {
  const XSTables& t;
  const uint64_t seed0;
  const int64_t first;
  uint64_t* __restrict__ const ver;
  const int32_t* __restrict__ const mats;
  const double* __restrict__ const concs;
  LcgMap J;
  uint64_t s;          // current lookup's seed state (after the E draw... recomputed)
  double E;
  int32_t mat, idx, nn, j;
  double m0, m1, m2, m3, m4;
  int32_t pc[P], kc[P];
  // next lookup's search: seed, bracket [lo, hi], pending probe (mid, val)
  uint64_t sn;
  double En;
  int32_t lo, hi, mid;
  double val;
  bool pend;

  __device__ __forceinline__ XSPrefetchLookup(const XSTables& tab, uint64_t seed, int64_t f,
                                              uint64_t* v, const int32_t* ms, const double* cs)
      : t(tab), seed0(seed), first(f), ver(v), mats(ms), concs(cs) {}

  // the next lookup's energy and its bins bracket (the search's first dependent load)
  __device__ __forceinline__ void search_init(uint64_t seed) {
    sn = seed;
    uint64_t q = seed;
    En = lcg_double(q);
    const int64_t H = 1ll << t.log2_bins;
    int64_t b = (int64_t)(En * (double)H);
    if (b > H - 1) b = H - 1;
    lo = __ldg(t.bins + b);
    hi = __ldg(t.bins + b + 1) + 1;
    if (hi > (int32_t)t.n_union - 1) hi = (int32_t)t.n_union - 1;
    pend = false;
  }
  // consume the pending probe (issued a step ago), issue the next one
  __device__ __forceinline__ void search_advance() {
    if constexpr (Early) {  // En from the seed (no register held across steps)
      uint64_t q = sn;
      En = lcg_double(q);
    }
    if (pend) {
      if (val > En) hi = mid;
      else lo = mid;
      pend = false;
    }
    if (hi - lo > 1) {
      mid = lo + ((hi - lo) >> 1);
      val = __ldg(t.unionized + mid);
      pend = true;
    }
  }
  __device__ __forceinline__ void search_finish() {
    if (pend) {
      if (val > En) hi = mid;
      else lo = mid;
      pend = false;
    }
    while (hi - lo > 1) {
      const int32_t m = lo + ((hi - lo) >> 1);
      if (__ldg(t.unionized + m) > En) hi = m;
      else lo = m;
    }
  }
  // start the lookup whose seed is sn and whose search state is (lo, hi, pend)
  __device__ __forceinline__ void start_from_next() {
    search_finish();
    uint64_t seed = sn;
    E = lcg_double(seed);
    mat = pick_mat(seed);
    idx = lo;
    nn = __ldg(t.num_nucs + mat);
    m0 = m1 = m2 = m3 = m4 = 0.0;
    j = 0;
    const int32_t* __restrict__ mrow = mats + mat * t.max_num_nucs;
    const uint16_t* __restrict__ irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
#pragma unroll
    for (int u = 0; u < P; ++u) {
      pc[u] = u < nn ? mrow[u] : 0;
      kc[u] = u < nn ? (int32_t)__ldg(irow + pc[u]) : 0;
    }
    s = sn;
    search_init(lcg_apply(J, s));  // the lookup after this one
  }
  template <class Idx>
  __device__ __forceinline__ void begin(Idx iv, Idx stride) {
    J = lcg_jump(2ull * (uint64_t)stride);
    search_init(lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv)));
    start_from_next();
  }
  template <class Idx>
  __device__ __forceinline__ void next(Idx) {
    start_from_next();
  }
  __device__ __forceinline__ bool step() {
    const int32_t* __restrict__ mrow = mats + mat * t.max_num_nucs;
    const double* __restrict__ crow = concs + mat * t.max_num_nucs;
    const uint16_t* __restrict__ irow = t.index_grid16 + (int64_t)idx * t.n_isotopes;
    if constexpr (Early) search_advance();
    int32_t pn[P], kn[P];
#pragma unroll
    for (int u = 0; u < P; ++u) {
      const int jj = j + P + u;
      pn[u] = jj < nn ? mrow[jj] : 0;
      kn[u] = jj < nn ? (int32_t)__ldg(irow + pn[u]) : 0;
    }
    double br[P][12];
#pragma unroll
    for (int u = 0; u < P; ++u) {
      if (j + u < nn) {
        int32_t k = kc[u];
        if (k == t.n_gridpoints - 1) --k;
        const double* g = t.brackets + ((int64_t)pc[u] * (t.n_gridpoints - 1) + k) * 12;
        ld_stream_v4f64(g, br[u][0], br[u][1], br[u][2], br[u][3]);
        ld_stream_v4f64(g + 4, br[u][4], br[u][5], br[u][6], br[u][7]);
        ld_stream_v4f64(g + 8, br[u][8], br[u][9], br[u][10], br[u][11]);
      }
    }
    if constexpr (!Early) search_advance();
#pragma unroll
    for (int u = 0; u < P; ++u) {
      if (j + u < nn) {
        const double conc = crow[j + u];
        xs_accumulate(E, conc, br[u][0], br[u][1], br[u][2], br[u][3], br[u][4], br[u][5],
                      br[u][6], br[u][7], br[u][8], br[u][9], br[u][10], br[u][11], m0, m1, m2,
                      m3, m4);
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
    ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
  }
};

template <class Body>
__device__ __forceinline__ void flat_loop(Body& lookup, int32_t count) {
  const int32_t stride = (int32_t)gridDim.x * (int32_t)blockDim.x;
  int32_t i = (int32_t)blockIdx.x * (int32_t)blockDim.x + (int32_t)threadIdx.x;
  if (i >= count) return;
  lookup.begin(i, stride);
  for (;;) {
    if (lookup.step()) continue;
    lookup.end(i);
    i += stride;
    if (i >= count) break;
    lookup.next(i);
  }
}

template <int V, int MINB>
__global__ void __launch_bounds__(kThreads, MINB)
    kern(const __grid_constant__ XSTables t, uint64_t seed, int64_t first, int32_t count,
         uint64_t* __restrict__ ver) {
  __shared__ int32_t sm[kMatSmem];
  __shared__ double sc[kMatSmem];
  for (int k = threadIdx.x; k < 12 * t.max_num_nucs; k += blockDim.x) {
    sm[k] = __ldg(t.mats + k);
    sc[k] = __ldg(t.concs + k);
  }
  __syncthreads();
  if constexpr (V == 0) {
    XSFlatLookup<false, true> lookup(t, seed, first, ver, sm, sc);
    flat_loop(lookup, count);
  } else if constexpr (V == 1) {
    XSPrefetchLookup<2> lookup(t, seed, first, ver, sm, sc);
    flat_loop(lookup, count);
  } else {
    XSPrefetchLookup<2, true> lookup(t, seed, first, ver, sm, sc);
    flat_loop(lookup, count);
  }
}

struct Var {
  void (*k)(XSTables, uint64_t, int64_t, int32_t, uint64_t*);
  int minb;
  bool window;
  const char* name;
};
static Var kVars[] = {{kern<0, 4>, 4, false, "V0_product_body"},
                      {kern<2, 4>, 4, false, "V2_early_next_search_4x256"},
                      {kern<2, 3>, 3, false, "V2_early_next_search_3x256"},
                      {kern<0, 4>, 4, true, "V0_product_body+L2window"},
                      {kern<2, 4>, 4, true, "V2_early_4x256+L2window"},
                      {kern<2, 3>, 3, true, "V2_early_3x256+L2window"}};

extern "C" int xsx_count() { return (int)(sizeof(kVars) / sizeof(kVars[0])); }
extern "C" const char* xsx_name(int v) { return kVars[v].name; }
extern "C" int xsx_regs(int v) {
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, kVars[v].k);
  return a.numRegs * 1000 + (int)a.localSizeBytes;
}
extern "C" int xsx_prepare(XSTables) { return 0; }
extern "C" int xsx_run(int v, XSTables t, uint64_t seed, int64_t first, int32_t n, void* ver,
                       void* stream) {
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaLaunchConfig_t cfg{};
  cudaLaunchAttribute attr[1];
  cfg.gridDim = dim3(sms * kVars[v].minb);
  cfg.blockDim = dim3(kThreads);
  cfg.stream = (cudaStream_t)stream;
  cfg.attrs = attr;
  cfg.numAttrs = 0;
  if (kVars[v].window) {  // the product's window: bracket records persisting
    int maxp = 0, maxwin = 0;
    cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev);
    cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, dev);
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)maxp);
    const size_t br = sizeof(double) * 12ull * t.n_isotopes * (t.n_gridpoints - 1);
    const size_t bytes = br < (size_t)maxwin ? br : (size_t)maxwin;
    cudaAccessPolicyWindow& w = attr[0].val.accessPolicyWindow;
    attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
    w.base_ptr = (void*)t.brackets;
    w.num_bytes = bytes;
    w.hitRatio = (float)((double)maxp / (double)bytes < 1.0 ? (double)maxp / (double)bytes : 1.0);
    w.hitProp = cudaAccessPropertyPersisting;
    w.missProp = cudaAccessPropertyStreaming;
    cfg.numAttrs = 1;
  }
  cudaLaunchKernelEx(&cfg, kVars[v].k, t, seed, first, n, (uint64_t*)ver);
  cudaError_t e = cudaGetLastError();
  if (kVars[v].window) {
    cudaStreamSynchronize((cudaStream_t)stream);
    cudaCtxResetPersistingL2Cache();
  }
  return e != cudaSuccess;
}
