// Exploration harness 8 (NOT part of libomprt.so): the index grid as PER-MATERIAL rows.
// The flattened XS kernel reads one 2-byte index entry per nuclide from the [n_union][68]
// row (15.5 scalar loads per lookup, ~23 % of the L1->L2 sector requests; profiles/r08).
// Here the same entries are stored per material, mi[m][e][j] = index_grid16[e][mats[m][j]],
// rows padded to 8 entries (16 B), so a lookup's entries are contiguous and arrive in one
// 16-byte load per 8 nuclides (V2) or one 32-bit load per pair (V1).  The table grows from
// 104.5 MB to ~381 MB (it no longer competes for L2; ~1.6 sectors per lookup from DRAM).
// Same arithmetic and order per lookup (bit-identical verification).
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/xs_body.cuh"
using namespace omprt_kernels;

constexpr int kThreads = 256;
constexpr int kMatSmem = 12 * 48;

struct MI {
  const uint16_t* tab;
  int64_t base[12];  // entry offset of material m's [n_union][stride_m] block
  int32_t stride[12];
};
static MI g_mi;
static uint16_t* g_mi_buf = nullptr;

__device__ __forceinline__ uint4 ld16(const uint16_t* p) {
  uint4 v;
  asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
      : "l"(p));
  return v;
}
__device__ __forceinline__ uint4 ld16_ef(const uint16_t* p) {
  uint4 v;
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
      : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
      : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ uint32_t ld4(const uint16_t* p) {
  uint32_t v;
  asm("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}

__device__ __forceinline__ void nuc(const XSTables& t, double E, double conc, int32_t p,
                                    int32_t k, double& m0, double& m1, double& m2, double& m3,
                                    double& m4) {
  if (k == t.n_gridpoints - 1) --k;
  const double* g = t.brackets + ((int64_t)p * (t.n_gridpoints - 1) + k) * 12;
  double le, lt, lel, la, lf, ln, he, ht, hel, ha, hf, hn;
  ld_stream_v4f64(g, le, he, lt, ht);
  ld_stream_v4f64(g + 4, lel, hel, la, ha);
  ld_stream_v4f64(g + 8, lf, hf, ln, hn);
  xs_accumulate(E, conc, le, he, lt, ht, lel, hel, la, ha, lf, hf, ln, hn, m0, m1, m2, m3, m4);
}

// V1 / V2 / V3 bodies in the resumable form of XSFlatLookup (begin/next/step/end).
template <int V>
struct MIFlat {
  const XSTables& t;
  const MI& mi;
  const uint64_t seed0;
  const int64_t first;
  uint64_t* __restrict__ const ver;
  const int32_t* __restrict__ const mats;
  const double* __restrict__ const concs;
  LcgMap J;
  uint64_t s;
  double E;
  int32_t mat, nn, j;
  const uint16_t* row;
  double m0, m1, m2, m3, m4;
  uint4 c, nx;      // V2/V3: the current and next 8-entry chunks
  uint32_t pr, pn;  // V1: the current and next pair

  __device__ __forceinline__ MIFlat(const XSTables& tab, const MI& m, uint64_t seed,
                                    int64_t f, uint64_t* v, const int32_t* ms,
                                    const double* cs)
      : t(tab), mi(m), seed0(seed), first(f), ver(v), mats(ms), concs(cs) {}

  __device__ __forceinline__ uint4 chunk(const uint16_t* p) const {
    if constexpr (V == 3) return ld16_ef(p);
    else return ld16(p);
  }
  __device__ __forceinline__ void start() {
    uint64_t seed = s;
    E = lcg_double(seed);
    mat = pick_mat(seed);
    const int32_t idx = binned_grid_search(t, E);
    nn = __ldg(t.num_nucs + mat);
    m0 = m1 = m2 = m3 = m4 = 0.0;
    j = 0;
    row = mi.tab + mi.base[mat] + (int64_t)idx * mi.stride[mat];
    if constexpr (V == 1) {
      pr = ld4(row);
      pn = nn > 2 ? ld4(row + 2) : 0u;
    } else {
      c = chunk(row);
      nx = nn > 8 ? chunk(row + 8) : make_uint4(0, 0, 0, 0);
    }
  }
  template <class Idx>
  __device__ __forceinline__ void begin(Idx iv, Idx stride) {
    J = lcg_jump(2ull * (uint64_t)stride);
    s = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv));
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
    uint32_t w;
    if constexpr (V == 1) {
      w = pr;
      pr = pn;
      pn = j + 4 < nn ? ld4(row + j + 4) : 0u;
    } else {
      w = c.x;
      c.x = c.y;
      c.y = c.z;
      c.z = c.w;
      c.w = 0u;
    }
    nuc(t, E, crow[j], mrow[j], (int32_t)(w & 0xFFFFu), m0, m1, m2, m3, m4);
    if (j + 1 < nn)
      nuc(t, E, crow[j + 1], mrow[j + 1], (int32_t)(w >> 16), m0, m1, m2, m3, m4);
    j += 2;
    if constexpr (V != 1) {
      if ((j & 7) == 0) {
        c = nx;
        if (j + 8 < nn) nx = chunk(row + j + 8);
      }
    }
    return j < nn;
  }
  template <class Idx>
  __device__ __forceinline__ void end(Idx iv) {
    ver[iv] = xs_argmax5(m0, m1, m2, m3, m4);
  }
};

// The twin's flattened Fig. 5 loop (cuda_xs_flat_twin, non-fused, static), around a body.
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

template <int V>
__global__ void __launch_bounds__(kThreads, 4)
    kern(const __grid_constant__ XSTables t, const __grid_constant__ MI mi, uint64_t seed,
         int64_t first, int32_t count, uint64_t* __restrict__ ver) {
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
  } else {
    MIFlat<V> lookup(t, mi, seed, first, ver, sm, sc);
    flat_loop(lookup, count);
  }
}

__global__ void build_mi(const uint16_t* __restrict__ idx16, int32_t n_iso, int64_t n_union,
                         const int32_t* __restrict__ mats, int32_t max_nn, int32_t m, int32_t nn,
                         int32_t stride, uint16_t* __restrict__ out) {
  const int64_t total = n_union * stride;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = i / stride;
    const int jj = (int)(i - e * stride);
    out[i] = jj < nn ? idx16[e * n_iso + mats[m * max_nn + jj]] : (uint16_t)0;
  }
}

struct Var {
  void (*k)(XSTables, MI, uint64_t, int64_t, int32_t, uint64_t*);
  const char* name;
};
static Var kVars[] = {{kern<0>, "V0_product_body"},
                      {kern<1>, "V1_mi_pair32"},
                      {kern<2>, "V2_mi_chunk16"},
                      {kern<3>, "V3_mi_chunk16_evict_first"},
                      {kern<0>, "V0_product_body+L2window"},
                      {kern<2>, "V2_mi_chunk16+L2window"},
                      {kern<3>, "V3_mi_chunk16_evict_first+L2window"}};

extern "C" int xsx_count() { return 7; }
extern "C" const char* xsx_name(int v) { return kVars[v].name; }
extern "C" int xsx_regs(int v) {
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, kVars[v].k);
  return a.numRegs * 1000 + (int)a.localSizeBytes;
}
extern "C" int xsx_prepare(XSTables t) {
  int32_t nn[12], mats[12 * 64];
  cudaMemcpy(nn, t.num_nucs, sizeof(nn), cudaMemcpyDeviceToHost);
  int64_t off = 0;
  for (int m = 0; m < 12; ++m) {
    g_mi.base[m] = off;
    g_mi.stride[m] = (nn[m] + 7) & ~7;
    off += (int64_t)g_mi.stride[m] * t.n_union + 8;  // + slack for the over-read chunk
  }
  (void)mats;
  if (cudaMalloc(&g_mi_buf, off * 2) != cudaSuccess) return 1;
  for (int m = 0; m < 12; ++m)
    build_mi<<<1184, 256>>>(t.index_grid16, t.n_isotopes, t.n_union, t.mats, t.max_num_nucs, m,
                            nn[m], g_mi.stride[m], g_mi_buf + g_mi.base[m]);
  g_mi.tab = g_mi_buf;
  printf("mi table %.1f MB\n", off * 2 / 1e6);
  return cudaDeviceSynchronize() != cudaSuccess;
}
extern "C" int xsx_run(int v, XSTables t, uint64_t seed, int64_t first, int32_t n, void* ver,
                       void* stream) {
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaLaunchConfig_t cfg{};
  cudaLaunchAttribute attr[1];
  cfg.gridDim = dim3(sms * 4);
  cfg.blockDim = dim3(kThreads);
  cfg.stream = (cudaStream_t)stream;
  cfg.attrs = attr;
  cfg.numAttrs = 0;
  if (v >= 4) {  // the product's window: bracket records persisting (omprt flat_launch)
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
  cudaLaunchKernelEx(&cfg, kVars[v].k, t, g_mi, seed, first, n, (uint64_t*)ver);
  cudaError_t e = cudaGetLastError();
  if (v >= 4) {
    cudaStreamSynchronize((cudaStream_t)stream);
    cudaCtxResetPersistingL2Cache();
  }
  return e != cudaSuccess;
}
