// Exploration harness 14 (NOT part of libomprt.so): the product's flattened XS body at more
// resident teams per SM -- 5 (51 registers) and 6 (42) teams of 256 under
// __launch_bounds__ -- against the product's 4 (64 registers): more warps to hide the L2
// latency, if ptxas can hold the body in fewer registers without spilling its prefetched
// index entries.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/xs_body.cuh"
using namespace omprt_kernels;

constexpr int kThreads = 256;
constexpr int kMatSmem = 12 * 48;

struct DI {
  int dummy;
};
static DI g_di;

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

template <int MINB, int P>
__global__ void __launch_bounds__(kThreads, MINB)
    kern(const __grid_constant__ XSTables t, const __grid_constant__ DI di, uint64_t seed,
         int64_t first, int32_t count, uint64_t* __restrict__ ver) {
  __shared__ int32_t sm[kMatSmem];
  __shared__ double sc[kMatSmem];
  for (int k = threadIdx.x; k < 12 * t.max_num_nucs; k += blockDim.x) {
    sm[k] = __ldg(t.mats + k);
    sc[k] = __ldg(t.concs + k);
  }
  __syncthreads();
  XSFlatLookup<false, true, false, P> lookup(t, seed, first, ver, sm, sc);
  flat_loop(lookup, count);
}

struct Var {
  void (*k)(XSTables, DI, uint64_t, int64_t, int32_t, uint64_t*);
  bool window;
  const char* name;
  int tpb = kThreads, minb = 4;
  unsigned dyn = 0;
};
static Var kVars[] = {
    {kern<4, 2>, true, "V0_product_body_4perSM", kThreads, 4, 0},
    {kern<5, 2>, true, "B5_5perSM_P2", kThreads, 5, 0},
    {kern<6, 2>, true, "B6_6perSM_P2", kThreads, 6, 0},
    {kern<5, 1>, true, "B5_5perSM_P1", kThreads, 5, 0},
    {kern<6, 1>, true, "B6_6perSM_P1", kThreads, 6, 0},
    {kern<4, 3>, true, "B4_4perSM_P3", kThreads, 4, 0},
    {kern<4, 2>, true, "V0_product_body_4perSM(again)", kThreads, 4, 0}};
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
  if (kVars[v].dyn)
    cudaFuncSetAttribute(kVars[v].k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)kVars[v].dyn);
  cudaLaunchConfig_t cfg{};
  cudaLaunchAttribute attr[1];
  cfg.gridDim = dim3(sms * kVars[v].minb);
  cfg.blockDim = dim3(kVars[v].tpb);
  cfg.dynamicSmemBytes = kVars[v].dyn;
  cfg.stream = (cudaStream_t)stream;
  cfg.attrs = attr;
  cfg.numAttrs = 0;
  if (kVars[v].window) {  // [unionized | bins | brackets], as the product's flat_launch
    int maxp = 0, maxwin = 0;
    cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev);
    cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, dev);
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)maxp);
    const size_t br = sizeof(double) * 12ull * t.n_isotopes * (t.n_gridpoints - 1);
    const uintptr_t hi = (uintptr_t)t.brackets + br;
    uintptr_t lo = (uintptr_t)t.unionized;
    if (lo > (uintptr_t)t.brackets || hi - lo > (size_t)maxp) lo = (uintptr_t)t.brackets;
    const size_t bytes = hi - lo;
    cudaAccessPolicyWindow& w = attr[0].val.accessPolicyWindow;
    attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
    w.base_ptr = (void*)lo;
    w.num_bytes = bytes;
    w.hitRatio = (float)((double)maxp / (double)bytes < 1.0 ? (double)maxp / (double)bytes : 1.0);
    w.hitProp = cudaAccessPropertyPersisting;
    w.missProp = cudaAccessPropertyStreaming;
    cfg.numAttrs = 1;
  }
  cudaLaunchKernelEx(&cfg, kVars[v].k, t, g_di, seed, first, n, (uint64_t*)ver);
  cudaError_t e = cudaGetLastError();
  if (kVars[v].window) {
    cudaStreamSynchronize((cudaStream_t)stream);
    cudaCtxResetPersistingL2Cache();
  }
  return e != cudaSuccess;
}
