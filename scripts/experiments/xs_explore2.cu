// Exploration harness 2 (NOT part of libomprt.so): the product XSBench body with the B200
// layouts under different launch bounds / unroll factors.
#include <cuda_runtime.h>
#include <cstdint>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/xs_body.cuh"
using namespace omprt_kernels;
#define K(NAME, TPB, MINB, U)                                                                  \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ XSTables t,        \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                \
    const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;                                   \
    if (i < n) ver[i] = xs_lookup_one<true, U>(t, seed, first + i);                            \
  }
K(a0, 256, 4, 4)
K(a1, 256, 4, 2)
K(a2, 256, 4, 3)
K(a3, 256, 3, 4)
K(a4, 256, 3, 6)
K(a5, 256, 3, 8)
K(a6, 128, 8, 4)
K(a7, 128, 6, 6)
K(a8, 256, 2, 8)
K(a9, 512, 2, 4)
K(a10, 256, 5, 2)
K(a11, 64, 16, 4)
typedef void (*KF)(XSTables, uint64_t, int64_t, int32_t, uint64_t*);
static KF kf[] = {a0, a1, a2, a3, a4, a5, a6, a7, a8, a9, a10, a11};
static int tpb[] = {256, 256, 256, 256, 256, 256, 128, 128, 256, 512, 256, 64};
extern "C" int xsx_count() { return (int)(sizeof(kf) / sizeof(kf[0])); }
extern "C" int xsx_regs(int v) { cudaFuncAttributes a; cudaFuncGetAttributes(&a, (const void*)kf[v]); return a.numRegs * 1000 + (int)a.localSizeBytes; }
extern "C" int xsx_prepare(XSTables) { return 0; }
extern "C" int xsx_run(int v, XSTables t, uint64_t seed, int64_t first, int32_t n, uint64_t* ver, void* stream) {
  kf[v]<<<(n + tpb[v] - 1) / tpb[v], tpb[v], 0, (cudaStream_t)stream>>>(t, seed, first, n, ver);
  return (int)cudaGetLastError();
}
