// Exploration harness (NOT part of libomprt.so): the PRODUCT's RSBench bodies
// (RSFlatLookup, RSQueuedLookup from rs_body.cuh) in the product's dynamic lock-step loop
// (omprt::distribute_parallel_for_dynamic_flat, warp-collective hook), at several launch
// bounds -- register budget vs occupancy for the pipelined pole loop.
#include <cuda_runtime.h>
#include <cstdint>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/omprt/device/omprt.cuh"
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/rs_body.cuh"
using namespace omprt_kernels;
using namespace omprt;

struct Tr : DefaultTraits {};

template <bool Q, int MINB>
__global__ void __launch_bounds__(128, MINB)
    kern(const __grid_constant__ RSTables t, uint64_t seed, int64_t first, int32_t n,
         uint64_t* ver, double* macro) {
  Team<Tr> team = init<Tr>();
  if constexpr (Q) {
    using L = RSQueuedLookup<true, 4>;
    L::init_queue();
    L b(t, seed, first, ver, macro);
    distribute_parallel_for_dynamic_flat<Tr, FlatSync::Lockstep>(team, n, 1, b);
  } else {
    RSFlatLookup<true> b(t, seed, first, ver, macro);
    distribute_parallel_for_dynamic_flat<Tr, FlatSync::Lockstep>(team, n, 1, b);
  }
}

typedef void (*KF)(RSTables, uint64_t, int64_t, int32_t, uint64_t*, double*);
struct Var { KF f; int tpb; const char* name; };
#ifdef OMPRT_RS_ABRAROV_NOINLINE
#define VN(x) x "_noinline"
#else
#define VN(x) x
#endif
static Var vars[] = {
  {kern<false, 5>, 128, VN("dflat_128x5")}, {kern<true, 5>, 128, VN("qflat_128x5")},
  {kern<false, 4>, 128, VN("dflat_128x4")}, {kern<true, 4>, 128, VN("qflat_128x4")},
  {kern<true, 3>, 128, VN("qflat_128x3")},
};
extern "C" int rsf_count() { return (int)(sizeof(vars) / sizeof(vars[0])); }
extern "C" const char* rsf_name(int v) { return vars[v].name; }
extern "C" int rsf_regs(int v) {
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, (const void*)vars[v].f);
  return a.numRegs * 1000 + (int)a.localSizeBytes;
}
extern "C" int rsf_run(int v, RSTables t, uint64_t seed, int64_t first, int32_t n, uint64_t* ver,
                       double* macro, void* stream) {
  int dev = 0, sms = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, vars[v].f, vars[v].tpb, 0);
  vars[v].f<<<sms * per, vars[v].tpb, 0, (cudaStream_t)stream>>>(t, seed, first, n, ver, macro);
  return (int)cudaGetLastError();
}
