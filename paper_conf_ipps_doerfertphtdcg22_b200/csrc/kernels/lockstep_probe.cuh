// Lock-step probe: checks the contract of the runtime's lock-step flattened loops and their
// warp-collective hook (omprt/device/workshare.cuh, FlatSync::Lockstep) with a synthetic
// body whose iteration i takes L(i) = 1 + (7 i mod 13) steps.  It records, per iteration,
// the steps it ran, and per thread, how many times the hook ran on it; any violation of
// "the hook runs after every trip on all 32 lanes, converged, and a lane's end() follows a
// hook call that reported done = true for it" increments *errors.  Tests only.
#pragma once
#include "../host/runtime.cuh"

namespace omprt_kernels {

using namespace omprt;

struct LockstepProbeBody {
  int32_t* steps;
  int32_t* errors;
  int64_t iv = -1;
  int32_t cnt = 0, len = 0, hooks = 0;
  bool last_done = false;

  __device__ __forceinline__ void start(int64_t i) {
    iv = i;
    cnt = 0;
    len = 1 + (int32_t)((7 * i) % 13);
    last_done = false;
  }
  template <class Idx>
  __device__ __forceinline__ void begin(Idx i, Idx) { start((int64_t)i); }
  template <class Idx>
  __device__ __forceinline__ void next(Idx i) { start((int64_t)i); }
  __device__ __forceinline__ bool step() {
    ++cnt;
    return cnt < len;
  }
  __device__ __forceinline__ void warp_collective(bool done) {
    ++hooks;
    if (__activemask() != 0xffffffffu) atomicAdd(errors, 1);
    // every lane took the same number of hook calls so far
    if (__shfl_sync(0xffffffffu, hooks, 0) != hooks) atomicAdd(errors, 1);
    // done is reported exactly once per iteration, on its last step
    if (done != (iv >= 0 && cnt == len && !last_done)) atomicAdd(errors, 1);
    last_done = last_done || done;
  }
  template <class Idx>
  __device__ __forceinline__ void end(Idx i) {
    if ((int64_t)i != iv || !last_done) atomicAdd(errors, 1);
    steps[i] = cnt;
    iv = -1;
  }
};

template <class Tr, bool Dyn>
__global__ void __launch_bounds__(1024)
    omprt_lockstep_probe_kernel(typename Tr::Idx n, int32_t* steps, int32_t* hooks,
                                int32_t* errors) {
  Team<Tr> team = init<Tr>();
  LockstepProbeBody body{steps, errors};
  if constexpr (Dyn)
    distribute_parallel_for_dynamic_flat<Tr, FlatSync::Lockstep>(team, n, (typename Tr::Idx)3,
                                                                 body);
  else
    distribute_parallel_for_flat<Tr, FlatSync::Lockstep>(team, n, body);
  hooks[(int64_t)blockIdx.x * blockDim.x + threadIdx.x] = body.hooks;
}

}  // namespace omprt_kernels

extern "C" int omprt_lockstep_probe(int64_t n, int32_t teams, int32_t threads, int32_t dynamic,
                                    int32_t* steps, int32_t* hooks, int32_t* errors,
                                    void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  OMPRT_CHECK_ARG(n >= 0 && n < (1ll << 30) && teams > 0 && threads > 0 && threads <= 1024 &&
                      threads % 32 == 0 && (n == 0 || steps) && hooks && errors,
                  "omprt_lockstep_probe: bad arguments");
  cudaStream_t s = as_stream(stream);
  if (dynamic)
    omprt_lockstep_probe_kernel<DefaultTraits, true><<<teams, threads, 0, s>>>(
        (int32_t)n, steps, hooks, errors);
  else
    omprt_lockstep_probe_kernel<DefaultTraits, false><<<teams, threads, 0, s>>>(
        (int32_t)n, steps, hooks, errors);
  return check_launch("omprt_lockstep_probe");
}
