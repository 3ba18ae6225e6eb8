// C1 (BASELINE configs[0]): SPMD `target teams distribute parallel for reduction(+:sum)`
//   for (i = 0; i < n; ++i) { a[i] = x*b[i] + c[i]; sum += a[i]; }
// runtime-driven (omprt) and bare-CUDA twin.  a[i] = fma(x, b[i], c[i]).
#pragma once
#include "../host/runtime.cuh"

namespace omprt_kernels {

using namespace omprt;

struct AxpyTraits : DefaultTraits {
  static constexpr unsigned unroll = 8;  // 8 independent iterations per trip (same owner)
};
struct AxpyTraitsAssume : AxpyTraits {
  static constexpr bool assume_teams_oversub = true;
};
struct AxpyTraitsDebug : AxpyTraits {
  static constexpr unsigned debug = dbg::Assert | dbg::Trace;
};
struct AxpyTraitsAssumeDebug : AxpyTraitsAssume {
  static constexpr unsigned debug = dbg::Assert | dbg::Trace;
};
// Runtime-driven kernel: the OpenMP region as the runtime executes it.
template <class Tr, bool Rec>
__global__ void __launch_bounds__(1024)
    omprt_axpy_rt(typename Tr::Idx n, double x, const double* __restrict__ b,
                  const double* __restrict__ c, double* __restrict__ a, double* sum_inout,
                  double* partials, unsigned* ticket, int32_t* owner, int32_t* count) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  double acc = 0.0;  // private copy, identity of +
  distribute_parallel_for(team, n, [&](Idx i) {
    const double v = fma(x, __ldg(b + i), __ldg(c + i));
    a[i] = v;
    acc += v;
    if constexpr (Rec) {
      owner[i] = get_team_num(team) * get_num_threads(team) + get_thread_num(team);
      atomicAdd(count + i, 1);
    }
  });
  league_reduce(team, team_reduce_to_main(team, acc, Plus{}), Plus{}, sum_inout, partials,
                ticket);
}

// Bare CUDA twin: grid-stride loop (the same cyclic assignment) and a hand-written copy of
// the same reduction algorithm (shfl.xor butterfly, warp partials, last-block combine).
template <class Idx, bool Rec>
__global__ void __launch_bounds__(1024)
    cuda_axpy_twin(Idx n, double x, const double* __restrict__ b, const double* __restrict__ c,
                   double* __restrict__ a, double* sum_inout, double* partials,
                   unsigned* ticket, int32_t* owner, int32_t* count) {
  const Idx stride = (Idx)gridDim.x * blockDim.x;
  const Idx gtid = (Idx)blockIdx.x * blockDim.x + threadIdx.x;
  double acc = 0.0;
  Idx i = gtid;
  for (; i + 7 * stride < n; i += 8 * stride) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const double v = fma(x, __ldg(b + i + u * stride), __ldg(c + i + u * stride));
      a[i + u * stride] = v;
      acc += v;
      if constexpr (Rec) {
        owner[i + u * stride] = (int32_t)gtid;
        atomicAdd(count + i + u * stride, 1);
      }
    }
  }
  for (; i < n; i += stride) {
    const double v = fma(x, __ldg(b + i), __ldg(c + i));
    a[i] = v;
    acc += v;
    if constexpr (Rec) {
      owner[i] = (int32_t)gtid;
      atomicAdd(count + i, 1);
    }
  }
  __shared__ double warp_sum[32];
  __shared__ unsigned is_last;
  for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
  const unsigned lane = threadIdx.x & 31u, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  if (lane == 0) warp_sum[wid] = acc;
  __syncthreads();
  double blk = 0.0;
  if (wid == 0) {
    blk = lane < nw ? warp_sum[lane] : 0.0;
    for (int off = 16; off > 0; off >>= 1) blk += __shfl_xor_sync(0xffffffffu, blk, off);
  }
  if (threadIdx.x == 0) {
    partials[blockIdx.x] = blk;
    __threadfence();
    is_last = (atomicAdd(ticket, 1u) == gridDim.x - 1) ? 1u : 0u;
  }
  __syncthreads();
  if (is_last) {
    __threadfence();
    double t = 0.0;
    for (unsigned k = threadIdx.x; k < gridDim.x; k += blockDim.x) t += __ldcg(partials + k);
    for (int off = 16; off > 0; off >>= 1) t += __shfl_xor_sync(0xffffffffu, t, off);
    if (lane == 0) warp_sum[wid] = t;
    __syncthreads();
    if (wid == 0) {
      double tt = lane < nw ? warp_sum[lane] : 0.0;
      for (int off = 16; off > 0; off >>= 1) tt += __shfl_xor_sync(0xffffffffu, tt, off);
      if (threadIdx.x == 0) {
        *sum_inout = *sum_inout + tt;
        *ticket = 0u;
      }
    }
  }
}

OMPRT_REGISTER_KERNEL(omprt_axpy_rt, omprt_axpy_rt<AxpyTraits, false>)
OMPRT_REGISTER_KERNEL(omprt_axpy_rt_assume, omprt_axpy_rt<AxpyTraitsAssume, false>)
OMPRT_REGISTER_KERNEL(omprt_axpy_rt_debug, omprt_axpy_rt<AxpyTraitsDebug, false>)
OMPRT_REGISTER_KERNEL(cuda_axpy_twin, cuda_axpy_twin<int32_t, false>)

template <class Tr, class Idx>
int launch_axpy_rt(int64_t n, double x, const double* b, const double* c, double* a,
                   double* sum, int32_t teams, int32_t threads, int32_t* owner, int32_t* count,
                   Workspace* w, cudaStream_t s) {
  static_assert(std::is_same<typename Tr::Idx, Idx>::value, "");
  if (owner)
    omprt_axpy_rt<Tr, true><<<teams, threads, 0, s>>>((Idx)n, x, b, c, a, sum,
                                                      (double*)w->partials, w->tickets + 0,
                                                      owner, count);
  else
    omprt_axpy_rt<Tr, false><<<teams, threads, 0, s>>>((Idx)n, x, b, c, a, sum,
                                                       (double*)w->partials, w->tickets + 0,
                                                       nullptr, nullptr);
  return check_launch("omprt_axpy_rt");
}

inline int axpy_validate(int64_t n, const double* b, const double* c, double* a, double* sum,
                         int32_t teams, int32_t threads, uint32_t flags, int32_t* owner,
                         int32_t* count, Workspace* w) {
  OMPRT_CHECK_ARG(n >= 0, "n must be >= 0");
  OMPRT_CHECK_ARG(teams > 0 && (uint64_t)teams <= w->opt.max_teams, "teams out of range");
  OMPRT_CHECK_ARG(threads > 0 && threads <= 1024 && threads % 32 == 0,
                  "threads must be a multiple of 32 in [32, 1024]");
  OMPRT_CHECK_ARG(sum != nullptr, "sum_inout is required");
  OMPRT_CHECK_ARG(n == 0 || (b && c && a), "null data pointer");
  OMPRT_CHECK_ARG(!(flags & OMPRT_RECORD_OWNER) || (owner && count),
                  "OMPRT_RECORD_OWNER needs owner and count");
  // the assumption is a promise; a call that breaks it is rejected
  OMPRT_CHECK_ARG(!(flags & OMPRT_ASSUME_OVERSUB) || (flags & OMPRT_UNCHECKED) ||
                      n <= (int64_t)teams * threads,
                  "oversubscription assumption violated: n=%lld > teams*threads=%lld",
                  (long long)n, (long long)teams * threads);
  return OMPRT_OK;
}

}  // namespace omprt_kernels

extern "C" int omprt_spmd_axpy_sum(int64_t n, double x, const double* b, const double* c,
                                   double* a, double* sum_inout, int32_t teams, int32_t threads,
                                   uint32_t flags, int32_t* owner, int32_t* count, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  if (int r = axpy_validate(n, b, c, a, sum_inout, teams, threads, flags, owner, count, w))
    return r;
  if (!(flags & OMPRT_RECORD_OWNER)) owner = count = nullptr;
  cudaStream_t s = as_stream(stream);
  const bool assume = flags & OMPRT_ASSUME_OVERSUB, debug = flags & OMPRT_DEBUG_BUILD;
  // 32-bit induction variable when n + (unroll+1)*T*N fits
  const bool i32 = n + 9 * (int64_t)teams * threads < INT32_MAX;
  if (i32) {
    if (assume)
      return debug ? launch_axpy_rt<AxpyTraitsAssumeDebug, int32_t>(n, x, b, c, a, sum_inout, teams,
                                                                   threads, owner, count, w, s)
                   : launch_axpy_rt<AxpyTraitsAssume, int32_t>(n, x, b, c, a, sum_inout, teams,
                                                              threads, owner, count, w, s);
    return debug ? launch_axpy_rt<AxpyTraitsDebug, int32_t>(n, x, b, c, a, sum_inout, teams,
                                                           threads, owner, count, w, s)
                 : launch_axpy_rt<AxpyTraits, int32_t>(n, x, b, c, a, sum_inout, teams, threads,
                                                      owner, count, w, s);
  }
  if (assume)
    return launch_axpy_rt<WithIdx64<AxpyTraitsAssume>, int64_t>(n, x, b, c, a, sum_inout, teams,
                                                                threads, owner, count, w, s);
  return launch_axpy_rt<WithIdx64<AxpyTraits>, int64_t>(n, x, b, c, a, sum_inout, teams, threads,
                                                        owner, count, w, s);
}

extern "C" int omprt_cuda_axpy_sum(int64_t n, double x, const double* b, const double* c,
                                   double* a, double* sum_inout, int32_t teams, int32_t threads,
                                   uint32_t flags, int32_t* owner, int32_t* count, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  if (int r = axpy_validate(n, b, c, a, sum_inout, teams, threads, flags, owner, count, w))
    return r;
  cudaStream_t s = as_stream(stream);
  const bool rec = flags & OMPRT_RECORD_OWNER;
  const bool i32 = n + 9 * (int64_t)teams * threads < INT32_MAX;
  double* p = (double*)w->partials;
  unsigned* t = w->tickets + 0;
  if (i32) {
    if (rec)
      cuda_axpy_twin<int32_t, true><<<teams, threads, 0, s>>>((int32_t)n, x, b, c, a, sum_inout,
                                                              p, t, owner, count);
    else
      cuda_axpy_twin<int32_t, false><<<teams, threads, 0, s>>>((int32_t)n, x, b, c, a,
                                                               sum_inout, p, t, nullptr, nullptr);
  } else {
    if (rec)
      cuda_axpy_twin<int64_t, true><<<teams, threads, 0, s>>>(n, x, b, c, a, sum_inout, p, t,
                                                              owner, count);
    else
      cuda_axpy_twin<int64_t, false><<<teams, threads, 0, s>>>(n, x, b, c, a, sum_inout, p, t,
                                                               nullptr, nullptr);
  }
  return check_launch("cuda_axpy_twin");
}
