// NEXT f3: C1 with a user-defined chunk --
//   #pragma omp target teams distribute parallel for dist_schedule(static, C) \
//                                                    schedule(static, C) reduction(+:sum)
// chunk k -> global thread k mod (T*N) (reading R-F3; C = 1 is Fig. 5).  A chunk is
// contiguous and owned by one thread, so with C = 4 and 32 B-aligned arrays the body moves
// it with 256-bit accesses (2 loads + 1 store per 4 iterations instead of 8 + 4).
#pragma once
#include "../host/runtime.cuh"
#include "axpy.cuh"
#include "vec.cuh"

namespace omprt_kernels {

using namespace omprt;

// The chunk body (user code, identical in both kernels): kVec4 = chunk is 4 and aligned.
template <bool kVec4, class Idx>
__device__ __forceinline__ double axpy_chunk_body(Idx lo, Idx cnt, double x,
                                                  const double* __restrict__ b,
                                                  const double* __restrict__ c,
                                                  double* __restrict__ a) {
  double acc = 0.0;
  if (kVec4 && cnt == 4) {
    double b0, b1, b2, b3, c0, c1, c2, c3;
    ld_stream_v4f64(b + lo, b0, b1, b2, b3);
    ld_stream_v4f64(c + lo, c0, c1, c2, c3);
    const double v0 = fma(x, b0, c0), v1 = fma(x, b1, c1), v2 = fma(x, b2, c2),
                 v3 = fma(x, b3, c3);
    st_v4f64(a + lo, v0, v1, v2, v3);
    acc += v0;
    acc += v1;
    acc += v2;
    acc += v3;
  } else {
    for (Idx i = lo; i < lo + cnt; ++i) {
      const double v = fma(x, __ldg(b + i), __ldg(c + i));
      a[i] = v;
      acc += v;
    }
  }
  return acc;
}

template <class Tr, bool kVec4, bool Rec>
__global__ void __launch_bounds__(1024)
    omprt_axpy_chunk_rt(typename Tr::Idx n, typename Tr::Idx chunk, double x,
                        const double* __restrict__ b, const double* __restrict__ c,
                        double* __restrict__ a, double* sum_inout, double* partials,
                        unsigned* ticket, int32_t* owner, int32_t* count) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  double acc = 0.0;
  distribute_parallel_for_chunks(team, n, chunk, [&](Idx lo, Idx cnt) {
    // the private copy accumulates in iteration order, chunk by chunk
    const double part = axpy_chunk_body<kVec4>(lo, cnt, x, b, c, a);
    acc += part;
    if constexpr (Rec) {
      for (Idx i = lo; i < lo + cnt; ++i) {
        owner[i] = get_team_num(team) * get_num_threads(team) + get_thread_num(team);
        atomicAdd(count + i, 1);
      }
    }
  });
  league_reduce_threads(team, acc, Plus{}, sum_inout, partials,
                ticket);
}

// Bare CUDA twin: the same chunk loop and the same hand-written reduction algorithm.
template <class Idx, bool kVec4, bool Rec>
__global__ void __launch_bounds__(1024)
    cuda_axpy_chunk_twin(Idx n, Idx chunk, double x, const double* __restrict__ b,
                         const double* __restrict__ c, double* __restrict__ a, double* sum_inout,
                         double* partials, unsigned* ticket, int32_t* owner, int32_t* count) {
  const Idx gtid = (Idx)blockIdx.x * blockDim.x + threadIdx.x;
  const Idx stride = (Idx)gridDim.x * blockDim.x * chunk;
  double acc = 0.0;
  Idx lo = gtid * chunk;
  for (; lo + 7 * stride + chunk <= n; lo += 8 * stride) {  // 8 whole chunks per trip
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      acc += axpy_chunk_body<kVec4>(lo + u * stride, chunk, x, b, c, a);
      if constexpr (Rec) {
        for (Idx i = lo + u * stride; i < lo + u * stride + chunk; ++i) {
          owner[i] = (int32_t)gtid;
          atomicAdd(count + i, 1);
        }
      }
    }
  }
  for (; lo < n; lo += stride) {
    const Idx cnt = n - lo < chunk ? n - lo : chunk;
    acc += axpy_chunk_body<kVec4>(lo, cnt, x, b, c, a);
    if constexpr (Rec) {
      for (Idx i = lo; i < lo + cnt; ++i) {
        owner[i] = (int32_t)gtid;
        atomicAdd(count + i, 1);
      }
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

// schedule(dynamic, C) (OMPRT_SCHED_DYNAMIC, reading R-D1): team blocks, chunks from a
// team-shared counter.  The per-thread sum order depends on which chunks a thread got, so
// the fp64 sum is compared with a tolerance; a[] is bit-exact.
template <class Tr, bool Rec>
__global__ void __launch_bounds__(1024)
    omprt_axpy_dyn_rt(typename Tr::Idx n, typename Tr::Idx chunk, double x,
                      const double* __restrict__ b, const double* __restrict__ c,
                      double* __restrict__ a, double* sum_inout, double* partials,
                      unsigned* ticket, int32_t* owner, int32_t* count) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  double acc = 0.0;
  distribute_parallel_for_dynamic_chunks(team, n, chunk, [&](Idx lo, Idx cnt) {
    acc += axpy_chunk_body<false>(lo, cnt, x, b, c, a);
    if constexpr (Rec) {
      for (Idx i = lo; i < lo + cnt; ++i) {
        owner[i] = get_team_num(team) * get_num_threads(team) + get_thread_num(team);
        atomicAdd(count + i, 1);
      }
    }
  });
  league_reduce_threads(team, acc, Plus{}, sum_inout, partials,
                ticket);
}

template <bool Rec>
__global__ void __launch_bounds__(1024)
    cuda_axpy_dyn_twin(int32_t n, int32_t chunk, double x, const double* __restrict__ b,
                       const double* __restrict__ c, double* __restrict__ a, double* sum_inout,
                       double* partials, unsigned* ticket, int32_t* owner, int32_t* count) {
  __shared__ unsigned next;
  __shared__ double warp_sum[32];
  __shared__ unsigned is_last;
  const int32_t per = (n + (int32_t)gridDim.x - 1) / (int32_t)gridDim.x;
  const int32_t blo = min((int32_t)blockIdx.x * per, n), bhi = min(blo + per, n);
  if (threadIdx.x == 0) next = blockDim.x;
  __syncthreads();
  double acc = 0.0;
  for (int32_t k = threadIdx.x;; k = (int32_t)atomicAdd(&next, 1u)) {
    const int32_t lo = blo + k * chunk;
    if (lo >= bhi) break;
    const int32_t cnt = min(chunk, bhi - lo);
    acc += axpy_chunk_body<false>(lo, cnt, x, b, c, a);
    if constexpr (Rec) {
      for (int32_t i = lo; i < lo + cnt; ++i) {
        owner[i] = (int32_t)(blockIdx.x * blockDim.x + threadIdx.x);
        atomicAdd(count + i, 1);
      }
    }
  }
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

OMPRT_REGISTER_KERNEL(omprt_axpy_dyn_rt, omprt_axpy_dyn_rt<AxpyTraits, false>)
OMPRT_REGISTER_KERNEL(cuda_axpy_dyn_twin, cuda_axpy_dyn_twin<false>)
OMPRT_REGISTER_KERNEL(omprt_axpy_chunk_rt, omprt_axpy_chunk_rt<AxpyTraits, true, false>)
OMPRT_REGISTER_KERNEL(cuda_axpy_chunk_twin, cuda_axpy_chunk_twin<int32_t, true, false>)

inline bool aligned32(const void* p) { return ((uintptr_t)p & 31u) == 0; }

}  // namespace omprt_kernels

extern "C" int omprt_spmd_axpy_sum_chunked(int64_t n, int64_t chunk, double x, const double* b,
                                           const double* c, double* a, double* sum_inout,
                                           int32_t teams, int32_t threads, uint32_t flags,
                                           int32_t* owner, int32_t* count, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  OMPRT_CHECK_ARG(chunk > 0, "chunk must be > 0");
  // the assumption for chunks: n <= T*N*C (checked here on the chunk count)
  const int64_t nchunks = (n + chunk - 1) / chunk;
  if (int r = axpy_validate(nchunks, b, c, a, sum_inout, teams, threads, flags, owner, count, w))
    return r;
  OMPRT_CHECK_ARG(n == 0 || (b && c && a), "null data pointer");
  const bool rec = flags & OMPRT_RECORD_OWNER, assume = flags & OMPRT_ASSUME_OVERSUB;
  if (!rec) owner = count = nullptr;
  cudaStream_t s = as_stream(stream);
  OMPRT_CHECK_ARG(n + (int64_t)(8 + 2) * teams * threads * chunk < INT32_MAX,
                  "iteration space too large for the chunked path");
  const bool v4 = chunk == 4 && aligned32(a) && aligned32(b) && aligned32(c);
  double* p = (double*)w->partials;
  unsigned* t = w->tickets + 0;
  const int32_t nn = (int32_t)n, cc = (int32_t)chunk;
  if (flags & OMPRT_SCHED_DYNAMIC) {
    OMPRT_CHECK_ARG(!assume, "OMPRT_SCHED_DYNAMIC: no oversubscription assumption");
    if (rec) omprt_axpy_dyn_rt<AxpyTraits, true><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, owner, count);
    else omprt_axpy_dyn_rt<AxpyTraits, false><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, owner, count);
    return check_launch("omprt_axpy_dyn_rt");
  }
#define OMPRT_AXC(TR, V, R)                                                                  \
  omprt_axpy_chunk_rt<TR, V, R><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, \
                                                         owner, count)
  if (assume) {
    if (v4) { if (rec) OMPRT_AXC(AxpyTraitsAssume, true, true); else OMPRT_AXC(AxpyTraitsAssume, true, false); }
    else { if (rec) OMPRT_AXC(AxpyTraitsAssume, false, true); else OMPRT_AXC(AxpyTraitsAssume, false, false); }
  } else {
    if (v4) { if (rec) OMPRT_AXC(AxpyTraits, true, true); else OMPRT_AXC(AxpyTraits, true, false); }
    else { if (rec) OMPRT_AXC(AxpyTraits, false, true); else OMPRT_AXC(AxpyTraits, false, false); }
  }
#undef OMPRT_AXC
  return check_launch("omprt_axpy_chunk_rt");
}

extern "C" int omprt_cuda_axpy_sum_chunked(int64_t n, int64_t chunk, double x, const double* b,
                                           const double* c, double* a, double* sum_inout,
                                           int32_t teams, int32_t threads, uint32_t flags,
                                           int32_t* owner, int32_t* count, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  OMPRT_CHECK_ARG(chunk > 0, "chunk must be > 0");
  const int64_t nchunks = (n + chunk - 1) / chunk;
  if (int r = axpy_validate(nchunks, b, c, a, sum_inout, teams, threads,
                            flags & ~OMPRT_ASSUME_OVERSUB, owner, count, w))
    return r;
  OMPRT_CHECK_ARG(n == 0 || (b && c && a), "null data pointer");
  const bool rec = flags & OMPRT_RECORD_OWNER;
  if (!rec) owner = count = nullptr;
  cudaStream_t s = as_stream(stream);
  OMPRT_CHECK_ARG(n + (int64_t)(8 + 2) * teams * threads * chunk < INT32_MAX,
                  "iteration space too large for the chunked path");
  const bool v4 = chunk == 4 && aligned32(a) && aligned32(b) && aligned32(c);
  double* p = (double*)w->partials;
  unsigned* t = w->tickets + 0;
  const int32_t nn = (int32_t)n, cc = (int32_t)chunk;
  if (flags & OMPRT_SCHED_DYNAMIC) {
    if (rec) cuda_axpy_dyn_twin<true><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, owner, count);
    else cuda_axpy_dyn_twin<false><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, owner, count);
    return check_launch("cuda_axpy_dyn_twin");
  }
  if (v4) {
    if (rec) cuda_axpy_chunk_twin<int32_t, true, true><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, owner, count);
    else cuda_axpy_chunk_twin<int32_t, true, false><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, owner, count);
  } else {
    if (rec) cuda_axpy_chunk_twin<int32_t, false, true><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, owner, count);
    else cuda_axpy_chunk_twin<int32_t, false, false><<<teams, threads, 0, s>>>(nn, cc, x, b, c, a, sum_inout, p, t, owner, count);
  }
  return check_launch("cuda_axpy_chunk_twin");
}
