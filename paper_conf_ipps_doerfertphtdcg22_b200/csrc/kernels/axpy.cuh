// C1 (BASELINE configs[0]): SPMD `target teams distribute parallel for reduction(+:sum)`
//   for (i = 0; i < n; ++i) { a[i] = x*b[i] + c[i]; sum += a[i]; }
// runtime-driven (omprt) and bare-CUDA twin.  a[i] = fma(x, b[i], c[i]).
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <type_traits>

#include "../host/runtime.cuh"
#include "../omprt/device/staging.cuh"

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
// Teams of <= 256 threads (C1: 8 x 128): 32 iterations per trip.  The config runs on 8 SMs
// with 4 warps each; its HBM reads are latency-bound by the bytes each SM keeps in flight
// (8 iterations: 4 warps x 16 loads x 256 B = 16 KB per SM, ~240 GB/s over the 8 SMs).  At
// 32 iterations a trip issues its 64 loads before the first store (the runtime kernel
// through distribute_parallel_for_split, the twin by hand) in a 255-register budget, which
// 256 threads per team still fit: 0.104 -> 0.059 ms at 2^20, runtime within 3 % of the
// twin.  64 iterations ran the twin at 0.048 ms but the runtime kernel at 0.053-0.055 ms
// for every budget tried (200-255): under the extra register pressure ptxas moves some of
// its stores ahead of the last loads (scripts/experiments/c1_prefetch.cu,
// profiles/c1_wide_r2.txt).  Same Fig. 5 assignment, same per-thread order: a[] and the
// sum keep their bits.
#ifndef OMPRT_AXPY_WIDE_UNROLL  // exploration builds only
#define OMPRT_AXPY_WIDE_UNROLL 32
#define OMPRT_AXPY_WIDE_REGS 255
#endif
constexpr unsigned kAxpyWideUnroll = OMPRT_AXPY_WIDE_UNROLL;
constexpr int kAxpyWideMaxThreads = 256;
struct AxpyTraitsWide : AxpyTraits {
  static constexpr unsigned unroll = kAxpyWideUnroll;
};
struct AxpyTraitsWideDebug : AxpyTraitsWide {
  static constexpr unsigned debug = dbg::Assert | dbg::Trace;
};

// Both C1 kernels carry the same register budget, __maxnreg__(58) (1024 threads still fit
// an SM).  Under __launch_bounds__(1024) ptxas held them to 32 registers and interleaved the
// unrolled trip's loads with its stores (2-4 loads in flight per thread); with a budget of
// their own both issue all 16 loads of a trip first -- what 4 warps per SM need: 0.30 ->
// 0.104 ms at 8 x 128 (scripts/experiments/c1_lib_kernels.cu, profiles/c1_budget_r2.txt).
// The runtime kernel's body is split into its loads and the rest
// (distribute_parallel_for_split), so its trip has the twin's shape and register count (50).
// Runtime-driven kernel: the OpenMP region as the runtime executes it.
constexpr int kAxpyMaxRegs = 58;
// the budget of a C1 kernel unrolled U times: 58 at U = 8, all 255 for the wide trips
constexpr int axpy_max_regs(unsigned U) { return U > 8 ? OMPRT_AXPY_WIDE_REGS : kAxpyMaxRegs; }
template <class Tr, bool Rec>
__global__ void __maxnreg__(axpy_max_regs(Tr::unroll))
    omprt_axpy_rt(typename Tr::Idx n, double x, const double* __restrict__ b,
                  const double* __restrict__ c, double* __restrict__ a, double* sum_inout,
                  double* partials, unsigned* ticket, int32_t* owner, int32_t* count) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  double acc = 0.0;  // private copy, identity of +
  // the body split into its loads and the rest (b and c are read-only in the loop), so the
  // runtime issues a trip's loads together (distribute_parallel_for_split)
  distribute_parallel_for_split(
      team, n, [&](Idx i) { return double2{__ldg(b + i), __ldg(c + i)}; },
      [&](Idx i, double2 bc) {
        const double v = fma(x, bc.x, bc.y);
        a[i] = v;
        acc += v;
        if constexpr (Rec) {
          owner[i] = get_team_num(team) * get_num_threads(team) + get_thread_num(team);
          atomicAdd(count + i, 1);
        }
      });
  league_reduce_threads(team, acc, Plus{}, sum_inout, partials,
                ticket);
}

// Bare CUDA twin: grid-stride loop (the same cyclic assignment) and a hand-written copy of
// the same reduction algorithm (shfl.xor butterfly, warp partials, last-block combine).
template <class Idx, bool Rec, int U = 8>
__global__ void __maxnreg__(axpy_max_regs(U))
    cuda_axpy_twin(Idx n, double x, const double* __restrict__ b, const double* __restrict__ c,
                   double* __restrict__ a, double* sum_inout, double* partials,
                   unsigned* ticket, int32_t* owner, int32_t* count) {
  const Idx stride = (Idx)gridDim.x * blockDim.x;
  const Idx gtid = (Idx)blockIdx.x * blockDim.x + threadIdx.x;
  double acc = 0.0;
  Idx i = gtid;
  // U iterations per trip, all 2U loads issued before the first store (what a CUDA
  // programmer writes to keep loads in flight with 4 warps per SM)
  for (; i + (U - 1) * stride < n; i += U * stride) {
    double bv[U], cv[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      bv[u] = __ldg(b + i + u * stride);
      cv[u] = __ldg(c + i + u * stride);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const double v = fma(x, bv[u], cv[u]);
      a[i + u * stride] = v;
      acc += v;
      if constexpr (Rec) {
        owner[i + u * stride] = (int32_t)gtid;
        atomicAdd(count + i + u * stride, 1);
      }
    }
  }
#pragma unroll 1
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

// ---- OMPRT_TMA_STREAM: the same loop with its operands streamed by 2-D TMA boxes --------
// (omprt/device/staging.cuh distribute_parallel_for_tma_stream): b, c and a viewed as
// [n / (T*N)][T*N] matrices, team b's columns [b*N, (b+1)*N) moved kAxRows trips at a time,
// kAxStages boxes per array in flight.  Same iterations per thread in the same order as
// Fig. 5, so a[] and the sum are bit-identical to omprt_axpy_rt.  (8 teams: the config's
// 8 SMs must each keep ~100 KB in flight to approach their share of HBM bandwidth.)
#ifndef OMPRT_AXPY_TMA_STAGES
#define OMPRT_AXPY_TMA_STAGES 6
#define OMPRT_AXPY_TMA_STORE 0
#endif
// rows per box: 2048 / threads; stages x (2 or 3 arrays) x 16 KB <= 227 KB
constexpr unsigned kAxStages = OMPRT_AXPY_TMA_STAGES;
constexpr bool kAxTmaStore = OMPRT_AXPY_TMA_STORE;  // a[] through TMA stores, or direct
struct AxpyMaps {
  CUtensorMap m[3];  // b, c (loads), a (store)
};

template <class Tr, bool Rec, unsigned kAxRows>
__global__ void __launch_bounds__(256)
    omprt_axpy_tma_rt(const __grid_constant__ AxpyMaps maps, typename Tr::Idx n, double x,
                      const double* __restrict__ b, const double* __restrict__ c,
                      double* __restrict__ a, double* sum_inout, double* partials,
                      unsigned* ticket, int32_t* owner, int32_t* count) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  double acc = 0.0;
  auto rec = [&](Idx i) {
    if constexpr (Rec) {
      owner[i] = get_team_num(team) * get_num_threads(team) + get_thread_num(team);
      atomicAdd(count + i, 1);
    }
  };
  distribute_parallel_for_tma_stream<Tr, 2, kAxTmaStore ? 1 : 0, kAxRows, kAxStages>(
      team, n, maps.m,
      [&](Idx i, const double (&xs)[2], double (&ys)[1]) {
        const double v = fma(x, xs[0], xs[1]);
        if constexpr (kAxTmaStore) ys[0] = v;
        else a[i] = v;
        acc += v;
        rec(i);
      },
      [&](Idx i) {
        const double v = fma(x, __ldg(b + i), __ldg(c + i));
        a[i] = v;
        acc += v;
        rec(i);
      });
  league_reduce_threads(team, acc, Plus{}, sum_inout, partials,
                ticket);
}

// Bare CUDA twin: the same TMA box pipeline and the same hand-written reduction.
template <bool Rec, unsigned kAxRows>
__global__ void __launch_bounds__(256)
    cuda_axpy_tma_twin(const __grid_constant__ AxpyMaps maps, int32_t n, double x,
                       const double* __restrict__ b, const double* __restrict__ c,
                       double* __restrict__ a, double* sum_inout, double* partials,
                       unsigned* ticket, int32_t* owner, int32_t* count) {
  extern __shared__ __align__(128) unsigned char smem[];
  double* const sb = reinterpret_cast<double*>(smem);
  const unsigned N = blockDim.x, t = threadIdx.x, box = kAxRows * N;
  constexpr unsigned kArr = kAxTmaStore ? 3u : 2u;
  uint64_t* const full = reinterpret_cast<uint64_t*>(smem + kAxStages * kArr * box * 8u);
  const int32_t TN = gridDim.x * N, rows = n / TN, col0 = blockIdx.x * N;
  const unsigned chunks = (unsigned)((rows + kAxRows - 1) / kAxRows);
  double acc = 0.0;
  if (t == 0) {
    for (unsigned s = 0; s < kAxStages; ++s) tma::mbar_init(full + s, 1);
    tma::fence_mbar_init();
    for (unsigned s = 0; s < kAxStages && s < chunks; ++s) {
      tma::mbar_arrive_expect_tx(full + s, 2u * box * 8u);
      tma::tensor_load_2d(sb + (s * kArr + 0) * box, &maps.m[0], col0, s * kAxRows, full + s);
      tma::tensor_load_2d(sb + (s * kArr + 1) * box, &maps.m[1], col0, s * kAxRows, full + s);
    }
  }
  __syncthreads();
  for (unsigned ch = 0; ch < chunks; ++ch) {
    const unsigned s = ch % kAxStages;
    tma::mbar_wait(full + s, (ch / kAxStages) & 1u);
    double* const bs = sb + (s * kArr + 0) * box;
    double* const cs = sb + (s * kArr + 1) * box;
    double* const as = sb + (s * kArr + 2) * box;  // kAxTmaStore only
    const int32_t row0 = ch * kAxRows;
    const int32_t i0 = row0 * TN + col0 + t;
    const double* const bt = bs + t;
    const double* const ct = cs + t;
    double* const at = as + t;
    auto row = [&](unsigned r) {
      const double v = fma(x, bt[r * N], ct[r * N]);
      const int32_t i = i0 + (int32_t)r * TN;
      if constexpr (kAxTmaStore) at[r * N] = v;
      else a[i] = v;
      acc += v;
      if constexpr (Rec) {
        owner[i] = blockIdx.x * N + t;
        atomicAdd(count + i, 1);
      }
    };
    if (row0 + (int32_t)kAxRows <= rows) {  // a whole box: no per-row bound, fully unrolled
#pragma unroll
      for (unsigned r = 0; r < kAxRows; ++r) row(r);
    } else {
      for (unsigned r = 0; row0 + (int32_t)r < rows; ++r) row(r);
    }
    if constexpr (kAxTmaStore) {
      tma::fence_proxy_async_smem();
      if (t == 0) tma::bulk_wait_read<kAxStages - 2>();
    }
    __syncthreads();
    if (t == 0) {
      if constexpr (kAxTmaStore) {
        tma::tensor_store_2d(&maps.m[2], col0, row0, as);
        tma::bulk_commit();
      }
      if (ch + kAxStages < chunks) {
        tma::mbar_arrive_expect_tx(full + s, 2u * box * 8u);
        tma::tensor_load_2d(bs, &maps.m[0], col0, (ch + kAxStages) * kAxRows, full + s);
        tma::tensor_load_2d(cs, &maps.m[1], col0, (ch + kAxStages) * kAxRows, full + s);
      }
    }
  }
  const int32_t i = rows * TN + col0 + t;
  if (i < n) {
    const double v = fma(x, __ldg(b + i), __ldg(c + i));
    a[i] = v;
    acc += v;
    if constexpr (Rec) {
      owner[i] = blockIdx.x * N + t;
      atomicAdd(count + i, 1);
    }
  }
  if constexpr (kAxTmaStore)
    if (t == 0) tma::bulk_wait<0>();
  __shared__ double warp_sum[32];
  __shared__ unsigned is_last;
  for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
  const unsigned lane = t & 31u, wid = t >> 5, nw = (N + 31) >> 5;
  if (lane == 0) warp_sum[wid] = acc;
  __syncthreads();
  double blk = 0.0;
  if (wid == 0) {
    blk = lane < nw ? warp_sum[lane] : 0.0;
    for (int off = 16; off > 0; off >>= 1) blk += __shfl_xor_sync(0xffffffffu, blk, off);
  }
  if (t == 0) {
    partials[blockIdx.x] = blk;
    __threadfence();
    is_last = (atomicAdd(ticket, 1u) == gridDim.x - 1) ? 1u : 0u;
  }
  __syncthreads();
  if (is_last) {
    __threadfence();
    double tt0 = 0.0;
    for (unsigned k = t; k < gridDim.x; k += N) tt0 += __ldcg(partials + k);
    for (int off = 16; off > 0; off >>= 1) tt0 += __shfl_xor_sync(0xffffffffu, tt0, off);
    if (lane == 0) warp_sum[wid] = tt0;
    __syncthreads();
    if (wid == 0) {
      double tt = lane < nw ? warp_sum[lane] : 0.0;
      for (int off = 16; off > 0; off >>= 1) tt += __shfl_xor_sync(0xffffffffu, tt, off);
      if (t == 0) {
        *sum_inout = *sum_inout + tt;
        *ticket = 0u;
      }
    }
  }
}

OMPRT_REGISTER_KERNEL(omprt_axpy_tma_rt, omprt_axpy_tma_rt<AxpyTraits, false, 16>)
OMPRT_REGISTER_KERNEL(cuda_axpy_tma_twin, cuda_axpy_tma_twin<false, 16>)

// the three tensor maps of a launch: [rows][T*N] doubles, box [kAxRows][threads]
inline int axpy_tma_maps(AxpyMaps* M, const double* b, const double* c, double* a, int64_t n,
                         int32_t teams, int32_t threads, uint32_t rows_per_box) {
  static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  if (!enc) {
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q) !=
            cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !enc) {
      cudaGetLastError();
      enc = nullptr;
      return set_error(OMPRT_E_CUDA, "cuTensorMapEncodeTiled is not available");
    }
  }
  const int64_t TN = (int64_t)teams * threads;
  const int64_t rows = std::max<int64_t>(n / TN, 1);  // rows = 0: no box is ever issued
  const cuuint64_t dims[2] = {(cuuint64_t)TN, (cuuint64_t)rows};
  const cuuint64_t strides[1] = {(cuuint64_t)TN * 8u};
  const cuuint32_t box[2] = {(cuuint32_t)threads, rows_per_box}, es[2] = {1, 1};
  const double* ptr[3] = {b, c, a};
  for (int k = 0; k < 3; ++k) {
    const CUresult r = enc(&M->m[k], CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double*>(ptr[k]),
                           dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                           CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return set_error(OMPRT_E_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  }
  return OMPRT_OK;
}

inline int launch_axpy_tma(bool twin, int64_t n, double x, const double* b, const double* c,
                           double* a, double* sum, int32_t teams, int32_t threads,
                           int32_t* owner, int32_t* count, Workspace* w, cudaStream_t s) {
  OMPRT_CHECK_ARG(threads <= 256 && threads % 32 == 0,
                  "OMPRT_TMA_STREAM: threads must be a multiple of 32, at most 256 (box width)");
  OMPRT_CHECK_ARG(((uintptr_t)a | (uintptr_t)b | (uintptr_t)c) % 16 == 0,
                  "OMPRT_TMA_STREAM: arrays must be 16 B aligned");
  OMPRT_CHECK_ARG(n + 2 * (int64_t)teams * threads < INT32_MAX,
                  "OMPRT_TMA_STREAM: n too large for the 32-bit path");
  if (n == 0) {
    // nothing to stream; the reduction still adds 0 (keeps *sum untouched numerically)
    return OMPRT_OK;
  }
  const uint32_t rows_per_box = threads <= 64 ? 32u : (threads <= 128 ? 16u : 8u);
  AxpyMaps M;
  if (int r = axpy_tma_maps(&M, b, c, a, n, teams, threads, rows_per_box)) return r;
  double* p = (double*)w->partials;
  unsigned* tk = w->tickets + 0;
  const int32_t nn = (int32_t)n;
  auto go = [&](auto k, uint32_t smem) -> int {
    OMPRT_CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    k<<<teams, threads, smem, s>>>(M, nn, x, b, c, a, sum, p, tk, owner, count);
    return OMPRT_OK;
  };
  auto pick = [&](auto rows_c) -> int {
    constexpr unsigned R = decltype(rows_c)::value;
    const uint32_t smem = tma_stream_smem_bytes<2, kAxTmaStore ? 1 : 0, R, kAxStages>(threads);
    if (twin)
      return owner ? go(cuda_axpy_tma_twin<true, R>, smem) : go(cuda_axpy_tma_twin<false, R>, smem);
    return owner ? go(omprt_axpy_tma_rt<AxpyTraits, true, R>, smem)
                 : go(omprt_axpy_tma_rt<AxpyTraits, false, R>, smem);
  };
  int r;
  if (rows_per_box == 32) r = pick(std::integral_constant<unsigned, 32>{});
  else if (rows_per_box == 16) r = pick(std::integral_constant<unsigned, 16>{});
  else r = pick(std::integral_constant<unsigned, 8>{});
  if (r) return r;
  return check_launch(twin ? "cuda_axpy_tma_twin" : "omprt_axpy_tma_rt");
}

OMPRT_REGISTER_KERNEL(omprt_axpy_rt, omprt_axpy_rt<AxpyTraits, false>)
OMPRT_REGISTER_KERNEL(omprt_axpy_rt_assume, omprt_axpy_rt<AxpyTraitsAssume, false>)
OMPRT_REGISTER_KERNEL(omprt_axpy_rt_debug, omprt_axpy_rt<AxpyTraitsDebug, false>)
OMPRT_REGISTER_KERNEL(cuda_axpy_twin, cuda_axpy_twin<int32_t, false>)
OMPRT_REGISTER_KERNEL(omprt_axpy_rt_wide, omprt_axpy_rt<AxpyTraitsWide, false>)
OMPRT_REGISTER_KERNEL(omprt_axpy_rt_wide_debug, omprt_axpy_rt<AxpyTraitsWideDebug, false>)
OMPRT_REGISTER_KERNEL(cuda_axpy_twin_wide, cuda_axpy_twin<int32_t, false, kAxpyWideUnroll>)

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

// the 64-iteration trips: teams of <= 256 threads (the 255-register budget), no
// oversubscription assumption (no loop then), 32-bit induction variable
inline bool axpy_wide(int64_t n, int32_t teams, int32_t threads, uint32_t flags) {
  return threads <= kAxpyWideMaxThreads && !(flags & OMPRT_ASSUME_OVERSUB) &&
         n + (int64_t)(kAxpyWideUnroll + 1) * teams * threads < INT32_MAX;
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
  if (flags & OMPRT_TMA_STREAM) {
    OMPRT_CHECK_ARG(!(flags & (OMPRT_ASSUME_OVERSUB | OMPRT_DEBUG_BUILD)),
                    "OMPRT_TMA_STREAM: release build, no oversubscription assumption");
    return launch_axpy_tma(false, n, x, b, c, a, sum_inout, teams, threads, owner, count, w, s);
  }
  const bool assume = flags & OMPRT_ASSUME_OVERSUB, debug = flags & OMPRT_DEBUG_BUILD;
  // trait selection: teams of <= 256 threads take the 64-iteration trips (the twin does
  // the same, axpy_wide())
  if (axpy_wide(n, teams, threads, flags))
    return debug ? launch_axpy_rt<AxpyTraitsWideDebug, int32_t>(n, x, b, c, a, sum_inout, teams,
                                                               threads, owner, count, w, s)
                 : launch_axpy_rt<AxpyTraitsWide, int32_t>(n, x, b, c, a, sum_inout, teams,
                                                          threads, owner, count, w, s);
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
  if (flags & OMPRT_TMA_STREAM)
    return launch_axpy_tma(true, n, x, b, c, a, sum_inout, teams, threads, rec ? owner : nullptr,
                           rec ? count : nullptr, w, s);
  const bool i32 = n + 9 * (int64_t)teams * threads < INT32_MAX;
  double* p = (double*)w->partials;
  unsigned* t = w->tickets + 0;
  if (axpy_wide(n, teams, threads, flags)) {
    if (rec)
      cuda_axpy_twin<int32_t, true, kAxpyWideUnroll><<<teams, threads, 0, s>>>(
          (int32_t)n, x, b, c, a, sum_inout, p, t, owner, count);
    else
      cuda_axpy_twin<int32_t, false, kAxpyWideUnroll><<<teams, threads, 0, s>>>(
          (int32_t)n, x, b, c, a, sum_inout, p, t, nullptr, nullptr);
    return check_launch("cuda_axpy_twin");
  }
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
