// C5 with shared-memory staging: OMPRT_WARP_STAGED (warp-cooperative cp.async) and
// OMPRT_TMA_TILED (one 2-D TMA tensor copy per warp tile).  The SU(3) site loop runs as a
// persistent `distribute parallel for` (Fig. 5 assignment) whose site records (576 B, AoS)
// are moved into padded shared-memory slots and back (omprt/device/staging.cuh), instead of
// 32-line-wide strided global accesses.  Each twin runs the same pipeline, written by hand.
// (A per-thread bulk-copy variant was measured slower -- 0.33 vs 0.20 ms -- and removed.)
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>

#include "../common/ptx_tma.cuh"
#include "../host/runtime.cuh"
#include "../omprt/device/staging.cuh"
#include "rs_su3.cuh"

namespace omprt_kernels {

using namespace omprt;

constexpr unsigned kSU3Rec = 576;   // 4 links x 3 x 3 complex fp64
constexpr unsigned kSU3Slot = 592;  // 148 words: 8 consecutive threads' 16 B loads hit
                                    // disjoint bank quads (conflict-free LDS.128)

// The body on a staged record (in place): C[l] = A[l] x B[l], the App. A.3 fma order, the
// same (l, r, c) accumulation of Re C as su3_site.
__device__ __forceinline__ double su3_site_slot(unsigned char* slot,
                                                const double2* __restrict__ B) {
  double2* v = reinterpret_cast<double2*>(slot);
  double re_sum = 0.0;
#pragma unroll
  for (int l = 0; l < 4; ++l) {
    double2 a[9];
#pragma unroll
    for (int e = 0; e < 9; ++e) a[e] = v[l * 9 + e];
#pragma unroll
    for (int r = 0; r < 3; ++r)
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        double re = 0.0, im = 0.0;
#pragma unroll
        for (int m = 0; m < 3; ++m) {
          const double2 x = a[r * 3 + m];
          const double2 y = __ldg(B + l * 9 + m * 3 + c);
          re = fma(x.x, y.x, re);
          re = fma(-x.y, y.y, re);
          im = fma(x.x, y.y, im);
          im = fma(x.y, y.x, im);
        }
        v[l * 9 + r * 3 + c] = make_double2(re, im);
        re_sum += re;
      }
  }
  return re_sum;
}

// The twins' hand-written league reduction (warp butterflies, per-block partial, last block
// by ticket folds the partials and adds to *checksum).
__device__ __forceinline__ void twin_ticket_sum(double acc, double* checksum, double* partials,
                                                unsigned* ticket) {
  const unsigned nt = blockDim.x, t = threadIdx.x;
  __shared__ double ws[32];
  __shared__ unsigned last;
  for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
  const unsigned lane = t & 31u, wid = t >> 5, nw = nt >> 5;
  if (lane == 0) ws[wid] = acc;
  __syncthreads();
  double b = 0.0;
  if (wid == 0) {
    b = lane < nw ? ws[lane] : 0.0;
    for (int off = 16; off > 0; off >>= 1) b += __shfl_xor_sync(0xffffffffu, b, off);
  }
  if (t == 0) {
    partials[blockIdx.x] = b;
    __threadfence();
    last = atomicAdd(ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (last) {
    __threadfence();
    double tt = 0.0;
    for (unsigned k = t; k < gridDim.x; k += nt) tt += __ldcg(partials + k);
    for (int off = 16; off > 0; off >>= 1) tt += __shfl_xor_sync(0xffffffffu, tt, off);
    if (lane == 0) ws[wid] = tt;
    __syncthreads();
    if (wid == 0) {
      double u = lane < nw ? ws[lane] : 0.0;
      for (int off = 16; off > 0; off >>= 1) u += __shfl_xor_sync(0xffffffffu, u, off);
      if (t == 0) {
        *checksum = *checksum + u;
        *ticket = 0u;
      }
    }
  }
}

struct SU3StagedTraits : DefaultTraits {};  // persistent grid: the loop stays

// ---- warp-cooperative staging (OMPRT_WARP_STAGED): coalesced cp.async in, STG.128 out ----
constexpr int kSU3WarpThreads = 192;  // 6 warps x 2 x 32 slots x 592 B = 222 KB per team

template <class Tr, bool Checksum>
__global__ void __launch_bounds__(kSU3WarpThreads, 1)
    omprt_su3_wstaged_rt(const double* __restrict__ A, const double2* __restrict__ B,
                         double* __restrict__ Cm, typename Tr::Idx n_sites, double* checksum,
                         double* partials, unsigned* ticket) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  double acc = 0.0;
  distribute_parallel_for_warp_staged<Tr, kSU3Rec, kSU3Slot>(
      team, n_sites, reinterpret_cast<const unsigned char*>(A),
      reinterpret_cast<unsigned char*>(Cm),
      [&](Idx, unsigned char* slot) { acc += su3_site_slot(slot, B); });
  if constexpr (Checksum)
    league_reduce_threads(team, acc, Plus{}, checksum, partials,
                  ticket);
}

// Bare CUDA twin: the same warp tile pipeline, by hand.
template <bool Checksum>
__global__ void __launch_bounds__(kSU3WarpThreads, 1)
    cuda_su3_wstaged_twin(const double* __restrict__ A, const double2* __restrict__ B,
                          double* __restrict__ Cm, int32_t n_sites, double* checksum,
                          double* partials, unsigned* ticket) {
  constexpr unsigned kCh = kSU3Rec / 16;  // 36 chunks per site
  extern __shared__ __align__(128) unsigned char smem[];
  const unsigned nt = blockDim.x, t = threadIdx.x, lane = t & 31u, w0 = t & ~31u;
  unsigned char* buf0 = smem + w0 * kSU3Slot;
  unsigned char* buf1 = smem + (nt + w0) * kSU3Slot;
  const unsigned char* in = reinterpret_cast<const unsigned char*>(A);
  unsigned char* out = reinterpret_cast<unsigned char*>(Cm);
  const int32_t stride = gridDim.x * nt;
  int32_t base = blockIdx.x * nt + w0;
  double acc = 0.0;
  const uint32_t s0 = tma::smem_addr(buf0), s1 = tma::smem_addr(buf1);
  auto fetch = [&](uint32_t b, int32_t wb) {  // zero-fill past the tile: no branches
    const unsigned nch = (unsigned)min(32, n_sites - wb) * kCh;
    const unsigned char* src = in + (size_t)wb * kSU3Rec;
#pragma unroll
    for (unsigned j = 0; j < kCh; ++j) {
      const unsigned c = lane + 32u * j;
      const unsigned r = c / kCh, q = c - r * kCh;  // record, 16 B chunk of the record
      tma::cp_async16_zfill(b + r * kSU3Slot + q * 16u, src + (c < nch ? c * 16u : 0u),
                            c < nch ? 16u : 0u);
    }
    tma::cp_async_commit();
  };
  if (base < n_sites) fetch(s0, base);
  for (unsigned k = 0; base < n_sites; base += stride, ++k) {
    unsigned char* cur = (k & 1) ? buf1 : buf0;
    if (base + stride < n_sites) {
      fetch((k & 1) ? s0 : s1, base + stride);
      tma::cp_async_wait<1>();
    } else {
      tma::cp_async_wait<0>();
    }
    __syncwarp();
    if (base + (int32_t)lane < n_sites) acc += su3_site_slot(cur + lane * kSU3Slot, B);
    __syncwarp();
    const unsigned nch = (unsigned)min(32, n_sites - base) * kCh;
    unsigned char* dst = out + (size_t)base * kSU3Rec;
#pragma unroll
    for (unsigned j = 0; j < kCh; ++j) {
      const unsigned c = lane + 32u * j;
      if (c < nch) {
        const unsigned r = c / kCh, q = c - r * kCh;
        *reinterpret_cast<uint4*>(dst + c * 16u) =
            *reinterpret_cast<const uint4*>(cur + r * kSU3Slot + q * 16u);
      }
    }
    __syncwarp();
  }
  if constexpr (Checksum) twin_ticket_sum(acc, checksum, partials, ticket);
}

OMPRT_REGISTER_KERNEL(omprt_su3_wstaged_rt, omprt_su3_wstaged_rt<SU3StagedTraits, true>)
OMPRT_REGISTER_KERNEL(cuda_su3_wstaged_twin, cuda_su3_wstaged_twin<true>)

// ---- TMA tensor tiles (OMPRT_TMA_TILED): one 2-D tensor copy per warp tile in and out ----
// A and C as tensors [n_sites][72] of doubles; boxes [32][74]: the two columns past the
// record are zero-filled on the load (592 B padded slots) and skipped on the store
// (omprt/device/staging.cuh distribute_parallel_for_tma_tiles).  6 warps per team, one
// team per SM: 6 x 2 x 32 x 592 B + barriers = 227.4 KB of shared memory.
#ifndef OMPRT_SU3_TILED_WARPS
#define OMPRT_SU3_TILED_WARPS 6
#define OMPRT_SU3_TILED_BUFFERS 2
#endif
constexpr int kSU3TiledThreads = 32 * OMPRT_SU3_TILED_WARPS;
constexpr unsigned kSU3TiledBuffers = OMPRT_SU3_TILED_BUFFERS;
constexpr unsigned kSU3SlotDoubles = kSU3Slot / 8;  // 74

template <class Tr, bool Checksum>
__global__ void __launch_bounds__(kSU3TiledThreads, 1)
    omprt_su3_tiled_rt(const __grid_constant__ CUtensorMap tin,
                       const __grid_constant__ CUtensorMap tout, const double2* __restrict__ B,
                       typename Tr::Idx n_sites, double* checksum, double* partials,
                       unsigned* ticket) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  double acc = 0.0;
  distribute_parallel_for_tma_tiles<Tr, kSU3Slot, kSU3TiledBuffers>(
      team, n_sites, &tin, &tout,
      [&](Idx, unsigned char* slot) { acc += su3_site_slot(slot, B); });
  if constexpr (Checksum)
    league_reduce_threads(team, acc, Plus{}, checksum, partials,
                  ticket);
}

// Bare CUDA twin: the same per-warp tensor-tile pipeline, by hand.
template <bool Checksum>
__global__ void __launch_bounds__(kSU3TiledThreads, 1)
    cuda_su3_tiled_twin(const __grid_constant__ CUtensorMap tin,
                        const __grid_constant__ CUtensorMap tout, const double2* __restrict__ B,
                        int32_t n_sites, double* checksum, double* partials, unsigned* ticket) {
  constexpr uint32_t kBox = 32u * kSU3Slot;
  constexpr unsigned K = kSU3TiledBuffers;
  extern __shared__ __align__(128) unsigned char smem[];
  const unsigned nt = blockDim.x, t = threadIdx.x, lane = t & 31u, w0 = t & ~31u;
  unsigned char* const buf = smem + w0 * kSU3Slot;
  const unsigned bstride = nt * kSU3Slot;
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + K * nt * kSU3Slot) + K * (t >> 5);
  if (lane == 0) {
    for (unsigned j = 0; j < K; ++j) tma::mbar_init(bar + j, 1);
    tma::fence_mbar_init();
  }
  __syncwarp();
  const int32_t stride = gridDim.x * nt;
  const int32_t first = blockIdx.x * nt + w0;
  double acc = 0.0;
  if (lane == 0)
    for (unsigned j = 0; j + 1 < K; ++j)
      if (first + (int32_t)j * stride < n_sites) {
        tma::mbar_arrive_expect_tx(bar + j, kBox);
        tma::tensor_load_2d(buf + j * bstride, &tin, 0, first + j * stride, bar + j);
      }
  unsigned phases = 0, j = 0;
  for (int32_t base = first; base < n_sites; base += stride) {
    const int32_t ahead = base + (int32_t)(K - 1) * stride;
    const unsigned ja = j == 0 ? K - 1 : j - 1;
    if (ahead < n_sites && lane == 0) {
      tma::bulk_wait_read<0>();
      tma::mbar_arrive_expect_tx(bar + ja, kBox);
      tma::tensor_load_2d(buf + ja * bstride, &tin, 0, ahead, bar + ja);
    }
    tma::mbar_wait(bar + j, (phases >> j) & 1u);
    phases ^= 1u << j;
    unsigned char* const cur = buf + j * bstride;
    if (base + (int32_t)lane < n_sites) acc += su3_site_slot(cur + lane * kSU3Slot, B);
    tma::fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
      tma::tensor_store_2d(&tout, 0, base, cur);
      tma::bulk_commit();
    }
    j = j + 1 == K ? 0 : j + 1;
  }
  if (lane == 0) tma::bulk_wait<0>();
  if constexpr (Checksum) twin_ticket_sum(acc, checksum, partials, ticket);
}

OMPRT_REGISTER_KERNEL(omprt_su3_tiled_rt, omprt_su3_tiled_rt<SU3StagedTraits, true>)
OMPRT_REGISTER_KERNEL(cuda_su3_tiled_twin, cuda_su3_tiled_twin<true>)

// CUtensorMap of a [n][72]-double AoS array with [32][74] boxes (driver entry point fetched
// once through the runtime; no libcuda link dependency)
inline int su3_tensor_map(CUtensorMap* m, const double* base, int64_t n) {
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
  const cuuint64_t dims[2] = {kSU3Rec / 8, (cuuint64_t)n};
  const cuuint64_t strides[1] = {kSU3Rec};
  const cuuint32_t box[2] = {kSU3SlotDoubles, 32}, es[2] = {1, 1};
  const CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double*>(base), dims,
                         strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error(OMPRT_E_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return OMPRT_OK;
}

inline int su3_tiled_launch(bool twin, const double* A, const double* B, double* Cm, int64_t n,
                            double* ck, int32_t teams, Workspace* w, cudaStream_t s) {
  OMPRT_CHECK_ARG(((uintptr_t)A | (uintptr_t)Cm) % 16 == 0, "A and C must be 16 B aligned");
  CUtensorMap tin, tout;
  if (int r = su3_tensor_map(&tin, A, n)) return r;
  if (int r = su3_tensor_map(&tout, Cm, n)) return r;
  const uint32_t smem = tma_tiles_smem_bytes<kSU3Slot, kSU3TiledBuffers>(kSU3TiledThreads);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (teams <= 0) teams = sms;
  OMPRT_CHECK_ARG(!ck || (uint64_t)teams <= w->opt.max_teams, "teams exceed max_teams");
  OMPRT_CHECK_ARG(n + 2 * (int64_t)teams * kSU3TiledThreads < INT32_MAX, "n_sites too large");
  auto* b2 = (const double2*)B;
  double* p = (double*)w->partials;
  unsigned* tk = w->tickets + 3;
  const int32_t nn = (int32_t)n;
  auto go = [&](auto k) -> int {
    OMPRT_CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    k<<<teams, kSU3TiledThreads, smem, s>>>(tin, tout, b2, nn, ck, p, tk);
    return OMPRT_OK;
  };
  int r;
  if (twin) r = ck ? go(cuda_su3_tiled_twin<true>) : go(cuda_su3_tiled_twin<false>);
  else r = ck ? go(omprt_su3_tiled_rt<SU3StagedTraits, true>)
              : go(omprt_su3_tiled_rt<SU3StagedTraits, false>);
  if (r) return r;
  return check_launch(twin ? "cuda_su3_tiled_twin" : "omprt_su3_tiled_rt");
}

// persistent geometry: one team per SM, warp-cooperative cp.async (192 threads, 222 KB).
template <class K>
inline int su3_staged_go(K k, uint32_t smem, int32_t teams, int threads, const double* A,
                         const double2* B, double* Cm, int32_t n, double* ck, double* p,
                         unsigned* tk, cudaStream_t s) {
  OMPRT_CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  k<<<teams, threads, smem, s>>>(A, B, Cm, n, ck, p, tk);
  return OMPRT_OK;
}

inline int su3_staged_launch(bool twin, const double* A, const double* B, double* Cm, int64_t n,
                             double* ck, int32_t teams, Workspace* w, cudaStream_t s) {
  const int threads = kSU3WarpThreads;
  const uint32_t smem = warp_staged_smem_bytes<kSU3Slot>(kSU3WarpThreads);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (teams <= 0) teams = sms;
  OMPRT_CHECK_ARG(!ck || (uint64_t)teams <= w->opt.max_teams, "teams exceed max_teams");
  OMPRT_CHECK_ARG(n + 2 * (int64_t)teams * threads < INT32_MAX, "n_sites too large");
  const int32_t nn = (int32_t)n;
  auto* b2 = (const double2*)B;
  double* p = (double*)w->partials;
  unsigned* tk = w->tickets + 3;
  int r;
  if (twin)
    r = su3_staged_go(ck ? cuda_su3_wstaged_twin<true> : cuda_su3_wstaged_twin<false>, smem,
                      teams, threads, A, b2, Cm, nn, ck, p, tk, s);
  else
    r = su3_staged_go(ck ? omprt_su3_wstaged_rt<SU3StagedTraits, true>
                         : omprt_su3_wstaged_rt<SU3StagedTraits, false>,
                      smem, teams, threads, A, b2, Cm, nn, ck, p, tk, s);
  if (r) return r;
  return check_launch(twin ? "cuda_su3_wstaged_twin" : "omprt_su3_wstaged_rt");
}

}  // namespace omprt_kernels
