// C3 (BASELINE configs[2], the headline): XSBench-shaped lookups as
//   #pragma omp target teams distribute parallel for
//   for (i = first; i < first + count; ++i) verification[i - first] = lookup(i);
// runtime-driven (omprt, with / without the oversubscription assumption) and
// the bare CUDA twin (XSBench's CUDA version: one lookup per thread).  The verification
// sum runs as a separate kernel (K11), or fused (OMPRT_FUSED_REDUCTION).  Both read
// either the tables as specified or their B200 layouts (omprt_xs_build_accel).
#pragma once
#include "../host/runtime.cuh"
#include "xs_body.cuh"
#include "xs_derive.cuh"

namespace omprt_kernels {

using namespace omprt;

struct XSTraits : DefaultTraits {};
struct XSTraitsAssume : DefaultTraits {
  static constexpr bool assume_teams_oversub = true;
};
struct XSTraitsDebug : DefaultTraits {
  static constexpr unsigned debug = dbg::Assert | dbg::Trace;
};
struct XSTraitsAssumeDebug : XSTraitsAssume {
  static constexpr unsigned debug = dbg::Assert | dbg::Trace;
};

constexpr int kXSThreads = 256;
static_assert(kXSThreads == kXSFlatThreads, "XSFlatLookup::flat_acc_slot is sized for it");
// 4 teams of 256 per SM (<= 64 registers): measured best occupancy / memory-parallelism
// trade-off for this latency-bound gather (scripts/experiments/xs_explore.*).
constexpr int kXSMinBlocks = 4;   // plain layout
constexpr int kXSMinBlocksAccel = 3;  // B200 layouts: 78 registers, no spills (x04)

template <class Tr, bool Fused, bool Accel, bool Macro = false>
__global__ void __launch_bounds__(kXSThreads, Accel ? kXSMinBlocksAccel : kXSMinBlocks)
    omprt_xs_rt(const __grid_constant__ XSTables t, uint64_t seed, int64_t first,
                typename Tr::Idx count, uint64_t* __restrict__ verification,
                unsigned long long* checksum, unsigned long long* partials, unsigned* ticket,
                double* __restrict__ macro = nullptr) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  unsigned long long acc = 0;
  distribute_parallel_for(team, count, [&](Idx iv) {
    const uint64_t v = xs_lookup_one<Accel, Macro>(t, seed, first + iv, macro + (int64_t)iv * 5);
    if constexpr (Fused) acc += v;
    else verification[iv] = v;
  });
  if constexpr (Fused)
    league_reduce_threads(team, acc, Plus{}, checksum, partials,
                  ticket);
}

// The twins' hand-written league reduction of a u64 (the same algorithm as the runtime's:
// warp butterflies, per-warp partials, block partial, ticket, last block folds in order).
// Every thread of the block calls it.
__device__ __forceinline__ void twin_u64_ticket_sum(unsigned long long v,
                                                    unsigned long long* checksum,
                                                    unsigned long long* partials,
                                                    unsigned* ticket) {
  __shared__ unsigned long long ws[32];
  __shared__ unsigned last;
  for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
  const unsigned lane = threadIdx.x & 31u, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (lane == 0) ws[wid] = v;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long b = 0;
    for (unsigned k = 0; k < nw; ++k) b += ws[k];
    partials[blockIdx.x] = b;
    __threadfence();
    last = atomicAdd(ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (last) {
    __threadfence();
    unsigned long long s = 0;
    for (unsigned k = threadIdx.x; k < gridDim.x; k += blockDim.x) s += __ldcg(partials + k);
    for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    __syncthreads();
    if (lane == 0) ws[wid] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long b = 0;
      for (unsigned k = 0; k < nw; ++k) b += ws[k];
      *checksum += b;
      *ticket = 0u;
    }
  }
}

// XSBench's CUDA kernel shape: one lookup per thread, early return past the end; the fused
// variant hand-codes the same reduction algorithm as the runtime.
template <bool Fused, bool Accel, bool Macro = false>
__global__ void __launch_bounds__(kXSThreads, Accel ? kXSMinBlocksAccel : kXSMinBlocks)
    cuda_xs_twin(const __grid_constant__ XSTables t, uint64_t seed, int64_t first, int32_t count,
                 uint64_t* __restrict__ verification, unsigned long long* checksum,
                 unsigned long long* partials, unsigned* ticket,
                 double* __restrict__ macro = nullptr) {
  const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if constexpr (!Fused) {
    if (i >= count) return;
    verification[i] = xs_lookup_one<Accel, Macro>(t, seed, first + i, macro + (int64_t)i * 5);
  } else {
    const unsigned long long v = i < count ? xs_lookup_one<Accel>(t, seed, first + i) : 0ull;
    twin_u64_ticket_sum(v, checksum, partials, ticket);
  }
}

// ---- flattened execution (OMPRT_XS_FLAT): a persistent grid, each thread runs its Fig. 5
// iterations through omprt::distribute_parallel_for_flat (B200 layouts required).  4 teams
// of 256 per SM (64 registers): measured best (profiles/xs_explore_x14*, x16*).  With
// Smem, the team first copies the material tables into team-shared memory (the runtime's
// team_local + for_static + team barrier; the twin: __shared__ + loop + __syncthreads).
constexpr int kXSMinBlocksFlat = 4;
constexpr int kXSMatSmem = 12 * 48;  // entries: up to 48 nuclides per material (small: 34)

constexpr unsigned kXSMatsSite = 10, kXSConcsSite = 11;  // team_local sites

// OMPRT_SCHED_DYNAMIC: schedule(dynamic, kXSDynChunk) instead of Fig. 5 (reading R-D1)
constexpr int kXSDynChunk = 8;

template <class Tr, bool Fused, bool Smem, bool Dyn = false, bool Macro = false>
__global__ void __launch_bounds__(kXSThreads, kXSMinBlocksFlat)
    omprt_xs_flat_rt(const __grid_constant__ XSTables t, uint64_t seed, int64_t first,
                     typename Tr::Idx count, uint64_t* __restrict__ verification,
                     unsigned long long* checksum, unsigned long long* partials,
                     unsigned* ticket, double* __restrict__ macro = nullptr) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  const int32_t* mats = t.mats;
  const double* concs = t.concs;
  if constexpr (Smem) {
    int32_t* sm = team_local<int32_t, kXSMatSmem, kXSMatsSite>();
    double* sc = team_local<double, kXSMatSmem, kXSConcsSite>();
    for_static(team, (Idx)(12 * t.max_num_nucs), [&](Idx k) {
      sm[k] = __ldg(t.mats + k);
      sc[k] = __ldg(t.concs + k);
    });
    aligned_barrier();
    mats = sm;
    concs = sc;
  }
  using Lookup = XSFlatLookup<Fused, Smem, Macro>;
  if constexpr (Fused) *Lookup::flat_acc_slot() = 0ull;
  Lookup lookup(t, seed, first, verification, mats, concs, macro);
  if constexpr (Dyn) distribute_parallel_for_dynamic_flat(team, count, (Idx)kXSDynChunk, lookup);
  else distribute_parallel_for_flat(team, count, lookup);
  if constexpr (Fused)
    league_reduce_threads(team, *Lookup::flat_acc_slot(), Plus{},
                  checksum, partials, ticket);
}

// Bare CUDA twin: the same flattened loop written by hand around the same body.
template <bool Fused, bool Smem, bool Dyn = false, bool Macro = false>
__global__ void __launch_bounds__(kXSThreads, kXSMinBlocksFlat)
    cuda_xs_flat_twin(const __grid_constant__ XSTables t, uint64_t seed, int64_t first,
                      int32_t count, uint64_t* __restrict__ verification,
                      unsigned long long* checksum, unsigned long long* partials,
                      unsigned* ticket, double* __restrict__ macro = nullptr) {
  const int32_t* mats = t.mats;
  const double* concs = t.concs;
  if constexpr (Smem) {
    __shared__ int32_t sm[kXSMatSmem];
    __shared__ double sc[kXSMatSmem];
    for (int k = threadIdx.x; k < 12 * t.max_num_nucs; k += blockDim.x) {
      sm[k] = __ldg(t.mats + k);
      sc[k] = __ldg(t.concs + k);
    }
    __syncthreads();
    mats = sm;
    concs = sc;
  }
  using Lookup = XSFlatLookup<Fused, Smem, Macro>;
  if constexpr (Fused) *Lookup::flat_acc_slot() = 0ull;
  Lookup lookup(t, seed, first, verification, mats, concs, macro);
  if constexpr (Dyn) {  // team block + team-shared chunk counter, by hand
    __shared__ unsigned next;
    const int32_t per = (count + (int32_t)gridDim.x - 1) / (int32_t)gridDim.x;
    const int32_t lo = min((int32_t)blockIdx.x * per, count);
    const int32_t hi = min(lo + per, count);
    if (threadIdx.x == 0) next = blockDim.x;
    __syncthreads();
    int32_t i = lo + (int32_t)threadIdx.x * kXSDynChunk;
    while (i < hi) {
      const int32_t end = min(i + kXSDynChunk, hi);
      lookup.begin(i, 1);
      for (;;) {
        if (lookup.step()) continue;
        lookup.end(i);
        if (++i >= end) break;
        lookup.next(i);
      }
      i = lo + (int32_t)atomicAdd(&next, 1u) * kXSDynChunk;
    }
    if constexpr (Fused)
      twin_u64_ticket_sum(*Lookup::flat_acc_slot(), checksum, partials, ticket);
    return;
  }
  const int32_t stride = (int32_t)gridDim.x * (int32_t)blockDim.x;
  int32_t i = (int32_t)blockIdx.x * (int32_t)blockDim.x + (int32_t)threadIdx.x;
  auto run = [&]() {
    lookup.begin(i, stride);
    for (;;) {
      if (lookup.step()) continue;
      lookup.end(i);
      i += stride;
      if (i >= count) break;
      lookup.next(i);
    }
  };
  if constexpr (!Fused) {
    if (i >= count) return;
    run();
  } else {
    if (i < count) run();
    twin_u64_ticket_sum(*Lookup::flat_acc_slot(), checksum, partials, ticket);
  }
}

// K11: verification sum, a runtime-driven SPMD reduction over a full-device grid.
struct SumTraits : DefaultTraits {
  static constexpr unsigned unroll = 8;
};
template <class Tr>
__global__ void __launch_bounds__(512)
    omprt_u64_sum_rt(const unsigned long long* __restrict__ v, typename Tr::Idx n,
                     unsigned long long* out, unsigned long long* partials, unsigned* ticket) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  unsigned long long acc = 0;
  distribute_parallel_for(team, n, [&](Idx i) { acc += __ldg(v + i); });
  league_reduce_threads(team, acc, Plus{}, out, partials, ticket);
}

OMPRT_REGISTER_KERNEL(omprt_xs_rt, omprt_xs_rt<XSTraits, false, false>)
OMPRT_REGISTER_KERNEL(omprt_xs_rt_assume, omprt_xs_rt<XSTraitsAssume, false, false>)
OMPRT_REGISTER_KERNEL(omprt_xs_rt_fused, omprt_xs_rt<XSTraitsAssume, true, false>)
OMPRT_REGISTER_KERNEL(omprt_xs_rt_debug, omprt_xs_rt<XSTraitsDebug, false, false>)
OMPRT_REGISTER_KERNEL(omprt_xs_rt_accel, omprt_xs_rt<XSTraits, false, true>)
OMPRT_REGISTER_KERNEL(omprt_xs_rt_assume_accel, omprt_xs_rt<XSTraitsAssume, false, true>)
OMPRT_REGISTER_KERNEL(omprt_xs_rt_fused_accel, omprt_xs_rt<XSTraitsAssume, true, true>)
OMPRT_REGISTER_KERNEL(omprt_xs_flat_rt, omprt_xs_flat_rt<XSTraits, false, true>)
OMPRT_REGISTER_KERNEL(omprt_xs_flat_rt_fused, omprt_xs_flat_rt<XSTraits, true, true>)
OMPRT_REGISTER_KERNEL(omprt_xs_flat_rt_gmem, omprt_xs_flat_rt<XSTraits, false, false>)
OMPRT_REGISTER_KERNEL(cuda_xs_flat_twin, cuda_xs_flat_twin<false, true>)
OMPRT_REGISTER_KERNEL(cuda_xs_flat_twin_fused, cuda_xs_flat_twin<true, true>)
OMPRT_REGISTER_KERNEL(cuda_xs_flat_twin_gmem, cuda_xs_flat_twin<false, false>)
OMPRT_REGISTER_KERNEL(omprt_xs_dflat_rt, omprt_xs_flat_rt<XSTraits, false, true, true>)
OMPRT_REGISTER_KERNEL(cuda_xs_dflat_twin, cuda_xs_flat_twin<false, true, true>)
OMPRT_REGISTER_KERNEL(cuda_xs_twin, cuda_xs_twin<false, false>)
OMPRT_REGISTER_KERNEL(cuda_xs_twin_fused, cuda_xs_twin<true, false>)
OMPRT_REGISTER_KERNEL(cuda_xs_twin_accel, cuda_xs_twin<false, true>)
OMPRT_REGISTER_KERNEL(cuda_xs_twin_fused_accel, cuda_xs_twin<true, true>)
OMPRT_REGISTER_KERNEL(omprt_u64_sum_rt, omprt_u64_sum_rt<SumTraits>)

inline XSTables to_dev(const omprt_xs_tables& a) {
  return XSTables{a.nuclide_grid, a.unionized, a.index_grid, a.num_nucs, a.mats, a.concs,
                  a.n_isotopes, a.n_gridpoints, a.max_num_nucs, 0, a.n_union,
                  a.bins, a.index_grid16, a.brackets, a.log2_bins, 0};
}

// Launch configuration of the flattened kernels: the persistent grid, plus (unless
// OMPRT_XS_NO_L2_PERSIST) an L2 access-policy window that makes the bracket records -- the
// bulk of the L2 sectors a lookup touches, 36.9 MB for the small problem -- persisting in
// the set-aside granted by omprt_l2_set_aside (none: no window), so the 16-bit index grid's misses cannot evict
// them; hitRatio scales down when the table exceeds the set-aside.  (Persisting lines
// outlive the launch: omprt_l2_reset_persisting returns them to normal.)
// The window is a STREAM attribute set around the one launch and restored after it (not a
// launch attribute): Nsight Compute drops launch attributes when it replays a kernel, so
// only this form lets ncu measure the launch exactly as it is timed (profiles/README.md).
struct FlatLaunch {
  cudaLaunchConfig_t cfg;
  bool window = false;
  cudaStreamAttrValue win{};
};
// Sets the window on the launch stream for the lifetime of the object, then restores the
// stream's previous window.
struct ScopedStreamWindow {
  cudaStream_t s;
  bool on;
  cudaStreamAttrValue prev{};
  ScopedStreamWindow(const FlatLaunch& L) : s(L.cfg.stream), on(L.window) {
    if (on && cudaStreamGetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &prev) ==
                  cudaSuccess)
      on = cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &L.win) ==
           cudaSuccess;
    else
      on = false;
    cudaGetLastError();  // a stream without attribute support just runs without the window
  }
  ~ScopedStreamWindow() {
    if (on && cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &prev) !=
                  cudaSuccess)
      cudaGetLastError();
  }
};
inline FlatLaunch flat_launch(const omprt_xs_tables& t, int32_t teams, int32_t threads,
                              uint32_t flags, const Workspace* w, cudaStream_t s) {
  FlatLaunch L{};
  L.cfg.gridDim = dim3((unsigned)teams);
  L.cfg.blockDim = dim3((unsigned)threads);
  L.cfg.dynamicSmemBytes = 0;
  L.cfg.stream = s;
  L.cfg.attrs = nullptr;
  L.cfg.numAttrs = 0;
  const size_t br = sizeof(double) * 12ull * t.n_isotopes * (t.n_gridpoints - 1);
  if (!(flags & OMPRT_XS_NO_L2_PERSIST) && w->l2_persist_bytes > 0 && t.brackets) {
    int dev = 0, maxwin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, dev);
    // the other hot read-only tables join the window when they lie just below the bracket
    // records (one allocation: [unionized | bins | brackets], XSDeviceTables' layout): the
    // bisection probes then hit persisting lines too
    uintptr_t lo = (uintptr_t)t.brackets;
    const uintptr_t hi = lo + br;
    auto join = [&](const void* p, size_t n) {
      const uintptr_t a = (uintptr_t)p;
      if (p && a < lo && a + n <= lo && lo - (a + n) <= 4096 && hi - a <= (size_t)maxwin &&
          hi - a <= (size_t)w->l2_persist_bytes)
        lo = a;
    };
    join(t.bins, sizeof(int32_t) * ((1ull << t.log2_bins) + 1));
    join(t.unionized, sizeof(double) * (size_t)t.n_union);
    const size_t bytes = std::min((size_t)(hi - lo), (size_t)std::max(maxwin, 0));
    if (bytes > 0) {
      cudaAccessPolicyWindow& win = L.win.accessPolicyWindow;
      win.base_ptr = (void*)lo;
      win.num_bytes = bytes;
      win.hitRatio = (float)std::min(1.0, (double)w->l2_persist_bytes / (double)bytes);
      win.hitProp = cudaAccessPropertyPersisting;
      win.missProp = cudaAccessPropertyStreaming;
      L.window = true;
    }
  }
  return L;
}

// the flattened kernels keep the material tables in team-shared memory when they fit
inline bool xs_mats_fit_smem(const omprt_xs_tables& t) {
  return 12ll * t.max_num_nucs <= kXSMatSmem;
}

// The flattened kernels: runtime-driven (Twin = false) or twin, by (fused, team-shared
// material tables, dynamic schedule, macroscopic-xs output of the test build).
template <bool Twin, bool F, bool S, bool D, bool M>
inline cudaError_t xs_flat_launch(const cudaLaunchConfig_t& cfg, const XSTables& d, uint64_t seed,
                                  int64_t first, int32_t n, uint64_t* ver, unsigned long long* ck,
                                  unsigned long long* p, unsigned* tk, double* mac) {
  if constexpr (Twin)
    return cudaLaunchKernelEx(&cfg, cuda_xs_flat_twin<F, S, D, M>, d, seed, first, n, ver, ck,
                              p, tk, mac);
  else
    return cudaLaunchKernelEx(&cfg, omprt_xs_flat_rt<XSTraits, F, S, D, M>, d, seed, first, n,
                              ver, ck, p, tk, mac);
}
template <bool Twin>
inline cudaError_t xs_flat_dispatch(uint32_t flags, bool fused, bool smem,
                                    const cudaLaunchConfig_t& cfg, const XSTables& d,
                                    uint64_t seed, int64_t first, int32_t n, uint64_t* ver,
                                    unsigned long long* ck, unsigned long long* p,
                                    unsigned* tk, double* mac) {
  const bool dyn = flags & OMPRT_SCHED_DYNAMIC;
  if (mac) {  // test build: unfused only (xs_validate)
    if (smem && dyn) return xs_flat_launch<Twin, false, true, true, true>(cfg, d, seed, first, n, ver, ck, p, tk, mac);
    if (smem) return xs_flat_launch<Twin, false, true, false, true>(cfg, d, seed, first, n, ver, ck, p, tk, mac);
    if (dyn) return xs_flat_launch<Twin, false, false, true, true>(cfg, d, seed, first, n, ver, ck, p, tk, mac);
    return xs_flat_launch<Twin, false, false, false, true>(cfg, d, seed, first, n, ver, ck, p, tk, mac);
  }
#define OMPRT_XSF(F, S, D) \
  if (fused == F && smem == S && dyn == D) \
    return xs_flat_launch<Twin, F, S, D, false>(cfg, d, seed, first, n, ver, ck, p, tk, mac);
#define OMPRT_XSF2(F, S) OMPRT_XSF(F, S, false) OMPRT_XSF(F, S, true)
  OMPRT_XSF2(false, false) OMPRT_XSF2(false, true) OMPRT_XSF2(true, false) OMPRT_XSF2(true, true)
#undef OMPRT_XSF2
#undef OMPRT_XSF
  return cudaErrorInvalidValue;
}

inline bool xs_has_accel(const omprt_xs_tables& t) {
  return t.bins != nullptr && t.index_grid16 != nullptr && t.brackets != nullptr;
}

inline int xs_validate(const omprt_xs_tables& t, int64_t count, uint64_t* ver, uint64_t* ck,
                       double* macro, int32_t& teams, int32_t threads, uint32_t flags,
                       Workspace* w) {
  OMPRT_CHECK_ARG(count >= 0 && count < (1ll << 31), "count must be in [0, 2^31)");
  OMPRT_CHECK_ARG(threads == kXSThreads, "threads must be %d", kXSThreads);
  OMPRT_CHECK_ARG(t.unionized && t.num_nucs && t.mats && t.concs && t.n_union >= 2 &&
                      t.n_union < (1ll << 31) && t.n_gridpoints >= 2 && t.n_isotopes > 0,
                  "bad XSBench tables");
  const bool accel = xs_has_accel(t);
  OMPRT_CHECK_ARG(accel || (t.nuclide_grid && t.index_grid), "bad XSBench tables");
  OMPRT_CHECK_ARG(!accel || (t.log2_bins >= 1 && t.log2_bins <= 28),
                  "accelerated layout: bad log2_bins");
  OMPRT_CHECK_ARG(accel || (!t.bins && !t.index_grid16 && !t.brackets),
                  "accelerated layout: bins, index_grid16 and brackets go together");
  const bool fused = flags & OMPRT_FUSED_REDUCTION;
  OMPRT_CHECK_ARG(!macro || (!fused && !(flags & OMPRT_DEBUG_BUILD)),
                  "macro (test build) is written by the unfused release kernels only");
  OMPRT_CHECK_ARG(fused ? ck != nullptr : (ver != nullptr || count == 0),
                  fused ? "fused reduction needs checksum_inout" : "verification is required");
  OMPRT_CHECK_ARG(!(flags & OMPRT_SCHED_DYNAMIC) || (flags & OMPRT_XS_FLAT),
                  "OMPRT_SCHED_DYNAMIC is implemented for the flattened loop (OMPRT_XS_FLAT)");
  if (flags & OMPRT_XS_FLAT) {
    OMPRT_CHECK_ARG(accel, "OMPRT_XS_FLAT needs the B200 layouts (omprt_xs_build_accel)");
    OMPRT_CHECK_ARG(!(flags & (OMPRT_ASSUME_OVERSUB | OMPRT_DEBUG_BUILD)),
                    "OMPRT_XS_FLAT runs a persistent grid (no assumption, release build)");
    if (teams <= 0) {  // persistent: the resident teams of the whole device
      int dev = 0, sms = 148, per_sm = kXSMinBlocksFlat;
      cudaGetDevice(&dev);
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(
          &per_sm, omprt_xs_flat_rt<XSTraits, false, true>, kXSThreads, 0);
      teams = (int32_t)std::max<int64_t>(
          1, std::min<int64_t>((int64_t)sms * std::max(per_sm, 1), ceil_div(count, threads)));
    }
  }
  if (teams <= 0) teams = (int32_t)std::max<int64_t>(1, ceil_div(count, threads));
  OMPRT_CHECK_ARG(!fused || (uint64_t)teams <= w->opt.max_teams, "teams exceed max_teams");
  OMPRT_CHECK_ARG(!(flags & OMPRT_ASSUME_OVERSUB) || count <= (int64_t)teams * threads,
                  "oversubscription assumption violated: count=%lld > teams*threads=%lld",
                  (long long)count, (long long)teams * threads);
  OMPRT_CHECK_ARG(count + 2 * (int64_t)teams * threads < INT32_MAX, "iteration space too large");
  return OMPRT_OK;
}

inline int launch_u64_sum(const uint64_t* v, int64_t n, uint64_t* out, Workspace* w,
                          cudaStream_t s) {
  OMPRT_CHECK_ARG(n >= 0 && out && (v || n == 0), "omprt_u64_sum: bad arguments");
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // a full-device grid: 4 teams of 512 per SM (sized in multiples of the SM count)
  int64_t teams = std::min<int64_t>((int64_t)sms * 4, std::max<int64_t>(1, ceil_div(n, 512)));
  if (n + 10 * teams * 512 < INT32_MAX)
    omprt_u64_sum_rt<SumTraits><<<(int)teams, 512, 0, s>>>(
        (const unsigned long long*)v, (int32_t)n, (unsigned long long*)out,
        (unsigned long long*)w->partials, w->tickets + 2);
  else
    omprt_u64_sum_rt<WithIdx64<SumTraits>><<<(int)teams, 512, 0, s>>>(
        (const unsigned long long*)v, n, (unsigned long long*)out,
        (unsigned long long*)w->partials, w->tickets + 2);
  return check_launch("omprt_u64_sum_rt");
}

inline int xs_accel_sizes(int32_t n_isotopes, int32_t n_gridpoints, int64_t n_union,
                          int32_t log2_bins, uint64_t* sizes) {
  OMPRT_CHECK_ARG(n_isotopes > 0 && n_gridpoints >= 2 && n_gridpoints <= 65536 &&
                      n_union >= 2 && log2_bins >= 1 && log2_bins <= 28 && sizes,
                  "omprt_xs_accel_sizes: bad arguments (n_gridpoints must be <= 65536)");
  sizes[0] = sizeof(int32_t) * ((1ull << log2_bins) + 1);
  sizes[1] = sizeof(uint16_t) * (uint64_t)n_union * n_isotopes;
  sizes[2] = sizeof(double) * 12ull * n_isotopes * (n_gridpoints - 1);
  return OMPRT_OK;
}

inline int launch_xs_accel(omprt_xs_tables* t, int32_t* bins, uint16_t* idx16, double* brackets,
                           int32_t log2_bins, cudaStream_t s) {
  uint64_t sz[3];
  if (int r = xs_accel_sizes(t->n_isotopes, t->n_gridpoints, t->n_union, log2_bins, sz)) return r;
  OMPRT_CHECK_ARG(t->nuclide_grid && t->unionized && t->index_grid && bins && idx16 && brackets,
                  "omprt_xs_build_accel: null pointer");
  OMPRT_CHECK_ARG((uintptr_t)brackets % 32 == 0, "brackets must be 32 B aligned");
  OMPRT_CHECK_ARG((uintptr_t)t->nuclide_grid % 16 == 0, "nuclide_grid must be 16 B aligned");
  xs_build_bins<<<1024, 256, 0, s>>>(t->unionized, (int32_t)t->n_union, log2_bins, bins);
  xs_build_index16<<<2048, 256, 0, s>>>(t->index_grid, idx16,
                                        (int64_t)t->n_union * t->n_isotopes);
  xs_build_brackets<<<2048, 256, 0, s>>>(t->nuclide_grid, brackets, t->n_isotopes,
                                         t->n_gridpoints);
  if (int r = check_launch("xs_build_accel")) return r;
  t->bins = bins;
  t->index_grid16 = idx16;
  t->brackets = brackets;
  t->log2_bins = log2_bins;
  return OMPRT_OK;
}

}  // namespace omprt_kernels

extern "C" int omprt_xs_lookup(omprt_xs_tables t, uint64_t seed, int64_t first, int64_t count,
                               uint64_t* verification, uint64_t* checksum_inout, double* macro,
                               int32_t teams, int32_t threads, uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  if (int r = xs_validate(t, count, verification, checksum_inout, macro, teams, threads, flags,
                          w))
    return r;
  if (count == 0) return OMPRT_OK;
  cudaStream_t s = as_stream(stream);
  const XSTables d = to_dev(t);
  const bool assume = flags & OMPRT_ASSUME_OVERSUB, fused = flags & OMPRT_FUSED_REDUCTION,
             debug = flags & OMPRT_DEBUG_BUILD, accel = xs_has_accel(t);
  auto* ck = (unsigned long long*)checksum_inout;
  auto* p = (unsigned long long*)w->partials;
  unsigned* tk = w->tickets + 1;
  const int32_t n = (int32_t)count;
  if (flags & OMPRT_XS_FLAT) {
    const bool smem = xs_mats_fit_smem(t);
    const FlatLaunch L = flat_launch(t, teams, threads, flags, w, s);
    ScopedStreamWindow sw(L);
    xs_flat_dispatch<false>(flags, fused, smem, L.cfg, d, seed, first, n, verification, ck, p,
                            tk, macro);
    return check_launch("omprt_xs_flat_rt");
  }
#define OMPRT_XS(TR, F, A) \
  omprt_xs_rt<TR, F, A><<<teams, threads, 0, s>>>(d, seed, first, n, verification, ck, p, tk)
#define OMPRT_XSM(TR, A) \
  omprt_xs_rt<TR, false, A, true><<<teams, threads, 0, s>>>(d, seed, first, n, verification, \
                                                           ck, p, tk, macro)
  if (macro) {  // test build: the macroscopic cross sections too
    if (accel && assume) OMPRT_XSM(XSTraitsAssume, true);
    else if (accel) OMPRT_XSM(XSTraits, true);
    else if (assume) OMPRT_XSM(XSTraitsAssume, false);
    else OMPRT_XSM(XSTraits, false);
  } else if (debug) {
    OMPRT_CHECK_ARG(!fused && !accel, "the debug build covers the plain, unfused kernel");
    if (assume) OMPRT_XS(XSTraitsAssumeDebug, false, false);
    else OMPRT_XS(XSTraitsDebug, false, false);
  } else if (accel) {
    if (fused && assume) OMPRT_XS(XSTraitsAssume, true, true);
    else if (fused) OMPRT_XS(XSTraits, true, true);
    else if (assume) OMPRT_XS(XSTraitsAssume, false, true);
    else OMPRT_XS(XSTraits, false, true);
  } else {
    if (fused && assume) OMPRT_XS(XSTraitsAssume, true, false);
    else if (fused) OMPRT_XS(XSTraits, true, false);
    else if (assume) OMPRT_XS(XSTraitsAssume, false, false);
    else OMPRT_XS(XSTraits, false, false);
  }
#undef OMPRT_XSM
#undef OMPRT_XS
  return check_launch("omprt_xs_rt");
}

extern "C" int omprt_cuda_xs_lookup(omprt_xs_tables t, uint64_t seed, int64_t first,
                                    int64_t count, uint64_t* verification,
                                    uint64_t* checksum_inout, double* macro, int32_t teams,
                                    int32_t threads, uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  // the twin runs one lookup per thread, or (OMPRT_XS_FLAT) the same persistent grid
  const bool flat = flags & OMPRT_XS_FLAT;
  int32_t tm = flat ? teams : 0;
  if (int r = xs_validate(t, count, verification, checksum_inout, macro, tm, threads,
                          flags & ~(OMPRT_ASSUME_OVERSUB | OMPRT_DEBUG_BUILD), w))
    return r;
  if (count == 0) return OMPRT_OK;
  cudaStream_t s = as_stream(stream);
  const XSTables d = to_dev(t);
  const bool fused = flags & OMPRT_FUSED_REDUCTION, accel = xs_has_accel(t);
  auto* ck = (unsigned long long*)checksum_inout;
  auto* p = (unsigned long long*)w->partials;
  unsigned* tk = w->tickets + 1;
  const int32_t n = (int32_t)count;
  if (flat) {  // the same launch (geometry, L2 window) as the runtime-driven kernel
    const bool smem = xs_mats_fit_smem(t);
    const FlatLaunch L = flat_launch(t, tm, threads, flags, w, s);
    ScopedStreamWindow sw(L);
    unsigned long long* nul = nullptr;
    unsigned* nult = nullptr;
    if (fused)
      xs_flat_dispatch<true>(flags, fused, smem, L.cfg, d, seed, first, n, verification, ck, p,
                             tk, macro);
    else
      xs_flat_dispatch<true>(flags, fused, smem, L.cfg, d, seed, first, n, verification, nul,
                             nul, nult, macro);
    return check_launch("cuda_xs_flat_twin");
  }
  if (macro && accel) cuda_xs_twin<false, true, true><<<tm, threads, 0, s>>>(d, seed, first, n, verification, nullptr, nullptr, nullptr, macro);
  else if (macro) cuda_xs_twin<false, false, true><<<tm, threads, 0, s>>>(d, seed, first, n, verification, nullptr, nullptr, nullptr, macro);
  else if (fused && accel) cuda_xs_twin<true, true><<<tm, threads, 0, s>>>(d, seed, first, n, verification, ck, p, tk);
  else if (fused) cuda_xs_twin<true, false><<<tm, threads, 0, s>>>(d, seed, first, n, verification, ck, p, tk);
  else if (accel) cuda_xs_twin<false, true><<<tm, threads, 0, s>>>(d, seed, first, n, verification, nullptr, nullptr, nullptr);
  else cuda_xs_twin<false, false><<<tm, threads, 0, s>>>(d, seed, first, n, verification, nullptr, nullptr, nullptr);
  return check_launch("cuda_xs_twin");
}

extern "C" int omprt_u64_sum(const uint64_t* v, int64_t n, uint64_t* out_inout, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  return launch_u64_sum(v, n, out_inout, w, as_stream(stream));
}

extern "C" int omprt_xs_accel_sizes(int32_t n_isotopes, int32_t n_gridpoints, int64_t n_union,
                                    int32_t log2_bins, uint64_t* sizes) {
  return omprt_kernels::xs_accel_sizes(n_isotopes, n_gridpoints, n_union, log2_bins, sizes);
}

extern "C" int omprt_xs_build_accel(omprt_xs_tables* t, int32_t* bins, uint16_t* index_grid16,
                                    double* brackets, int32_t log2_bins, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  OMPRT_CHECK_ARG(t != nullptr, "omprt_xs_build_accel: null tables");
  return launch_xs_accel(t, bins, index_grid16, brackets, log2_bins, as_stream(stream));
}

// End to end with HOST tables, `steps` times (an OpenMP `target map(to: tables)
// map(from: checksum)` per step): H2D of the tables -> the B200 layouts built on the device
// (bins always; the 16-bit index grid and the bracket records unless the host already holds
// them in that layout) -> lookups with the fused checksum -> D2H of the checksum.  Two
// device table slots, a copy stream and per-slot events let the H2D of step s+1 run while
// step s computes (`target nowait` with dependences).  Synchronous: returns when all steps
// are done.  Host tables should be pinned (pageable copies serialize).
extern "C" int omprt_xs_run_host_steps(omprt_xs_tables h, uint64_t seed, int64_t first,
                                       int64_t count, int32_t threads, uint32_t flags,
                                       int32_t steps, uint64_t* checksums_host,
                                       uint64_t* h2d_bytes, uint64_t* d2h_bytes, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  // derive: only the raw data crosses PCIe; the unionized and index grids are built here
  const bool derive = !h.unionized && !h.index_grid && !h.index_grid16;
  OMPRT_CHECK_ARG(checksums_host && steps >= 1 && steps <= kMaxE2ESteps && h.num_nucs &&
                      h.mats && h.concs && (h.nuclide_grid || h.brackets) &&
                      (derive ? h.nuclide_grid != nullptr
                              : (h.unionized && (h.index_grid || h.index_grid16))),
                  "omprt_xs_run_host_steps: bad arguments");
  OMPRT_CHECK_ARG(!derive || (int64_t)h.n_isotopes * h.n_gridpoints == h.n_union,
                  "derived tables: n_union must be n_isotopes * n_gridpoints");
  const bool accel =
      derive || (flags & (OMPRT_XS_ACCEL | OMPRT_XS_FLAT)) || h.index_grid16 || h.brackets;
  OMPRT_CHECK_ARG(accel || (h.index_grid && h.nuclide_grid),
                  "the plain path needs the int32 index grid and the nuclide grid");
  OMPRT_CHECK_ARG(!accel || h.n_gridpoints <= 65536, "16-bit index: n_gridpoints > 65536");
  // the material tables are host memory here: every listed nuclide must exist (a table
  // built for fewer nuclides than the material lists name would read past the grids)
  OMPRT_CHECK_ARG(h.max_num_nucs > 0, "omprt_xs_run_host_steps: max_num_nucs must be > 0");
  for (int m = 0; m < 12; ++m) {
    OMPRT_CHECK_ARG(h.num_nucs[m] >= 0 && h.num_nucs[m] <= h.max_num_nucs,
                    "material %d: num_nucs out of range", m);
    for (int k = 0; k < h.num_nucs[m]; ++k) {
      const int32_t q = h.mats[m * h.max_num_nucs + k];
      OMPRT_CHECK_ARG(q >= 0 && q < h.n_isotopes, "material %d lists nuclide %d of %d", m, q,
                      h.n_isotopes);
    }
  }
  cudaStream_t s = as_stream(stream);
  const int32_t log2_bins = 18;  // 2^18 search bins: ~1.5 bisection probes (profiles/l2_pack_x57.txt)
  uint64_t asz[3] = {0, 0, 0};
  if (accel) xs_accel_sizes(h.n_isotopes, h.n_gridpoints, h.n_union, log2_bins, asz);
  const bool up16 = accel && h.index_grid16, upbr = accel && h.brackets;
  const size_t n_grid = upbr ? 0 : (size_t)h.n_isotopes * h.n_gridpoints * 6 * sizeof(double);
  const size_t n_br = upbr ? asz[2] : 0;
  const size_t n_uni = derive ? 0 : (size_t)h.n_union * sizeof(double);
  const size_t n_idx =
      derive ? 0 : (up16 ? asz[1] : (size_t)h.n_union * h.n_isotopes * sizeof(int32_t));
  const size_t built_uni = derive ? (size_t)h.n_union * sizeof(double) : 0;
  if (derive) {
    uint64_t tb = 0;
    if (int r = omprt_xs_derive_tmp_bytes(h.n_isotopes, h.n_gridpoints, &tb)) return r;
    if (w->derive_tmp_bytes < tb) {
      OMPRT_CUDA_TRY(cudaDeviceSynchronize());
      cudaFree(w->derive_tmp);
      w->derive_tmp = nullptr;
      w->derive_tmp_bytes = 0;
      if (cudaMalloc(&w->derive_tmp, tb) != cudaSuccess) {
        cudaGetLastError();
        return set_error(OMPRT_E_NOMEM, "omprt_xs_run_host_steps: cannot allocate %llu B",
                         (unsigned long long)tb);
      }
      w->derive_tmp_bytes = tb;
    }
  }
  const size_t n_num = 12 * sizeof(int32_t);
  const size_t n_mat = (size_t)12 * h.max_num_nucs * sizeof(int32_t);
  const size_t n_con = (size_t)12 * h.max_num_nucs * sizeof(double);
  auto al = [](size_t b) { return (b + 255) & ~size_t(255); };
  // slot layout: uploaded tables, then the device-built layouts
  const size_t built16 = (accel && !up16) ? asz[1] : 0, builtbr = (accel && !upbr) ? asz[2] : 0;
  const size_t total = al(n_grid) + al(n_br) + al(n_uni) + al(n_idx) + al(n_num) + al(n_mat) +
                       al(n_con);
  const size_t total_built =
      accel ? al(asz[0]) + al(built16) + al(builtbr) + al(built_uni) : 0;
  if (w->xs_built_bytes < total_built) {
    OMPRT_CUDA_TRY(cudaDeviceSynchronize());
    for (int k = 0; k < 2; ++k) {
      cudaFree(w->xs_built[k]);
      w->xs_built[k] = nullptr;
    }
    w->xs_built_bytes = 0;
    if (cudaMalloc(&w->xs_built[0], total_built) != cudaSuccess ||
        cudaMalloc(&w->xs_built[1], total_built) != cudaSuccess) {
      cudaGetLastError();
      return set_error(OMPRT_E_NOMEM, "omprt_xs_run_host_steps: cannot allocate 2 x %zu B",
                       total_built);
    }
    w->xs_built_bytes = total_built;
  }
  if (!w->copy_stream) {
    OMPRT_CUDA_TRY(cudaStreamCreateWithFlags(&w->copy_stream, cudaStreamNonBlocking));
    for (int k = 0; k < 2; ++k) {
      OMPRT_CUDA_TRY(cudaEventCreateWithFlags(&w->copy_done[k], cudaEventDisableTiming));
      OMPRT_CUDA_TRY(cudaEventCreateWithFlags(&w->compute_done[k], cudaEventDisableTiming));
    }
    OMPRT_CUDA_TRY(cudaHostAlloc(&w->pinned_ck, kMaxE2ESteps * sizeof(uint64_t),
                                 cudaHostAllocDefault));
    OMPRT_CUDA_TRY(cudaMalloc(&w->dev_ck, kMaxE2ESteps * sizeof(uint64_t)));
  }
  if ((flags & OMPRT_XS_FLAT) && w->e2e_ver_n < (size_t)count) {
    OMPRT_CUDA_TRY(cudaDeviceSynchronize());
    cudaFree(w->e2e_ver);
    w->e2e_ver = nullptr;
    w->e2e_ver_n = 0;
    if (cudaMalloc(&w->e2e_ver, std::max<size_t>(count, 1) * sizeof(uint64_t)) != cudaSuccess) {
      cudaGetLastError();
      return set_error(OMPRT_E_NOMEM, "omprt_xs_run_host_steps: cannot allocate verification");
    }
    w->e2e_ver_n = std::max<size_t>(count, 1);
  }
  if (w->xs_buf_bytes < total) {
    OMPRT_CUDA_TRY(cudaDeviceSynchronize());
    for (int k = 0; k < 2; ++k) {
      cudaFree(w->xs_buf[k]);
      w->xs_buf[k] = nullptr;
    }
    w->xs_buf_bytes = 0;
    if (cudaMalloc(&w->xs_buf[0], total) != cudaSuccess ||
        cudaMalloc(&w->xs_buf[1], total) != cudaSuccess) {
      cudaGetLastError();
      return set_error(OMPRT_E_NOMEM, "omprt_xs_run_host_steps: cannot allocate 2 x %zu B",
                       total);
    }
    w->xs_buf_bytes = total;
  }
  // the previous call's work on the user stream is ordered before this call's copies
  OMPRT_CUDA_TRY(cudaEventRecord(w->compute_done[0], s));
  OMPRT_CUDA_TRY(cudaEventRecord(w->compute_done[1], s));
  OMPRT_CUDA_TRY(cudaMemsetAsync(w->dev_ck, 0, steps * sizeof(uint64_t), s));
  for (int32_t st = 0; st < steps; ++st) {
    const int b = st & 1;
    unsigned char* base = (unsigned char*)w->xs_buf[b];
    size_t off = 0;
    bool ok = true;
    cudaStream_t cs = w->copy_stream;
    ok = ok && cudaStreamWaitEvent(cs, w->compute_done[b], 0) == cudaSuccess;
    auto put = [&](const void* src, size_t bytes) -> void* {
      void* dst = base + off;
      off += al(bytes);
      if (bytes) ok = ok && cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, cs) ==
                                cudaSuccess;
      return dst;
    };
    omprt_xs_tables d = h;
    d.nuclide_grid = upbr ? nullptr : (const double*)put(h.nuclide_grid, n_grid);
    double* br = (double*)put(upbr ? h.brackets : nullptr, n_br);
    d.unionized = (const double*)put(h.unionized, n_uni);
    void* idx = put(up16 ? (const void*)h.index_grid16 : (const void*)h.index_grid, n_idx);
    d.num_nucs = (const int32_t*)put(h.num_nucs, n_num);
    d.mats = (const int32_t*)put(h.mats, n_mat);
    d.concs = (const double*)put(h.concs, n_con);
    if (!ok) return set_error(OMPRT_E_CUDA, "omprt_xs_run_host_steps: H2D copy failed");
    d.index_grid = (up16 || derive) ? nullptr : (const int32_t*)idx;
    d.bins = nullptr;
    d.index_grid16 = nullptr;
    d.brackets = nullptr;
    // the slot's device-built layouts are made on the copy stream too, right after its
    // H2D, so they overlap the previous step's lookups (two slots of built layouts)
    if (accel) {
      // [unionized | bins | brackets | index]: the hot read-only tables adjacent, so the
      // flattened launch's L2 window covers all three (flat_launch)
      unsigned char* bb = (unsigned char*)w->xs_built[b];
      size_t bo = 0;
      double* U = (double*)(bb + bo);
      bo += al(built_uni);
      int32_t* bins = (int32_t*)(bb + bo);
      bo += al(asz[0]);
      double* brk = upbr ? br : (double*)(bb + bo);
      bo += al(builtbr);
      uint16_t* i16 = up16 ? (uint16_t*)idx : (uint16_t*)(bb + bo);
      bo += al(built16);
      if (derive) {
        if (int r = xs_derive(d.nuclide_grid, d.n_isotopes, d.n_gridpoints, U, i16,
                              w->derive_tmp, w->derive_tmp_bytes, cs))
          return r;
        d.unionized = U;
      } else if (!up16) {
        xs_build_index16<<<2048, 256, 0, cs>>>(d.index_grid, i16,
                                               (int64_t)d.n_union * d.n_isotopes);
      }
      xs_build_bins<<<1024, 256, 0, cs>>>(d.unionized, (int32_t)d.n_union, log2_bins, bins);
      if (!upbr)
        xs_build_brackets<<<2048, 256, 0, cs>>>(d.nuclide_grid, brk, d.n_isotopes,
                                                d.n_gridpoints);
      if (int r = check_launch("xs_build_accel")) return r;
      d.bins = bins;
      d.index_grid16 = i16;
      d.brackets = brk;
      d.log2_bins = log2_bins;
    }
    OMPRT_CUDA_TRY(cudaEventRecord(w->copy_done[b], cs));
    OMPRT_CUDA_TRY(cudaStreamWaitEvent(s, w->copy_done[b], 0));
    if (flags & OMPRT_XS_FLAT) {
      // flattened: per-lookup verification + K11 sum (the fused flat kernel spills: its
      // extra live state does not fit the 64 registers of 4 teams per SM)
      if (int r = omprt_xs_lookup(d, seed, first, count, w->e2e_ver, nullptr, nullptr, 0, threads,
                                  flags & ~OMPRT_XS_ACCEL, stream))
        return r;
      if (int r = launch_u64_sum(w->e2e_ver, count, w->dev_ck + st, w, s)) return r;
    } else if (int r = omprt_xs_lookup(d, seed, first, count, nullptr, w->dev_ck + st, nullptr, 0,
                                       threads,
                                       (flags & ~OMPRT_XS_ACCEL) | OMPRT_FUSED_REDUCTION |
                                           OMPRT_ASSUME_OVERSUB,
                                       stream)) {
      return r;
    }
    OMPRT_CUDA_TRY(cudaMemcpyAsync(w->pinned_ck + st, w->dev_ck + st, sizeof(uint64_t),
                                   cudaMemcpyDeviceToHost, s));
    OMPRT_CUDA_TRY(cudaEventRecord(w->compute_done[b], s));
  }
  OMPRT_CUDA_TRY(cudaStreamSynchronize(s));
  memcpy(checksums_host, w->pinned_ck, steps * sizeof(uint64_t));
  if (h2d_bytes)
    *h2d_bytes = n_grid + n_br + n_uni + n_idx + n_num + n_mat + n_con;  // per step
  if (d2h_bytes) *d2h_bytes = sizeof(uint64_t);
  return OMPRT_OK;
}

extern "C" int omprt_xs_run_host(omprt_xs_tables h, uint64_t seed, int64_t first, int64_t count,
                                 int32_t threads, uint32_t flags, uint64_t* checksum_host,
                                 uint64_t* h2d_bytes, uint64_t* d2h_bytes, void* stream) {
  return omprt_xs_run_host_steps(h, seed, first, count, threads, flags, 1, checksum_host,
                                 h2d_bytes, d2h_bytes, stream);
}
