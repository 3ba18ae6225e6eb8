// C4 (BASELINE configs[3]): RSBench-shaped lookups, and C5 (configs[4]): SU(3) link
// multiply (GridMini-shaped), each as an SPMD
// `target teams distribute parallel for` driven by omprt plus its bare CUDA twin.
#pragma once
#include "../host/runtime.cuh"
#include "rs_body.cuh"

namespace omprt_kernels {

using namespace omprt;

// ---------------------------------------------------------------------------- RSBench
struct RSTraits : DefaultTraits {};
struct RSTraitsAssume : DefaultTraits {
  static constexpr bool assume_teams_oversub = true;
};
constexpr int kRSThreads = 128;
static_assert(kRSThreads == kRSBodyThreads, "rs_nuclide's shared-memory slots");
// 4 teams of 128 per SM (<= 128 registers, no spills): the round-1 choice of 5 (96
// registers) was 10 % faster for the round-1 body; with the round-2 body it spilled 120-216 B
// per thread and ran no faster (185.3 ms at 4 vs 186.2 ms at 5 per SM, 10M lookups).
constexpr int kRSMinBlocks = 4;
// The flattened kernels: 4 teams of 128 per SM (<= 128 registers, no spills).  With the
// prefetched pole loop (and, queued, the Abrarov drain) in one loop body the 96-register
// budget of 5 teams spills inside the pole loop: queued 106 ms vs 77.8 ms, dynamic 82.8 vs
// 81.9 ms at 10M lookups (profiles/rs_q_explore_x33.txt).
constexpr int kRSFlatMinBlocks = 4;

template <class Tr, bool Macro>
__global__ void __launch_bounds__(kRSThreads, kRSMinBlocks)
    omprt_rs_rt(const __grid_constant__ RSTables t, uint64_t seed, int64_t first,
                typename Tr::Idx count, uint64_t* __restrict__ verification,
                double* __restrict__ macro) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  distribute_parallel_for(team, count, [&](Idx iv) {
    verification[iv] = rs_lookup_one<Macro>(t, seed, first + iv, macro + (int64_t)iv * 4);
  });
}

template <bool Macro>
__global__ void __launch_bounds__(kRSThreads, kRSMinBlocks)
    cuda_rs_twin(const __grid_constant__ RSTables t, uint64_t seed, int64_t first, int32_t count,
                 uint64_t* __restrict__ verification, double* __restrict__ macro) {
  const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= count) return;
  verification[i] = rs_lookup_one<Macro>(t, seed, first + i, macro + (int64_t)i * 4);
}

// Flattened execution (OMPRT_FLAT): a persistent grid of the device's resident teams, each
// thread running its Fig. 5 lookups through omprt::distribute_parallel_for_flat with one
// nuclide per step (RSFlatLookup), so lanes are not held by the warp's longest material.
template <class Tr, bool Macro>
__global__ void __launch_bounds__(kRSThreads, kRSFlatMinBlocks)
    omprt_rs_flat_rt(const __grid_constant__ RSTables t, uint64_t seed, int64_t first,
                     typename Tr::Idx count, uint64_t* __restrict__ verification,
                     double* __restrict__ macro) {
  Team<Tr> team = init<Tr>();
  RSFlatLookup<Macro> lookup(t, seed, first, verification, macro);
  distribute_parallel_for_flat<Tr, FlatSync::Lockstep>(team, count, lookup);
}

// Bare CUDA twin: the same flattened loop written by hand around the same body.
template <bool Macro>
__global__ void __launch_bounds__(kRSThreads, kRSFlatMinBlocks)
    cuda_rs_flat_twin(const __grid_constant__ RSTables t, uint64_t seed, int64_t first,
                      int32_t count, uint64_t* __restrict__ verification,
                      double* __restrict__ macro) {
  RSFlatLookup<Macro> lookup(t, seed, first, verification, macro);
  const int32_t stride = (int32_t)gridDim.x * (int32_t)blockDim.x;
  int32_t i = (int32_t)blockIdx.x * (int32_t)blockDim.x + (int32_t)threadIdx.x;
  bool live = i < count;
  if (live) lookup.begin(i, stride);
  while (__any_sync(0xffffffffu, live)) {  // lanes step together (warp vote per trip)
    if (live && !lookup.step()) {
      lookup.end(i);
      i += stride;
      live = i < count;
      if (live) lookup.next(i);
    }
  }
}

// schedule(dynamic, kRSDynChunk) + flattened (OMPRT_FLAT | OMPRT_SCHED_DYNAMIC): the same
// body; a thread that drew cheap lookups (few nuclides) requests more of its team's block
// instead of the static schedule's fixed share (a thread's fuel lookups -- 321 nuclides,
// 14 % of lookups -- vary by +-25 % between threads, and the warp waits for its slowest).
constexpr int kRSDynChunk = 1;

template <class Tr, bool Macro>
__global__ void __launch_bounds__(kRSThreads, kRSFlatMinBlocks)
    omprt_rs_dflat_rt(const __grid_constant__ RSTables t, uint64_t seed, int64_t first,
                      typename Tr::Idx count, uint64_t* __restrict__ verification,
                      double* __restrict__ macro) {
  Team<Tr> team = init<Tr>();
  RSFlatLookup<Macro> lookup(t, seed, first, verification, macro);
  distribute_parallel_for_dynamic_flat<Tr, FlatSync::Lockstep>(team, count,
                                                               (typename Tr::Idx)kRSDynChunk,
                                                               lookup);
}

template <bool Macro>
__global__ void __launch_bounds__(kRSThreads, kRSFlatMinBlocks)
    cuda_rs_dflat_twin(const __grid_constant__ RSTables t, uint64_t seed, int64_t first,
                       int32_t count, uint64_t* __restrict__ verification,
                       double* __restrict__ macro) {
  __shared__ unsigned next;
  const int32_t per = (count + (int32_t)gridDim.x - 1) / (int32_t)gridDim.x;
  const int32_t lo = min((int32_t)blockIdx.x * per, count);
  const int32_t hi = min(lo + per, count);
  if (threadIdx.x == 0) next = blockDim.x;
  __syncthreads();
  RSFlatLookup<Macro> lookup(t, seed, first, verification, macro);
  int32_t i = lo + (int32_t)threadIdx.x * kRSDynChunk;
  int32_t end = min(i + kRSDynChunk, hi);
  bool live = i < hi;
  if (live) lookup.begin(i, 1);
  while (__any_sync(0xffffffffu, live)) {
    if (live && !lookup.step()) {
      lookup.end(i);
      if (++i < end) {
        lookup.next(i);
      } else {
        i = lo + (int32_t)atomicAdd(&next, 1u) * kRSDynChunk;
        end = min(i + kRSDynChunk, hi);
        live = i < hi;
        if (live) lookup.begin(i, 1);
      }
    }
  }
}

// OMPRT_RS_QUEUE (with OMPRT_FLAT | OMPRT_SCHED_DYNAMIC): the same dynamic lock-step loop
// around RSQueuedLookup -- Abrarov poles queued per warp and drained by the runtime's
// warp-collective hook (reading R-A8).  One queue per warp in team-shared memory.
template <class Tr, bool Macro>
__global__ void __launch_bounds__(kRSThreads, kRSFlatMinBlocks)
    omprt_rs_qflat_rt(const __grid_constant__ RSTables t, uint64_t seed, int64_t first,
                      typename Tr::Idx count, uint64_t* __restrict__ verification,
                      double* __restrict__ macro) {
  Team<Tr> team = init<Tr>();
  using Lookup = RSQueuedLookup<Macro, kRSThreads / 32>;
  Lookup::init_queue();  // published by the loop's team barrier (dynamic_init)
  Lookup lookup(t, seed, first, verification, macro);
  distribute_parallel_for_dynamic_flat<Tr, FlatSync::Lockstep>(team, count,
                                                               (typename Tr::Idx)kRSDynChunk,
                                                               lookup);
}

template <bool Macro>
__global__ void __launch_bounds__(kRSThreads, kRSFlatMinBlocks)
    cuda_rs_qflat_twin(const __grid_constant__ RSTables t, uint64_t seed, int64_t first,
                       int32_t count, uint64_t* __restrict__ verification,
                       double* __restrict__ macro) {
  __shared__ unsigned next;
  using Lookup = RSQueuedLookup<Macro, kRSThreads / 32>;
  const int32_t per = (count + (int32_t)gridDim.x - 1) / (int32_t)gridDim.x;
  const int32_t lo = min((int32_t)blockIdx.x * per, count);
  const int32_t hi = min(lo + per, count);
  if (threadIdx.x == 0) next = blockDim.x;
  Lookup::init_queue();
  __syncthreads();
  Lookup lookup(t, seed, first, verification, macro);
  int32_t i = lo + (int32_t)threadIdx.x * kRSDynChunk;
  int32_t end = min(i + kRSDynChunk, hi);
  bool live = i < hi;
  if (live) lookup.begin(i, 1);
  while (__any_sync(0xffffffffu, live)) {
    const bool done = live && !lookup.step();
    __syncwarp();
    lookup.warp_collective(done);
    if (done) {
      lookup.end(i);
      if (++i < end) {
        lookup.next(i);
      } else {
        i = lo + (int32_t)atomicAdd(&next, 1u) * kRSDynChunk;
        end = min(i + kRSDynChunk, hi);
        live = i < hi;
        if (live) lookup.begin(i, 1);
      }
    }
  }
}

OMPRT_REGISTER_KERNEL(omprt_rs_dflat_rt, omprt_rs_dflat_rt<RSTraits, false>)
OMPRT_REGISTER_KERNEL(omprt_rs_qflat_rt, omprt_rs_qflat_rt<RSTraits, false>)
OMPRT_REGISTER_KERNEL(cuda_rs_qflat_twin, cuda_rs_qflat_twin<false>)
OMPRT_REGISTER_KERNEL(cuda_rs_dflat_twin, cuda_rs_dflat_twin<false>)
OMPRT_REGISTER_KERNEL(omprt_rs_flat_rt, omprt_rs_flat_rt<RSTraits, false>)
OMPRT_REGISTER_KERNEL(cuda_rs_flat_twin, cuda_rs_flat_twin<false>)
OMPRT_REGISTER_KERNEL(omprt_rs_rt, omprt_rs_rt<RSTraits, false>)
OMPRT_REGISTER_KERNEL(omprt_rs_rt_assume, omprt_rs_rt<RSTraitsAssume, false>)
OMPRT_REGISTER_KERNEL(cuda_rs_twin, cuda_rs_twin<false>)

inline RSTables to_dev(const omprt_rs_tables& a) {
  return RSTables{a.poles,    a.pole_l,  a.windows, a.win_range,  a.win_off,
                  a.n_windows, a.k0rs,   a.num_nucs, a.mats,      a.concs,
                  a.matnuc,    a.n_nuclides, a.numL, a.max_num_nucs, a.prepared};
}

// Persistent grid of the flattened kernels: teams = 0 -> every SM's resident teams (of the
// queued kernel with OMPRT_RS_QUEUE: fewer per SM, more registers).
inline int32_t rs_flat_teams(int32_t teams, uint32_t flags = 0) {
  if (teams > 0) return teams;
  int dev = 0, sms = 148, per_sm = kRSMinBlocks;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (flags & OMPRT_RS_QUEUE)
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, omprt_rs_qflat_rt<RSTraits, false>,
                                                  kRSThreads, 0);
  else
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, omprt_rs_flat_rt<RSTraits, false>,
                                                  kRSThreads, 0);
  return sms * std::max(1, per_sm);
}

inline int rs_validate(const omprt_rs_tables& t, int64_t count, uint64_t* ver, int32_t& teams,
                       int32_t threads, uint32_t flags) {
  OMPRT_CHECK_ARG(count >= 0 && count < (1ll << 31), "count must be in [0, 2^31)");
  OMPRT_CHECK_ARG(threads == kRSThreads, "threads must be %d", kRSThreads);
  OMPRT_CHECK_ARG(t.numL == 4, "numL must be 4");
  OMPRT_CHECK_ARG(t.prepared == 1 && t.matnuc && ((uintptr_t)t.matnuc & 31) == 0,
                  "RSBench tables not prepared (omprt_rs_prepare)");
  OMPRT_CHECK_ARG(t.poles && t.pole_l && t.windows && t.win_range && t.win_off && t.n_windows &&
                      t.k0rs && t.num_nucs && t.mats && t.concs,
                  "bad RSBench tables");
  OMPRT_CHECK_ARG(ver != nullptr || count == 0, "verification is required");
  OMPRT_CHECK_ARG((((uintptr_t)t.poles | (uintptr_t)t.windows) & 31) == 0,
                  "poles and windows must be 32 B aligned (256-bit loads)");
  OMPRT_CHECK_ARG(!(flags & OMPRT_XS_FLAT) || !(flags & OMPRT_ASSUME_OVERSUB),
                  "OMPRT_XS_FLAT runs a persistent grid (no oversubscription assumption)");
  OMPRT_CHECK_ARG(!(flags & OMPRT_SCHED_DYNAMIC) || (flags & OMPRT_XS_FLAT),
                  "OMPRT_SCHED_DYNAMIC is implemented for the flattened loop (OMPRT_FLAT)");
  OMPRT_CHECK_ARG(!(flags & OMPRT_RS_QUEUE) ||
                      ((flags & OMPRT_XS_FLAT) && (flags & OMPRT_SCHED_DYNAMIC)),
                  "OMPRT_RS_QUEUE requires OMPRT_FLAT | OMPRT_SCHED_DYNAMIC");
  if (flags & OMPRT_XS_FLAT) teams = rs_flat_teams(teams, flags);
  if (teams <= 0) teams = (int32_t)std::max<int64_t>(1, ceil_div(count, threads));
  OMPRT_CHECK_ARG(!(flags & OMPRT_ASSUME_OVERSUB) || count <= (int64_t)teams * threads,
                  "oversubscription assumption violated");
  OMPRT_CHECK_ARG(count + 2 * (int64_t)teams * threads < INT32_MAX, "iteration space too large");
  return OMPRT_OK;
}

// ---------------------------------------------------------------------------- SU(3)
// 256-bit global accesses (sm_100: LDG/STG.E.ENL2.256): a site is 576 B = 18 x 32 B, so a
// pair of links (288 B) moves in 9 instructions per thread instead of 18 x 16 B ones --
// half the L1 wavefronts of the strided AoS access.
// One site: C[l] = A[l] x B[l] for the 4 links; complex MAC = 4 fmas in fixed order
// (App. A.3), so C is bit-identical to the oracle.  Row r of C[l] needs only row r of A[l],
// so it overwrites it in registers.  Returns sum of Re C over the site in (l, r, c) order.
__device__ __forceinline__ double su3_site(const double* __restrict__ A,
                                           const double2* __restrict__ B,
                                           double* __restrict__ Cs) {
  double re_sum = 0.0;
#pragma unroll
  for (int lp = 0; lp < 2; ++lp) {
    double v[36];
#pragma unroll
    for (int q = 0; q < 9; ++q)
      ld_stream_v4f64(A + lp * 36 + 4 * q, v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
#pragma unroll
    for (int li = 0; li < 2; ++li) {
      const int l = 2 * lp + li, base = 18 * li;
#pragma unroll
      for (int r = 0; r < 3; ++r) {
        double out[6];
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          double re = 0.0, im = 0.0;
#pragma unroll
          for (int m = 0; m < 3; ++m) {
            const double xr = v[base + (r * 3 + m) * 2], xi = v[base + (r * 3 + m) * 2 + 1];
            const double2 y = __ldg(B + l * 9 + m * 3 + c);
            re = fma(xr, y.x, re);
            re = fma(-xi, y.y, re);
            im = fma(xr, y.y, im);
            im = fma(xi, y.x, im);
          }
          out[2 * c] = re;
          out[2 * c + 1] = im;
          re_sum += re;
        }
#pragma unroll
        for (int e = 0; e < 6; ++e) v[base + r * 6 + e] = out[e];
      }
    }
#pragma unroll
    for (int q = 0; q < 9; ++q)
      st_cs_v4f64(Cs + lp * 36 + 4 * q, v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
  }
  return re_sum;
}

struct SU3Traits : DefaultTraits {
  static constexpr bool assume_teams_oversub = true;  // one site per thread
};
struct SU3TraitsLoop : DefaultTraits {};
constexpr int kSU3Threads = 128;

template <class Tr, bool Checksum>
__global__ void __launch_bounds__(kSU3Threads)
    omprt_su3_rt(const double* __restrict__ A, const double2* __restrict__ B,
                 double* __restrict__ Cm, typename Tr::Idx n_sites, double* checksum,
                 double* partials, unsigned* ticket) {
  using Idx = typename Tr::Idx;
  Team<Tr> team = init<Tr>();
  double acc = 0.0;
  distribute_parallel_for(team, n_sites, [&](Idx s) {
    acc += su3_site(A + (int64_t)s * 72, B, Cm + (int64_t)s * 72);
  });
  if constexpr (Checksum)
    league_reduce_threads(team, acc, Plus{}, checksum, partials,
                  ticket);
}

template <bool Checksum>
__global__ void __launch_bounds__(kSU3Threads)
    cuda_su3_twin(const double* __restrict__ A, const double2* __restrict__ B,
                  double* __restrict__ Cm, int32_t n_sites, double* checksum, double* partials,
                  unsigned* ticket) {
  const int32_t s = blockIdx.x * blockDim.x + threadIdx.x;
  double acc = 0.0;
  if (s < n_sites) acc = su3_site(A + (int64_t)s * 72, B, Cm + (int64_t)s * 72);
  if constexpr (Checksum) {
    __shared__ double ws[32];
    __shared__ unsigned last;
    for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
    const unsigned lane = threadIdx.x & 31u, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    if (lane == 0) ws[wid] = acc;
    __syncthreads();
    double b = 0.0;
    if (wid == 0) {
      b = lane < nw ? ws[lane] : 0.0;
      for (int off = 16; off > 0; off >>= 1) b += __shfl_xor_sync(0xffffffffu, b, off);
    }
    if (threadIdx.x == 0) {
      partials[blockIdx.x] = b;
      __threadfence();
      last = atomicAdd(ticket, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (last) {
      __threadfence();
      double t = 0.0;
      for (unsigned k = threadIdx.x; k < gridDim.x; k += blockDim.x) t += __ldcg(partials + k);
      for (int off = 16; off > 0; off >>= 1) t += __shfl_xor_sync(0xffffffffu, t, off);
      if (lane == 0) ws[wid] = t;
      __syncthreads();
      if (wid == 0) {
        double tt = lane < nw ? ws[lane] : 0.0;
        for (int off = 16; off > 0; off >>= 1) tt += __shfl_xor_sync(0xffffffffu, tt, off);
        if (threadIdx.x == 0) {
          *checksum = *checksum + tt;
          *ticket = 0u;
        }
      }
    }
  }
}

OMPRT_REGISTER_KERNEL(omprt_su3_rt, omprt_su3_rt<SU3Traits, true>)
OMPRT_REGISTER_KERNEL(omprt_su3_rt_loop, omprt_su3_rt<SU3TraitsLoop, true>)
OMPRT_REGISTER_KERNEL(cuda_su3_twin, cuda_su3_twin<true>)

// staged variants (su3_staged.cuh)
inline int su3_staged_launch(bool twin, const double* A, const double* B, double* Cm, int64_t n,
                             double* ck, int32_t teams, Workspace* w, cudaStream_t s);
inline int su3_tiled_launch(bool twin, const double* A, const double* B, double* Cm, int64_t n,
                            double* ck, int32_t teams, Workspace* w, cudaStream_t s);

inline int su3_validate(const double* A, const double* B, double* Cm, int64_t n,
                        int32_t& teams, int32_t threads, uint32_t flags, double* ck,
                        Workspace* w) {
  OMPRT_CHECK_ARG(n >= 0 && n < (1ll << 30), "n_sites out of range");
  OMPRT_CHECK_ARG(threads == kSU3Threads, "threads must be %d", kSU3Threads);
  OMPRT_CHECK_ARG(n == 0 || (A && B && Cm), "null data pointer");
  OMPRT_CHECK_ARG(((uintptr_t)A | (uintptr_t)Cm) % 32 == 0 && (uintptr_t)B % 16 == 0,
                  "A and C must be 32 B aligned (256-bit accesses), B 16 B aligned");
  if (teams <= 0) teams = (int32_t)std::max<int64_t>(1, ceil_div(n, threads));
  OMPRT_CHECK_ARG(!ck || (uint64_t)teams <= w->opt.max_teams, "teams exceed max_teams");
  OMPRT_CHECK_ARG(!(flags & OMPRT_ASSUME_OVERSUB) || n <= (int64_t)teams * threads,
                  "oversubscription assumption violated");
  return OMPRT_OK;
}

}  // namespace omprt_kernels

namespace omprt_kernels {
// the prepared pole records (omprt_rs_prepare): EA.re / 2, (0 - EA.im) / 2, RT, RA, RF
__device__ __forceinline__ void rs_prepare_record(const double* __restrict__ r,
                                                  double* __restrict__ o) {
  o[0] = __dmul_rn(r[0], 0.5);
  o[1] = __dmul_rn(__dsub_rn(0.0, r[1]), 0.5);
#pragma unroll
  for (int k = 2; k < 8; ++k) o[k] = r[k];
}
__global__ void rs_prepare_poles(const double* __restrict__ in, double* __restrict__ out,
                                 int64_t n) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    rs_prepare_record(in + p * 8, out + p * 8);
}
// one thread per window (reading R-A12): the window's prepared records stably sorted by l
// (a counting sort: l = 0 first, each run in the input order), and the window record
// (T, A, F, runs) with runs = c1 | c2 << 21 | c3 << 42, c_k = the number of the window's
// poles with l < k.  Rejected (bit 0 of *err): a window range outside [0, n_poles), one
// that starts before the previous window ends (overlapping windows cannot be sorted
// independently), a window of 2^21 poles or more, an l outside [0, 4).
__global__ void rs_prepare_windows(const double* __restrict__ poles,
                                   const int32_t* __restrict__ pole_l,
                                   const int32_t* __restrict__ win_range,
                                   const double* __restrict__ windows, int64_t n_poles,
                                   int64_t n_windows, double* __restrict__ out_poles,
                                   double* __restrict__ out_windows,
                                   unsigned long long* __restrict__ err) {
  const int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (w >= n_windows) return;
  const int64_t s = win_range[2 * w], e = win_range[2 * w + 1];
  bool bad = s < 0 || e < s || e > n_poles || e - s >= (1 << 21) ||
             (w > 0 && s < (int64_t)win_range[2 * w - 1]);
  int64_t c[4] = {0, 0, 0, 0};
  for (int64_t p = s; !bad && p < e; ++p) {
    const int32_t l = pole_l[p];
    if (l < 0 || l > 3) bad = true;
    else ++c[l];
  }
  if (bad) {
    atomicOr(err, 1ull);
    return;
  }
  int64_t pos[4] = {s, s + c[0], s + c[0] + c[1], s + c[0] + c[1] + c[2]};
  for (int64_t p = s; p < e; ++p) rs_prepare_record(poles + p * 8, out_poles + 8 * pos[pole_l[p]]++);
  const uint64_t runs = (uint64_t)c[0] | (uint64_t)(c[0] + c[1]) << 21 |
                        (uint64_t)(c[0] + c[1] + c[2]) << 42;
  out_windows[4 * w] = windows[4 * w];
  out_windows[4 * w + 1] = windows[4 * w + 1];
  out_windows[4 * w + 2] = windows[4 * w + 2];
  out_windows[4 * w + 3] = __longlong_as_double((long long)runs);
}
// one thread per material entry (reading R-A13): the 64 B record of (m, j) -- k0rs of its
// nuclide, conc, the nuclide's window offset | count << 32 -- zeros past num_nucs[m].
// Rejected: a nuclide id outside [0, n_nuclides), num_nucs outside [0, max_num_nucs], a
// nuclide whose windows are not all among the n_windows_total prepared ones (or none).
__global__ void rs_prepare_matnuc(const int32_t* __restrict__ num_nucs,
                                  const int32_t* __restrict__ mats,
                                  const double* __restrict__ concs,
                                  const double* __restrict__ k0rs,
                                  const int32_t* __restrict__ win_off,
                                  const int32_t* __restrict__ n_windows, int32_t n_mats,
                                  int32_t max_num_nucs, int32_t n_nuclides,
                                  int64_t n_windows_total, double* __restrict__ out,
                                  unsigned long long* err) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= (int64_t)n_mats * max_num_nucs) return;
  const int m = (int)(i / max_num_nucs), j = (int)(i % max_num_nucs);
  double* o = out + i * 8;
#pragma unroll
  for (int k = 0; k < 8; ++k) o[k] = 0.0;
  const int nn = num_nucs[m];
  if (nn < 0 || nn > max_num_nucs) {
    atomicOr(err, 2ull);
    return;
  }
  if (j >= nn) return;
  const int nuc = mats[i];
  if (nuc < 0 || nuc >= n_nuclides || win_off[nuc] < 0 || n_windows[nuc] < 1 ||
      (int64_t)win_off[nuc] + n_windows[nuc] > n_windows_total) {
    atomicOr(err, 2ull);
    return;
  }
#pragma unroll
  for (int l = 0; l < 4; ++l) o[l] = k0rs[nuc * 4 + l];
  o[4] = concs[i];
  o[5] = __longlong_as_double((long long)(uint32_t)win_off[nuc] |
                              (long long)((uint64_t)(uint32_t)n_windows[nuc] << 32));
}
}  // namespace omprt_kernels

extern "C" int omprt_rs_prepare(omprt_rs_tables* t, int64_t n_poles, int64_t n_windows,
                                int32_t n_mats, double* prepared_poles,
                                double* prepared_windows, double* prepared_matnuc,
                                void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  OMPRT_CHECK_ARG(t && t->poles && t->pole_l && t->windows && t->win_range && t->win_off &&
                      t->n_windows && t->k0rs && t->num_nucs && t->mats && t->concs &&
                      prepared_poles && prepared_windows && prepared_matnuc && n_poles > 0 &&
                      n_windows > 0 && n_mats > 0 && t->max_num_nucs > 0 &&
                      (((uintptr_t)prepared_poles | (uintptr_t)prepared_windows |
                        (uintptr_t)prepared_matnuc) & 31) == 0,
                  "omprt_rs_prepare: bad arguments");
  OMPRT_CHECK_ARG(t->prepared == 0, "omprt_rs_prepare: the tables are already prepared");
  OMPRT_CHECK_ARG(t->numL == 4, "omprt_rs_prepare: numL must be 4");
  cudaStream_t st = as_stream(stream);
  unsigned long long* err = (unsigned long long*)w->scratch_u64;
  OMPRT_CUDA_TRY(cudaMemsetAsync(err, 0, sizeof(*err), st));
  rs_prepare_poles<<<1024, 256, 0, st>>>(t->poles, prepared_poles, n_poles);
  if (int r = check_launch("rs_prepare_poles")) return r;
  rs_prepare_windows<<<(unsigned)ceil_div(n_windows, 256), 256, 0, st>>>(
      t->poles, t->pole_l, t->win_range, t->windows, n_poles, n_windows, prepared_poles,
      prepared_windows, err);
  if (int r = check_launch("rs_prepare_windows")) return r;
  rs_prepare_matnuc<<<(unsigned)ceil_div((int64_t)n_mats * t->max_num_nucs, 256), 256, 0, st>>>(
      t->num_nucs, t->mats, t->concs, t->k0rs, t->win_off, t->n_windows, n_mats,
      t->max_num_nucs, t->n_nuclides, n_windows, prepared_matnuc, err);
  if (int r = check_launch("rs_prepare_matnuc")) return r;
  unsigned long long bad = 0;
  OMPRT_CUDA_TRY(cudaMemcpyAsync(&bad, err, sizeof(bad), cudaMemcpyDeviceToHost, st));
  OMPRT_CUDA_TRY(cudaStreamSynchronize(st));
  OMPRT_CHECK_ARG(bad == 0,
                  "omprt_rs_prepare: windows overlap / out of range / >= 2^21 poles, l "
                  "outside [0, 4), or a material entry outside [0, n_nuclides) (code %llu)",
                  bad);
  t->poles = prepared_poles;
  t->windows = prepared_windows;
  t->matnuc = prepared_matnuc;
  t->prepared = 1;
  return OMPRT_OK;
}

extern "C" int omprt_rs_lookup(omprt_rs_tables t, uint64_t seed, int64_t first, int64_t count,
                               uint64_t* verification, double* macro, int32_t teams,
                               int32_t threads, uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  if (int r = rs_validate(t, count, verification, teams, threads, flags)) return r;
  if (count == 0) return OMPRT_OK;
  cudaStream_t s = as_stream(stream);
  const RSTables d = to_dev(t);
  const int32_t n = (int32_t)count;
  if (flags & OMPRT_RS_QUEUE) {
    if (macro) omprt_rs_qflat_rt<RSTraits, true><<<teams, threads, 0, s>>>(d, seed, first, n, verification, macro);
    else omprt_rs_qflat_rt<RSTraits, false><<<teams, threads, 0, s>>>(d, seed, first, n, verification, nullptr);
    return check_launch("omprt_rs_qflat_rt");
  }
  if ((flags & OMPRT_XS_FLAT) && (flags & OMPRT_SCHED_DYNAMIC)) {
    if (macro) omprt_rs_dflat_rt<RSTraits, true><<<teams, threads, 0, s>>>(d, seed, first, n, verification, macro);
    else omprt_rs_dflat_rt<RSTraits, false><<<teams, threads, 0, s>>>(d, seed, first, n, verification, nullptr);
    return check_launch("omprt_rs_dflat_rt");
  }
  if (flags & OMPRT_XS_FLAT) {
    const int32_t tm = rs_flat_teams(teams);
    if (macro) omprt_rs_flat_rt<RSTraits, true><<<tm, threads, 0, s>>>(d, seed, first, n, verification, macro);
    else omprt_rs_flat_rt<RSTraits, false><<<tm, threads, 0, s>>>(d, seed, first, n, verification, nullptr);
    return check_launch("omprt_rs_flat_rt");
  }
  if (flags & OMPRT_ASSUME_OVERSUB) {
    if (macro) omprt_rs_rt<RSTraitsAssume, true><<<teams, threads, 0, s>>>(d, seed, first, n, verification, macro);
    else omprt_rs_rt<RSTraitsAssume, false><<<teams, threads, 0, s>>>(d, seed, first, n, verification, nullptr);
  } else {
    if (macro) omprt_rs_rt<RSTraits, true><<<teams, threads, 0, s>>>(d, seed, first, n, verification, macro);
    else omprt_rs_rt<RSTraits, false><<<teams, threads, 0, s>>>(d, seed, first, n, verification, nullptr);
  }
  return check_launch("omprt_rs_rt");
}

extern "C" int omprt_cuda_rs_lookup(omprt_rs_tables t, uint64_t seed, int64_t first,
                                    int64_t count, uint64_t* verification, double* macro,
                                    int32_t teams, int32_t threads, uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  const bool flat = flags & OMPRT_XS_FLAT;
  int32_t tm = flat ? teams : 0;
  if (int r = rs_validate(t, count, verification, tm, threads,
                          flags & (OMPRT_XS_FLAT | OMPRT_SCHED_DYNAMIC | OMPRT_RS_QUEUE)))
    return r;
  if (count == 0) return OMPRT_OK;
  cudaStream_t s = as_stream(stream);
  const RSTables d = to_dev(t);
  if (flags & OMPRT_RS_QUEUE) {
    if (macro) cuda_rs_qflat_twin<true><<<tm, threads, 0, s>>>(d, seed, first, (int32_t)count, verification, macro);
    else cuda_rs_qflat_twin<false><<<tm, threads, 0, s>>>(d, seed, first, (int32_t)count, verification, nullptr);
    return check_launch("cuda_rs_qflat_twin");
  }
  if (flat && (flags & OMPRT_SCHED_DYNAMIC)) {
    if (macro) cuda_rs_dflat_twin<true><<<tm, threads, 0, s>>>(d, seed, first, (int32_t)count, verification, macro);
    else cuda_rs_dflat_twin<false><<<tm, threads, 0, s>>>(d, seed, first, (int32_t)count, verification, nullptr);
    return check_launch("cuda_rs_dflat_twin");
  }
  if (flat) {  // the same persistent geometry as the runtime-driven kernel
    tm = rs_flat_teams(teams);
    if (macro) cuda_rs_flat_twin<true><<<tm, threads, 0, s>>>(d, seed, first, (int32_t)count, verification, macro);
    else cuda_rs_flat_twin<false><<<tm, threads, 0, s>>>(d, seed, first, (int32_t)count, verification, nullptr);
    return check_launch("cuda_rs_flat_twin");
  }
  if (macro) cuda_rs_twin<true><<<tm, threads, 0, s>>>(d, seed, first, (int32_t)count, verification, macro);
  else cuda_rs_twin<false><<<tm, threads, 0, s>>>(d, seed, first, (int32_t)count, verification, nullptr);
  return check_launch("cuda_rs_twin");
}

extern "C" int omprt_su3_mult(const double* A, const double* B, double* Cm, int64_t n_sites,
                              double* checksum_inout, int32_t teams, int32_t threads,
                              uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  if (flags & OMPRT_TMA_TILED) {
    OMPRT_CHECK_ARG(!(flags & (OMPRT_ASSUME_OVERSUB | OMPRT_WARP_STAGED)),
                    "OMPRT_TMA_TILED: persistent grid, exclusive with the other stagings");
    int32_t tm = 1;
    if (int r = su3_validate(A, B, Cm, n_sites, tm, threads, 0, checksum_inout, w)) return r;
    if (n_sites == 0) return OMPRT_OK;
    return su3_tiled_launch(false, A, B, Cm, n_sites, checksum_inout, teams, w,
                            as_stream(stream));
  }
  if (flags & OMPRT_WARP_STAGED) {
    OMPRT_CHECK_ARG(threads == kSU3Threads && !(flags & OMPRT_ASSUME_OVERSUB),
                    "the staged variant runs a persistent grid (no assumption)");
    int32_t tm = 1;
    if (int r = su3_validate(A, B, Cm, n_sites, tm, threads, 0, checksum_inout, w)) return r;
    if (n_sites == 0) return OMPRT_OK;
    return su3_staged_launch(false, A, B, Cm, n_sites, checksum_inout, teams, w,
                             as_stream(stream));
  }
  if (int r = su3_validate(A, B, Cm, n_sites, teams, threads, flags, checksum_inout, w)) return r;
  if (n_sites == 0) return OMPRT_OK;
  cudaStream_t s = as_stream(stream);
  auto* a = A;
  auto* b = (const double2*)B;
  auto* c = Cm;
  double* p = (double*)w->partials;
  unsigned* tk = w->tickets + 3;
  const int32_t n = (int32_t)n_sites;
  if (flags & OMPRT_ASSUME_OVERSUB) {
    if (checksum_inout) omprt_su3_rt<SU3Traits, true><<<teams, threads, 0, s>>>(a, b, c, n, checksum_inout, p, tk);
    else omprt_su3_rt<SU3Traits, false><<<teams, threads, 0, s>>>(a, b, c, n, nullptr, p, tk);
  } else {
    if (checksum_inout) omprt_su3_rt<SU3TraitsLoop, true><<<teams, threads, 0, s>>>(a, b, c, n, checksum_inout, p, tk);
    else omprt_su3_rt<SU3TraitsLoop, false><<<teams, threads, 0, s>>>(a, b, c, n, nullptr, p, tk);
  }
  return check_launch("omprt_su3_rt");
}

extern "C" int omprt_cuda_su3_mult(const double* A, const double* B, double* Cm, int64_t n_sites,
                                   double* checksum_inout, int32_t teams, int32_t threads,
                                   uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  int32_t tm = 0;
  if (int r = su3_validate(A, B, Cm, n_sites, tm, threads, 0, checksum_inout, w)) return r;
  if (flags & OMPRT_TMA_TILED) {
    OMPRT_CHECK_ARG(!(flags & OMPRT_WARP_STAGED),
                    "OMPRT_TMA_TILED is exclusive with the other staging");
    if (n_sites == 0) return OMPRT_OK;
    return su3_tiled_launch(true, A, B, Cm, n_sites, checksum_inout, teams, w,
                            as_stream(stream));
  }
  if (flags & OMPRT_WARP_STAGED) {
    if (n_sites == 0) return OMPRT_OK;
    return su3_staged_launch(true, A, B, Cm, n_sites, checksum_inout, teams, w,
                             as_stream(stream));
  }
  (void)teams;
  (void)flags;
  if (n_sites == 0) return OMPRT_OK;
  cudaStream_t s = as_stream(stream);
  if (checksum_inout)
    cuda_su3_twin<true><<<tm, threads, 0, s>>>(A, (const double2*)B, Cm,
                                               (int32_t)n_sites, checksum_inout,
                                               (double*)w->partials, w->tickets + 3);
  else
    cuda_su3_twin<false><<<tm, threads, 0, s>>>(A, (const double2*)B, Cm,
                                                (int32_t)n_sites, nullptr, nullptr, nullptr);
  return check_launch("cuda_su3_twin");
}
