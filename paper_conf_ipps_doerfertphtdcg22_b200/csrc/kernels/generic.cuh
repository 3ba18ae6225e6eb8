// C2 (BASELINE configs[1]): a generic-mode target region:
//   #pragma omp target teams num_teams(T) thread_limit(N)
//   { double w[256]; int perm[256]; double s = 0;            // shared with the region:
//     for (k...) { w[k] = in[t*256+k]*(t+1); s += w[k]; perm[k] = (17k+t) % 256; }  // globalized
//     #pragma omp parallel for
//     for (j...) out[t*256+j] = w[perm[j]] / s + w[j]; }
// (SURVEY App. A.4).  Runtime-driven: main thread + custom (or general) state machine +
// alloc_shared stack; twin: __shared__ arrays, thread 0 prologue, one __syncthreads.
// Products that feed adds use __dmul_rn/__dadd_rn so nvcc cannot contract them (Q12).
//
// Also: the ICV probe kernel (Fig. 3/4 semantics).
#pragma once
#include "../common/ptx_tma.cuh"
#include "../host/runtime.cuh"

namespace omprt_kernels {

using namespace omprt;

template <class Base, bool GeneralSM>
struct GenSM : Base {
  static constexpr bool custom_state_machine = !GeneralSM;
};

struct GenericTraits : DefaultTraits {
  static constexpr Mode mode = Mode::Generic;
  static constexpr unsigned stack_bytes = 4096;  // SURVEY Q9 default
  static constexpr bool assume_threads_oversub = true;  // inner_n <= team size
};
struct GenericTraitsLoop : GenericTraits {
  static constexpr bool assume_threads_oversub = false;
};
// stack in dynamic shared memory (fallback tests: 4 KiB / 2 KiB / 0 B at launch)
struct GenericTraitsDyn : GenericTraitsLoop {
  static constexpr unsigned stack_bytes = 0;
  static constexpr bool dynamic_stack = true;
};
struct GenericTraitsDebug : GenericTraitsLoop {
  static constexpr unsigned debug = dbg::Assert | dbg::Trace;
};

// The sequential prologue (user code, identical in the runtime kernel and the twin): the
// team's main thread fills the arrays the parallel region reads.  One thread reading its
// team's row of `in` load by load waits a memory latency per batch of loads (16 batches of
// 16 for 256 elements: ~1 us each on B200); instead the thread moves the row into a
// shared-memory staging buffer with ONE bulk copy (TMA, cp.async.bulk + mbarrier; SASS
// UBLKCP) of its 16 B-aligned span -- one wait, no per-element copy instructions -- and
// runs the sequential loop from shared memory.  Same values, same order.  `in` must be
// 16 B aligned (host-checked), so [a, e) below never leaves the array.
constexpr int32_t kGenStage = 256;
__device__ __forceinline__ double gen_prologue(const double* __restrict__ tin, int32_t t,
                                               int32_t inner_n, double* w, int32_t* perm) {
  __shared__ __align__(16) double stage[kGenStage + 2];
  __shared__ __align__(8) uint64_t bar;
  const double tp1 = (double)(t + 1);
  double s = 0.0;
  const int32_t step = inner_n > 0 ? 17 % inner_n : 0;
  int32_t pk = inner_n > 0 ? t % inner_n : 0;
  omprt::tma::mbar_init(&bar, 1);
  omprt::tma::fence_mbar_init();
  uint32_t phase = 0;
  for (int32_t k0 = 0; k0 < inner_n; k0 += kGenStage) {
    const int32_t m = inner_n - k0 < kGenStage ? inner_n - k0 : kGenStage;
    // [a, e): the 16 B-aligned span from src rounded down to the end rounded down; the
    // element before src (off = 1) belongs to the previous row, the last element of the
    // chunk is read separately when the end is not aligned
    const uintptr_t src = reinterpret_cast<uintptr_t>(tin + k0);
    const uintptr_t a = src & ~(uintptr_t)15, e = (src + 8u * (uint32_t)m) & ~(uintptr_t)15;
    const int32_t off = (int32_t)((src - a) >> 3);
    const uint32_t bytes = (uint32_t)(e - a);
    if (bytes > 0) {
      omprt::tma::fence_proxy_async_smem();  // the previous chunk's reads of stage first
      omprt::tma::mbar_arrive_expect_tx(&bar, bytes);
      omprt::tma::bulk_load(stage, reinterpret_cast<const void*>(a), bytes, &bar);
    }
    if (e < src + 8u * (uint32_t)m) stage[off + m - 1] = __ldg(tin + k0 + m - 1);
    if (bytes > 0) {
      omprt::tma::mbar_wait(&bar, phase);
      phase ^= 1u;
    }
    const double* st = stage + off;
    // 4 elements per trip with 16-byte shared / generic accesses (w and perm come from
    // alloc_shared: 16 B aligned; k0 is a multiple of 4): 5 memory instructions per 4
    // elements instead of 12 on this single-thread critical path
    int32_t u = 0;
    for (; off == 0 && u + 4 <= m; u += 4) {
      const int32_t k = k0 + u;
      const double2 a = *reinterpret_cast<const double2*>(st + u);
      const double2 b = *reinterpret_cast<const double2*>(st + u + 2);
      const double x0 = __dmul_rn(a.x, tp1), x1 = __dmul_rn(a.y, tp1);
      const double x2 = __dmul_rn(b.x, tp1), x3 = __dmul_rn(b.y, tp1);
      *reinterpret_cast<double2*>(w + k) = make_double2(x0, x1);
      *reinterpret_cast<double2*>(w + k + 2) = make_double2(x2, x3);
      s = __dadd_rn(__dadd_rn(__dadd_rn(__dadd_rn(s, x0), x1), x2), x3);
      int4 pv;
      pv.x = pk;  // (k * 17 + t) mod inner_n, carried (no integer division per element)
      pk += step; if (pk >= inner_n) pk -= inner_n;
      pv.y = pk;
      pk += step; if (pk >= inner_n) pk -= inner_n;
      pv.z = pk;
      pk += step; if (pk >= inner_n) pk -= inner_n;
      pv.w = pk;
      pk += step; if (pk >= inner_n) pk -= inner_n;
      *reinterpret_cast<int4*>(perm + k) = pv;
    }
    for (; u < m; ++u) {
      const int32_t k = k0 + u;
      const double x = __dmul_rn(st[u], tp1);
      w[k] = x;
      s = __dadd_rn(s, x);
      perm[k] = pk;
      pk += step;
      if (pk >= inner_n) pk -= inner_n;
    }
  }
  return s;
}

// The parallel region: team `for` over j (Fig. 5 with NumBlocks = 1).
template <bool Rec, bool Join>
struct GenRegion {
  struct Args {
    const double* w;
    const int32_t* perm;
    double s;
    double* out;
    int32_t* owner;
    int32_t inner_n;
  };
  static constexpr bool terminal = true;  // the only region of the kernel
  static constexpr bool join = Join;      // postlogue reads `out` after the region
  template <class Tr>
  __device__ __forceinline__ void operator()(Team<Tr>& team, const Args& a) const {
    for_static(team, (typename Tr::Idx)a.inner_n, [&](int j) {
      a.out[j] = __dadd_rn(__ddiv_rn(a.w[a.perm[j]], a.s), a.w[j]);
      if constexpr (Rec) a.owner[j] = get_thread_num(team);
    });
  }
};

constexpr int kGenericMaxThreads = 256;
// 8 teams of 256 per SM (<= 32 registers) for the runtime kernel AND the twin, so neither
// comparison side is limited by a register count the other escapes.
constexpr int kGenericMinBlocks = 8;

template <class Tr, int kInner, bool Rec, bool Post>
__global__ void __launch_bounds__(kGenericMaxThreads, kGenericMinBlocks)
    omprt_generic_rt(int32_t inner_n_rt, const double* __restrict__ in, double* __restrict__ out,
                     int32_t* owner, double* post) {
  using R = GenRegion<Rec, Post>;
  using L = RegionList<R>;
  const int32_t inner_n = kInner > 0 ? kInner : inner_n_rt;
  Team<Tr> team = init<Tr>();
  if (!is_main(team)) {  // workers: wait for the main thread's parallel region
    worker_state_machine<Tr, L>(team);
    return;
  }
  // ---- sequential part: the team's main thread alone ----
  const int32_t t = (int32_t)blockIdx.x;
  double* w = static_cast<double*>(alloc_shared(team, (uint32_t)inner_n * 8u));
  int32_t* perm = static_cast<int32_t*>(alloc_shared(team, (uint32_t)inner_n * 4u));
  const double s = gen_prologue(in + (int64_t)t * inner_n, t, inner_n, w, perm);
  double* tout = out + (int64_t)t * inner_n;
  parallel<Tr, L, R>(team, typename R::Args{w, perm, s, tout,
                                            Rec ? owner + (int64_t)t * inner_n : nullptr,
                                            inner_n});
  if constexpr (Post) {  // after the join the main thread sees the region's writes
    double acc = 0.0;
    for (int32_t j = 0; j < inner_n; ++j) acc = __dadd_rn(acc, tout[j]);
    post[t] = acc;
  }
  free_shared(team, perm, (uint32_t)inner_n * 4u);
  free_shared(team, w, (uint32_t)inner_n * 8u);
  deinit<Tr, L, true>(team);
}

// Bare CUDA twin.
template <int kInner, bool Rec, bool Post>
__global__ void __launch_bounds__(kGenericMaxThreads, kGenericMinBlocks)
    cuda_generic_twin(int32_t inner_n_rt, const double* __restrict__ in,
                      double* __restrict__ out, int32_t* owner, double* post) {
  __shared__ __align__(16) double w[256];
  __shared__ __align__(16) int32_t perm[256];
  __shared__ double s_sh;
  const int32_t inner_n = kInner > 0 ? kInner : inner_n_rt;
  const int32_t t = (int32_t)blockIdx.x;
  if (threadIdx.x == 0) s_sh = gen_prologue(in + (int64_t)t * inner_n, t, inner_n, w, perm);
  __syncthreads();
  const double s = s_sh;
  double* tout = out + (int64_t)t * inner_n;
  for (int32_t j = threadIdx.x; j < inner_n; j += blockDim.x) {
    tout[j] = __dadd_rn(__ddiv_rn(w[perm[j]], s), w[j]);
    if constexpr (Rec) owner[(int64_t)t * inner_n + j] = threadIdx.x;
  }
  if constexpr (Post) {
    __syncthreads();
    if (threadIdx.x == 0) {
      double acc = 0.0;
      for (int32_t j = 0; j < inner_n; ++j) acc = __dadd_rn(acc, tout[j]);
      post[t] = acc;
    }
  }
}

// ---- NEXT f2: deglobalized generic-mode kernel ---------------------------
// The globalized arrays have compile-time sizes, so they become static team-local smem
// arrays (no stack, no cursor, no fallback) and the region names them directly; only `s`
// travels through the argument sharing space.  The state machine is unchanged.
template <class Base>
struct Deglob : Base {
  static constexpr unsigned stack_bytes = 0;
  static constexpr bool dynamic_stack = false;
  static constexpr bool stack_fallback = false;
};
constexpr unsigned kGenMaxInner = 256;

template <bool Rec, bool Join>
struct GenRegionDeglob {
  struct Args {
    double s;
    double* out;
    int32_t* owner;
    int32_t inner_n;
  };
  static constexpr bool terminal = true;
  static constexpr bool join = Join;
  template <class Tr>
  __device__ __forceinline__ void operator()(Team<Tr>& team, const Args& a) const {
    const double* w = team_local<double, kGenMaxInner, 0>();
    const int32_t* perm = team_local<int32_t, kGenMaxInner, 1>();
    for_static(team, (typename Tr::Idx)a.inner_n, [&](int j) {
      a.out[j] = __dadd_rn(__ddiv_rn(w[perm[j]], a.s), w[j]);
      if constexpr (Rec) a.owner[j] = get_thread_num(team);
    });
  }
};

template <class Tr, int kInner, bool Rec, bool Post>
__global__ void __launch_bounds__(kGenericMaxThreads, kGenericMinBlocks)
    omprt_generic_deglob_rt(int32_t inner_n_rt, const double* __restrict__ in,
                            double* __restrict__ out, int32_t* owner, double* post) {
  using R = GenRegionDeglob<Rec, Post>;
  using L = RegionList<R>;
  const int32_t inner_n = kInner > 0 ? kInner : inner_n_rt;
  Team<Tr> team = init<Tr>();
  if (!is_main(team)) {
    worker_state_machine<Tr, L>(team);
    return;
  }
  const int32_t t = (int32_t)blockIdx.x;
  double* w = team_local<double, kGenMaxInner, 0>();
  int32_t* perm = team_local<int32_t, kGenMaxInner, 1>();
  const double s = gen_prologue(in + (int64_t)t * inner_n, t, inner_n, w, perm);
  double* tout = out + (int64_t)t * inner_n;
  parallel<Tr, L, R>(team, typename R::Args{s, tout, Rec ? owner + (int64_t)t * inner_n : nullptr,
                                            inner_n});
  if constexpr (Post) {
    double acc = 0.0;
    for (int32_t j = 0; j < inner_n; ++j) acc = __dadd_rn(acc, tout[j]);
    post[t] = acc;
  }
  deinit<Tr, L, true>(team);
}

// ---- NEXT f1: SPMDized kernel -----------------------------------------------------
// The same target region in SPMD mode: the sequential prologue is guarded (thread 0 runs
// it, an aligned barrier broadcasts w, perm and s), then all threads run the team `for`.
template <class Base>
struct Spmdized : Base {
  static constexpr Mode mode = Mode::SPMD;
  static constexpr unsigned stack_bytes = 0;
  static constexpr bool dynamic_stack = false;
  static constexpr bool stack_fallback = false;
};

template <class Tr, int kInner, bool Rec, bool Post>
__global__ void __launch_bounds__(kGenericMaxThreads, kGenericMinBlocks)
    omprt_generic_spmd_rt(int32_t inner_n_rt, const double* __restrict__ in,
                          double* __restrict__ out, int32_t* owner, double* post) {
  const int32_t inner_n = kInner > 0 ? kInner : inner_n_rt;
  Team<Tr> team = init<Tr>();
  const int32_t t = (int32_t)blockIdx.x;
  double* w = team_local<double, kGenMaxInner, 0>();
  int32_t* perm = team_local<int32_t, kGenMaxInner, 1>();
  double* s_sh = team_local<double, 1, 2>();
  guarded(team, [&] { s_sh[0] = gen_prologue(in + (int64_t)t * inner_n, t, inner_n, w, perm); });
  const double s = s_sh[0];
  double* tout = out + (int64_t)t * inner_n;
  for_static(team, (typename Tr::Idx)inner_n, [&](int j) {
    tout[j] = __dadd_rn(__ddiv_rn(w[perm[j]], s), w[j]);
    if constexpr (Rec) owner[(int64_t)t * inner_n + j] = get_thread_num(team);
  });
  if constexpr (Post) {
    aligned_barrier();  // the region's writes are visible to thread 0
    if (team.thread_num == 0) {
      double acc = 0.0;
      for (int32_t j = 0; j < inner_n; ++j) acc = __dadd_rn(acc, tout[j]);
      post[t] = acc;
    }
  }
}

// Variant 1: deglobalized (generic mode), 2: SPMDized.
template <int Variant, class Tr, int KI, bool R, bool P>
inline void launch_gv(int32_t teams, int32_t threads, int32_t inner_n, const double* in,
                      double* out, int32_t* owner, double* post, cudaStream_t s) {
  if constexpr (Variant == 1)
    omprt_generic_deglob_rt<Tr, KI, R, P><<<teams, threads, 0, s>>>(inner_n, in, out, owner, post);
  else
    omprt_generic_spmd_rt<Tr, KI, R, P><<<teams, threads, 0, s>>>(inner_n, in, out, owner, post);
}

template <int Variant, class Tr>
inline void launch_generic_variant(int32_t teams, int32_t threads, int32_t inner_n,
                                   const double* in, double* out, int32_t* owner, double* post,
                                   cudaStream_t s) {
  const bool rec = owner != nullptr, pst = post != nullptr;
#define OMPRT_GV(KI, R, P) \
  launch_gv<Variant, Tr, KI, R, P>(teams, threads, inner_n, in, out, owner, post, s)
  if (inner_n == 256) {
    if (rec && pst) OMPRT_GV(256, true, true);
    else if (rec) OMPRT_GV(256, true, false);
    else if (pst) OMPRT_GV(256, false, true);
    else OMPRT_GV(256, false, false);
  } else {
    if (rec && pst) OMPRT_GV(0, true, true);
    else if (rec) OMPRT_GV(0, true, false);
    else if (pst) OMPRT_GV(0, false, true);
    else OMPRT_GV(0, false, false);
  }
#undef OMPRT_GV
}

OMPRT_REGISTER_KERNEL(omprt_generic_deglob_rt,
                      omprt_generic_deglob_rt<Deglob<GenSM<GenericTraits, false>>, 256, false, false>)
OMPRT_REGISTER_KERNEL(omprt_generic_spmd_rt,
                      omprt_generic_spmd_rt<Spmdized<GenericTraits>, 256, false, false>)
OMPRT_REGISTER_KERNEL(omprt_generic_rt, omprt_generic_rt<GenSM<GenericTraits, false>, 256, false, false>)
OMPRT_REGISTER_KERNEL(omprt_generic_rt_general_sm,
                      omprt_generic_rt<GenSM<GenericTraits, true>, 256, false, false>)
OMPRT_REGISTER_KERNEL(cuda_generic_twin, cuda_generic_twin<256, false, false>)

template <class Tr, int kInner>
inline void launch_generic_rt(int32_t teams, int32_t threads, int32_t inner_n, const double* in,
                              double* out, int32_t* owner, double* post, uint32_t dyn,
                              cudaStream_t s) {
  const bool rec = owner != nullptr, pst = post != nullptr;
  if (rec && pst)
    omprt_generic_rt<Tr, kInner, true, true><<<teams, threads, dyn, s>>>(inner_n, in, out, owner, post);
  else if (rec)
    omprt_generic_rt<Tr, kInner, true, false><<<teams, threads, dyn, s>>>(inner_n, in, out, owner, post);
  else if (pst)
    omprt_generic_rt<Tr, kInner, false, true><<<teams, threads, dyn, s>>>(inner_n, in, out, owner, post);
  else
    omprt_generic_rt<Tr, kInner, false, false><<<teams, threads, dyn, s>>>(inner_n, in, out, owner, post);
}

template <class Tr>
inline void launch_generic_rt_any(int32_t teams, int32_t threads, int32_t inner_n,
                                  const double* in, double* out, int32_t* owner, double* post,
                                  uint32_t dyn, cudaStream_t s) {
  if (inner_n == 256)
    launch_generic_rt<Tr, 256>(teams, threads, inner_n, in, out, owner, post, dyn, s);
  else
    launch_generic_rt<Tr, 0>(teams, threads, inner_n, in, out, owner, post, dyn, s);
}

template <class Tr>
inline void launch_generic_sm(bool general, int32_t teams, int32_t threads, int32_t inner_n,
                              const double* in, double* out, int32_t* owner, double* post,
                              uint32_t dyn, cudaStream_t s) {
  if (general)
    launch_generic_rt_any<GenSM<Tr, true>>(teams, threads, inner_n, in, out, owner, post, dyn, s);
  else
    launch_generic_rt_any<GenSM<Tr, false>>(teams, threads, inner_n, in, out, owner, post, dyn, s);
}

inline uint64_t stack_round_host(uint64_t b) { return (b + 15) & ~uint64_t(15); }

inline int generic_validate(int32_t teams, int32_t threads, int32_t inner_n, const double* in,
                            double* out, double* post, uint32_t flags, Workspace* w,
                            bool twin) {
  OMPRT_CHECK_ARG(teams > 0 && teams <= 2147483647, "teams must be > 0");
  OMPRT_CHECK_ARG(threads > 0 && threads <= kGenericMaxThreads, "threads must be in [1, %d]",
                  kGenericMaxThreads);
  OMPRT_CHECK_ARG(inner_n >= 0 && inner_n <= 65536, "inner_n out of range");
  OMPRT_CHECK_ARG(!twin || inner_n <= 256, "the CUDA twin supports inner_n <= 256");
  OMPRT_CHECK_ARG(inner_n == 0 || (in && out), "null data pointer");
  OMPRT_CHECK_ARG(((uintptr_t)in & 15) == 0, "in must be 16 B aligned (bulk-copied rows)");
  OMPRT_CHECK_ARG(!(flags & OMPRT_POSTLOGUE) || post, "OMPRT_POSTLOGUE needs postlogue");
  OMPRT_CHECK_ARG(!(flags & OMPRT_ASSUME_OVERSUB) || inner_n <= threads,
                  "threads-oversubscription assumption violated: inner_n=%d > threads=%d",
                  inner_n, threads);
  if (!twin) {
    // bytes of the globalized arrays (16 B granules) against stack + this team's pool slice
    const uint64_t need = stack_round_host((uint64_t)inner_n * 8) +
                          stack_round_host((uint64_t)inner_n * 4);
    const uint64_t cap = (flags & OMPRT_NO_STACK) ? 0 : (flags & OMPRT_SMALL_STACK) ? 2048 : 4096;
    if (need > cap) {
      OMPRT_CHECK_ARG((uint64_t)teams <= w->opt.pool_teams,
                      "teams (%d) exceed the fallback pool's pool_teams (%llu)", teams,
                      (unsigned long long)w->opt.pool_teams);
      if (need > cap + w->opt.pool_bytes_per_team)
        return set_error(OMPRT_E_STACK,
                         "globalized arrays (%llu B) exceed stack (%llu B) + pool slice (%llu B)",
                         (unsigned long long)need, (unsigned long long)cap,
                         (unsigned long long)w->opt.pool_bytes_per_team);
    }
  }
  return OMPRT_OK;
}

}  // namespace omprt_kernels

extern "C" int omprt_generic_team(int32_t teams, int32_t threads, int32_t inner_n,
                                  const double* in, double* out, int32_t* owner,
                                  double* postlogue, uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  if (int r = generic_validate(teams, threads, inner_n, in, out, postlogue, flags, w, false))
    return r;
  cudaStream_t s = as_stream(stream);
  double* post = (flags & OMPRT_POSTLOGUE) ? postlogue : nullptr;
  const bool general = flags & OMPRT_GENERAL_SM;
  if (flags & (OMPRT_SPMDIZE | OMPRT_DEGLOBALIZE)) {
    OMPRT_CHECK_ARG(inner_n <= (int32_t)kGenMaxInner,
                    "SPMDized / deglobalized variants need inner_n <= %u", kGenMaxInner);
    OMPRT_CHECK_ARG(!(flags & (OMPRT_SMALL_STACK | OMPRT_NO_STACK | OMPRT_DEBUG_BUILD)),
                    "SPMDized / deglobalized variants have no stack and no debug build");
    const bool assume = flags & OMPRT_ASSUME_OVERSUB;
    if (flags & OMPRT_SPMDIZE) {
      if (assume) launch_generic_variant<2, Spmdized<GenericTraits>>(teams, threads, inner_n, in, out, owner, post, s);
      else launch_generic_variant<2, Spmdized<GenericTraitsLoop>>(teams, threads, inner_n, in, out, owner, post, s);
    } else if (general) {
      if (assume) launch_generic_variant<1, Deglob<GenSM<GenericTraits, true>>>(teams, threads, inner_n, in, out, owner, post, s);
      else launch_generic_variant<1, Deglob<GenSM<GenericTraitsLoop, true>>>(teams, threads, inner_n, in, out, owner, post, s);
    } else {
      if (assume) launch_generic_variant<1, Deglob<GenSM<GenericTraits, false>>>(teams, threads, inner_n, in, out, owner, post, s);
      else launch_generic_variant<1, Deglob<GenSM<GenericTraitsLoop, false>>>(teams, threads, inner_n, in, out, owner, post, s);
    }
    return check_launch("omprt_generic_variant");
  }
  if (flags & (OMPRT_SMALL_STACK | OMPRT_NO_STACK)) {
    const uint32_t dyn = (flags & OMPRT_NO_STACK) ? 0u : 2048u;
    launch_generic_sm<GenericTraitsDyn>(general, teams, threads, inner_n, in, out, owner, post,
                                        dyn, s);
  } else if (stack_round_host((uint64_t)inner_n * 8) + stack_round_host((uint64_t)inner_n * 4) >
             4096) {
    // does not fit the static 4 KiB stack: spill to the pool through a 4 KiB dynamic stack
    const uint32_t dyn = 4096;
    launch_generic_sm<GenericTraitsDyn>(general, teams, threads, inner_n, in, out, owner, post,
                                        dyn, s);
  } else if (flags & OMPRT_DEBUG_BUILD) {
    launch_generic_sm<GenericTraitsDebug>(general, teams, threads, inner_n, in, out, owner, post,
                                          0, s);
  } else if (flags & OMPRT_ASSUME_OVERSUB) {
    launch_generic_sm<GenericTraits>(general, teams, threads, inner_n, in, out, owner, post, 0,
                                     s);
  } else {
    launch_generic_sm<GenericTraitsLoop>(general, teams, threads, inner_n, in, out, owner, post,
                                         0, s);
  }
  return check_launch("omprt_generic_rt");
}

extern "C" int omprt_cuda_generic_team(int32_t teams, int32_t threads, int32_t inner_n,
                                       const double* in, double* out, int32_t* owner,
                                       double* postlogue, uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  if (int r = generic_validate(teams, threads, inner_n, in, out, postlogue, flags, w, true))
    return r;
  cudaStream_t s = as_stream(stream);
  const bool rec = owner != nullptr, pst = (flags & OMPRT_POSTLOGUE) != 0;
#define OMPRT_TWIN_LAUNCH(K)                                                               \
  do {                                                                                     \
    if (rec && pst)                                                                        \
      cuda_generic_twin<K, true, true><<<teams, threads, 0, s>>>(inner_n, in, out, owner,   \
                                                                 postlogue);              \
    else if (rec)                                                                          \
      cuda_generic_twin<K, true, false><<<teams, threads, 0, s>>>(inner_n, in, out, owner,  \
                                                                  postlogue);             \
    else if (pst)                                                                          \
      cuda_generic_twin<K, false, true><<<teams, threads, 0, s>>>(inner_n, in, out, owner,  \
                                                                  postlogue);             \
    else                                                                                   \
      cuda_generic_twin<K, false, false><<<teams, threads, 0, s>>>(inner_n, in, out, owner, \
                                                                   postlogue);            \
  } while (0)
  if (inner_n == 256) OMPRT_TWIN_LAUNCH(256);
  else OMPRT_TWIN_LAUNCH(0);
#undef OMPRT_TWIN_LAUNCH
  return check_launch("cuda_generic_twin");
}

// ---------------------------------------------------------------------------------------
// ICV probe: records the ICV queries at the prologue, in the region, inside a
// serialized nested parallel and after it.
// ---------------------------------------------------------------------------------------
namespace omprt_kernels {

template <class Tr>
__device__ __forceinline__ void icv_record(const Team<Tr>& t, int32_t* r) {
  r[0] = get_thread_num(t);
  r[1] = get_num_threads(t);
  r[2] = get_level(t);
  r[3] = get_active_level(t);
  r[4] = in_parallel(t);
  r[5] = get_team_num(t);
  r[6] = get_num_teams(t);
}

struct IcvNested {
  struct Args {
    int32_t* rec;
  };
  static constexpr bool terminal = true;
  static constexpr bool join = false;
  template <class Tr>
  __device__ __forceinline__ void operator()(Team<Tr>& team, const Args& a) const {
    icv_record(team, a.rec);
  }
};

struct IcvOuter {
  struct Args {
    int32_t* team_rec;  // this team's records
    int32_t nthreads;
    int32_t nested_request;
  };
  static constexpr bool terminal = true;
  static constexpr bool join = false;
  template <class Tr>
  __device__ __forceinline__ void operator()(Team<Tr>& team, const Args& a) const {
    const int k = get_thread_num(team);
    icv_record(team, a.team_rec + (1 + k) * 7);
    parallel<Tr, RegionList<IcvNested>, IcvNested>(
        team, IcvNested::Args{a.team_rec + (1 + a.nthreads + k) * 7}, a.nested_request);
    icv_record(team, a.team_rec + (1 + 2 * a.nthreads + k) * 7);
  }
};

struct IcvTraits : DefaultTraits {
  static constexpr Mode mode = Mode::Generic;
  // thread ICV states (48 B each after rounding) come from per-thread slices; slices
  // that are too small spill to the global pool
  static constexpr unsigned stack_bytes = 1024 * 24;
};
template <class Base>
struct WithThreadStates : Base {
  static constexpr bool uses_thread_states = true;
};
template <class Base>
struct WithDebug : Base {
  static constexpr unsigned debug = dbg::Assert | dbg::Trace;
};

template <class Tr>
__global__ void __launch_bounds__(1024) omprt_icv_probe_kernel(int32_t nthreads, int32_t nested,
                                                               int32_t* rec) {
  using L = RegionList<IcvOuter>;
  Team<Tr> team = init<Tr>();
  if (!is_main(team)) {
    worker_state_machine<Tr, L>(team);
    return;
  }
  int32_t* team_rec = rec + (int64_t)blockIdx.x * (1 + 3 * nthreads) * 7;
  icv_record(team, team_rec);
  parallel<Tr, L, IcvOuter>(team, IcvOuter::Args{team_rec, nthreads, nested}, nthreads);
  deinit<Tr, L, true>(team);
}

}  // namespace omprt_kernels

extern "C" int omprt_icv_probe(int32_t teams, int32_t threads, int32_t nested_request,
                               int32_t* rec, uint32_t flags, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  OMPRT_CHECK_ARG(teams > 0 && threads > 0 && threads <= 1024 && rec && nested_request > 0,
                  "omprt_icv_probe: bad arguments");
  cudaStream_t s = as_stream(stream);
  const bool ts = flags & OMPRT_THREAD_STATES, dbgb = flags & OMPRT_DEBUG_BUILD,
             gen = flags & OMPRT_GENERAL_SM;
#define OMPRT_ICV(...) omprt_icv_probe_kernel<__VA_ARGS__><<<teams, threads, 0, s>>>(threads, nested_request, rec)
  if (ts && dbgb) OMPRT_ICV(WithDebug<WithThreadStates<IcvTraits>>);
  else if (ts && gen) OMPRT_ICV(GenSM<WithThreadStates<IcvTraits>, true>);
  else if (ts) OMPRT_ICV(WithThreadStates<IcvTraits>);
  else if (dbgb) OMPRT_ICV(WithDebug<IcvTraits>);
  else if (gen) OMPRT_ICV(GenSM<IcvTraits, true>);
  else OMPRT_ICV(IcvTraits);
#undef OMPRT_ICV
  return check_launch("omprt_icv_probe");
}
