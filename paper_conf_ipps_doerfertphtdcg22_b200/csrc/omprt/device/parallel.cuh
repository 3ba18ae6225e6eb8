// omprt device runtime -- generic-mode `parallel` and the worker state machine.
//
// P:87, §II-C: each team starts with a single main thread; workers wait in a state
// machine (Bertolli et al.) until the main thread reaches a `parallel`, which hands them
// the region.  P:481 §VII: `parallel` needs barriers at its start and end; §IV-D:
// these are non-aligned (the main thread arrives from a different place than the workers).
// P:476 / §IV-A: a "custom" state machine compares against the known regions instead of
// calling through a function pointer.
//
// Here the region list is a compile-time type list, so the custom state machine is an
// if-cascade over inlined region bodies, and whatever the list proves is dropped: with a
// single region the region id is not even read; after a region marked `terminal` the
// workers exit, so there is no terminate round-trip; a region that is not `join` and is
// terminal has no end barrier (C11's effect).  The general state machine
// (Traits::custom_state_machine = false) publishes a function pointer and always joins.
//
// Region protocol (a stateless functor type):
//   struct R {
//     struct Args { ... };                 // trivially copyable, passed through smem
//     static constexpr bool terminal = ...; // no region follows: workers exit after it
//     static constexpr bool join = ...;     // main reads the region's results afterwards
//     template <class Tr> __device__ void operator()(omprt::Team<Tr>&, const Args&) const;
//   };
#pragma once
#include <cstring>
#include <type_traits>

#include "stack.cuh"
#include "state.cuh"

namespace omprt {

template <class... Rs>
struct RegionList {
  static constexpr unsigned size = sizeof...(Rs);
};

namespace detail {

template <class R, class L>
struct RegionIndex;
template <class R, class... Rs>
struct RegionIndex<R, RegionList<R, Rs...>> {
  static constexpr unsigned value = 0;
};
template <class R, class S, class... Rs>
struct RegionIndex<R, RegionList<S, Rs...>> {
  static constexpr unsigned value = 1 + RegionIndex<R, RegionList<Rs...>>::value;
};

template <class L>
struct FirstRegion;
template <class R, class... Rs>
struct FirstRegion<RegionList<R, Rs...>> {
  using type = R;
};

// Workers must read the published region id unless the list is a single terminal region.
template <class L>
inline constexpr bool kNeedRegionId = !(L::size == 1 && FirstRegion<L>::type::terminal);

template <class... Rs>
__host__ __device__ constexpr size_t max_args_bytes(RegionList<Rs...>*) {
  size_t m = 16;
  ((m = sizeof(typename Rs::Args) > m ? sizeof(typename Rs::Args) : m), ...);
  return (m + 15) & ~size_t(15);
}

// Sharing space for region arguments: one per (kernel, region list), in static smem.
template <class L>
__device__ __forceinline__ unsigned char* sharing_space() {
  constexpr size_t N = max_args_bytes(static_cast<L*>(nullptr));
  __shared__ __align__(16) unsigned char omprt_sharing[N];
  return omprt_sharing;
}

// Context of thread k inside a region of `size` threads (level 1 of the team).
template <class Tr>
__device__ __forceinline__ Team<Tr> region_context(const Team<Tr>& outer, uint32_t k,
                                                   uint32_t size, uint32_t stack_top,
                                                   uint32_t pool_top) {
  Team<Tr> t = outer;
  t.thread_num = (int32_t)k;
  t.team_size = (int32_t)size;
  t.level = 1;
  t.active_level = size > 1 ? 1 : 0;
  stack_enter_region<Tr>(t, stack_top, pool_top, k, size);
  return t;
}

template <class Tr, class R>
__device__ __noinline__ void outlined_region(void* team, const void* args) {
  R{}(*static_cast<Team<Tr>*>(team), *static_cast<const typename R::Args*>(args));
}

template <class Tr, class R>
__device__ __forceinline__ void worker_run(Team<Tr>& team, GenericShared<Tr>* g,
                                           const unsigned char* share) {
  const uint32_t size = g->team_size;
  const uint32_t k = threadIdx.x;
  if (k < size) {
    Team<Tr> t = region_context(team, k, size, g->stack_top, g->pool_top);
    R{}(t, *reinterpret_cast<const typename R::Args*>(share));
  }
}

template <class Tr, class L, unsigned I>
struct Dispatch;
template <class Tr, unsigned I, class R, class... Rs>
struct Dispatch<Tr, RegionList<R, Rs...>, I> {
  // returns true when the workers must leave the state machine
  __device__ __forceinline__ static bool run(uint32_t id, Team<Tr>& team, GenericShared<Tr>* g,
                                             const unsigned char* share) {
    if (sizeof...(Rs) == 0 || id == I) {
      worker_run<Tr, R>(team, g, share);
      if constexpr (R::join || !R::terminal) unaligned_barrier(kJoinBarrierId);
      return R::terminal;
    }
    if constexpr (sizeof...(Rs) > 0)
      return Dispatch<Tr, RegionList<Rs...>, I + 1>::run(id, team, g, share);
    return true;
  }
};

// Nested parallel: serialized on the encountering thread, in a new data
// environment.  With thread states the environment is a ThreadICVState on the stack,
// linked into the thread-states array (Fig. 3); without them it is the register context.
template <class Tr, class R>
__device__ __forceinline__ void nested_parallel(Team<Tr>& team, const typename R::Args& args) {
  OMPRT_TRACE(Tr, "parallel (nested, serialized)");
  Team<Tr> inner = team;
  inner.thread_num = 0;
  inner.team_size = 1;
  inner.level = team.level + 1;
  inner.active_level = team.active_level;
  if constexpr (Tr::uses_thread_states) {
    ThreadICVState*& slot = team.tstates->slot[threadIdx.x];
    ThreadICVState* ts =
        static_cast<ThreadICVState*>(alloc_shared(team, (uint32_t)sizeof(ThreadICVState)));
    // copy from the most recent state (the team view if this thread has none yet)
    if (slot != nullptr) {
      *ts = *slot;
    } else {
      ts->icv = ICVState{team.team_size, team.level, team.active_level, 1, 1, 0};
      ts->thread_num = team.thread_num;
      ts->team_size = team.team_size;
    }
    ts->icv.levels_var += 1;
    ts->thread_num = 0;
    ts->team_size = 1;
    ts->prev = slot;
    slot = ts;
    inner.stack = team.stack;
    R{}(inner, args);
    slot = ts->prev;
    free_shared(team, ts, (uint32_t)sizeof(ThreadICVState));
  } else {
    R{}(inner, args);
  }
}

}  // namespace detail

// `parallel` with an optional num_threads clause (0 = none: team size = nthreads-var).
// Called by the main thread in sequential code (generic mode), or by any thread inside a
// region (nested -> serialized).
template <class Tr, class L, class R>
__device__ __forceinline__ void parallel(Team<Tr>& team, const typename R::Args& args,
                                         int32_t num_threads = 0) {
  static_assert(std::is_trivially_copyable<typename R::Args>::value, "Args must be POD");
  if constexpr (Tr::mode == Mode::SPMD) {
    // SPMD kernels are already inside the (only) parallel region: nested -> serialized
    detail::nested_parallel<Tr, R>(team, args);
    return;
  } else {
    if (team.level > 0) {
      detail::nested_parallel<Tr, R>(team, args);
      return;
    }
    OMPRT_TRACE(Tr, "parallel");
    GenericShared<Tr>* g = team.gshared;
    unsigned char* share = detail::sharing_space<L>();
    uint32_t size = num_threads > 0 ? (uint32_t)num_threads : (uint32_t)g->icv.nthreads_var;
    size = size < blockDim.x ? size : blockDim.x;
    uint32_t stack_top = 0, pool_top = 0;
    if constexpr (kHasStack<Tr>) {
      stack_top = team.stack.top;
      pool_top = team.stack.ptop;
    }
    // publish the region (Fig. 8 levels_var update)
    if constexpr (!Tr::custom_state_machine) {
      g->fn = &detail::outlined_region<Tr, R>;
      g->args = share;
    } else if constexpr (detail::kNeedRegionId<L>) {
      g->region = detail::RegionIndex<R, L>::value;
    }
    g->team_size = size;
    g->stack_top = stack_top;
    g->pool_top = pool_top;
    g->icv.levels_var = 1;
    g->icv.active_levels_var = size > 1 ? 1 : 0;
    memcpy(share, &args, sizeof(args));
    unaligned_barrier(kStateMachineBarrierId);  // release the workers
    // the main thread is OpenMP thread 0 of the region
    Team<Tr> t = detail::region_context(team, 0u, size, stack_top, pool_top);
    R{}(t, args);
    if constexpr (!Tr::custom_state_machine || R::join || !R::terminal)
      unaligned_barrier(kJoinBarrierId);  // join: the region's writes are visible
    g->icv.levels_var = 0;
    g->icv.active_levels_var = 0;
  }
}

// Worker side of the state machine: called by every thread except the main thread of a
// generic-mode team; returns when the team terminates (after a terminal region, or when
// deinit publishes "terminate").
template <class Tr, class L>
__device__ __forceinline__ void worker_state_machine(Team<Tr>& team) {
  static_assert(Tr::mode == Mode::Generic, "state machine is generic-mode only");
  OMPRT_TRACE(Tr, "worker_state_machine");
  GenericShared<Tr>* g = team.gshared;
  for (;;) {
    unaligned_barrier(kStateMachineBarrierId);
    if constexpr (Tr::custom_state_machine) {
      const uint32_t id = detail::kNeedRegionId<L> ? g->region : 0u;
      if (detail::kNeedRegionId<L> && id == kRegionTerminate) return;
      if (detail::Dispatch<Tr, L, 0>::run(id, team, g, detail::sharing_space<L>())) return;
    } else {
      void (*fn)(void*, const void*) = g->fn;
      if (fn == nullptr) return;
      const uint32_t size = g->team_size;
      const uint32_t k = threadIdx.x;
      if (k < size) {
        Team<Tr> t = detail::region_context(team, k, size, g->stack_top, g->pool_top);
        fn(&t, g->args);
      }
      unaligned_barrier(kJoinBarrierId);
    }
  }
}

// NEXT f1 -- SPMDization (§IV-A3): sequential code of a generic-mode region executed
// in SPMD mode, "guarded for single threaded execution": the team's thread 0 runs `fn`
// (its side effects happen once), then an aligned barrier broadcasts them.  No state
// machine, no region hand-off.
template <class Tr, class Fn>
__device__ __forceinline__ void guarded(Team<Tr>& team, Fn&& fn) {
  static_assert(Tr::mode == Mode::SPMD, "guarded execution is the SPMD form of sequential code");
  OMPRT_TRACE(Tr, "guarded");
  if (team.thread_num == 0) fn();
  aligned_barrier();
}

// Runtime de-initialization: release the workers unless the last region was
// terminal (then they already left).  `last_was_terminal` is a compile-time fact of the
// kernel's control flow.
template <class Tr, class L, bool LastWasTerminal>
__device__ __forceinline__ void deinit(Team<Tr>& team) {
  OMPRT_TRACE(Tr, "deinit");
  if constexpr (Tr::mode == Mode::Generic && !(Tr::custom_state_machine && LastWasTerminal)) {
    GenericShared<Tr>* g = team.gshared;
    if constexpr (Tr::custom_state_machine) g->region = kRegionTerminate;
    else g->fn = nullptr;
    unaligned_barrier(kStateMachineBarrierId);
  }
}

}  // namespace omprt
