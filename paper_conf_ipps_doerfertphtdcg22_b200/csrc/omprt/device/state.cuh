// omprt device runtime -- team / thread state and runtime initialization.
//
// P:96-119 §III.  The paper keeps the runtime state in static shared memory and relies on
// inter-procedural value propagation (§IV-B) to fold it away.  This runtime keeps
// each thread's view of the ICVs in a small per-thread context object (`Team<Tr>`, held in
// registers, passed by reference into every runtime call) and puts into shared memory only
// what other threads must observe:
//   * generic mode: the team ICV state and the parallel-region hand-off;
//   * Traits::uses_thread_states: the thread-states array of Fig. 3;
//   * Traits::stack_bytes: the shared-memory stack (stack.cuh).
// Values known at compile time (SPMD mode, levels inside a region, ...) are never stored, so
// a stateless SPMD kernel has 0 B of runtime shared memory and no init barrier -- the
// paper's "11,304 B -> 0 B" by construction rather than by optimization.
#pragma once
#include <cstdint>
#include <type_traits>

#include "config.cuh"
#include "env.cuh"
#include "sync.cuh"

namespace omprt {

// OpenMP ICVs tracked per data environment.
struct ICVState {
  int32_t nthreads_var;           // requested team size of the next parallel region
  int32_t levels_var;             // enclosing parallel regions
  int32_t active_levels_var;      // enclosing active (team size > 1) parallel regions
  int32_t max_active_levels_var;  // 1: nested regions are serialized
  int32_t run_sched_var;          // schedule kind (static = 1)
  int32_t run_sched_chunk;        // 0 = no chunk (Fig. 5)
};

// P:108 §III-C: a thread ICV state, created on demand from the shared-memory stack, copied
// from the most recent state and chained to it (nested data environments, Fig. 3).
struct ThreadICVState {
  ICVState icv;
  int32_t thread_num;     // omp_get_thread_num inside this data environment
  int32_t team_size;      // omp_get_num_threads inside this data environment
  ThreadICVState* prev;   // previous (enclosing) thread state, NULL -> team state
};

inline constexpr unsigned kMaxThreadsPerTeam = 1024;
inline constexpr uint32_t kRegionTerminate = 0xffffffffu;

// Team state in shared memory for generic mode (P:102-104, P:92 state machine hand-off).
template <class Tr>
struct GenericShared {
  ICVState icv;                          // team ICV state
  uint32_t region;                       // custom state machine: index in the region list
  uint32_t team_size;                    // threads that execute the published region
  void (*fn)(void*, const void*);        // general state machine: outlined region
  const void* args;                      // where the region's arguments were published
  uint32_t stack_top;                    // team stack cursor when the region started
  uint32_t pool_top;                     // team pool cursor when the region started
};

// Thread-states array of Fig. 3, present only with Traits::uses_thread_states.
struct ThreadStatesArray {
  ThreadICVState* slot[kMaxThreadsPerTeam];
};

// Cursor of one thread into the shared-memory stack (smem part) and its global fallback
// (pool part).  Per-thread, in registers; see stack.cuh.
struct StackCursor {
  unsigned char* base;   // smem area owned by this thread (team area for the main thread)
  uint32_t cap;          // bytes in that area
  uint32_t top;          // bytes in use
  unsigned char* pbase;  // pool area owned by this thread
  uint32_t pcap;
  uint32_t ptop;
};

struct Empty {};

// Per-thread runtime context.  Every runtime entry point takes it by reference; it is a
// plain aggregate of registers, so whatever the kernel never reads is dead code.
template <class Tr>
struct Team {
  int32_t thread_num;     // omp_get_thread_num
  int32_t team_size;      // omp_get_num_threads
  int32_t level;          // omp_get_level
  int32_t active_level;   // omp_get_active_level
  std::conditional_t<Tr::mode == Mode::Generic, GenericShared<Tr>*, Empty> gshared;
  std::conditional_t<Tr::uses_thread_states, ThreadStatesArray*, Empty> tstates;
  std::conditional_t<kHasStack<Tr>, StackCursor, Empty> stack;
};

namespace detail {

template <class Tr>
__device__ __forceinline__ unsigned char* stack_storage(uint32_t& cap) {
  if constexpr (Tr::dynamic_stack) {
    extern __shared__ __align__(16) unsigned char omprt_dyn_stack[];
    cap = dynamic_smem_size() & ~(kStackAlign - 1);
    return omprt_dyn_stack;
  } else if constexpr (Tr::stack_bytes > 0) {
    static_assert(Tr::stack_bytes % kStackAlign == 0, "stack_bytes must be a multiple of 16");
    __shared__ __align__(16) unsigned char omprt_stack[Tr::stack_bytes];
    cap = Tr::stack_bytes;
    return omprt_stack;
  } else {
    cap = 0;
    return nullptr;
  }
}

template <class Tr>
__device__ __forceinline__ void stack_init(Team<Tr>& team, bool team_area) {
  if constexpr (kHasStack<Tr>) {
    uint32_t cap;
    unsigned char* s = stack_storage<Tr>(cap);
    unsigned char* pool = nullptr;
    uint32_t pcap = 0;
    if constexpr (Tr::stack_fallback) {
      if (omprt_env.pool != nullptr && blockIdx.x < omprt_env.pool_teams) {
        pool = omprt_env.pool + (uint64_t)blockIdx.x * omprt_env.pool_bytes_per_team;
        pcap = (uint32_t)omprt_env.pool_bytes_per_team;
      }
    }
    if (team_area) {
      // generic mode: the main thread owns the whole team stack in sequential code
      team.stack = StackCursor{s, cap, 0u, pool, pcap, 0u};
    } else {
      // SPMD: every thread owns a 16 B-aligned slice ("track the usage ... by each
      // thread")
      const uint32_t n = blockDim.x, t = threadIdx.x;
      const uint32_t sl = (cap / n) & ~(kStackAlign - 1);
      const uint32_t psl = (pcap / n) & ~(kStackAlign - 1);
      team.stack = StackCursor{s + t * sl, sl, 0u, pool ? pool + (uint64_t)t * psl : nullptr,
                               psl, 0u};
    }
  }
}

}  // namespace detail

// Runtime initialization of a team.  Returns this thread's context.
//  SPMD: all threads are active; ICVs are the parallel region's (level 1).  No shared
//        memory is written unless thread states are used, and then each thread writes
//        only its own slot, so no barrier is needed (C11's effect).
//  Generic: the main thread (CTA thread 0) initializes the team ICV state;
//        workers see it only after the first state-machine barrier, so again no barrier.
template <class Tr>
__device__ __forceinline__ Team<Tr> init() {
  OMPRT_TRACE(Tr, "init");
  static_assert(!(Tr::dynamic_stack && Tr::stack_bytes > 0), "pick one stack placement");
  Team<Tr> team{};
  if constexpr (Tr::uses_thread_states) {
    __shared__ ThreadStatesArray omprt_thread_states;
    team.tstates = &omprt_thread_states;
    team.tstates->slot[threadIdx.x] = nullptr;  // NULL: use the team state
  }
  if constexpr (Tr::mode == Mode::SPMD) {
    team.thread_num = (int32_t)threadIdx.x;
    team.team_size = (int32_t)blockDim.x;
    team.level = 1;
    team.active_level = blockDim.x > 1 ? 1 : 0;
    detail::stack_init<Tr>(team, false);
  } else {
    __shared__ GenericShared<Tr> omprt_team_state;
    team.gshared = &omprt_team_state;
    team.thread_num = 0;
    team.team_size = 1;
    team.level = 0;
    team.active_level = 0;
    if (threadIdx.x == 0) {
      ICVState icv{(int32_t)blockDim.x, 0, 0, 1, 1, 0};
      omprt_team_state.icv = icv;
    }
    detail::stack_init<Tr>(team, threadIdx.x == 0);
  }
  return team;
}

// Main thread of the team in generic mode (the one that runs sequential code).
template <class Tr>
__device__ __forceinline__ bool is_main(const Team<Tr>&) {
  if constexpr (Tr::mode == Mode::Generic) return threadIdx.x == 0;
  return true;
}

}  // namespace omprt
