// omprt device runtime -- compile-time configuration ("Traits").
//
// The paper prunes unused runtime features with LLVM passes over runtime bitcode linked into
// the application (§IV), fed by user assumptions given as compiler flags
// (§III-F) and by a debug flag (§III-G).  Here the same information is a
// constexpr trait struct the kernel is instantiated with: a feature whose trait is off is
// never instantiated, so it costs no register, no shared memory and no instruction
// (`if constexpr`), which is the effect the paper's optimizations aim for.
//
// A kernel writes its own traits by deriving from DefaultTraits and overriding fields:
//   struct MyTraits : omprt::DefaultTraits {
//     static constexpr omprt::Mode mode = omprt::Mode::Generic;
//     static constexpr unsigned stack_bytes = 4096;
//   };
#pragma once
#include <cstdint>

namespace omprt {

// P:98-100 §III-A: SPMD vs generic execution (§II-C).  A template parameter here,
// stronger than the paper's by-value flag: nothing is stored and nothing is loaded.
enum class Mode : int { SPMD = 0, Generic = 1 };

// P:131 §III-G: debug features selected by a bit-field.  Compile-time bits decide what is
// compiled in; the runtime bits (env OMPRT_DEBUG, read by omprt_init) decide what runs.
namespace dbg {
enum : unsigned { None = 0u, Assert = 1u, Trace = 2u };
}

struct DefaultTraits {
  static constexpr Mode mode = Mode::SPMD;
  // P:125 §III-F "-fopenmp-assume-teams-oversubscription": n <= #teams * #threads for a
  // combined distribute parallel for, so each thread runs at most one iteration.
  static constexpr bool assume_teams_oversub = false;
  // P:125 "-fopenmp-assume-threads-oversubscription": n <= #threads for a team `for`.
  static constexpr bool assume_threads_oversub = false;
  // P:106-108 §III-C: per-thread ICV state pointers (smem array, NULL = team state).
  static constexpr bool uses_thread_states = false;
  // P:110-112 §III-D: team shared-memory stack capacity in bytes (static smem), 0 = none.
  static constexpr unsigned stack_bytes = 0;
  // the stack lives in dynamic shared memory, sized at launch (%dynamic_smem_size).
  static constexpr bool dynamic_stack = false;
  // spill to the global-memory pool when the stack is full.
  static constexpr bool stack_fallback = true;
  // P:129-131 §III-G: compile-time debug bits (dbg::Assert | dbg::Trace).
  static constexpr unsigned debug = dbg::None;
  // Generic mode: compile-time "custom" state machine over a static region list
  // (direct, inlinable dispatch), or the general one (function pointer published in smem).
  static constexpr bool custom_state_machine = true;
  // Loop unroll of the Fig. 5 do-while that keeps the iteration -> thread assignment.
  static constexpr unsigned unroll = 1;
  // Record, per iteration, which global thread ran it (test builds only).
  static constexpr bool record_owner = false;
  // Iteration-variable type (int32 when n + T*N < 2^31, host-selected).
  using Idx = int32_t;
};

// The same traits with a 64-bit loop index (when n + T*N does not fit int32).
template <class Base>
struct WithIdx64 : Base {
  using Idx = int64_t;
};

// OMPRT_STRIP_DEBUG (a verification build, tests/test_release_pruning.py): the debug
// machinery does not exist at all -- no kernel is debug-instrumented whatever its traits,
// and env.cuh defines neither the assertion nor the trace functions.  Every release kernel
// of the normal build must compile to the same SASS as in this build (§III-G: "the
// debugging code paths will be trivially dead and removed statically").
#ifdef OMPRT_STRIP_DEBUG
template <class Tr>
inline constexpr bool kDebugAssert = false;
template <class Tr>
inline constexpr bool kDebugTrace = false;
#else
template <class Tr>
inline constexpr bool kDebugAssert = (Tr::debug & dbg::Assert) != 0;
template <class Tr>
inline constexpr bool kDebugTrace = (Tr::debug & dbg::Trace) != 0;
#endif
template <class Tr>
inline constexpr bool kHasStack = Tr::stack_bytes > 0 || Tr::dynamic_stack;

// Shared-memory stack allocation granule (16 B alignment).
inline constexpr unsigned kStackAlign = 16;

// Named hardware barriers.  Fig. 6 puts the runtime's aligned barrier on
// barrier 8 to keep it apart from the user's __syncthreads (barrier 0).  On sm_100 a CTA
// reserves (highest id + 1) barriers from the SM's pool, so ids 8-10 cap residency at
// 6 CTAs/SM (ncu launch__occupancy_limit_barriers = 6, profiles/ncu_generic_x01): the
// aligned barrier uses barrier 0 (it is a full-CTA aligned barrier, exactly what
// __syncthreads is) and the state machine ids 1 and 2 -- 3 barriers per CTA.
inline constexpr unsigned kAlignedBarrierId = 0;
inline constexpr unsigned kStateMachineBarrierId = 1;
inline constexpr unsigned kJoinBarrierId = 2;

// Error codes shared with the host ABI (include/omprt.h).
enum : int {
  kOK = 0,
  kErrInval = -1,
  kErrCuda = -2,
  kErrNoMem = -3,
  kErrStack = -4,
  kErrAssert = -5,
  kErrNotInit = -6,
};

}  // namespace omprt
