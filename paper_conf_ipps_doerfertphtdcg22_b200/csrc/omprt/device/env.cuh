// omprt device runtime -- per-device environment, debug/assert/trace machinery.
//
// P:127-133 §III-G: one runtime with debugging "with zero overhead for release builds":
// debug code is compiled in by a compile-time flag and enabled at run time by an
// environment variable; in release builds an assertion becomes an assumption
// (`__builtin_assume`).  Here: Traits::debug (compile time) and DeviceEnv::debug_bits
// (runtime, from OMPRT_DEBUG at omprt_init).  With Traits::debug == 0 every macro below
// expands to nothing but a compiler assumption.
#pragma once
#include <cstdint>
#include <cstdio>

#include "config.cuh"

namespace omprt {

// Written once per device by omprt_init (cudaMemcpyToSymbol) and read through the constant
// cache; only cold paths (stack overflow, debug) touch it.
struct DeviceEnv {
  unsigned char* pool;              // global fallback pool for the smem stack
  uint64_t pool_bytes_per_team;     // per-team slice
  uint64_t pool_teams;              // number of slices
  int* error_word;                  // mapped pinned host memory: first device error code
  int* error_info;                  // [4] team, thread, line, extra
  unsigned debug_bits;              // runtime debug bits (OMPRT_DEBUG)
  unsigned pad;
};

}  // namespace omprt

// Single definition: the library is one translation unit (src/libomprt.cu).
__constant__ omprt::DeviceEnv omprt_env;

namespace omprt {

// Fatal device error: record the first error in the mapped error word, then trap
// ("__assert_fail ... provides the same functionality as a regular assertion").
__device__ __noinline__ void fatal(int code, int line, int extra) {
  int* w = omprt_env.error_word;
  if (w != nullptr) {
    if (atomicCAS(w, 0, code) == 0 && omprt_env.error_info != nullptr) {
      omprt_env.error_info[0] = (int)blockIdx.x;
      omprt_env.error_info[1] = (int)threadIdx.x;
      omprt_env.error_info[2] = line;
      omprt_env.error_info[3] = extra;
    }
    __threadfence_system();
  }
  __trap();
}

#ifndef OMPRT_STRIP_DEBUG
__device__ __noinline__ void assert_fail(const char* msg, int line) {
  printf("[omprt] assertion failed (line %d, team %d, thread %d): %s\n", line,
         (int)blockIdx.x, (int)threadIdx.x, msg);
  fatal(kErrAssert, line, 0);
}

__device__ __noinline__ void trace_call(const char* fn) {
  printf("[omprt] team %d thread %d: %s\n", (int)blockIdx.x, (int)threadIdx.x, fn);
}

#endif  // OMPRT_STRIP_DEBUG

}  // namespace omprt

// OMPRT_ASSERT(Traits, cond, msg): checked in debug builds with the runtime Assert bit set;
// otherwise an assumption.  __builtin_assume drops conditions with side effects,
// so `cond` must be side-effect free.
#ifdef OMPRT_STRIP_DEBUG
// The stripped build: an assertion is only its release meaning (an assumption), a trace
// point nothing.
#define OMPRT_ASSERT(TR, COND, MSG) __builtin_assume(COND)
#define OMPRT_TRACE(TR, NAME) \
  do {                        \
  } while (0)
#else
#define OMPRT_ASSERT(TR, COND, MSG)                                                  \
  do {                                                                               \
    if constexpr (::omprt::kDebugAssert<TR>) {                                       \
      if ((omprt_env.debug_bits & ::omprt::dbg::Assert) && !(COND))                  \
        ::omprt::assert_fail(MSG, __LINE__);                                         \
    } else {                                                                         \
      __builtin_assume(COND);                                                        \
    }                                                                                \
  } while (0)

// Runtime-call tracing ("runtime call function tracing").
#define OMPRT_TRACE(TR, NAME)                                                        \
  do {                                                                               \
    if constexpr (::omprt::kDebugTrace<TR>) {                                        \
      if (omprt_env.debug_bits & ::omprt::dbg::Trace) ::omprt::trace_call(NAME);     \
    }                                                                                \
  } while (0)
#endif  // OMPRT_STRIP_DEBUG
