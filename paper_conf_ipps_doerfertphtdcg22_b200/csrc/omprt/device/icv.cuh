// omprt device runtime -- ICV queries (OpenMP 5.1 omp_get_* inside target regions).
//
// P:102-108 §III-B/C, Fig. 3: a lookup goes to the thread's own ICV state if it has
// one, else to the team state.  Without Traits::uses_thread_states the thread state does
// not exist and a query is a read of the per-thread context (a register, usually a
// constant after inlining).  Values: SURVEY §8(c) C3.
#pragma once
#include "state.cuh"

namespace omprt {

namespace detail {
template <class Tr>
__device__ __forceinline__ const ThreadICVState* thread_state(const Team<Tr>& t) {
  if constexpr (Tr::uses_thread_states) return t.tstates->slot[threadIdx.x];
  return nullptr;
}
}  // namespace detail

template <class Tr>
__device__ __forceinline__ int get_thread_num(const Team<Tr>& t) {
  if (const ThreadICVState* s = detail::thread_state(t)) return s->thread_num;
  return t.thread_num;
}
template <class Tr>
__device__ __forceinline__ int get_num_threads(const Team<Tr>& t) {
  if (const ThreadICVState* s = detail::thread_state(t)) return s->team_size;
  return t.team_size;
}
template <class Tr>
__device__ __forceinline__ int get_level(const Team<Tr>& t) {
  if (const ThreadICVState* s = detail::thread_state(t)) return s->icv.levels_var;
  return t.level;
}
template <class Tr>
__device__ __forceinline__ int get_active_level(const Team<Tr>& t) {
  if (const ThreadICVState* s = detail::thread_state(t)) return s->icv.active_levels_var;
  return t.active_level;
}
template <class Tr>
__device__ __forceinline__ int in_parallel(const Team<Tr>& t) {
  return get_active_level(t) > 0 ? 1 : 0;
}
template <class Tr>
__device__ __forceinline__ int get_team_num(const Team<Tr>&) {
  return (int)blockIdx.x;
}
template <class Tr>
__device__ __forceinline__ int get_num_teams(const Team<Tr>&) {
  return (int)gridDim.x;
}
template <class Tr>
__device__ __forceinline__ int get_max_active_levels(const Team<Tr>&) {
  return 1;  // nested parallel regions are serialized
}

}  // namespace omprt
