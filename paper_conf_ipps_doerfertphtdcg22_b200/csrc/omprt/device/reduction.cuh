// omprt device runtime -- team and league reductions.
//
// The paper did not redesign reductions; this is a new design from north_star:
// thread-private accumulators (identity-initialized) -> warp shfl.xor butterfly (5 fixed
// steps; every lane ends with the same bits) -> one partial per warp in shared memory ->
// warp 0 combines the warp partials -> per-team partial in global memory -> release fence +
// ticket atomic -> the last team to arrive combines all team partials in a fixed order,
// adds the reduction variable's original value (OpenMP: orig (+) private copies), writes it
// and re-arms the ticket.  The order depends only on the launch geometry, so results are
// deterministic run to run.
#pragma once
#include <cstdint>

#include "state.cuh"
#include "sync.cuh"

namespace omprt {

struct Plus {
  template <class T>
  __device__ __forceinline__ T operator()(T a, T b) const { return a + b; }
  template <class T>
  __device__ __forceinline__ static constexpr T identity() { return T(0); }
};
struct Times {
  template <class T>
  __device__ __forceinline__ T operator()(T a, T b) const { return a * b; }
  template <class T>
  __device__ __forceinline__ static constexpr T identity() { return T(1); }
};
struct Min {
  template <class T>
  __device__ __forceinline__ T operator()(T a, T b) const { return b < a ? b : a; }
  template <class T>
  __device__ __forceinline__ static constexpr T identity();
};
struct Max {
  template <class T>
  __device__ __forceinline__ T operator()(T a, T b) const { return b > a ? b : a; }
  template <class T>
  __device__ __forceinline__ static constexpr T identity();
};
template <>
__device__ __forceinline__ constexpr double Min::identity<double>() { return 1.7976931348623157e308; }
template <>
__device__ __forceinline__ constexpr double Max::identity<double>() { return -1.7976931348623157e308; }
template <>
__device__ __forceinline__ constexpr unsigned long long Min::identity<unsigned long long>() {
  return ~0ull;
}
template <>
__device__ __forceinline__ constexpr unsigned long long Max::identity<unsigned long long>() {
  return 0ull;
}

// Warp butterfly: after 5 xor steps every lane holds op over the 32 lanes (the operands of
// each step are the same pair on both lanes, so all lanes agree bit for bit).
template <class T, class Op>
__device__ __forceinline__ T warp_reduce(T v, Op op) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) v = op(v, __shfl_xor_sync(0xffffffffu, v, off));
  return v;
}

namespace detail {
// Team reduction over all threads of the CTA; the result is valid in warp 0.  One aligned
// barrier, none after it: the per-warp slots are free again only after the caller's next
// aligned barrier (league_reduce has one right after; its last-team combine is the final
// use of the slots).
template <class T, class Op>
__device__ __forceinline__ T team_reduce_to_warp0(T v, Op op) {
  __shared__ T omprt_warp_partial[32];
  v = warp_reduce(v, op);
  const uint32_t w = threadIdx.x >> 5, l = threadIdx.x & 31u;
  const uint32_t nw = (blockDim.x + 31u) >> 5;
  if (l == 0) omprt_warp_partial[w] = v;
  aligned_barrier();
  T r = Op::template identity<T>();
  if (w == 0) {
    r = l < nw ? omprt_warp_partial[l] : Op::template identity<T>();
    r = warp_reduce(r, op);
  }
  return r;
}
}  // namespace detail

// Team reduction over all threads of the CTA; the result is valid in warp 0 (thread 0 is
// what the league reduction uses).  Ends with an aligned barrier, so back-to-back calls
// cannot overwrite a slot warp 0 is still reading.
template <class Tr, class T, class Op>
__device__ __forceinline__ T team_reduce_to_main(Team<Tr>&, T v, Op op) {
  const T r = detail::team_reduce_to_warp0(v, op);
  aligned_barrier();
  return r;
}

// Team reduction whose result is valid in every thread (SURVEY §8(b) team_reduce).
template <class Tr, class T, class Op>
__device__ __forceinline__ T team_reduce(Team<Tr>& team, T v, Op op) {
  __shared__ T omprt_team_result;
  T r = detail::team_reduce_to_warp0(v, op);
  if (threadIdx.x == 0) omprt_team_result = r;
  aligned_barrier();
  r = omprt_team_result;
  aligned_barrier();  // the slot may be reused by a later reduction
  return r;
}

// League reduction: *inout = *inout (op) (op over the teams' values).  `team_val` must be
// valid in thread 0.  partials: >= gridDim.x slots; ticket: zero before the launch, zero
// again after it.  Every thread of every team must call it.
template <class Tr, class T, class Op>
__device__ __forceinline__ void league_reduce(Team<Tr>& team, T team_val, Op op, T* inout,
                                              T* partials, unsigned* ticket) {
  OMPRT_TRACE(Tr, "league_reduce");
  __shared__ uint32_t omprt_is_last;
  if (threadIdx.x == 0) {
    partials[blockIdx.x] = team_val;
    __threadfence();  // release: the partial is visible before the ticket
    const unsigned prev = atomicAdd(ticket, 1u);
    omprt_is_last = (prev == gridDim.x - 1) ? 1u : 0u;
  }
  aligned_barrier();
  if (omprt_is_last) {
    __threadfence();  // acquire side
    T acc = Op::template identity<T>();
    for (uint32_t k = threadIdx.x; k < gridDim.x; k += blockDim.x)
      acc = op(acc, __ldcg(partials + k));
    const T total = detail::team_reduce_to_warp0(acc, op);  // last use of the slots
    if (threadIdx.x == 0) {
      *inout = op(*inout, total);
      *ticket = 0u;
    }
  }
}

// Team + league reduction of every thread's private value v (the combined-construct form
// `reduction(op: x)`): the team reduction feeds the league's ticket protocol directly, whose
// aligned barrier also frees the team reduction's slots -- one barrier fewer than
// league_reduce(team, team_reduce_to_main(...)).  Every thread of every team must call it.
template <class Tr, class T, class Op>
__device__ __forceinline__ void league_reduce_threads(Team<Tr>& team, T v, Op op, T* inout,
                                                      T* partials, unsigned* ticket) {
  league_reduce(team, detail::team_reduce_to_warp0(v, op), op, inout, partials, ticket);
}

}  // namespace omprt
