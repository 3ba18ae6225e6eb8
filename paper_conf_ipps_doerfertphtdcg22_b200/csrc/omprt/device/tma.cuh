// omprt device runtime -- bulk (TMA) staging of per-iteration records through shared
// memory (sm_90+ cp.async.bulk + mbarrier; SASS UBLKCP / SYNCS).
//
// north_star: "shared-memory or TMA staging".  A loop whose iteration i reads a fixed-size
// record in[i] and writes a record out[i] of an AoS array (SU(3): 576 B per site) makes
// every warp-wide load touch 32 different cache lines.  The runtime instead moves each
// record with one bulk copy into a padded shared-memory slot owned by the thread that runs
// iteration i under the Fig. 5 assignment, the body works on the slot, and the runtime
// bulk-stores the slot to out[i].  Every thread runs its own double-buffered pipeline
// (own mbarriers, own bulk groups), so no CTA-wide barrier is involved.
#pragma once
#include <cstdint>

#include "../../common/ptx_tma.cuh"
#include "state.cuh"

namespace omprt {


// Shared-memory footprint of distribute_parallel_for_staged for `team_size` threads.
template <unsigned kSlotBytes, unsigned kBuffers>
__host__ __device__ constexpr uint32_t staged_smem_bytes(uint32_t team_size) {
  return team_size * (kBuffers * kSlotBytes + kBuffers * 8u);
}

// `distribute parallel for` (Fig. 5 assignment) whose iteration i reads the kRecBytes record
// in + i*kRecBytes and writes the record out + i*kRecBytes: the runtime stages the record
// into this thread's slot (kSlotBytes >= kRecBytes, padded against bank conflicts), calls
// body(i, slot) -- which computes in place -- and bulk-stores the slot.  Double buffered:
// the record of the thread's next iteration is in flight while the body runs.
// Needs staged_smem_bytes<kSlotBytes, 2>(team_size) bytes of dynamic shared memory.
template <class Tr, unsigned kRecBytes, unsigned kSlotBytes, class Body>
__device__ __forceinline__ void distribute_parallel_for_staged(Team<Tr>& team,
                                                               typename Tr::Idx n,
                                                               const unsigned char* in,
                                                               unsigned char* out, Body&& body) {
  using Idx = typename Tr::Idx;
  static_assert(kRecBytes % 16 == 0 && kSlotBytes % 16 == 0 && kSlotBytes >= kRecBytes,
                "bulk copies move multiples of 16 B into 16 B-aligned slots");
  OMPRT_TRACE(Tr, "distribute_parallel_for_staged");
  extern __shared__ __align__(128) unsigned char omprt_stage_smem[];
  const uint32_t nt = (uint32_t)team.team_size, t = (uint32_t)team.thread_num;
  unsigned char* slot[2] = {omprt_stage_smem + (0 * nt + t) * kSlotBytes,
                            omprt_stage_smem + (1 * nt + t) * kSlotBytes};
  uint64_t* bar = reinterpret_cast<uint64_t*>(omprt_stage_smem + 2 * nt * kSlotBytes) + 2 * t;
  tma::mbar_init(bar + 0, 1);
  tma::mbar_init(bar + 1, 1);
  tma::fence_mbar_init();
  const Idx total = (Idx)gridDim.x * (Idx)nt;
  Idx iv = (Idx)blockIdx.x * (Idx)nt + (Idx)t;
  if (Tr::assume_teams_oversub) OMPRT_ASSERT(Tr, n <= total, "oversubscription assumption violated");
  // prologue: the first iteration's record
  if (iv < n) {
    tma::mbar_arrive_expect_tx(bar + 0, kRecBytes);
    tma::bulk_load(slot[0], in + (size_t)iv * kRecBytes, kRecBytes, bar + 0);
  }
  uint32_t k = 0, phase0 = 0, phase1 = 0;
  for (; iv < n; iv += total, ++k) {
    const uint32_t b = k & 1u;
    const Idx nx = iv + total;
    if (!Tr::assume_teams_oversub && nx < n) {
      // the next record goes to the other slot once its previous store has read it
      tma::bulk_wait_read<0>();
      tma::mbar_arrive_expect_tx(bar + (b ^ 1u), kRecBytes);
      tma::bulk_load(slot[b ^ 1u], in + (size_t)nx * kRecBytes, kRecBytes, bar + (b ^ 1u));
    }
    tma::mbar_wait(bar + b, b ? phase1 : phase0);
    if (b) phase1 ^= 1u;
    else phase0 ^= 1u;
    body(iv, slot[b]);
    tma::fence_proxy_async_smem();
    tma::bulk_store(out + (size_t)iv * kRecBytes, slot[b], kRecBytes);
    tma::bulk_commit();
    if (Tr::assume_teams_oversub) break;
  }
  tma::bulk_wait<0>();  // stores complete before the thread exits
}

}  // namespace omprt
