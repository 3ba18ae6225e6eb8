// omprt device runtime -- staging of per-iteration records through shared memory:
// warp-cooperative 16 B cp.async (SASS LDGSTS), 2-D TMA tensor tiles per warp (SASS
// UTMALDG / UTMASTG) and TMA-streamed columns of the Fig. 5 assignment.
//
// north_star: "shared-memory or TMA staging".  A loop whose iteration i reads a fixed-size
// record in[i] and writes a record out[i] of an AoS array (SU(3): 576 B per site) makes
// every warp-wide load touch 32 different cache lines.  The runtime instead moves the
// records of a warp's iterations (under Fig. 5, 32 consecutive ones) into padded
// shared-memory slots, each lane's body works on its slot, and the runtime writes the
// slots back -- per warp, double buffered, with no CTA-wide barrier.
#pragma once
#include <cstdint>

#include "../../common/ptx_tma.cuh"
#include "state.cuh"
#include "sync.cuh"

namespace omprt {


// ---- warp-cooperative staging (cp.async / LDGSTS) ---------------------------------------
// Under the Fig. 5 assignment the 32 lanes of a warp run 32 consecutive iterations, so the
// warp's 32 records are one contiguous byte range.  The warp copies that range with
// coalesced 16 B cp.async (each warp instruction moves 512 contiguous bytes) into 32 padded
// slots, each lane runs body(i, slot) on its own slot, and the warp writes the slots back
// with coalesced 16 B stores.  Double buffered per warp: the next tile's range is in flight
// while the body runs.  Only __syncwarp orders the lanes; the team never synchronizes.

template <unsigned kSlotBytes>
__host__ __device__ constexpr uint32_t warp_staged_smem_bytes(uint32_t team_size) {
  return team_size * 2u * kSlotBytes;
}

namespace detail {
// chunk c (16 B) of the tile's byte range belongs to record c / kChunks
template <unsigned kRecBytes, unsigned kSlotBytes>
__device__ __forceinline__ void warp_stage_in(uint32_t sbuf, const unsigned char* src,
                                              uint32_t cnt, uint32_t lane) {
  constexpr uint32_t kChunks = kRecBytes / 16;
  const uint32_t nch = cnt * kChunks;
#pragma unroll
  for (uint32_t j = 0; j < kChunks; ++j) {
    const uint32_t c = lane + 32u * j;
    const uint32_t r = c / kChunks, q = c - r * kChunks;
    // chunks past the tile's last record zero-fill their (unused) slot bytes: branch-free
    const bool in_tile = c < nch;
    tma::cp_async16_zfill(sbuf + r * kSlotBytes + q * 16u, src + (in_tile ? c * 16u : 0u),
                          in_tile ? 16u : 0u);
  }
  tma::cp_async_commit();
}
template <unsigned kRecBytes, unsigned kSlotBytes>
__device__ __forceinline__ void warp_stage_out(const unsigned char* buf, unsigned char* dst,
                                               uint32_t cnt, uint32_t lane) {
  constexpr uint32_t kChunks = kRecBytes / 16;
  const uint32_t nch = cnt * kChunks;
#pragma unroll
  for (uint32_t j = 0; j < kChunks; ++j) {
    const uint32_t c = lane + 32u * j;
    if (c < nch) {
      const uint32_t r = c / kChunks, q = c - r * kChunks;
      const uint4 v = *reinterpret_cast<const uint4*>(buf + r * kSlotBytes + q * 16u);
      *reinterpret_cast<uint4*>(dst + c * 16u) = v;
    }
  }
}
}  // namespace detail

// `distribute parallel for` (Fig. 5 assignment) over records of kRecBytes, staged per warp.
// Needs warp_staged_smem_bytes<kSlotBytes>(team_size) bytes of dynamic shared memory and a
// team size that is a multiple of 32.
template <class Tr, unsigned kRecBytes, unsigned kSlotBytes, class Body>
__device__ __forceinline__ void distribute_parallel_for_warp_staged(Team<Tr>& team,
                                                                    typename Tr::Idx n,
                                                                    const unsigned char* in,
                                                                    unsigned char* out,
                                                                    Body&& body) {
  using Idx = typename Tr::Idx;
  static_assert(kRecBytes % 16 == 0 && kSlotBytes % 16 == 0 && kSlotBytes >= kRecBytes,
                "16 B copies into 16 B-aligned slots");
  OMPRT_TRACE(Tr, "distribute_parallel_for_warp_staged");
  extern __shared__ __align__(128) unsigned char omprt_stage_smem[];
  const uint32_t nt = (uint32_t)team.team_size, t = (uint32_t)team.thread_num;
  OMPRT_ASSERT(Tr, nt % 32u == 0, "warp staging needs whole warps");
  const uint32_t lane = t & 31u, w0 = t & ~31u;
  unsigned char* const buf0 = omprt_stage_smem + w0 * kSlotBytes;
  unsigned char* const buf1 = omprt_stage_smem + (nt + w0) * kSlotBytes;
  const Idx total = (Idx)gridDim.x * (Idx)nt;
  Idx base = (Idx)blockIdx.x * (Idx)nt + (Idx)w0;  // the warp's first iteration
  if (Tr::assume_teams_oversub) OMPRT_ASSERT(Tr, n <= total, "oversubscription assumption violated");
  const uint32_t sbuf0 = tma::smem_addr(buf0), sbuf1 = tma::smem_addr(buf1);
  auto tile = [&](Idx b) { return n - b < (Idx)32 ? (uint32_t)(n - b) : 32u; };
  if (base < n)
    detail::warp_stage_in<kRecBytes, kSlotBytes>(sbuf0, in + (size_t)base * kRecBytes,
                                                 tile(base), lane);
  for (uint32_t k = 0; base < n; base += total, ++k) {
    unsigned char* const cur = (k & 1u) ? buf1 : buf0;
    const Idx nx = base + total;
    if (!Tr::assume_teams_oversub && nx < n) {
      detail::warp_stage_in<kRecBytes, kSlotBytes>((k & 1u) ? sbuf0 : sbuf1,
                                                   in + (size_t)nx * kRecBytes, tile(nx), lane);
      tma::cp_async_wait<1>();
    } else {
      tma::cp_async_wait<0>();
    }
    __syncwarp();
    const Idx iv = base + (Idx)lane;
    if (iv < n) body(iv, cur + lane * kSlotBytes);
    __syncwarp();
    detail::warp_stage_out<kRecBytes, kSlotBytes>(cur, out + (size_t)base * kRecBytes,
                                                  tile(base), lane);
    __syncwarp();  // the slots are refilled by the fetch two tiles on
    if (Tr::assume_teams_oversub) break;
  }
}

// ---- TMA tensor tiles ----------------------------------------------------------------
// The records of a warp's 32 consecutive iterations (Fig. 5) as ONE 2-D tensor copy: the
// records are a tensor [n][kRecBytes / 8] of doubles, the box is [32][kSlotBytes / 8].  The
// box's extra columns lie outside the tensor, so TMA zero-fills them on the load -- every
// record lands in its own padded kSlotBytes slot (conflict-free per-lane shared-memory
// access) -- and skips them on the store.  One lane of the warp issues the copies; each
// lane runs body(i, slot) on its record in place; the warp's tiles are double buffered (the
// next tile's load is in flight while the body runs).  No team barrier; the tensor maps
// (tmap_in, tmap_out: generic addresses of __grid_constant__ CUtensorMap parameters) are
// encoded on the host.  Needs tma_tiles_smem_bytes<kSlotBytes>(team_size) bytes of dynamic
// shared memory and a team size that is a multiple of 32.
template <unsigned kSlotBytes, unsigned kBuffers = 2>
__host__ __device__ constexpr uint32_t tma_tiles_smem_bytes(uint32_t team_size) {
  return team_size * kBuffers * kSlotBytes + (team_size / 32u) * kBuffers * 8u;
}

template <class Tr, unsigned kSlotBytes, unsigned kBuffers = 2, class Body>
__device__ __forceinline__ void distribute_parallel_for_tma_tiles(Team<Tr>& team,
                                                                  typename Tr::Idx n,
                                                                  const void* tmap_in,
                                                                  const void* tmap_out,
                                                                  Body&& body) {
  using Idx = typename Tr::Idx;
  static_assert(kSlotBytes % 16 == 0, "TMA boxes have 16 B multiples per row");
  static_assert(kBuffers >= 2 && kBuffers <= 4, "2..4 tile buffers per warp");
  constexpr uint32_t kBox = 32u * kSlotBytes;  // bytes a tile load writes (zero fill included)
  OMPRT_TRACE(Tr, "distribute_parallel_for_tma_tiles");
  extern __shared__ __align__(128) unsigned char omprt_stage_smem[];
  const uint32_t nt = (uint32_t)team.team_size, t = (uint32_t)team.thread_num;
  OMPRT_ASSERT(Tr, nt % 32u == 0, "TMA tiles need whole warps");
  const uint32_t lane = t & 31u, w0 = t & ~31u;
  // buffer j of this warp: omprt_stage_smem + (j * nt + w0) * kSlotBytes
  unsigned char* const buf = omprt_stage_smem + w0 * kSlotBytes;
  const uint32_t buf_stride = nt * kSlotBytes;
  uint64_t* const bar = reinterpret_cast<uint64_t*>(omprt_stage_smem + kBuffers * nt * kSlotBytes) +
                        kBuffers * (t >> 5);
  if (lane == 0) {
#pragma unroll
    for (unsigned j = 0; j < kBuffers; ++j) tma::mbar_init(bar + j, 1);
    tma::fence_mbar_init();
  }
  __syncwarp();
  const Idx total = (Idx)gridDim.x * (Idx)nt;
  const Idx first = (Idx)blockIdx.x * (Idx)nt + (Idx)w0;  // the warp's first iteration
  if (Tr::assume_teams_oversub) OMPRT_ASSERT(Tr, n <= total, "oversubscription assumption violated");
  // prologue: the warp's first kBuffers - 1 tiles in flight
  if (lane == 0) {
#pragma unroll
    for (unsigned j = 0; j + 1 < kBuffers; ++j) {
      const Idx b0 = first + (Idx)j * total;
      if (b0 < n && (j == 0 || !Tr::assume_teams_oversub)) {
        tma::mbar_arrive_expect_tx(bar + j, kBox);
        tma::tensor_load_2d(buf + j * buf_stride, tmap_in, 0, (int32_t)b0, bar + j);
      }
    }
  }
  uint32_t phases = 0;  // bit j: parity of buffer j's next completion
  uint32_t j = 0;       // this tile's buffer
  for (Idx base = first; base < n; base += total) {
    // the tile kBuffers - 1 ahead goes into the buffer the previous tile used, once that
    // tile's store has read it
    const Idx ahead = base + (Idx)(kBuffers - 1) * total;
    const uint32_t ja = j == 0 ? kBuffers - 1 : j - 1;
    if (!Tr::assume_teams_oversub && ahead < n && lane == 0) {
      tma::bulk_wait_read<0>();
      tma::mbar_arrive_expect_tx(bar + ja, kBox);
      tma::tensor_load_2d(buf + ja * buf_stride, tmap_in, 0, (int32_t)ahead, bar + ja);
    }
    tma::mbar_wait(bar + j, (phases >> j) & 1u);
    phases ^= 1u << j;
    unsigned char* const cur = buf + j * buf_stride;
    const Idx iv = base + (Idx)lane;
    if (iv < n) body(iv, cur + lane * kSlotBytes);
    tma::fence_proxy_async_smem();  // this lane's slot writes -> the async proxy
    __syncwarp();
    if (lane == 0) {
      tma::tensor_store_2d(tmap_out, 0, (int32_t)base, cur);
      tma::bulk_commit();
    }
    if (Tr::assume_teams_oversub) break;
    j = j + 1 == kBuffers ? 0 : j + 1;
  }
  if (lane == 0) tma::bulk_wait<0>();  // the stores are complete before the warp exits
}

// ---- TMA streaming of element-wise loops under the Fig. 5 assignment -------------------
// For a `distribute parallel for` whose iteration i reads element i of kIn arrays and
// writes element i of kOut arrays (fp64).  Fig. 5 hands iteration i to global thread
// i mod (T*N), so viewed as a row-major matrix [n / (T*N)][T*N] (row = trip, column = global
// thread), team b owns the N columns [b*N, (b+1)*N) of every row: one 2-D TMA box
// [kRows][N] per array moves kRows trips of the whole team.  kStages boxes per array are in
// flight (the HBM latency is covered by the bytes in flight, not by the team's few warps);
// thread t computes column t of each row in row order -- exactly its Fig. 5 iterations, in
// its Fig. 5 order -- and its outputs go back with one TMA store per array and stage.  The
// trailing n mod (T*N) iterations (a partial row, not a box) run from global memory via
// tail(i).  maps[0 .. kIn) load, maps[kIn .. kIn+kOut) store: generic addresses of
// __grid_constant__ CUtensorMaps of shape [rows = n / (T*N)][T*N] with box [kRows][N].
// body(i, const double (&x)[kIn], double (&y)[kOut]); with kOut = 0 the body writes its
// outputs itself (y is a dummy) -- coalesced direct stores need no staging.  Needs
// tma_stream_smem_bytes<kIn, kOut, kRows, kStages>(N) bytes of dynamic shared memory.
template <unsigned kIn, unsigned kOut, unsigned kRows, unsigned kStages>
__host__ __device__ constexpr uint32_t tma_stream_smem_bytes(uint32_t team_size) {
  return kStages * (kIn + kOut) * kRows * team_size * 8u + kStages * 8u;
}

template <class Tr, unsigned kIn, unsigned kOut, unsigned kRows, unsigned kStages, class Maps,
          class Body, class Tail>
__device__ __forceinline__ void distribute_parallel_for_tma_stream(Team<Tr>& team,
                                                                   typename Tr::Idx n,
                                                                   const Maps* maps, Body&& body,
                                                                   Tail&& tail) {
  using Idx = typename Tr::Idx;
  static_assert(kStages >= 2, "at least double buffered");
  OMPRT_TRACE(Tr, "distribute_parallel_for_tma_stream");
  extern __shared__ __align__(128) unsigned char omprt_stage_smem[];
  double* const sbuf = reinterpret_cast<double*>(omprt_stage_smem);
  const uint32_t N = (uint32_t)team.team_size, t = (uint32_t)team.thread_num;
  const uint32_t box = kRows * N;  // doubles per array per stage
  uint64_t* const full =
      reinterpret_cast<uint64_t*>(omprt_stage_smem + kStages * (kIn + kOut) * box * 8u);
  auto stage_buf = [&](uint32_t s, uint32_t k) { return sbuf + (s * (kIn + kOut) + k) * box; };
  const Idx TN = (Idx)gridDim.x * (Idx)N;
  const Idx rows = n / TN;  // whole trips: the TMA part
  const int32_t col0 = (int32_t)(blockIdx.x * N);
  const uint32_t chunks = (uint32_t)((rows + kRows - 1) / kRows);
  if (t == 0) {
#pragma unroll
    for (uint32_t s = 0; s < kStages; ++s) tma::mbar_init(full + s, 1);
    tma::fence_mbar_init();
#pragma unroll
    for (uint32_t s = 0; s < kStages; ++s)
      if (s < chunks) {
        tma::mbar_arrive_expect_tx(full + s, kIn * box * 8u);
#pragma unroll
        for (uint32_t k = 0; k < kIn; ++k)
          tma::tensor_load_2d(stage_buf(s, k), maps + k, col0, (int32_t)(s * kRows), full + s);
      }
  }
  aligned_barrier();  // barriers initialized before anyone waits on them
  for (uint32_t c = 0; c < chunks; ++c) {
    const uint32_t s = c % kStages;
    tma::mbar_wait(full + s, (c / kStages) & 1u);
    const Idx row0 = (Idx)c * kRows;
    const Idx iv0 = row0 * TN + (Idx)col0 + (Idx)t;  // this thread's iteration in row r: + r*TN
    const double* xin[kIn];
    double* yout[kOut > 0 ? kOut : 1];
#pragma unroll
    for (uint32_t k = 0; k < kIn; ++k) xin[k] = stage_buf(s, k) + t;
#pragma unroll
    for (uint32_t k = 0; k < kOut; ++k) yout[k] = stage_buf(s, kIn + k) + t;
    auto row = [&](uint32_t r) {
      double x[kIn], y[kOut > 0 ? kOut : 1];
#pragma unroll
      for (uint32_t k = 0; k < kIn; ++k) x[k] = xin[k][r * N];
      body(iv0 + (Idx)r * TN, x, y);
#pragma unroll
      for (uint32_t k = 0; k < kOut; ++k) yout[k][r * N] = y[k];
    };
    if (row0 + (Idx)kRows <= rows) {  // a whole box: no per-row bound, fully unrolled
#pragma unroll
      for (uint32_t r = 0; r < kRows; ++r) row(r);
    } else {
      for (uint32_t r = 0; row0 + (Idx)r < rows; ++r) row(r);
    }
    if constexpr (kOut > 0) {
      tma::fence_proxy_async_smem();  // this thread's outputs -> the async proxy
      if (t == 0) tma::bulk_wait_read<kStages - 2>();  // chunk c+1 may rewrite chunk c+1-K's
    }
    aligned_barrier();
    if (t == 0) {
      if constexpr (kOut > 0) {
#pragma unroll
        for (uint32_t k = 0; k < kOut; ++k)
          tma::tensor_store_2d(maps + kIn + k, col0, (int32_t)row0, stage_buf(s, kIn + k));
        tma::bulk_commit();
      }
      if (c + kStages < chunks) {  // this stage's inputs are consumed: refill it
        tma::mbar_arrive_expect_tx(full + s, kIn * box * 8u);
#pragma unroll
        for (uint32_t k = 0; k < kIn; ++k)
          tma::tensor_load_2d(stage_buf(s, k), maps + k, col0, (int32_t)((c + kStages) * kRows),
                              full + s);
      }
    }
  }
  const Idx iv = rows * TN + (Idx)col0 + (Idx)t;  // this thread's last Fig. 5 iteration
  if (iv < n) tail(iv);
  if constexpr (kOut > 0)
    if (t == 0) tma::bulk_wait<0>();
}

}  // namespace omprt
