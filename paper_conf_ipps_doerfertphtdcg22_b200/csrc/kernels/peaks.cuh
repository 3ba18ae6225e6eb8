// Measurement probes -- NOT the hot path.  bench.py times them next to the kernels to get
// the roofs their roofline fractions are taken against where MEASURED_PEAKS.json has none:
//   * L2 -> SM read bandwidth: an L2-resident buffer read with the same 256-bit,
//     L1-non-allocating loads (LDG.E.ENL2.256) the XSBench bracket loads use, either
//     streaming (every 32 B sector of the buffer in order, the hardware's best case) or as
//     random 32 B sectors / random 96 B records (3 adjacent sectors: the bracket record of a
//     lookup's nuclide) -- the access pattern that bounds C3;
//   * FP64 FMA throughput: 8 independent DFMA chains per thread on a full-device grid, the
//     roof of the RSBench lookup ("compute bound");
//   * HBM -> SM streaming read bandwidth of a given number of SMs: one team per SM moving
//     its contiguous slice of a buffer larger than L2 by bulk copies (cp.async.bulk, 16 KB
//     each, 8 in flight) into shared memory -- the most an SM can pull from HBM, the roof of
//     a config that by definition runs on few SMs (C1: 8 teams).
// Each probe folds what it reads into a value written to `sink` only under a condition that
// never holds, so no load or fma can be removed.
#pragma once
#include <cstdint>

#include "../common/ptx_tma.cuh"
#include "../host/runtime.cuh"
#include "vec.cuh"

namespace omprt_kernels {

constexpr int kProbeThreads = 256;

// the bracket loads' instruction (LDG.E.NA.ENL2.256), volatile so that a batch of them is
// issued back to back (all in flight) before any result is consumed
__device__ __forceinline__ void probe_ld(const double* p, unsigned long long& a,
                                         unsigned long long& b, unsigned long long& c,
                                         unsigned long long& d) {
  asm volatile("ld.global.nc.L1::no_allocate.v4.u64 {%0,%1,%2,%3}, [%4];"
               : "=l"(a), "=l"(b), "=l"(c), "=l"(d)
               : "l"(p));
}

__device__ __forceinline__ uint32_t probe_hash(uint32_t x) {  // lowbias32
  x ^= x >> 16;
  x *= 0x7feb352du;
  x ^= x >> 15;
  x *= 0x846ca68bu;
  x ^= x >> 16;
  return x;
}

// mode 0: stream all sectors; 1: random 32 B sectors; 2: random 96 B records (3 sectors).
// Every thread issues `per_thread` accesses per rep in the random modes (8 in flight).
// 2 teams of 256 per SM: up to 128 registers, so a batch of 8 random records (96 registers
// of load data) is in flight at once (at the 32 registers of full occupancy ptxas issues
// one record at a time).
template <int Mode>
__global__ void __launch_bounds__(kProbeThreads, 2)
    probe_l2_read(const double* __restrict__ buf, int64_t n_sectors, int32_t reps,
                  int32_t per_thread, double* sink) {
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t nthreads = (int64_t)gridDim.x * blockDim.x;
  unsigned long long acc = 0;  // xor of every word read (integer: off the fp64 pipe)
  if constexpr (Mode == 0) {
    for (int32_t r = 0; r < reps; ++r) {
      for (int64_t i = tid; i < n_sectors; i += 4 * nthreads) {
        unsigned long long a[4][4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int64_t k = i + u * nthreads;
          const int64_t kk = k < n_sectors ? k : i;
          probe_ld(buf + kk * 4, a[u][0], a[u][1], a[u][2], a[u][3]);
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) acc ^= a[u][0] ^ a[u][1] ^ a[u][2] ^ a[u][3];
      }
    }
  } else {
    constexpr int W = Mode == 1 ? 4 : 12;
    const int64_t n_rec = Mode == 1 ? n_sectors : n_sectors / 3;
    for (int32_t r = 0; r < reps; ++r) {
      for (int32_t j = 0; j < per_thread; j += 8) {
        unsigned long long a[8][W];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const uint32_t h =
              probe_hash((uint32_t)tid * 0x9E3779B9u ^ (uint32_t)(r * per_thread + j + u));
          const int64_t rec = (int64_t)(((uint64_t)h * (uint64_t)n_rec) >> 32);
          const double* p = buf + rec * W;
          probe_ld(p, a[u][0], a[u][1], a[u][2], a[u][3]);
          if constexpr (Mode == 2) {
            probe_ld(p + 4, a[u][4], a[u][5], a[u][6], a[u][7]);
            probe_ld(p + 8, a[u][8], a[u][9], a[u][10], a[u][11]);
          }
        }
#pragma unroll
        for (int u = 0; u < 8; ++u)
#pragma unroll
          for (int e = 0; e < W; ++e) acc ^= a[u][e];
      }
    }
  }
  if (acc == 0x9E3779B97F4A7C15ull) *sink = (double)acc;
}

// 8 independent fma chains per thread, `iters` steps each: 16 * iters flops per thread.
__global__ void __launch_bounds__(kProbeThreads) probe_fp64_fma(int64_t iters, double seed,
                                                                double* sink) {
  double x[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) x[k] = seed + threadIdx.x * 1e-9 + k;
  const double m = 0.999999999, c = 1e-9;
  for (int64_t i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = fma(x[k], m, c);
  }
  double acc = 0.0;
#pragma unroll
  for (int k = 0; k < 8; ++k) acc += x[k];
  if (acc == -1.2345e300) *sink = acc;
}

// HBM stream probe: team b reads bytes [b * slice, (b + 1) * slice) in kHbmChunk pieces,
// 8 bulk copies in flight on a ring of kHbmStages mbarriers (one issuing thread).  Mode 1 also
// writes every second landed chunk back to `dst` (bulk store from shared memory): 2 bytes
// read per byte written, C1's mix (b and c read, a written).
constexpr uint32_t kHbmChunk = 16384;
constexpr int kHbmStages = 12;  // 8 loads in flight + 4 stages whose stores are reading
template <int Mode>
__global__ void __launch_bounds__(32, 1)
    probe_hbm_stream(const unsigned char* __restrict__ buf, unsigned char* __restrict__ dst,
                     int64_t slice, double* sink) {
  extern __shared__ __align__(128) unsigned char ring[];
  __shared__ uint64_t bars[kHbmStages];
  namespace tma = omprt::tma;
  if (threadIdx.x != 0) return;
  for (int k = 0; k < kHbmStages; ++k) tma::mbar_init(&bars[k], 1);
  tma::fence_mbar_init();
  const unsigned char* src = buf + (int64_t)blockIdx.x * slice;
  unsigned char* out = Mode == 1 ? dst + (int64_t)blockIdx.x * (slice / 2) : nullptr;
  const int64_t chunks = slice / kHbmChunk;
  uint32_t phase = 0;
  // chunk c has landed in stage c % kHbmStages: mode 1 writes the odd ones out.  Landings
  // are taken kLag = 8 chunks behind the loads (8 loads in flight), so a stage's store has
  // had 4 loads' time to read it before the stage is refilled.
  constexpr int64_t kLag = 8;
  auto landed = [&](int64_t c) {
    const int k = (int)(c % kHbmStages);
    tma::mbar_wait(&bars[k], phase >> k & 1u);
    phase ^= 1u << k;
    if constexpr (Mode == 1) {
      if (c & 1) {
        tma::bulk_store(out + (c >> 1) * kHbmChunk, ring + (size_t)k * kHbmChunk, kHbmChunk);
        tma::bulk_commit();
      }
    }
  };
  for (int64_t c = 0; c < chunks; ++c) {
    const int k = (int)(c % kHbmStages);
    if (c >= kLag) landed(c - kLag);
    if constexpr (Mode == 1) {
      // the store of chunk c - kHbmStages (if any) has read its stage: at most the
      // (kHbmStages - kLag) / 2 stores committed after it may still be reading
      if (c >= kHbmStages) tma::bulk_wait_read<(kHbmStages - kLag) / 2>();
    }
    tma::mbar_arrive_expect_tx(&bars[k], kHbmChunk);
    tma::bulk_load(ring + (size_t)k * kHbmChunk, src + c * kHbmChunk, kHbmChunk, &bars[k]);
  }
  for (int64_t c = chunks > kLag ? chunks - kLag : 0; c < chunks; ++c) landed(c);
  if constexpr (Mode == 1) tma::bulk_wait<0>();
  const double v = *reinterpret_cast<const double*>(ring);
  if (v == -1.2345e300) *sink = v;
}

}  // namespace omprt_kernels

// bytes: size of the L2-resident buffer (>= 96, 32 B aligned); reps: passes (mode 0) or
// rounds of per_thread accesses (modes 1, 2); teams = 0: 2 per SM.  The caller times the
// launch on `stream`; bytes read = reps * bytes (mode 0), reps * per_thread * threads * 32
// or * 96 (modes 1, 2).
extern "C" int omprt_probe_l2_read(const double* buf, uint64_t bytes, int32_t mode, int32_t reps,
                                   int32_t per_thread, int32_t teams, double* sink,
                                   void* stream) {
  using namespace omprt_kernels;
  OMPRT_CHECK_ARG(buf && sink && bytes >= 96 && ((uintptr_t)buf & 31) == 0 && reps > 0 &&
                      mode >= 0 && mode <= 2 && (mode == 0 || (per_thread > 0 && per_thread % 8 == 0)),
                  "omprt_probe_l2_read: bad arguments");
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (teams <= 0) teams = 2 * sms;
  const int64_t ns = (int64_t)(bytes / 32);
  cudaStream_t s = as_stream(stream);
  if (mode == 0) probe_l2_read<0><<<teams, kProbeThreads, 0, s>>>(buf, ns, reps, per_thread, sink);
  else if (mode == 1) probe_l2_read<1><<<teams, kProbeThreads, 0, s>>>(buf, ns, reps, per_thread, sink);
  else probe_l2_read<2><<<teams, kProbeThreads, 0, s>>>(buf, ns, reps, per_thread, sink);
  return check_launch("probe_l2_read");
}

// flops = 16 * iters * teams * 256; teams = 0: 8 per SM.
extern "C" int omprt_probe_fp64_fma(int64_t iters, int32_t teams, double* sink, void* stream) {
  using namespace omprt_kernels;
  OMPRT_CHECK_ARG(iters > 0 && sink, "omprt_probe_fp64_fma: bad arguments");
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (teams <= 0) teams = 8 * sms;
  probe_fp64_fma<<<teams, kProbeThreads, 0, as_stream(stream)>>>(iters, 1.0, sink);
  return check_launch("probe_fp64_fma");
}

// bytes read = teams * slice, slice = (bytes / teams) rounded down to 16 KB; one team of 32
// threads per SM (teams <= the SM count), 192 KB of dynamic shared memory each.  Use a
// buffer larger than L2 (126 MB) so the reads come from HBM.  dst (mode 1 only): bytes / 2
// writable bytes; bytes written = teams * slice / 2.
extern "C" int omprt_probe_hbm_stream(const void* buf, void* dst, uint64_t bytes, int32_t mode,
                                      int32_t teams, double* sink, void* stream) {
  using namespace omprt_kernels;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t slice =
      teams > 0 ? (int64_t)(bytes / (uint64_t)teams) / (2 * kHbmChunk) * (2 * kHbmChunk) : 0;
  OMPRT_CHECK_ARG(buf && sink && ((uintptr_t)buf & 15) == 0 && teams > 0 && teams <= sms &&
                      slice >= (int64_t)(2 * kHbmChunk) && (mode == 0 || mode == 1) &&
                      (mode == 0 || (dst && ((uintptr_t)dst & 15) == 0)),
                  "omprt_probe_hbm_stream: bad arguments");
  const int smem = (int)kHbmChunk * kHbmStages;
  const auto k = mode == 0 ? probe_hbm_stream<0> : probe_hbm_stream<1>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k<<<teams, 32, smem, as_stream(stream)>>>(static_cast<const unsigned char*>(buf),
                                           static_cast<unsigned char*>(dst), slice, sink);
  return check_launch("probe_hbm_stream");
}
