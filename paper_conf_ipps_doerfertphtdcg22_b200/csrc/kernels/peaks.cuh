// Measurement probes -- NOT the hot path.  bench.py times them next to the kernels to get
// the roofs their roofline fractions are taken against where MEASURED_PEAKS.json has none:
//   * L2 -> SM read bandwidth: an L2-resident buffer read with the same 256-bit,
//     L1-non-allocating loads (LDG.E.ENL2.256) the XSBench bracket loads use, either
//     streaming (every 32 B sector of the buffer in order, the hardware's best case) or as
//     random 32 B sectors / random 96 B records (3 adjacent sectors: the bracket record of a
//     lookup's nuclide) -- the access pattern that bounds C3;
//   * FP64 FMA throughput: 8 independent DFMA chains per thread on a full-device grid, the
//     roof of the RSBench lookup ("compute bound").
// Each probe folds what it reads into a value written to `sink` only under a condition that
// never holds, so no load or fma can be removed.
#pragma once
#include <cstdint>

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
