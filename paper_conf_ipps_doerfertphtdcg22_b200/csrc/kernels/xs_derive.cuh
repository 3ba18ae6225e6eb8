// XSBench's derived tables built on the device from the nuclide grids (SURVEY App. A.1:
// "unionized grid: all energies, sorted; index grid: per unionized energy and nuclide, the
// lower bracket index"), so an end-to-end step ships only the raw problem data (nuclide
// grids + materials, 36.9 MB for the small problem) instead of 147.6 MB of tables.
//
//   unionized[e]       = the e-th smallest of all n_iso * n_gp energies (a stable merge of the
//                        n_iso per-nuclide sorted runs of the energies' order-preserving
//                        64-bit keys, ceil(log2 n_iso) merge-path levels; the same order as
//                        a stable radix sort, 90 vs 131 us for the small problem)
//   index_grid[e][q]   = clip(#{k : E_q[k] <= unionized[e]} - 1, 0, n_gp - 2)
//
// The index rows are a column-wise prefix count over the sorted order: row e differs from
// row e-1 only in the column of the nuclide that energy e came from.  Rows are cut into
// chunks of kDeriveRows; (A) counts each chunk's nuclide ids, (B) scans the counts over the
// chunks per nuclide, (C) walks each chunk with one thread per nuclide column, writing whole
// rows (n_iso x 2 B, coalesced).  Equal energies (ties) are handled exactly: a row whose
// energy equals the next rows' also counts those rows (`<=`), by a look-ahead that only runs
// at ties.  Energies must be finite and not -0.0 (the proxy app draws them from [0, 1)).
#pragma once
#include <cub/block/block_scan.cuh>

#include "../host/runtime.cuh"

namespace omprt_kernels {

constexpr int kDeriveRows = 256;  // rows per chunk
constexpr int kDeriveMaxIso = 4096;

__global__ void xs_derive_keys(const double* __restrict__ g, int32_t n_gp, int64_t n,
                               unsigned long long* __restrict__ keys,
                               uint16_t* __restrict__ ids) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long b = (unsigned long long)__double_as_longlong(__ldg(g + i * 6));
    keys[i] = (b >> 63) ? ~b : (b | (1ull << 63));  // IEEE order as unsigned order
    ids[i] = (uint16_t)(i / n_gp);
  }
}

__global__ void xs_derive_unionized(const unsigned long long* __restrict__ keys, int64_t n,
                                    double* __restrict__ U) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n;
       e += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = keys[e];
    U[e] = __longlong_as_double((long long)((k >> 63) ? (k & ~(1ull << 63)) : ~k));
  }
}

// The union as a merge of the per-nuclide runs: every nuclide's energies are sorted (the
// index grid's definition presumes it), so the keys in nuclide-major order are n_iso sorted
// runs of n_gp.  ceil(log2 n_iso) levels of pairwise merges (runs of L -> 2L; the last run
// of a level may be short or alone) give the same order as a stable sort of the keys: ties
// go to the lower run, i.e. the lower nuclide, then the lower k -- CUB's stable radix order.
// Each thread writes kMergeItems consecutive outputs: the merge-path co-rank of its first
// output by bisection, then a sequential merge.
constexpr int kMergeItems = 4;
__global__ void xs_derive_merge(const unsigned long long* __restrict__ kin,
                                const uint16_t* __restrict__ iin,
                                unsigned long long* __restrict__ kout,
                                uint16_t* __restrict__ iout, int64_t n, int64_t L) {
  const int64_t o0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * kMergeItems;
  if (o0 >= n) return;
  const int64_t o1 = o0 + kMergeItems < n ? o0 + kMergeItems : n;
  int64_t o = o0;
  while (o < o1) {
    // the pair of runs [a0, a0+la) and [b0, b0+lb) that output position o belongs to
    const int64_t a0 = (o / (2 * L)) * (2 * L);
    const int64_t b0 = a0 + L < n ? a0 + L : n;
    const int64_t la = b0 - a0, lb = (b0 + L < n ? b0 + L : n) - b0;
    const int64_t pend = b0 + lb;  // end of this pair's output
    const int64_t d = o - a0;
    int64_t lo = d - lb > 0 ? d - lb : 0, hi = d < la ? d : la;
    while (lo < hi) {  // #A among the first d outputs (A wins ties)
      const int64_t i = (lo + hi) >> 1;
      if (__ldg(kin + a0 + i) <= __ldg(kin + b0 + (d - i - 1))) lo = i + 1;
      else hi = i;
    }
    int64_t i = lo, j = d - lo;
    const int64_t stop = o1 < pend ? o1 : pend;
    // heads of both runs in registers (an exhausted run's head is +inf: never taken)
    constexpr unsigned long long kInf = ~0ull;
    unsigned long long ka = i < la ? __ldg(kin + a0 + i) : kInf;
    unsigned long long kb = j < lb ? __ldg(kin + b0 + j) : kInf;
    for (; o < stop; ++o) {
      const bool takeA = j >= lb || (i < la && ka <= kb);
      if (takeA) {
        kout[o] = ka;
        iout[o] = __ldg(iin + a0 + i);
        ++i;
        ka = i < la ? __ldg(kin + a0 + i) : kInf;
      } else {
        kout[o] = kb;
        iout[o] = __ldg(iin + b0 + j);
        ++j;
        kb = j < lb ? __ldg(kin + b0 + j) : kInf;
      }
    }
  }
}

// (A) per chunk: how many of its rows come from each nuclide
__global__ void xs_derive_hist(const uint16_t* __restrict__ ids, int64_t n, int32_t n_iso,
                               uint32_t* __restrict__ hist) {
  __shared__ uint32_t h[kDeriveMaxIso];
  for (int q = threadIdx.x; q < n_iso; q += blockDim.x) h[q] = 0;
  __syncthreads();
  const int64_t r0 = (int64_t)blockIdx.x * kDeriveRows;
  const int64_t r1 = r0 + kDeriveRows < n ? r0 + kDeriveRows : n;
  for (int64_t e = r0 + threadIdx.x; e < r1; e += blockDim.x) atomicAdd(&h[ids[e]], 1u);
  __syncthreads();
  for (int q = threadIdx.x; q < n_iso; q += blockDim.x)
    hist[(int64_t)blockIdx.x * n_iso + q] = h[q];
}

// (B) per nuclide (one block each): exclusive scan of the chunk counts, in place
constexpr int kScanThreads = 1024;
__global__ void __launch_bounds__(kScanThreads)
    xs_derive_scan(uint32_t* __restrict__ hist, int32_t n_chunks, int32_t n_iso) {
  using Scan = cub::BlockScan<uint32_t, kScanThreads>;
  __shared__ typename Scan::TempStorage tmp;
  const int q = blockIdx.x;
  uint32_t carry = 0;
  for (int c0 = 0; c0 < n_chunks; c0 += kScanThreads) {
    const int c = c0 + threadIdx.x;
    const uint32_t v = c < n_chunks ? hist[(int64_t)c * n_iso + q] : 0u;
    uint32_t ex, tot;
    Scan(tmp).ExclusiveSum(v, ex, tot);
    if (c < n_chunks) hist[(int64_t)c * n_iso + q] = carry + ex;
    carry += tot;
    __syncthreads();  // tmp is reused by the next tile
  }
}

// (C) per chunk, one thread per nuclide column: the running count -> index rows
__global__ void xs_derive_index(const uint16_t* __restrict__ ids, const double* __restrict__ U,
                                const uint32_t* __restrict__ start, int64_t n, int32_t n_iso,
                                int32_t n_gp, uint16_t* __restrict__ index16) {
  __shared__ uint16_t sid[kDeriveRows];
  __shared__ double su[kDeriveRows + 1];
  const int64_t r0 = (int64_t)blockIdx.x * kDeriveRows;
  const int rows = (int)(r0 + kDeriveRows < n ? kDeriveRows : n - r0);
  for (int k = threadIdx.x; k < rows; k += blockDim.x) sid[k] = ids[r0 + k];
  for (int k = threadIdx.x; k <= rows; k += blockDim.x) su[k] = r0 + k < n ? U[r0 + k] : 0.0;
  __syncthreads();
  const int32_t kmax = n_gp - 2;
  for (int q = threadIdx.x; q < n_iso; q += blockDim.x) {
    int64_t cnt = start[(int64_t)blockIdx.x * n_iso + q];
    for (int k = 0; k < rows; ++k) {
      cnt += sid[k] == q;
      int64_t v = cnt;
      if (r0 + k + 1 < n && su[k + 1] == su[k]) {  // tie: count the equal rows ahead too
        for (int64_t e2 = r0 + k + 1; e2 < n && U[e2] == su[k]; ++e2) v += ids[e2] == q;
      }
      v -= 1;
      index16[(r0 + k) * n_iso + q] = (uint16_t)(v < 0 ? 0 : (v > kmax ? kmax : v));
    }
  }
}

// (C') the same rows for an even n_iso <= kDeriveBallotIso with every thread busy: thread
// t owns the column pair (2p, 2p+1), p = t mod n_iso/2, over one of the chunk's row segments
// (t div n_iso/2) and writes both entries of a row with one 32-bit store (a warp: one
// contiguous row piece).  A segment's starting counts come from per-(warp, nuclide) ballot
// masks of the chunk's rows (popc of the rows before the segment), then the thread walks its
// rows as (C) does.  Ties as in (C).
constexpr int kDeriveBallotIso = 256;
constexpr int kDeriveWords = kDeriveRows / 32;
__global__ void __launch_bounds__(kDeriveRows)
    xs_derive_index_pairs(const uint16_t* __restrict__ ids, const double* __restrict__ U,
                          const uint32_t* __restrict__ start, int64_t n, int32_t n_iso,
                          int32_t n_gp, uint16_t* __restrict__ index16) {
  __shared__ uint32_t mask[kDeriveWords][kDeriveBallotIso];
  __shared__ uint16_t sidt[kDeriveRows];  // nuclide id | 0x8000 when the next energy ties
  const int64_t r0 = (int64_t)blockIdx.x * kDeriveRows;
  const int rows = (int)(r0 + kDeriveRows < n ? kDeriveRows : n - r0);
  const int k = threadIdx.x, w = k >> 5;
  const int my = k < rows ? (int)ids[r0 + k] : -1;
  if (k < rows) {
    const bool tie = r0 + k + 1 < n && U[r0 + k + 1] == U[r0 + k];
    sidt[k] = (uint16_t)(my | (tie ? 0x8000 : 0));
  }
  for (int q = 0; q < n_iso; ++q) {
    const uint32_t m = __ballot_sync(0xffffffffu, my == q);
    if ((k & 31) == 0) mask[w][q] = m;
  }
  __syncthreads();
  const int pairs = n_iso >> 1, segs = kDeriveRows / pairs;
  const int seg = k / pairs, q0 = 2 * (k - seg * pairs), q1 = q0 + 1;
  if (seg >= segs) return;
  const int per = (rows + segs - 1) / segs;
  const int rs = seg * per, re = rs + per < rows ? rs + per : rows;
  // counts of rows < rs of this chunk, per column (<= n_gp: int32)
  int c0 = (int)start[(int64_t)blockIdx.x * n_iso + q0];
  int c1 = (int)start[(int64_t)blockIdx.x * n_iso + q1];
  for (int j = 0; j < (rs >> 5); ++j) {
    c0 += __popc(mask[j][q0]);
    c1 += __popc(mask[j][q1]);
  }
  if (rs & 31) {
    const uint32_t below = (1u << (rs & 31)) - 1u;
    c0 += __popc(mask[rs >> 5][q0] & below);
    c1 += __popc(mask[rs >> 5][q1] & below);
  }
  const int kmax = n_gp - 2;
  uint32_t* out = reinterpret_cast<uint32_t*>(index16 + (r0 + rs) * n_iso + q0);
#pragma unroll 4
  for (int r = rs; r < re; ++r, out += pairs) {
    const int v = sidt[r], id = v & 0x7fff;
    c0 += id == q0;
    c1 += id == q1;
    int v0 = c0, v1 = c1;
    if (v & 0x8000) {  // tie: count the equal rows ahead too
      const double u = U[r0 + r];
      for (int64_t e2 = r0 + r + 1; e2 < n && U[e2] == u; ++e2) {
        v0 += ids[e2] == q0;
        v1 += ids[e2] == q1;
      }
    }
    v0 = min(max(v0 - 1, 0), kmax);
    v1 = min(max(v1 - 1, 0), kmax);
    *out = (uint32_t)v0 | ((uint32_t)v1 << 16);
  }
}

struct DeriveLayout {
  size_t keys_in, keys_out, ids_in, ids_out, hist, total;
};
inline size_t al256(size_t b) { return (b + 255) & ~size_t(255); }

inline int xs_derive_layout(int32_t n_iso, int32_t n_gp, DeriveLayout* L) {
  OMPRT_CHECK_ARG(n_iso > 0 && n_iso <= kDeriveMaxIso && n_gp >= 2 && n_gp <= 65536 &&
                      (int64_t)n_iso * n_gp < (1ll << 31),
                  "omprt_xs_derive: need 0 < n_isotopes <= %d, 2 <= n_gridpoints <= 65536",
                  kDeriveMaxIso);
  const int64_t n = (int64_t)n_iso * n_gp;
  const int64_t chunks = (n + kDeriveRows - 1) / kDeriveRows;
  size_t off = 0;
  L->keys_in = off;
  off += al256(8 * n);
  L->keys_out = off;
  off += al256(8 * n);
  L->ids_in = off;
  off += al256(2 * n);
  L->ids_out = off;
  off += al256(2 * n);
  L->hist = off;
  off += al256(4 * chunks * n_iso);
  L->total = off;
  return OMPRT_OK;
}

inline int xs_derive(const double* nuclide_grid, int32_t n_iso, int32_t n_gp, double* U,
                     uint16_t* index16, void* tmp, size_t tmp_bytes, cudaStream_t s) {
  DeriveLayout L;
  if (int r = xs_derive_layout(n_iso, n_gp, &L)) return r;
  OMPRT_CHECK_ARG(nuclide_grid && U && index16 && tmp, "omprt_xs_derive: null pointer");
  OMPRT_CHECK_ARG(tmp_bytes >= L.total, "omprt_xs_derive: tmp needs %zu B", L.total);
  const int64_t n = (int64_t)n_iso * n_gp;
  const int32_t chunks = (int32_t)((n + kDeriveRows - 1) / kDeriveRows);
  unsigned char* b = (unsigned char*)tmp;
  auto* kin = (unsigned long long*)(b + L.keys_in);
  auto* kout = (unsigned long long*)(b + L.keys_out);
  auto* iin = (uint16_t*)(b + L.ids_in);
  auto* iout = (uint16_t*)(b + L.ids_out);
  auto* hist = (uint32_t*)(b + L.hist);
  xs_derive_keys<<<1024, 256, 0, s>>>(nuclide_grid, n_gp, n, kin, iin);
  // merge levels, ping-ponging between the two key/id buffers; the result ends in kout/iout
  const unsigned mblocks = (unsigned)((n + 256 * kMergeItems - 1) / (256 * kMergeItems));
  int levels = 0;
  for (int64_t run = n_gp; run < n; run *= 2) ++levels;
  if (levels == 0) {
    OMPRT_CUDA_TRY(cudaMemcpyAsync(kout, kin, n * sizeof(unsigned long long),
                                   cudaMemcpyDeviceToDevice, s));
    OMPRT_CUDA_TRY(cudaMemcpyAsync(iout, iin, n * sizeof(uint16_t), cudaMemcpyDeviceToDevice, s));
  }
  {
    // an odd number of levels starts in (kin -> kout), an even one in (kout <- kin copied)
    unsigned long long* ks[2] = {kin, kout};
    uint16_t* is[2] = {iin, iout};
    int src = (levels % 2 == 0) ? 1 : 0;  // so that the last level writes kout/iout
    if (levels > 0 && src == 1) {
      OMPRT_CUDA_TRY(cudaMemcpyAsync(kout, kin, n * sizeof(unsigned long long),
                                     cudaMemcpyDeviceToDevice, s));
      OMPRT_CUDA_TRY(cudaMemcpyAsync(iout, iin, n * sizeof(uint16_t), cudaMemcpyDeviceToDevice,
                                     s));
    }
    for (int64_t run = n_gp; run < n; run *= 2) {
      xs_derive_merge<<<mblocks, 256, 0, s>>>(ks[src], is[src], ks[src ^ 1], is[src ^ 1], n, run);
      src ^= 1;
    }
  }
  xs_derive_unionized<<<1024, 256, 0, s>>>(kout, n, U);
  xs_derive_hist<<<chunks, 256, 0, s>>>(iout, n, n_iso, hist);
  xs_derive_scan<<<n_iso, kScanThreads, 0, s>>>(hist, chunks, n_iso);
  if (n_iso <= kDeriveBallotIso && n_iso % 2 == 0 && ((uintptr_t)index16 & 3) == 0)
    xs_derive_index_pairs<<<chunks, kDeriveRows, 0, s>>>(iout, U, hist, n, n_iso, n_gp, index16);
  else
    xs_derive_index<<<chunks, 128, 0, s>>>(iout, U, hist, n, n_iso, n_gp, index16);
  return check_launch("omprt_xs_derive");
}

}  // namespace omprt_kernels

extern "C" int omprt_xs_derive_tmp_bytes(int32_t n_isotopes, int32_t n_gridpoints,
                                         uint64_t* bytes) {
  using namespace omprt_kernels;
  OMPRT_CHECK_ARG(bytes != nullptr, "omprt_xs_derive_tmp_bytes: null output");
  DeriveLayout L;
  if (int r = xs_derive_layout(n_isotopes, n_gridpoints, &L)) return r;
  *bytes = L.total;
  return OMPRT_OK;
}

extern "C" int omprt_xs_derive(const double* nuclide_grid, int32_t n_isotopes,
                               int32_t n_gridpoints, double* unionized, uint16_t* index_grid16,
                               void* tmp, uint64_t tmp_bytes, void* stream) {
  using namespace omprt_kernels;
  Workspace* w;
  if (int r = current_ws(&w)) return r;
  return xs_derive(nuclide_grid, n_isotopes, n_gridpoints, unionized, index_grid16, tmp,
                   tmp_bytes, as_stream(stream));
}
