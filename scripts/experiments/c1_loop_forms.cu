// C1 exploration (r2 x06): why does the runtime's unrolled Fig. 5 loop run slower than the
// twin's hand-written grid-stride loop under the same register budget?  Four loop forms of
// a[i] = fma(x, b[i], c[i]); acc += a[i] on 8 teams x 128 threads, n = 2^20, L2 flushed
// before every launch, CUDA events, median of 21.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o c1_loop_forms c1_loop_forms.cu
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

template <class Idx>
__device__ __forceinline__ void fin(double acc, double* out) { if (acc == 1.2345) *out = acc; }

// A: the twin's form (signed index, 8 loads of b and c then 8 fma/store)
template <class Idx>
__global__ void __maxnreg__(56) formA(Idx n, double x, const double* __restrict__ b,
    const double* __restrict__ c, double* __restrict__ a, double* out) {
  const Idx stride = (Idx)gridDim.x * blockDim.x;
  Idx i = (Idx)blockIdx.x * blockDim.x + threadIdx.x;
  double acc = 0.0;
  for (; i + 7 * stride < n; i += 8 * stride) {
    double bv[8], cv[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) { bv[u] = __ldg(b + i + u * stride); cv[u] = __ldg(c + i + u * stride); }
#pragma unroll
    for (int u = 0; u < 8; ++u) { const double v = fma(x, bv[u], cv[u]); a[i + u * stride] = v; acc += v; }
  }
  for (; i < n; i += stride) { const double v = fma(x, __ldg(b + i), __ldg(c + i)); a[i] = v; acc += v; }
  fin<Idx>(acc, out);
}
// C: the runtime's form (a per-iteration body called 8 times per trip, then the remainder)
template <class Idx>
__global__ void __maxnreg__(56) formC(Idx n, double x, const double* __restrict__ b,
    const double* __restrict__ c, double* __restrict__ a, double* out) {
  const Idx total = (Idx)gridDim.x * blockDim.x;
  Idx iv = (Idx)blockIdx.x * blockDim.x + threadIdx.x;
  double acc = 0.0;
  auto body = [&](Idx i) { const double v = fma(x, __ldg(b + i), __ldg(c + i)); a[i] = v; acc += v; };
  while (iv + 7 * total < n) {
#pragma unroll
    for (int u = 0; u < 8; ++u) body(iv + (Idx)u * total);
    iv += 8 * total;
  }
#pragma unroll 1
  for (; iv < n; iv += total) body(iv);
  fin<Idx>(acc, out);
}
// E: the runtime's form with the trip's loads hoisted by the body split into load / use
template <class Idx>
__global__ void __maxnreg__(56) formE(Idx n, double x, const double* __restrict__ b,
    const double* __restrict__ c, double* __restrict__ a, double* out) {
  const Idx total = (Idx)gridDim.x * blockDim.x;
  Idx iv = (Idx)blockIdx.x * blockDim.x + threadIdx.x;
  double acc = 0.0;
  while (iv + 7 * total < n) {
    const double* bp = b + iv; const double* cp = c + iv; double* ap = a + iv;
    double bv[8], cv[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) { bv[u] = __ldg(bp + (Idx)u * total); cv[u] = __ldg(cp + (Idx)u * total); }
#pragma unroll
    for (int u = 0; u < 8; ++u) { const double v = fma(x, bv[u], cv[u]); ap[(Idx)u * total] = v; acc += v; }
    iv += 8 * total;
  }
  for (; iv < n; iv += total) { const double v = fma(x, __ldg(b + iv), __ldg(c + iv)); a[iv] = v; acc += v; }
  fin<Idx>(acc, out);
}

int main() {
  const int n = 1 << 20, T = 8, N = 128;
  double *b, *c, *a, *o; float* scrub;
  cudaMalloc(&b, n * 8); cudaMalloc(&c, n * 8); cudaMalloc(&a, n * 8); cudaMalloc(&o, 8);
  cudaMalloc(&scrub, 256 << 20);
  cudaMemset(b, 0, n * 8); cudaMemset(c, 0, n * 8);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  auto run = [&](const char* name, auto k) {
    std::vector<float> t;
    for (int r = 0; r < 23; ++r) {
      cudaMemsetAsync(scrub, r, 256 << 20);
      cudaEventRecord(e0); k(); cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (r >= 2) t.push_back(ms);
    }
    std::sort(t.begin(), t.end());
    printf("{\"form\": \"%s\", \"median_ms\": %.5f, \"min_ms\": %.5f}\n", name, t[t.size() / 2], t[0]);
  };
  for (int pass = 0; pass < 2; ++pass) {
    run("A_twin_signed", [&] { formA<int><<<T, N>>>(n, 1.5, b, c, a, o); });
    run("A_twin_unsigned", [&] { formA<unsigned><<<T, N>>>(n, 1.5, b, c, a, o); });
    run("C_runtime_signed", [&] { formC<int><<<T, N>>>(n, 1.5, b, c, a, o); });
    run("C_runtime_unsigned", [&] { formC<unsigned><<<T, N>>>(n, 1.5, b, c, a, o); });
    run("E_runtime_split_signed", [&] { formE<int><<<T, N>>>(n, 1.5, b, c, a, o); });
  }
  return cudaDeviceSynchronize() != cudaSuccess;
}
