// C1 exploration (r2 x07): the library's own runtime-driven and twin C1 kernels launched from
// a standalone harness (same TU as libomprt.cu), next to the loop forms of c1_loop_forms.cu:
// does the runtime kernel's extra time come from the kernel or from its surroundings?
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I ../../include \
//        -o c1_lib_kernels c1_lib_kernels.cu
#include <algorithm>
#include <cstdio>
#include <vector>

#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/host/runtime.cuh"
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/host/api.cuh"
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/axpy.cuh"

using namespace omprt_kernels;

// bisection of omprt_axpy_rt: F1 = the runtime's loop, no reduction; F2 = a hand loop + the
// runtime's team/league reduction
__global__ void __maxnreg__(kAxpyMaxRegs) F1(int n, double x, const double* __restrict__ b,
    const double* __restrict__ c, double* __restrict__ a, double* out) {
  Team<AxpyTraits> team = init<AxpyTraits>();
  double acc = 0.0;
  distribute_parallel_for(team, n, [&](int i) {
    const double v = fma(x, __ldg(b + i), __ldg(c + i));
    a[i] = v;
    acc += v;
  });
  if (acc == 1.2345) *out = acc;
}
__global__ void __maxnreg__(kAxpyMaxRegs) F2(int n, double x, const double* __restrict__ b,
    const double* __restrict__ c, double* __restrict__ a, double* sum, double* partials,
    unsigned* ticket) {
  Team<AxpyTraits> team = init<AxpyTraits>();
  const int total = gridDim.x * blockDim.x;
  int iv = blockIdx.x * blockDim.x + threadIdx.x;
  double acc = 0.0;
  auto body = [&](int i) { const double v = fma(x, __ldg(b + i), __ldg(c + i)); a[i] = v; acc += v; };
  while (iv + 7 * total < n) {
#pragma unroll
    for (int u = 0; u < 8; ++u) body(iv + u * total);
    iv += 8 * total;
  }
  for (; iv < n; iv += total) body(iv);
  league_reduce_threads(team, acc, Plus{}, sum, partials, ticket);
}

int main() {
  const int n = 1 << 20, T = 8, N = 128;
  double *b, *c, *a, *s, *p;
  unsigned* tk;
  float* scrub;
  cudaMalloc(&b, n * 8); cudaMalloc(&c, n * 8); cudaMalloc(&a, n * 8);
  cudaMalloc(&s, 8); cudaMalloc(&p, 4096 * 8); cudaMalloc(&tk, 64);
  cudaMemset(tk, 0, 64); cudaMemset(s, 0, 8);
  cudaMalloc(&scrub, 256 << 20);
  std::vector<double> h(n);
  for (int i = 0; i < n; ++i) h[i] = (i % 1000) * 1e-3;
  cudaMemcpy(b, h.data(), n * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(c, h.data(), n * 8, cudaMemcpyHostToDevice);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  auto run = [&](const char* name, auto k) {
    std::vector<float> t;
    for (int r = 0; r < 23; ++r) {
      cudaMemsetAsync(scrub, r, 256 << 20);
      cudaEventRecord(e0); k(); cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (r >= 2) t.push_back(ms);
    }
    std::sort(t.begin(), t.end());
    printf("{\"kernel\": \"%s\", \"median_ms\": %.5f, \"min_ms\": %.5f}\n", name, t[t.size() / 2], t[0]);
  };
  for (int pass = 0; pass < 2; ++pass) {
    run("omprt_axpy_rt", [&] { omprt_axpy_rt<AxpyTraits, false><<<T, N>>>(n, 1.5, b, c, a, s, p, tk, nullptr, nullptr); });
    run("cuda_axpy_twin", [&] { cuda_axpy_twin<int32_t, false><<<T, N>>>(n, 1.5, b, c, a, s, p, tk, nullptr, nullptr); });
    run("F1_runtime_loop_no_reduction", [&] { F1<<<T, N>>>(n, 1.5, b, c, a, s); });
    run("F2_hand_loop_runtime_reduction", [&] { F2<<<T, N>>>(n, 1.5, b, c, a, s, p, tk); });
  }
  printf("err %d\n", (int)cudaDeviceSynchronize());
  return 0;
}
