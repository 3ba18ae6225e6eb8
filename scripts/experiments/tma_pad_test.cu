// Does a 2-D TMA box wider than the tensor's inner dimension give a padded smem layout?
// tensor [n rows][72 doubles] (row stride 576 B), box [32 rows][74 doubles]: expect smem
// rows of 592 B with elements 72, 73 zero-filled (out of bounds), and a store of the same
// box writing only the 72 in-bounds elements of each in-bounds row.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

__global__ void k(const __grid_constant__ CUtensorMap tin, const __grid_constant__ CUtensorMap tout,
                  int y0, double* dump) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ __align__(8) uint64_t bar;
  double* buf = (double*)sm;
  const uint32_t sbar = (uint32_t)__cvta_generic_to_shared(&bar);
  const uint32_t sbuf = (uint32_t)__cvta_generic_to_shared(buf);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sbar));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sbar), "r"(32 * 74 * 8));
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(sbuf), "l"(&tin), "r"(0), "r"(y0), "r"(sbar) : "memory");
  }
  __syncthreads();
  asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}" ::"r"(sbar));
  for (int i = threadIdx.x; i < 32 * 74; i += blockDim.x) dump[i] = buf[i];
  __syncthreads();
  for (int i = threadIdx.x; i < 32 * 74; i += blockDim.x) buf[i] = -buf[i] - 1.0;
  asm volatile("fence.proxy.async.shared::cta;");
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.tile.bulk_group [%0, {%1, %2}], [%3];"
                 ::"l"(&tout), "r"(0), "r"(y0), "r"(sbuf) : "memory");
    asm volatile("cp.async.bulk.commit_group;");
    asm volatile("cp.async.bulk.wait_group 0;");
  }
}

int main() {
  const int n = 40;  // rows: second tile (y0 = 32) has 8 in-bounds rows
  double *g, *o, *dump;
  cudaMalloc(&g, n * 72 * 8 + 4096);
  cudaMalloc(&o, n * 72 * 8 + 4096);
  cudaMalloc(&dump, 32 * 74 * 8);
  double h[n * 72 + 512];
  for (int i = 0; i < n * 72 + 512; ++i) h[i] = i + 1;
  cudaMemcpy(g, h, sizeof h, cudaMemcpyHostToDevice);
  for (int i = 0; i < n * 72 + 512; ++i) h[i] = 7.0;
  cudaMemcpy(o, h, sizeof h, cudaMemcpyHostToDevice);
  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  CUtensorMap tin, tout;
  cuuint64_t dims[2] = {72, (cuuint64_t)n}, strides[1] = {576};
  cuuint32_t box[2] = {74, 32}, es[2] = {1, 1};
  CUresult r1 = enc(&tin, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, g, dims, strides, box, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                    CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  CUresult r2 = enc(&tout, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, o, dims, strides, box, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                    CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode %d %d\n", (int)r1, (int)r2);
  int bad = 0;
  for (int y0 : {0, 32}) {
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 32 * 74 * 8);
    k<<<1, 128, 32 * 74 * 8>>>(tin, tout, y0, dump);
    cudaError_t e = cudaDeviceSynchronize();
    printf("y0=%d kernel %s\n", y0, cudaGetErrorString(e));
    double d[32 * 74];
    cudaMemcpy(d, dump, sizeof d, cudaMemcpyDeviceToHost);
    for (int r = 0; r < 32; ++r)
      for (int c = 0; c < 74; ++c) {
        const int row = y0 + r;
        const double want = (c < 72 && row < n) ? (double)(row * 72 + c + 1) : 0.0;
        if (d[r * 74 + c] != want) { if (bad < 10) printf("smem r%d c%d got %g want %g\n", r, c, d[r * 74 + c], want); ++bad; }
      }
  }
  double ho[n * 72 + 512];
  cudaMemcpy(ho, o, sizeof ho, cudaMemcpyDeviceToHost);
  for (int i = 0; i < n * 72 + 512; ++i) {
    const double want = i < n * 72 ? -(double)(i + 1) - 1.0 : 7.0;
    if (ho[i] != want) { if (bad < 20) printf("out %d got %g want %g\n", i, ho[i], want); ++bad; }
  }
  printf("TMA_PAD_TEST %s (%d mismatches)\n", bad ? "FAIL" : "PASS", bad);
  return bad != 0;
}
