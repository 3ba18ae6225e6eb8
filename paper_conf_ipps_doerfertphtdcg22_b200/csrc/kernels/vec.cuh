// 256-bit global memory accesses (sm_100: LDG.E.ENL2.256 / STG.E.ENL2.256).  Addresses must
// be 32 B aligned.  Used by the loop bodies (user code) of the kernels, identically in the
// runtime-driven kernels and their twins.
#pragma once

namespace omprt_kernels {

__device__ __forceinline__ void ld_nc_v4f64(const double* p, double& a, double& b, double& c,
                                            double& d) {
  asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];" : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
}
// streaming read: no L1 allocation (data used once)
__device__ __forceinline__ void ld_stream_v4f64(const double* p, double& a, double& b, double& c,
                                                double& d) {
  asm("ld.global.nc.L1::no_allocate.v4.f64 {%0,%1,%2,%3}, [%4];"
      : "=d"(a), "=d"(b), "=d"(c), "=d"(d)
      : "l"(p));
}
// Stores carry no "memory" clobber so read-only (ld.global.nc) loads of later iterations
// can be hoisted above them: the kernels never read what these stores write.
__device__ __forceinline__ void st_v4f64(double* p, double a, double b, double c, double d) {
  asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(p), "d"(a), "d"(b), "d"(c), "d"(d));
}
// streaming store (evict-first)
__device__ __forceinline__ void st_cs_v4f64(double* p, double a, double b, double c, double d) {
  asm volatile("st.global.cs.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(p), "d"(a), "d"(b), "d"(c),
               "d"(d));
}

}  // namespace omprt_kernels
