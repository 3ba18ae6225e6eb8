// Exploration harness (NOT part of libomprt.so): RSBench body variants x launch bounds.
#include <cuda_runtime.h>
#include <cstdint>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/rs_body.cuh"
using namespace omprt_kernels;
__device__ __forceinline__ uint64_t rs_old(const RSTables& t, uint64_t seed0, int64_t i,
                                                  double* macro_out) {
  uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)i);
  const double E = lcg_double(seed);
  const int mat = pick_mat(seed);
  const double sqrtE = sqrt(E);
  const int nn = __ldg(t.num_nucs + mat);
  double M0 = 0.0, M1 = 0.0, M2 = 0.0, M3 = 0.0;
  for (int j = 0; j < nn; ++j) {
    const int nuc = __ldg(t.mats + mat * t.max_num_nucs + j);
    const double conc = __ldg(t.concs + mat * t.max_num_nucs + j);
    const int nw = __ldg(t.n_windows + nuc);
    const double spacing = 1.0 / nw;
    int w = (int)(E / spacing);
    if (w >= nw) w = nw - 1;
    // sigT factors for l = 0..3 (numL = 4)
    cplx f[4];
#pragma unroll
    for (int l = 0; l < 4; ++l) {
      double phi = __ldg(t.k0rs + nuc * 4 + l) * sqrtE;
      if (l == 1) phi -= -atan(phi);
      else if (l == 2) phi -= atan(3.0 * phi / (3.0 - phi * phi));
      else if (l == 3) phi -= atan(phi * (15.0 - phi * phi) / (15.0 - 6.0 * phi * phi));
      phi *= 2.0;
      double sn, cs;
      sincos(phi, &sn, &cs);
      f[l] = {cs, -sn};
    }
    const int64_t wi = (int64_t)__ldg(t.win_off + nuc) + w;
    const double2 TA = __ldg(reinterpret_cast<const double2*>(t.windows + wi * 4));
    const double Fw = __ldg(t.windows + wi * 4 + 2);
    const int2 rg = __ldg(reinterpret_cast<const int2*>(t.win_range + wi * 2));
    double sigT = E * TA.x, sigA = E * TA.y, sigF = E * Fw;
    for (int p = rg.x; p < rg.y; ++p) {
      const double2* P = reinterpret_cast<const double2*>(t.poles + (int64_t)p * 8);
      const double2 EA = __ldg(P + 0), RT = __ldg(P + 1), RA = __ldg(P + 2), RF = __ldg(P + 3);
      const int l = __ldg(t.pole_l + p);
      const cplx Z = {(E - EA.x) * 0.5, (0.0 - EA.y) * 0.5};
      const cplx W = faddeeva_w(Z);
      const cplx fl = l == 0 ? f[0] : l == 1 ? f[1] : l == 2 ? f[2] : f[3];
      const cplx Wf = cmul(W, fl);
      sigT += RT.x * Wf.r - RT.y * Wf.i;
      sigA += RA.x * W.r - RA.y * W.i;
      sigF += RF.x * W.r - RF.y * W.i;
    }
    M0 += sigT * conc;
    M1 += sigA * conc;
    M2 += sigF * conc;
    M3 += (sigT - sigA) * conc;
  }
  if constexpr (false) {
    macro_out[0] = M0;
    macro_out[1] = M1;
    macro_out[2] = M2;
    macro_out[3] = M3;
  }
  double mx = -1.0;
  uint64_t v = 1;
  if (M0 > mx) { mx = M0; v = 1; }
  if (M1 > mx) { mx = M1; v = 2; }
  if (M2 > mx) { mx = M2; v = 3; }
  if (M3 > mx) { mx = M3; v = 4; }
  return v;
}

__device__ __forceinline__ uint64_t rs_polepf(const RSTables& t, uint64_t seed0, int64_t i,
                                                  double* macro_out) {
  uint64_t seed = lcg_fast_forward(seed0, 2ull * (uint64_t)i);
  const double E = lcg_double(seed);
  const int mat = pick_mat(seed);
  const double sqrtE = sqrt(E);
  const int nn = __ldg(t.num_nucs + mat);
  double M0 = 0.0, M1 = 0.0, M2 = 0.0, M3 = 0.0;
  for (int j = 0; j < nn; ++j) {
    const int nuc = __ldg(t.mats + mat * t.max_num_nucs + j);
    const double conc = __ldg(t.concs + mat * t.max_num_nucs + j);
    const int nw = __ldg(t.n_windows + nuc);
    const double spacing = 1.0 / nw;
    int w = (int)(E / spacing);
    if (w >= nw) w = nw - 1;
    // sigT factors for l = 0..3 (numL = 4)
    cplx f[4];
#pragma unroll
    for (int l = 0; l < 4; ++l) {
      double phi = __ldg(t.k0rs + nuc * 4 + l) * sqrtE;
      if (l == 1) phi -= -atan(phi);
      else if (l == 2) phi -= atan(3.0 * phi / (3.0 - phi * phi));
      else if (l == 3) phi -= atan(phi * (15.0 - phi * phi) / (15.0 - 6.0 * phi * phi));
      phi *= 2.0;
      double sn, cs;
      sincos(phi, &sn, &cs);
      f[l] = {cs, -sn};
    }
    const int64_t wi = (int64_t)__ldg(t.win_off + nuc) + w;
    const double2 TA = __ldg(reinterpret_cast<const double2*>(t.windows + wi * 4));
    const double Fw = __ldg(t.windows + wi * 4 + 2);
    const int2 rg = __ldg(reinterpret_cast<const int2*>(t.win_range + wi * 2));
    double sigT = E * TA.x, sigA = E * TA.y, sigF = E * Fw;
    double2 nEA = {0.0, 0.0}, nRT = nEA, nRA = nEA, nRF = nEA;
    int nl = 0;
    if (rg.x < rg.y) {
      const double2* P = reinterpret_cast<const double2*>(t.poles + (int64_t)rg.x * 8);
      nEA = __ldg(P + 0); nRT = __ldg(P + 1); nRA = __ldg(P + 2); nRF = __ldg(P + 3);
      nl = __ldg(t.pole_l + rg.x);
    }
    for (int p = rg.x; p < rg.y; ++p) {
      const double2 EA = nEA, RT = nRT, RA = nRA, RF = nRF;
      const int l = nl;
      if (p + 1 < rg.y) {
        const double2* P = reinterpret_cast<const double2*>(t.poles + (int64_t)(p + 1) * 8);
        nEA = __ldg(P + 0); nRT = __ldg(P + 1); nRA = __ldg(P + 2); nRF = __ldg(P + 3);
        nl = __ldg(t.pole_l + p + 1);
      }
      const cplx Z = {(E - EA.x) * 0.5, (0.0 - EA.y) * 0.5};
      const cplx W = faddeeva_w(Z);
      const cplx fl = l == 0 ? f[0] : l == 1 ? f[1] : l == 2 ? f[2] : f[3];
      const cplx Wf = cmul(W, fl);
      sigT += RT.x * Wf.r - RT.y * Wf.i;
      sigA += RA.x * W.r - RA.y * W.i;
      sigF += RF.x * W.r - RF.y * W.i;
    }
    M0 += sigT * conc;
    M1 += sigA * conc;
    M2 += sigF * conc;
    M3 += (sigT - sigA) * conc;
  }
  if constexpr (false) {
    macro_out[0] = M0;
    macro_out[1] = M1;
    macro_out[2] = M2;
    macro_out[3] = M3;
  }
  double mx = -1.0;
  uint64_t v = 1;
  if (M0 > mx) { mx = M0; v = 1; }
  if (M1 > mx) { mx = M1; v = 2; }
  if (M2 > mx) { mx = M2; v = 3; }
  if (M3 > mx) { mx = M3; v = 4; }
  return v;
}

__device__ __forceinline__ uint64_t rs_new(const RSTables& t, uint64_t s, int64_t i) { return rs_lookup_one<false>(t, s, i, nullptr); }
#define K(NAME, TPB, MINB, FN)                                                                   \
  __global__ void __launch_bounds__(TPB, MINB) NAME(const __grid_constant__ RSTables t,          \
      uint64_t seed, int64_t first, int32_t n, uint64_t* ver) {                                  \
    const int32_t i = blockIdx.x * blockDim.x + threadIdx.x;                                     \
    if (i < n) ver[i] = FN(t, seed, first + i);                                                  \
  }
#define KO(NAME, TPB, MINB) K(NAME, TPB, MINB, rs_old_w)
#define KP(NAME, TPB, MINB) K(NAME, TPB, MINB, rs_polepf_w)
#define KN(NAME, TPB, MINB) K(NAME, TPB, MINB, rs_new)
__device__ __forceinline__ uint64_t rs_old2(const RSTables& t, uint64_t s, int64_t i, double*) { return 0; }

__device__ __forceinline__ uint64_t rs_old_w(const RSTables& t, uint64_t s, int64_t i) { return rs_old(t, s, i, nullptr); }
__device__ __forceinline__ uint64_t rs_polepf_w(const RSTables& t, uint64_t s, int64_t i) { return rs_polepf(t, s, i, nullptr); }
KO(o4, 128, 4) KO(o3, 128, 3) KO(o5, 128, 5) KO(o6, 64, 8)
KP(p4, 128, 4) KP(p3, 128, 3) KP(p5, 128, 5)
KN(n4, 128, 4) KN(n3, 128, 3) KN(n1, 128, 1)
typedef void (*KF)(RSTables, uint64_t, int64_t, int32_t, uint64_t*);
static KF kf[] = {o4, o3, o5, o6, p4, p3, p5, n4, n3, n1};
static int tpb[] = {128, 128, 128, 64, 128, 128, 128, 128, 128, 128};
extern "C" int rsx_count() { return (int)(sizeof(kf) / sizeof(kf[0])); }
extern "C" int rsx_regs(int v) { cudaFuncAttributes a; cudaFuncGetAttributes(&a, (const void*)kf[v]); return a.numRegs * 1000 + (int)a.localSizeBytes; }
extern "C" int rsx_run(int v, RSTables t, uint64_t seed, int64_t first, int32_t n, uint64_t* ver, void* stream) {
  kf[v]<<<(n + tpb[v] - 1) / tpb[v], tpb[v], 0, (cudaStream_t)stream>>>(t, seed, first, n, ver);
  return (int)cudaGetLastError();
}
