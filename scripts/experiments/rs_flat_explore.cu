// Exploration harness (NOT part of libomprt.so): the flattened, lock-step, dynamic-schedule
// RSBench kernel with Faddeeva evaluation variants x launch bounds.
//   V0  the library body (rs_body.cuh faddeeva_w: 2 complex divisions / 4 fp64 divides)
//   V1  asymptotic branch as one complex quotient: i Z (a (Z^2-d) + c (Z^2-b)) /
//       ((Z^2-b)(Z^2-d)), one real reciprocal of |den|^2
//   V2  V1 + the Abrarov terms through one real reciprocal each
#include <cuda_runtime.h>
#include <cstdint>
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/omprt/device/omprt.cuh"
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/rs_body.cuh"
#include "../../paper_conf_ipps_doerfertphtdcg22_b200/csrc/kernels/vec.cuh"
using namespace omprt_kernels;
using namespace omprt;

__device__ __forceinline__ cplx cdiv_rcp(cplx a, cplx b) {
  const double r = 1.0 / (b.r * b.r + b.i * b.i);
  return {(a.r * b.r + a.i * b.i) * r, (a.i * b.r - a.r * b.i) * r};
}

template <int V>
__device__ __forceinline__ cplx faddeeva_v(cplx Z) {
  if constexpr (V == 0) return faddeeva_w(Z);
  const double absz = sqrt(__dadd_rn(__dmul_rn(Z.r, Z.r), __dmul_rn(Z.i, Z.i)));
  if (absz < 6.0) {
    if constexpr (V == 1) return faddeeva_w(Z);
    constexpr double tau = 12.0;
    constexpr double an[10] = {0.27584023329217705,   0.22457395522461585,
                               0.1594149382739117,    0.0986657664154542,
                               0.053244140787639394,  0.02505215000539365,
                               0.01027746567053954,   0.0036761643328448498,
                               0.001146493641242233,  0.0003117570150461973};
    constexpr double npi2[10] = {9.869604401089358,  39.47841760435743,  88.82643960980423,
                                 157.91367041742973, 246.74011002723395, 355.3057584392169,
                                 483.61061565337855, 631.6546816697189,  799.437956488238,
                                 986.9604401089358};
    constexpr double prefactor = 81.24330003087691;
    const cplx tZ = {tau * Z.r, tau * Z.i};
    const double ex = rs_fast_exp(-tau * Z.i);
    double sn, cs;
    sincos(tau * Z.r, &sn, &cs);
    const cplx e = {ex * cs, ex * sn};
    cplx W = cdiv_rcp({e.i, 1.0 - e.r}, tZ);
    const cplx Z2 = cmul(Z, Z);
    cplx sum = {0.0, 0.0};
#pragma unroll
    for (int n = 0; n < 10; ++n) {
      const double sgn = (n & 1) ? 1.0 : -1.0;
      const cplx top = {sgn * e.r - 1.0, sgn * e.i};
      const cplx bot = {npi2[n] - tau * tau * Z2.r, -tau * tau * Z2.i};
      const cplx q = cdiv_rcp(top, bot);
      sum.r += an[n] * q.r;
      sum.i += an[n] * q.i;
    }
    const cplx zs = cmul(Z, sum);
    W.r += -prefactor * zs.i;
    W.i += prefactor * zs.r;
    return W;
  }
  constexpr double a = 0.512424224754768462984202823134979415014943561548661637413182;
  constexpr double b = 0.275255128608410950901357962647054304017026259671664935783653;
  constexpr double c = 0.051765358792987823963876628425793170829107067780337219430904;
  constexpr double d = 2.724744871391589049098642037352945695982973740328335064216346;
  const cplx Z2 = cmul(Z, Z);
  const cplx u = {Z2.r - b, Z2.i}, v = {Z2.r - d, Z2.i};
  const cplx num = {a * v.r + c * u.r, a * v.i + c * u.i};
  const cplx q = cdiv_rcp(num, cmul(u, v));
  return cmul({-Z.i, Z.r}, q);
}

// V >= 3: 256-bit pole loads (2 x LDG.256 per 64 B pole); V >= 4: the Abrarov branch
// deferred to the end of the window (one pending pole per lane; its contribution is added
// last -- a different summation order, within the tolerance contract)
template <int V>
__device__ __forceinline__ void nuclide_v(const RSTables& t, double E, double sqrtE, int nuc,
                                          double& sigT, double& sigA, double& sigF) {
  const int nw = __ldg(t.n_windows + nuc);
  const double spacing = 1.0 / nw;
  int w = (int)(E / spacing);
  if (w >= nw) w = nw - 1;
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
  sigT = E * TA.x;
  sigA = E * TA.y;
  sigF = E * Fw;
  int pend = -1;
  cplx Zp = {0.0, 0.0};
  auto add = [&](int p, double rtr, double rti, double rar, double rai, double rfr, double rfi,
                 cplx W) {
    const int l = __ldg(t.pole_l + p);
    const cplx fl = l == 0 ? f[0] : l == 1 ? f[1] : l == 2 ? f[2] : f[3];
    const cplx Wf = cmul(W, fl);
    sigT += rtr * Wf.r - rti * Wf.i;
    sigA += rar * W.r - rai * W.i;
    sigF += rfr * W.r - rfi * W.i;
  };
  for (int p = rg.x; p < rg.y; ++p) {
    const double* P = t.poles + (int64_t)p * 8;
    double ear, eai, rtr, rti, rar, rai, rfr, rfi;
    if constexpr (V >= 3) {
      ld_nc_v4f64(P, ear, eai, rtr, rti);
      ld_nc_v4f64(P + 4, rar, rai, rfr, rfi);
    } else {
      const double2* Q = reinterpret_cast<const double2*>(P);
      const double2 EA = __ldg(Q + 0), RT = __ldg(Q + 1), RA = __ldg(Q + 2), RF = __ldg(Q + 3);
      ear = EA.x; eai = EA.y; rtr = RT.x; rti = RT.y; rar = RA.x; rai = RA.y; rfr = RF.x; rfi = RF.y;
    }
    const cplx Z = {(E - ear) * 0.5, (0.0 - eai) * 0.5};
    if constexpr (V >= 4) {
      const double absz = sqrt(__dadd_rn(__dmul_rn(Z.r, Z.r), __dmul_rn(Z.i, Z.i)));
      if (absz < 6.0 && pend < 0) {  // defer (one per lane)
        pend = p;
        Zp = Z;
        continue;
      }
    }
    add(p, rtr, rti, rar, rai, rfr, rfi, faddeeva_v<(V >= 2 ? 2 : V)>(Z));
  }
  if constexpr (V >= 4) {
    if (pend >= 0) {
      const double* P = t.poles + (int64_t)pend * 8;
      double ear, eai, rtr, rti, rar, rai, rfr, rfi;
      ld_nc_v4f64(P, ear, eai, rtr, rti);
      ld_nc_v4f64(P + 4, rar, rai, rfr, rfi);
      add(pend, rtr, rti, rar, rai, rfr, rfi, faddeeva_v<2>(Zp));
    }
  }
}

template <int V>
struct Body {
  const RSTables& t;
  uint64_t seed0;
  int64_t first;
  uint64_t* ver;
  double* macro;
  LcgMap J;
  uint64_t s;
  double E, sqrtE;
  int32_t mat, nn, j;
  double M0, M1, M2, M3;
  __device__ Body(const RSTables& tt, uint64_t sd, int64_t f, uint64_t* v, double* m)
      : t(tt), seed0(sd), first(f), ver(v), macro(m) {}
  __device__ __forceinline__ void start() {
    uint64_t seed = s;
    E = lcg_double(seed);
    mat = pick_mat(seed);
    sqrtE = sqrt(E);
    nn = __ldg(t.num_nucs + mat);
    j = 0;
    M0 = M1 = M2 = M3 = 0.0;
  }
  template <class Idx> __device__ __forceinline__ void begin(Idx iv, Idx stride) {
    J = lcg_jump(2ull * (uint64_t)stride);
    s = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv));
    start();
  }
  template <class Idx> __device__ __forceinline__ void next(Idx) {
    s = lcg_apply(J, s);
    start();
  }
  __device__ __forceinline__ bool step() {
    if (j < nn) {
      const int nuc = __ldg(t.mats + mat * t.max_num_nucs + j);
      const double conc = __ldg(t.concs + mat * t.max_num_nucs + j);
      double sigT, sigA, sigF;
      nuclide_v<V>(t, E, sqrtE, nuc, sigT, sigA, sigF);
      rs_accumulate(conc, sigT, sigA, sigF, M0, M1, M2, M3);
    }
    return ++j < nn;
  }
  template <class Idx> __device__ __forceinline__ void end(Idx iv) {
    double* m = macro + (int64_t)iv * 4;
    m[0] = M0; m[1] = M1; m[2] = M2; m[3] = M3;
    ver[iv] = rs_argmax4(M0, M1, M2, M3);
  }
};

struct Tr : DefaultTraits {};

template <int V, int TPB, int MINB, bool DYN>
__global__ void __launch_bounds__(TPB, MINB)
    kern(const __grid_constant__ RSTables t, uint64_t seed, int64_t first, int32_t n,
         uint64_t* ver, double* macro) {
  Team<Tr> team = init<Tr>();
  Body<V> b(t, seed, first, ver, macro);
  if constexpr (DYN) distribute_parallel_for_dynamic_flat<Tr, FlatSync::Lockstep>(team, n, 1, b);
  else distribute_parallel_for_flat<Tr, FlatSync::Lockstep>(team, n, b);
}


// ---- V5: the Abrarov branch through a per-warp shared-memory QUEUE -----------------------
// A lane whose pole has |Z| < 6 appends (Z, f_l, conc, pole, link) to its warp's queue and
// moves on; the asymptotic poles never wait for it.  After every lock-step trip the whole
// warp (all 32 lanes, converged) flushes the queue when it holds >= 32 entries or when a
// lane that is about to finish its lookup has entries pending: every lane evaluates one
// queued Abrarov pole, writes conc * (dT, dA, dF, dT - dA) into the slot, and each owner
// adds its own entries in push order (a linked list per lane: deterministic).  The
// contributions reach M0..M3 per pole instead of through sigT..sigF of their nuclide: a
// different summation order, within the tolerance contract.
constexpr int kQCap = 64;
struct WarpQ {
  double zr[kQCap], zi[kQCap], fr[kQCap], fi[kQCap], cc[kQCap];
  int p[kQCap], nxt[kQCap];
  int count;
};

struct QBody {
  const RSTables& t;
  uint64_t seed0;
  int64_t first;
  uint64_t* ver;
  double* macro;
  WarpQ& q;
  LcgMap J;
  uint64_t s;
  double E, sqrtE;
  int32_t mat, nn, j;
  int32_t qhead, qtail;
  double M0, M1, M2, M3;
  __device__ QBody(const RSTables& tt, uint64_t sd, int64_t f, uint64_t* v, double* m, WarpQ& qq)
      : t(tt), seed0(sd), first(f), ver(v), macro(m), q(qq), qhead(-1), qtail(-1) {}
  __device__ __forceinline__ void start() {
    uint64_t seed = s;
    E = lcg_double(seed);
    mat = pick_mat(seed);
    sqrtE = sqrt(E);
    nn = __ldg(t.num_nucs + mat);
    j = 0;
    M0 = M1 = M2 = M3 = 0.0;
  }
  template <class Idx> __device__ __forceinline__ void begin(Idx iv, Idx stride) {
    J = lcg_jump(2ull * (uint64_t)stride);
    s = lcg_fast_forward(seed0, 2ull * (uint64_t)(first + iv));
    start();
  }
  template <class Idx> __device__ __forceinline__ void next(Idx) {
    s = lcg_apply(J, s);
    start();
  }
  __device__ __forceinline__ void nuclide(int nuc, double conc, double& sigT, double& sigA,
                                          double& sigF) {
    const int nw = __ldg(t.n_windows + nuc);
    const double spacing = 1.0 / nw;
    int w = (int)(E / spacing);
    if (w >= nw) w = nw - 1;
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
    sigT = E * TA.x;
    sigA = E * TA.y;
    sigF = E * Fw;
    for (int p = rg.x; p < rg.y; ++p) {
      const double* P = t.poles + (int64_t)p * 8;
      double ear, eai, rtr, rti, rar, rai, rfr, rfi;
      ld_nc_v4f64(P, ear, eai, rtr, rti);
      ld_nc_v4f64(P + 4, rar, rai, rfr, rfi);
      const int l = __ldg(t.pole_l + p);
      const cplx fl = l == 0 ? f[0] : l == 1 ? f[1] : l == 2 ? f[2] : f[3];
      const cplx Z = {(E - ear) * 0.5, (0.0 - eai) * 0.5};
      const double absz = sqrt(__dadd_rn(__dmul_rn(Z.r, Z.r), __dmul_rn(Z.i, Z.i)));
      if (absz < 6.0) {
        const int slot = atomicAdd(&q.count, 1);
        if (slot < kQCap) {
          q.zr[slot] = Z.r; q.zi[slot] = Z.i; q.fr[slot] = fl.r; q.fi[slot] = fl.i;
          q.cc[slot] = conc; q.p[slot] = p; q.nxt[slot] = -1;
          if (qtail >= 0) q.nxt[qtail] = slot;
          else qhead = slot;
          qtail = slot;
          continue;
        }
      }
      const cplx W = faddeeva_v<2>(Z);
      const cplx Wf = cmul(W, fl);
      sigT += rtr * Wf.r - rti * Wf.i;
      sigA += rar * W.r - rai * W.i;
      sigF += rfr * W.r - rfi * W.i;
    }
  }
  __device__ __forceinline__ bool step() {
    if (j < nn) {
      const int nuc = __ldg(t.mats + mat * t.max_num_nucs + j);
      const double conc = __ldg(t.concs + mat * t.max_num_nucs + j);
      double sigT, sigA, sigF;
      nuclide(nuc, conc, sigT, sigA, sigF);
      rs_accumulate(conc, sigT, sigA, sigF, M0, M1, M2, M3);
    }
    return ++j < nn;
  }
  // all 32 lanes, converged, after every lock-step trip
  __device__ __forceinline__ void collective(bool done) {
    __syncwarp();
    const int n = min(*(volatile int*)&q.count, kQCap);
    if (!__any_sync(0xffffffffu, done && qhead >= 0) && n < 32) return;
    const int lane = threadIdx.x & 31;
    for (int k = lane; k < n; k += 32) {
      const cplx Z = {q.zr[k], q.zi[k]}, fl = {q.fr[k], q.fi[k]};
      const double conc = q.cc[k];
      const double* P = t.poles + (int64_t)q.p[k] * 8;
      double ear, eai, rtr, rti, rar, rai, rfr, rfi;
      ld_nc_v4f64(P, ear, eai, rtr, rti);
      ld_nc_v4f64(P + 4, rar, rai, rfr, rfi);
      const cplx W = faddeeva_v<2>(Z);
      const cplx Wf = cmul(W, fl);
      const double dT = rtr * Wf.r - rti * Wf.i;
      const double dA = rar * W.r - rai * W.i;
      const double dF = rfr * W.r - rfi * W.i;
      q.zr[k] = dT * conc;
      q.zi[k] = dA * conc;
      q.fr[k] = dF * conc;
      q.fi[k] = (dT - dA) * conc;
    }
    __syncwarp();
    for (int k = qhead; k >= 0; k = q.nxt[k]) {
      M0 += q.zr[k];
      M1 += q.zi[k];
      M2 += q.fr[k];
      M3 += q.fi[k];
    }
    qhead = qtail = -1;
    __syncwarp();
    if (lane == 0) q.count = 0;
    __syncwarp();
  }
  template <class Idx> __device__ __forceinline__ void end(Idx iv) {
    double* m = macro + (int64_t)iv * 4;
    m[0] = M0; m[1] = M1; m[2] = M2; m[3] = M3;
    ver[iv] = rs_argmax4(M0, M1, M2, M3);
  }
};

// the lock-step dynamic loop (cuda_rs_dflat_twin) with the warp-collective hook per trip
template <int TPB, int MINB>
__global__ void __launch_bounds__(TPB, MINB)
    kernq(const __grid_constant__ RSTables t, uint64_t seed, int64_t first, int32_t count,
          uint64_t* ver, double* macro) {
  __shared__ unsigned next;
  __shared__ WarpQ qs[TPB / 32];
  const int32_t per = (count + (int32_t)gridDim.x - 1) / (int32_t)gridDim.x;
  const int32_t lo = min((int32_t)blockIdx.x * per, count);
  const int32_t hi = min(lo + per, count);
  if (threadIdx.x == 0) next = blockDim.x;
  if ((threadIdx.x & 31) == 0) qs[threadIdx.x >> 5].count = 0;
  __syncthreads();
  QBody b(t, seed, first, ver, macro, qs[threadIdx.x >> 5]);
  int32_t i = lo + (int32_t)threadIdx.x;
  bool live = i < hi;
  if (live) b.begin(i, 1);
  while (__any_sync(0xffffffffu, live)) {
    const bool done = live && !b.step();
    b.collective(done);
    if (done) {
      b.end(i);
      i = lo + (int32_t)atomicAdd(&next, 1u);
      live = i < hi;
      if (live) b.begin(i, 1);
    }
  }
}

typedef void (*KF)(RSTables, uint64_t, int64_t, int32_t, uint64_t*, double*);
struct Var { KF f; int tpb; const char* name; };
static Var vars[] = {
  {kernq<128, 5>, 128, "V5_queue_128x5_dyn"},
  {kernq<128, 4>, 128, "V5_queue_128x4_dyn"},
  {kern<3, 128, 5, true>, 128, "V3_128x5_dyn"},

};
extern "C" int rsf_count() { return (int)(sizeof(vars) / sizeof(vars[0])); }
extern "C" const char* rsf_name(int v) { return vars[v].name; }
extern "C" int rsf_regs(int v) {
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, (const void*)vars[v].f);
  return a.numRegs * 1000 + (int)a.localSizeBytes;
}
extern "C" int rsf_run(int v, RSTables t, uint64_t seed, int64_t first, int32_t n, uint64_t* ver,
                       double* macro, void* stream) {
  int dev = 0, sms = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, vars[v].f, vars[v].tpb, 0);
  vars[v].f<<<sms * per, vars[v].tpb, 0, (cudaStream_t)stream>>>(t, seed, first, n, ver, macro);
  return (int)cudaGetLastError();
}
