// Exploration record (NOT part of libomprt.so; r2 x12-x14): the RSBench flattened body
// with each lock-step trip's poles shared out over the warp -- a warp scan numbers the
// trip's poles of all 32 lanes, the lanes evaluate them 32 at a time, and each lane sums
// its own window's contributions from a warp buffer in window order (bit-identical sums).
// Correct (1.3e-15 normwise against the unqueued kernel, same checksum over 10M lookups)
// but SLOWER: 94.3 ms vs 58.1 ms for the product's queued body at 10M lookups
// (profiles/rs_body_variants_r2.txt).  The owner search (5 dependent shared-memory
// loads before a pole record can be requested), the serial per-lane sums and the
// 37 KB of shared memory per team (66 B of spills at 128 registers) cost more than the
// ~1/3 of lanes the one-lane-per-window loop leaves idle.  It was compiled into the
// library (rs_body.cuh, instantiated by omprt_rs_qflat_rt<Tr, Macro, true> under the flag
// OMPRT_RS_WARP_POLES) when measured; kept here as written.
// ---- the flattened body with each trip's poles shared out over the warp (reading R-A9) ---
// In the lock-step loop a trip takes every live lane through one nuclide, and its pole loop
// runs as long as the longest window among the 32 lanes: with ~10 poles per window (9..14)
// and lanes idle once their own window is done, ncu counted 20.7 of 32 lanes active per
// instruction.  Here a trip only SETS UP each lane's nuclide (step(): window, sigT
// factors, pole range); the runtime's warp-collective hook then numbers the trip's poles
// of all lanes 0..C-1 (a warp scan of the window lengths) and the 32 lanes evaluate them
// k = lane, lane + 32, ... -- ceil(C / 32) iterations with all lanes busy instead of
// max(window) iterations with ~2/3 of them.  A pole's contributions (dT, dA, dF) go to a
// warp buffer in pole order and each lane adds its own window's, in window order, to its
// sigT..sigF: every contribution is computed by the same explicit operations on whatever
// lane, so each lookup's sums are bit-for-bit those of the one-lane-per-window loop.  Poles
// on the Abrarov branch are queued (as R-A8) with their owner lane, queue slots allocated
// in pole order (ballot), so a lookup's queued poles are drained in a fixed order too.
constexpr int kRSRound = 128;  // poles per round of the warp's contribution buffer
struct RSWarpPoleBuf {
  int32_t incl[32];        // inclusive end of lane l's poles in the trip's numbering
  int32_t base[32];        // pole k of lane l is pole base[l] + k of the table
  double E[32];            // lane l's lookup energy
  double conc[32];         // lane l's nuclide concentration (for its queued poles)
  double c[3][kRSRound];   // dT, dA, dF of the round's poles, by k - round base
  uint8_t queued[kRSRound];
  int32_t qcnt[32];        // lane l's poles waiting in the queue
};
struct RSOwnerQueue {
  double zr[kRSQueueCap], zi[kRSQueueCap], fr[kRSQueueCap], fi[kRSQueueCap], cc[kRSQueueCap];
  int32_t p[kRSQueueCap], owner[kRSQueueCap];
  int32_t count, pad;
};

template <bool kMacro, int kWarps>
struct RSWarpPolesLookup : RSFlatLookup<kMacro> {
  using Base = RSFlatLookup<kMacro>;
  bool pending = false;     // this trip set up a nuclide whose poles are not yet summed
  int32_t pstart = 0, pcount = 0;
  double sT = 0.0, sA = 0.0, sF = 0.0, pconc = 0.0;

  __device__ __forceinline__ RSWarpPolesLookup(const RSTables& tab, uint64_t seed,
                                               int64_t first_, uint64_t* verification,
                                               double* macro_)
      : Base(tab, seed, first_, verification, macro_) {}

  static __device__ __forceinline__ RSWarpPoleBuf& pbuf() {
    __shared__ RSWarpPoleBuf b[kWarps];
    return b[threadIdx.x >> 5];
  }
  static __device__ __forceinline__ RSOwnerQueue& queue() {
    __shared__ RSOwnerQueue q[kWarps];
    return q[threadIdx.x >> 5];
  }
  // before the loop, then a team barrier
  static __device__ __forceinline__ void init_queue() {
    if ((threadIdx.x & 31u) == 0) queue().count = 0;
    pbuf().qcnt[threadIdx.x & 31u] = 0;
  }

  __device__ __forceinline__ bool step() {
    const RSTables& t = this->t;
    if (this->j < this->nn) {
      const int nuc = __ldg(t.mats + this->mat * t.max_num_nucs + this->j);
      pconc = __ldg(t.concs + this->mat * t.max_num_nucs + this->j);
      const int2 rg = rs_nuclide_setup(t, this->E, this->sqrtE, nuc, sT, sA, sF);
      pstart = rg.x;
      pcount = rg.y - rg.x;
      pending = true;
    }
    return ++this->j < this->nn;
  }

  // one pole of the trip's numbering (owner lane o, table index p, buffer slot `slot`):
  // its contributions into the buffer, or into the queue on the Abrarov branch.  Called by
  // all 32 lanes together (`valid` false for the lanes past the round's end).
  __device__ __forceinline__ void eval(RSWarpPoleBuf& w, RSOwnerQueue& q, const RSPole& x,
                                       int p, int o, bool valid, int slot) {
    const unsigned lane = threadIdx.x & 31u;
    cplx Z = {dmul(dsub(w.E[o], x.ear), 0.5), dmul(dsub(0.0, x.eai), 0.5)};
    if (!valid) Z = {8.0, 8.0};  // a harmless point on the asymptotic branch
    const cplx fl = rs_fsh()[x.l & 3][(threadIdx.x & ~31u) + o];
    const bool abr = valid && rs_abrarov_branch(Z);
    const unsigned m = __ballot_sync(0xffffffffu, abr);
    bool queued = false;
    if (m) {  // warp-uniform: slots in pole order
      const int qb = *(volatile int32_t*)&q.count;
      const int qs = qb + __popc(m & ((1u << lane) - 1u));
      queued = abr && qs < kRSQueueCap;
      if (queued) {
        q.zr[qs] = Z.r;
        q.zi[qs] = Z.i;
        q.fr[qs] = fl.r;
        q.fi[qs] = fl.i;
        q.cc[qs] = w.conc[o];
        q.p[qs] = p;
        q.owner[qs] = o;
        atomicAdd(&w.qcnt[o], 1);
      }
      __syncwarp();
      if (lane == 0) q.count = min(kRSQueueCap, qb + __popc(m));
      __syncwarp();
    }
    if (valid) {
      double dT = 0.0, dA = 0.0, dF = 0.0;
      if (!queued) {
        const cplx W = abr ? faddeeva_abrarov(Z) : faddeeva_asym(Z);
        const cplx Wf = cmul(W, fl);
        dT = fma(x.rtr, Wf.r, -dmul(x.rti, Wf.i));
        dA = fma(x.rar, W.r, -dmul(x.rai, W.i));
        dF = fma(x.rfr, W.r, -dmul(x.rfi, W.i));
      }
      w.c[0][slot] = dT;
      w.c[1][slot] = dA;
      w.c[2][slot] = dF;
      w.queued[slot] = queued ? 1 : 0;
    }
  }

  // all 32 lanes, converged (omprt's lock-step hook), after every trip
  __device__ __forceinline__ void warp_collective(bool done) {
    const unsigned lane = threadIdx.x & 31u;
    RSWarpPoleBuf& w = pbuf();
    RSOwnerQueue& q = queue();
    const RSTables& t = this->t;
    const int cnt = pending ? pcount : 0;
    int incl = cnt;  // the trip's pole numbering: inclusive warp scan of the window lengths
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int v = __shfl_up_sync(0xffffffffu, incl, o);
      if ((int)lane >= o) incl += v;
    }
    const int C = __shfl_sync(0xffffffffu, incl, 31);
    const int excl = incl - cnt;
    if (C > 0) {
      w.incl[lane] = incl;
      w.base[lane] = pstart - excl;
      w.E[lane] = this->E;
      w.conc[lane] = pconc;
      __syncwarp();
      auto locate = [&](int k, int& o) {  // owner: the first lane whose range ends past k
        int lo = 0;
#pragma unroll
        for (int s2 = 16; s2 > 0; s2 >>= 1)
          if (w.incl[lo + s2 - 1] <= k) lo += s2;
        o = lo;
        return w.base[lo] + k;
      };
      for (int rb = 0; rb < C; rb += kRSRound) {
        const int re = min(C, rb + kRSRound);
        // k = rb + lane + 32 i; the next k's record is in flight while this one is evaluated
        RSPole A{}, B{};
        int oa = 0, ob = 0, pa = 0, pb = 0;
        bool va = rb + (int)lane < re, vb = false;
        if (va) {
          pa = locate(rb + (int)lane, oa);
          rs_load_pole(t, A, pa);
        }
        for (int kb = rb; kb < re; kb += 64) {
          vb = kb + 32 + (int)lane < re;
          if (vb) {
            pb = locate(kb + 32 + (int)lane, ob);
            rs_load_pole(t, B, pb);
          }
          eval(w, q, A, pa, oa, va, kb - rb + (int)lane);
          if (kb + 32 >= re) break;
          va = kb + 64 + (int)lane < re;
          if (va) {
            pa = locate(kb + 64 + (int)lane, oa);
            rs_load_pole(t, A, pa);
          }
          eval(w, q, B, pb, ob, vb, kb + 32 - rb + (int)lane);
        }
        __syncwarp();
        if (pending) {  // this lane's window, in window order
          const int k1 = min(incl, re);
          for (int k = max(excl, rb); k < k1; ++k) {
            if (w.queued[k - rb]) continue;
            sT = dadd(sT, w.c[0][k - rb]);
            sA = dadd(sA, w.c[1][k - rb]);
            sF = dadd(sF, w.c[2][k - rb]);
          }
        }
        __syncwarp();
      }
    }
    if (pending) {
      rs_accumulate(pconc, sT, sA, sF, this->M0, this->M1, this->M2, this->M3);
      pending = false;
    }
    // the Abrarov queue: drained by all lanes when full enough, or when a lane that
    // finished its lookup in this trip still has poles in it (its end() needs them)
    const int n = min(*(volatile int32_t*)&q.count, kRSQueueCap);
    const bool mine = w.qcnt[lane] > 0;
    if (!__any_sync(0xffffffffu, done && mine) && n < 32) return;
    for (int k = (int)lane; k < n; k += 32) {
      const cplx Z = {q.zr[k], q.zi[k]}, fl = {q.fr[k], q.fi[k]};
      const double conc = q.cc[k];
      RSPole x;
      rs_load_pole(t, x, q.p[k]);
      const cplx W = faddeeva_abrarov(Z);  // queued only when |Z| < 6
      const cplx Wf = cmul(W, fl);
      const double dT = fma(x.rtr, Wf.r, -dmul(x.rti, Wf.i));
      const double dA = fma(x.rar, W.r, -dmul(x.rai, W.i));
      const double dF = fma(x.rfr, W.r, -dmul(x.rfi, W.i));
      q.zr[k] = dmul(dT, conc);
      q.zi[k] = dmul(dA, conc);
      q.fr[k] = dmul(dF, conc);
      q.fi[k] = dmul(dsub(dT, dA), conc);
    }
    __syncwarp();
    if (mine) {  // this lane's entries, in queue (= pole) order
      for (int k = 0; k < n; ++k) {
        if (q.owner[k] != (int)lane) continue;
        this->M0 = dadd(this->M0, q.zr[k]);
        this->M1 = dadd(this->M1, q.zi[k]);
        this->M2 = dadd(this->M2, q.fr[k]);
        this->M3 = dadd(this->M3, q.fi[k]);
      }
      w.qcnt[lane] = 0;
    }
    __syncwarp();
    if (lane == 0) q.count = 0;
    __syncwarp();
  }
};

