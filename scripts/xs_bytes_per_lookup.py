"""Algorithmic bytes per XSBench-shaped lookup over the full BASELINE configs[2] workload
(17M lookups, small problem), for the roofline's per-unit figure.  Writes
profiles/xs_algorithmic_bytes.json, which bench.py reads.

* "plain" (the tables as specified) -- counted by the CPU oracle (oracle_xs_bytes): one 8 B
  energy per binary-search probe, 4 B num_nucs, per nuclide 4 B mats + 8 B concs + 4 B
  index + two 48 B gridpoints, plus the 8 B verification store.
* "accel" (the B200 layouts of omprt_xs_build_accel) -- the same lookups with the binned
  search (8 B for the two adjacent bin entries + 8 B per probe of the bisection over the
  bin's bracket, counted exactly here with numpy over all lookups), a 2 B index entry and a
  96 B bracket record per nuclide; the per-nuclide and fixed terms are the oracle's.
"""
import json
import os
import sys
import threading

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gen  # noqa: E402
import oracle  # noqa: E402

N = 17_000_000
LOG2_BINS = 18


def plain_bytes(t):
    parts = os.cpu_count() or 1
    res = [0] * parts

    def run(k):
        a, b = N * k // parts, N * (k + 1) // parts
        res[k] = oracle.xs_bytes(t, a, b - a, seed=gen.XS_LOOKUP_SEED)

    ths = [threading.Thread(target=run, args=(k,)) for k in range(parts)]
    for th in ths:
        th.start()
    for th in ths:
        th.join()
    return int(sum(res))


def accel_bytes(t):
    st = gen.lcg_states(gen.XS_LOOKUP_SEED, 2 * N)
    E = st[0::2].astype(np.float64) * 2.0 ** -63
    roll = st[1::2].astype(np.float64) * 2.0 ** -63
    del st
    dist = gen.MAT_DIST
    running = []
    for i in range(12):  # summed in XSBench's order: dist[i] + dist[i-1] + ... + dist[1]
        r = 0.0
        for j in range(i, 0, -1):
            r += dist[j]
        running.append(r)
    mat = np.zeros(N, np.int64)
    done = np.zeros(N, bool)
    for i in range(12):
        hit = (~done) & (roll < running[i])
        mat[hit] = i
        done |= hit
    nn = t.num_nucs[mat].astype(np.int64)
    U = t.unionized
    H = 1 << LOG2_BINS
    edges = np.arange(H + 1, dtype=np.float64) / H
    R = np.clip(np.searchsorted(U, edges, side="right") - 1, 0, U.size - 2)
    b = np.minimum((E * H).astype(np.int64), H - 1)
    lo = R[b].astype(np.int64)
    hi = np.minimum(R[b + 1].astype(np.int64) + 1, U.size - 1)
    probes = np.zeros(N, np.int64)
    active = hi - lo > 1
    while active.any():
        mid = lo + (hi - lo) // 2
        go_hi = U[mid] > E
        hi = np.where(active & go_hi, mid, hi)
        lo = np.where(active & ~go_hi, mid, lo)
        probes += active
        active = hi - lo > 1
    per = 8 + 8 * probes + 4 + nn * (4 + 8 + 2 + 96) + 8
    return int(per.sum()), float(probes.mean())


def main():
    t = gen.XSTables(**gen.XS_SMALL)
    plain = plain_bytes(t)
    accel, mean_probes = accel_bytes(t)
    out = {"workload": "XSBench small, 17M lookups, seed 1070", "lookups": N,
           "total_bytes": plain, "bytes_per_lookup": plain / N,
           "accel": {"total_bytes": accel, "bytes_per_lookup": accel / N, "log2_bins": LOG2_BINS,
                     "mean_probes": mean_probes},
           "source": "scripts/xs_bytes_per_lookup.py (plain: oracle_xs_bytes; accel: numpy)"}
    with open(os.path.join(ROOT, "profiles", "xs_algorithmic_bytes.json"), "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
