"""Algorithmic bytes per XSBench-shaped lookup over the full BASELINE configs[2] workload
(17M lookups, small problem), counted by the CPU oracle (oracle_xs_bytes: every table
element a lookup reads -- one 8 B energy per binary-search probe, num_nucs, and per
nuclide mats 4 B + concs 8 B + index 4 B + two 48 B gridpoints -- plus the 8 B
verification store).  Writes profiles/xs_algorithmic_bytes.json, which bench.py reads for
the roofline's per-unit figure.  Calls only oracle/ and gen/."""
import json
import os
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gen  # noqa: E402
import oracle  # noqa: E402


def main():
    t = gen.XSTables(**gen.XS_SMALL)
    n = 17_000_000
    parts = os.cpu_count() or 1
    res = [0] * parts

    def run(k):
        a, b = n * k // parts, n * (k + 1) // parts
        res[k] = oracle.xs_bytes(t, a, b - a, seed=gen.XS_LOOKUP_SEED)

    ths = [threading.Thread(target=run, args=(k,)) for k in range(parts)]
    for th in ths:
        th.start()
    for th in ths:
        th.join()
    out = {"workload": "XSBench small, 17M lookups, seed 1070", "lookups": n,
           "total_bytes": int(sum(res)), "bytes_per_lookup": sum(res) / n,
           "source": "scripts/xs_bytes_per_lookup.py (oracle_xs_bytes)"}
    path = os.path.join(ROOT, "profiles", "xs_algorithmic_bytes.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
