"""Algorithmic fp64 operations per RSBench-shaped lookup (BASELINE configs[3], the default
"large" shape, seed 1070), for the C4 roofline's per-unit figure: the CPU
oracle's instrumented pass (oracle_rs_count: every add/sub, mul, div, sqrt and
transcendental call of App. A.2's cross-section computation, counted where the oracle writes
it) over a contiguous sample of lookups spread over the 10M.  Writes
profiles/rs_algorithmic_flops.json, which bench.py reads.

flops = add + mul + div + sqrt (+ 2 fma; the definition has none); transcendental calls
(sin, cos, atan) are reported beside them, not as flops.
  python scripts/rs_flops_per_lookup.py [samples_per_block]"""
import json
import os
import sys
import threading

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import gen  # noqa: E402
import oracle  # noqa: E402

N = 10_000_000


def main():
    per_block = int(sys.argv[1]) if len(sys.argv) > 1 else 2000
    t = gen.RSTables()
    blocks = 50  # 50 contiguous blocks at evenly spaced starts over the 10M lookups
    starts = [b * (N // blocks) for b in range(blocks)]
    res = [None] * blocks

    def run(k):
        res[k] = oracle.rs_count(t, starts[k], per_block)

    th = [threading.Thread(target=run, args=(k,)) for k in range(blocks)]
    for x in th:
        x.start()
    for x in th:
        x.join()
    ops = np.sum(res, axis=0)
    n = blocks * per_block
    names = ["add", "mul", "div", "sqrt", "trans", "faddeeva", "abrarov", "poles", "pairs", "fma"]
    per = {k: float(v) / n for k, v in zip(names, ops)}
    flops = per["add"] + per["mul"] + per["div"] + per["sqrt"] + 2 * per["fma"]
    out = {"workload": "RSBench large (355 nuclides, ~1000 poles / 100 windows each), seed 1070",
           "sample": f"{blocks} blocks of {per_block} contiguous lookups, evenly spaced over {N}",
           "lookups_counted": n, "per_lookup": per, "flops_per_lookup": flops,
           "source": "scripts/rs_flops_per_lookup.py (oracle_rs_count)"}
    path = os.path.join(ROOT, "profiles", "rs_algorithmic_flops.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
