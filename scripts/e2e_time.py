"""Host-clock time per step of the end-to-end XS offload (omprt_xs_run_host_steps, derived
tables, flattened lookups), with and without the L2 set-aside.
  python scripts/e2e_time.py [steps] [lib.so]   (A/B: one process per library build)"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_ipps_doerfertphtdcg22_b200 import omprt  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
if len(sys.argv) > 2:
    omprt.load(sys.argv[2])
torch.cuda.set_device(0)
omprt.omprt_init(0)
t = gen.XSTables(**gen.XS_SMALL)
raw = {k: torch.from_numpy(getattr(t, k)).pin_memory()
       for k in ("nuclide_grid", "num_nucs", "mats", "concs")}
hs = omprt.xs_host_struct(t, raw, derive=True)
res = {}
for aside in (1 << 40, 0):
    got = omprt.omprt_l2_set_aside(aside)
    omprt.omprt_xs_run_host_steps(hs, gen.XS_LOOKUP_SEED, 0, 17_000_000, 3,
                                  flags=omprt.OMPRT_XS_FLAT)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    cks, h2d, d2h = omprt.omprt_xs_run_host_steps(hs, gen.XS_LOOKUP_SEED, 0, 17_000_000, steps,
                                                  flags=omprt.OMPRT_XS_FLAT)
    ms = 1000 * (time.perf_counter() - t0) / steps
    res[f"aside_{got >> 20}MB"] = {"ms_per_step": ms, "lookups_per_s": 17e6 / ms * 1e3,
                                   "checksums_equal": len(set(cks)) == 1, "h2d": h2d}
print(json.dumps(res))
