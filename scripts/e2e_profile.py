"""Run the end-to-end XS steps once per host-table mode (for an ncu launch list).
  python scripts/e2e_profile.py [steps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_ipps_doerfertphtdcg22_b200 import omprt  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 2
torch.cuda.set_device(0)
omprt.omprt_init(0)
t = gen.XSTables(**gen.XS_SMALL)
raw = {k: torch.from_numpy(getattr(t, k)).pin_memory()
       for k in ("nuclide_grid", "num_nucs", "mats", "concs")}
hs = omprt.xs_host_struct(t, raw, derive=True)
print(omprt.omprt_xs_run_host_steps(hs, gen.XS_LOOKUP_SEED, 0, 17_000_000, steps,
                                    flags=omprt.OMPRT_XS_FLAT))
