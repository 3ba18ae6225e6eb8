"""Static SASS instruction mix of the kernels whose mangled name matches a substring.
  python scripts/sass_stats.py <substring> [<substring> ...]"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_ipps_doerfertphtdcg22_b200", "libomprt.so")
sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
for blk in sass.split("Function : ")[1:]:
    name = blk.split("\n", 1)[0]
    if not any(p in name for p in sys.argv[1:]):
        continue
    ins = re.findall(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]+)", blk)
    c = collections.Counter(i.split(".")[0] for i in ins)
    print(name[:70], len(ins), dict(c.most_common(12)))
