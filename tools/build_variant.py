"""Build the current csrc/ tree into tools/_libs/<name>.so (for tools/ab_time.py).

    python tools/build_variant.py NAME [-DMACRO ...]
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_andersonbdk11_b200 import build  # noqa: E402

name, defs = sys.argv[1], sys.argv[2:]
os.makedirs(os.path.join(ROOT, "tools", "_libs"), exist_ok=True)
out = os.path.join(ROOT, "tools", "_libs", name + ".so")
cmd = build.nvcc_cmd(out)
cmd[1:1] = defs
r = subprocess.run(cmd, capture_output=True, text=True)
print(out if r.returncode == 0 else r.stdout + r.stderr)
sys.exit(r.returncode)
