"""A/B timing of alternative libcaqr builds (development tool).

    python tools/ab_time.py LIB1.so LIB2.so ... [--m M --n N --reps R --rounds K]

Each library runs in its own subprocess (CAQR_LIB_PATH), rounds interleaved;
per call: A restored from a pristine copy and a 256 MiB L2 flush outside the
CUDA-event window (the bench.py protocol).  Prints the median ms per library.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import os, sys, json, torch
sys.path.insert(0, ROOT)
from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads
m, n, reps, dt = M, N, REPS, DT
dtype = torch.float32 if dt == "f32" else torch.float64
A0 = workloads.device_gaussian(m, n, seed=0, dtype=dtype, device="cuda").t()
A = caqr.colmajor_empty(m, n, dtype)
flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
ts = []
for r in range(reps + 3):
    A.copy_(A0); flush.fill_(r); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); R, ws = caqr.caqr_factor(A); e1.record(); torch.cuda.synchronize()
    if r >= 3: ts.append(e0.elapsed_time(e1))
ts.sort()
print(json.dumps({"median": ts[len(ts) // 2], "min": ts[0]}))
'''


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("libs", nargs="+")
    ap.add_argument("--m", type=int, default=1_000_000)
    ap.add_argument("--n", type=int, default=192)
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--reps", type=int, default=15)
    ap.add_argument("--rounds", type=int, default=3)
    a = ap.parse_args()
    code = (CHILD.replace("ROOT", repr(ROOT)).replace("M, N, REPS, DT", f"{a.m}, {a.n}, {a.reps}, {a.dtype!r}"))
    res = {l: [] for l in a.libs}
    for _ in range(a.rounds):
        for l in a.libs:
            env = dict(os.environ, CAQR_LIB_PATH=os.path.abspath(l))
            out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True)
            line = [x for x in out.stdout.splitlines() if x.startswith("{")]
            if not line:
                print(l, "FAILED", out.stderr[-800:])
                continue
            res[l].append(json.loads(line[-1])["median"])
    for l, v in res.items():
        v.sort()
        print(f"{os.path.basename(l):30s} {a.m}x{a.n} {a.dtype}: median {v[len(v) // 2] if v else float('nan'):.4f} ms  all {['%.4f' % x for x in v]}")


if __name__ == "__main__":
    main()
