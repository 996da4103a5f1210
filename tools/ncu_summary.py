"""Summarise an ncu report: key metrics + per-source-line stall/instruction shares."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30


def run(*a):
    return subprocess.run(["ncu", "-i", rep, *a], capture_output=True, text=True).stdout


det = list(csv.reader(io.StringIO(run("--page", "details", "--csv"))))
h = det[0]
want = ["Duration", "Elapsed Cycles", "SM Frequency", "DRAM Throughput", "Compute (SM) Throughput",
        "Executed Ipc Active", "Issued Instructions", "Achieved Occupancy", "Registers Per Thread",
        "L2 Hit Rate", "L1/TEX Hit Rate", "Memory Throughput", "Warp Cycles Per Issued Instruction",
        "Grid Size", "Dynamic Shared Memory Per Block"]
for row in det[1:]:
    d = dict(zip(h, row))
    if d.get("Metric Name") in want:
        print(f"{d['Metric Name']:40s} {d['Metric Value']:>16s} {d['Metric Unit']}")
raw = list(csv.reader(io.StringIO(run("--page", "raw", "--csv"))))
if len(raw) > 2:
    rh, units, vals = raw[0], raw[1], raw[2]
    for k in ["dram__bytes_read.sum", "dram__bytes_write.sum", "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
              "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
              "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
              "sm__inst_executed_pipe_uma.avg.pct_of_peak_sustained_active",
              "sm__warps_active.avg.pct_of_peak_sustained_active",
              "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
              "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
              "smsp__average_warp_latency_issue_stalled_barrier", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
              "lts__t_bytes.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]:
        if k in rh:
            i = rh.index(k)
            print(f"{k:60s} {vals[i]:>16s} {units[i]}")
src = list(csv.reader(io.StringIO(run("--page", "source", "--csv", "--print-source", "cuda,sass"))))
hdr = None
out = []
cur = None
for r in src:
    if len(r) >= 2 and r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if len(r) > 3 and r[0] == "Line No":
        hdr = r
        continue
    if hdr and len(r) == len(hdr) and r[0].isdigit() and r[2] == "-":
        d = dict(zip(hdr, r))
        out.append((int(r[4] or 0), int(d["Instructions Executed"] or 0), cur, int(r[0]), r[1][:80]))
ts = sum(o[0] for o in out) or 1
ti = sum(o[1] for o in out) or 1
print(f"--- top source lines by stall samples (total {ts} samples, {ti} warp-instr)")
for o in sorted(out, reverse=True)[:top]:
    print(f"{o[0]/ts*100:5.1f}% smp {o[1]/ti*100:5.1f}% ins  {o[2]}:{o[3]}  {o[4]}")

# region aggregation (function line ranges of tsqr_fused.cuh, optional argv[3] = "a-b:name,...")
if len(sys.argv) > 3:
    regions = []
    for spec in sys.argv[3].split(","):
        rng, name = spec.split(":")
        a, b = map(int, rng.split("-"))
        regions.append((a, b, name))
    agg = {}
    for smp, ins, f, ln, _ in out:
        name = "other"
        if f == "tsqr_fused.cuh":
            for a, b, nm in regions:
                if a <= ln <= b:
                    name = nm
        elif f and "kernels" in f:
            name = "tsqr_kernels.cuh"
        elif f:
            name = f
        d = agg.setdefault(name, [0, 0])
        d[0] += smp
        d[1] += ins
    print("--- regions")
    for k, (smp, ins) in sorted(agg.items(), key=lambda kv: -kv[1][0]):
        print(f"{k:25s} {smp/ts*100:5.1f}% samples {ins/ti*100:5.1f}% instr")
