#!/usr/bin/env python
"""Benchmark: QR GFLOP/s (LAPACK count 2mn^2 - 2n^3/3) of the B200 TSQR/CAQR
path on BASELINE.json's headline workload, 1,000,000 x 192 fp32 (config C4).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config NAME] [--impl caqr|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...      (row-sharded, weak scaling)
    python bench.py --gpus N ...   (N > 1 without torchrun: re-launches itself
                                    under torch.distributed.run; exits 1 if fewer
                                    than N GPUs are visible)

One step = one caqr_factor (TSQR leaves + tree + R extraction) of a fresh copy
of the synthetic input that is already resident in HBM.  A is restored from a
pristine copy and a 256 MiB buffer is written (L2 flush) before every step,
outside the CUDA events that time the step; inputs (768 MB) exceed L2 anyway.
Rank 0 prints ONE JSON line.  Beside the headline (weak scaling: 1M rows per
GPU) it carries "strong_scaling" (config C4' 8,000,000 x 192 split over the N
ranks; at N = 1 the whole 6.1 GB matrix on one GPU) and, at N = 1, "configs":
the other BASELINE configs (C1, C2, C3, C4 fp64, C5) timed with the same
protocol.  `--impl reference` times the CPU oracle (the reference arm of this
tier: the paper ships no code) on a bounded row sample -- the same sample the
cpu_baseline leg uses.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "QR GFLOP/s (2mn^2-2n^3/3) on 1M x 192 fp32 and % of HBM/FP32 roofline, 1-8 GPUs"
UNIT = "GFLOP/s"
FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback ("of fallback")
SMS, FP32_LANES, FP64_LANES = 148, 128, 64  # per-SM FMA lanes (B200)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="caqr", choices=["caqr", "reference"])
    ap.add_argument("--config", default="c4_1Mx192_f32")
    ap.add_argument("--leaf-rows", type=int, default=0)
    ap.add_argument("--panel-cols", type=int, default=0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-chunks", type=int, default=16, help="row chunks of caqr_factor_host in the e2e leg")
    ap.add_argument("--cpu-sample-rows", type=int, default=0)
    ap.add_argument("--no-extra", action="store_true", help="skip the strong-scaling and extra-config legs")
    return ap.parse_args()


def cpu_info():
    """`lscpu` model name and the host's core count (nproc)."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"model": model, "nproc": os.cpu_count()}


def sample_rows(cfg, override=0):
    """Rows of the CPU oracle's bounded sample of a workload (both the
    reference arm and the cpu_baseline leg): ~8 GFLOP per step, i.e. ~4 s of
    single-thread oracle at its ~2 GFLOP/s."""
    m, n = cfg["m"], cfg["n"]
    return int(override or min(m, max(n, 8e9 / (2.0 * n * n))))


def relaunch_distributed(args):
    """--gpus N > 1 without a torch.distributed environment: re-run this script
    under torch.distributed.run with N ranks on this node (never a silent
    one-GPU measurement); exit 1 if fewer than N GPUs are visible."""
    import subprocess

    import torch

    have = torch.cuda.device_count()
    if have < args.gpus:
        sys.stderr.write(f"bench.py: --gpus {args.gpus} requested but only {have} GPU(s) visible\n")
        raise SystemExit(1)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(29500 + os.getpid() % 1000), __file__] + sys.argv[1:]
    raise SystemExit(subprocess.call(cmd))


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return dict(hbm_gbs=float(d["hbm_gbs"]), sm_max_mhz=float(d.get("sm_max_mhz", 1965.0)),
                    source="measured (MEASURED_PEAKS.json)")
    except Exception:
        return dict(hbm_gbs=FALLBACK_HBM_GBS, sm_max_mhz=1965.0, source="fallback (B200_PROFILING.md)")


def alu_peak_tflops(dtype: str, sm_max_mhz: float) -> float:
    """FP32/FP64 FMA peak from unit counts and the max SM clock:
    148 SMs x {128 fp32 | 64 fp64} FMA lanes x 2 flop x clock."""
    lanes = FP32_LANES if dtype == "f32" else FP64_LANES
    return SMS * lanes * 2 * sm_max_mhz * 1e6 / 1e12


def workload(name):
    from paper_conf_ipps_andersonbdk11_b200 import workloads

    if name not in workloads.CONFIGS:
        raise SystemExit(f"unknown config {name}; one of {sorted(workloads.CONFIGS)}")
    return dict(workloads.CONFIGS[name])


# ---- clocks during the timed region (NVML, same source as nvidia-smi) --------
class ClockSampler:
    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
        0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
        0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, index: int, period_s: float = 0.002):
        self.samples, self.reasons, self.max_mhz = [], 0, None
        self.period = period_s
        self._stop = threading.Event()
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover
            self.nv = None
            self.err = str(e)

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                self.reasons |= nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.nv:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        reasons = [v for k, v in self.REASONS.items() if self.reasons & k and v != "gpu_idle"]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": reasons, "samples": len(self.samples)}


# ---- reference arm: the CPU oracle -------------------------------------------
def run_reference(args, rank):
    if rank != 0:
        return
    import numpy as np

    import oracle
    from paper_conf_ipps_andersonbdk11_b200 import workloads

    cfg = workload(args.config)
    m, n, dt = cfg["m"], cfg["n"], cfg["dtype"]
    rows = sample_rows(cfg, args.cpu_sample_rows)
    acc = "d" if dt == "f32" else "ld"
    npdt = np.float32 if dt == "f32" else np.float64
    A = workloads.gaussian(rows, n, seed=0, dtype=npdt).astype(np.float64)
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.qr(A, want_q=False, acc=acc)
        dt_s = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt_s)
    flops = 2.0 * rows * n * n - 2.0 * n ** 3 / 3.0
    t = sum(times) / len(times)
    val = flops / t / 1e9
    sample = f"oracle_qr_{acc} (xGEQR2, 1 thread) on the first {rows} rows of the {m}x{n} {dt} input, per step"
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": dt, "data": "synthetic",
        "config": {"workload": args.config, "m": m, "n": n, "sample_rows": rows},
        "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                         "cpu": cpu_info()},
        "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(cfg, rows_override=0):
    """The oracle as it stands, 1 thread, on a bounded row sample (~10-30 s)."""
    import numpy as np

    import oracle
    from paper_conf_ipps_andersonbdk11_b200 import workloads

    m, n, dt = cfg["m"], cfg["n"], cfg["dtype"]
    rows = sample_rows(cfg, rows_override)  # the reference arm's sample
    acc = "d" if dt == "f32" else "ld"
    A = workloads.gaussian(rows, n, seed=0, dtype=np.float32 if dt == "f32" else np.float64)
    A = A.astype(np.float64)
    t0 = time.perf_counter()
    oracle.qr(A, want_q=False, acc=acc)
    t = time.perf_counter() - t0
    flops = 2.0 * rows * n * n - 2.0 * n ** 3 / 3.0
    return {"value": flops / t / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"oracle_qr_{acc} (single-thread Householder, C) on rows [0,{rows}) x {n} of a "
                      f"{dt} Gaussian, {t:.1f} s (same sample as one --impl reference step)",
            "cpu": cpu_info()}


# ---- extra legs: strong scaling (C4') and the other BASELINE configs ----------
def make_input(cfg, seed, dev, rows=None):
    """Synthetic input of a config as a column-major device tensor: Gaussian
    drawn on the device; the s-step Krylov basis and the video matrix built on
    the host (workloads.py recipes) and uploaded."""
    import numpy as np
    import torch

    from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

    m, n = rows or cfg["m"], cfg["n"]
    tdt = torch.float32 if cfg["dtype"] == "f32" else torch.float64
    if cfg["kind"] == "gaussian":
        return workloads.device_gaussian(m, n, seed=seed, dtype=tdt, device=dev).t()
    host = (workloads.krylov_basis(grid=2000, s=n, seed=seed, shifted=True) if cfg["kind"] == "krylov"
            else workloads.video(seed=seed)).astype(np.float32 if cfg["dtype"] == "f32" else np.float64)
    A0 = caqr.colmajor_empty(host.shape[0], host.shape[1], tdt, dev)
    A0.copy_(torch.from_numpy(np.ascontiguousarray(host)))
    return A0


def timed_steps(step, prep, warmup, steps, stream):
    """Same protocol as the headline: >= 3 warm-ups, prep (A restore + L2
    flush) outside the CUDA events, events on the launching stream."""
    import torch

    for _ in range(max(warmup, 3)):
        prep()
        step()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    for a, b in evs:
        prep()
        a.record(stream)
        step()
        b.record(stream)
    torch.cuda.synchronize()
    return sum(a.elapsed_time(b) for a, b in evs) / steps


def extra_configs_leg(args, dev, flush, peaks):
    """N = 1: the other BASELINE configs with the headline's protocol."""
    import torch

    from paper_conf_ipps_andersonbdk11_b200 import caqr

    out = {}
    stream = torch.cuda.current_stream()
    for name in ("c1_4096x16_f32", "c2_krylov_4Mx8_f32", "c3_video_110592x100_f32", "c4_1Mx192_f64",
                 "c5_8192x8192_f32"):
        cfg = workload(name)
        m, n, dt = cfg["m"], cfg["n"], cfg["dtype"]
        esz = 4 if dt == "f32" else 8
        opts = caqr.make_opts(0, cfg.get("nb", 0))
        A0 = make_input(cfg, 0, dev)
        A = caqr.colmajor_empty(m, n, A0.dtype, dev)
        code = caqr.CAQR_F32 if dt == "f32" else caqr.CAQR_F64
        R = caqr.colmajor_empty(n, n, A0.dtype, dev)
        ws = torch.empty(max(caqr.caqr_workspace_bytes(m, n, code, opts), 1), dtype=torch.uint8, device=dev)

        def prep():
            A.copy_(A0)
            flush.zero_()

        steps = min(args.steps, 5 if m * n > 5e7 else 20)
        step = lambda: caqr.caqr_factor(A, R=R, ws=ws, opts=opts)  # noqa: E731
        ms = timed_steps(step, prep, args.warmup, steps, stream)
        # the same C-ABI call replayed from a CUDA graph: the device time
        # without the ~25 us of host work per call (Python + ctypes + plan +
        # launches), which dominates the small configs (C1, C2)
        gms = None
        try:
            g = torch.cuda.CUDAGraph()
            side = torch.cuda.Stream()
            side.wait_stream(stream)
            with torch.cuda.stream(side):
                prep()
                step()
            stream.wait_stream(side)
            with torch.cuda.graph(g):
                step()
            gms = timed_steps(g.replay, prep, args.warmup, steps, stream)
            del g
        except Exception as exc:  # noqa: BLE001 -- reported, the eager number stands
            gms = f"graph capture failed: {exc}"
        fl = 2.0 * m * n * n - 2.0 * n ** 3 / 3.0
        alu = alu_peak_tflops(dt, peaks["sm_max_mhz"])
        t_roof = max(2.0 * m * n * esz / (peaks["hbm_gbs"] * 1e9), fl / (alu * 1e12))
        out[name] = {"ms_per_step": ms, "value": fl / (ms * 1e-3) / 1e9, "unit": UNIT, "steps": steps,
                     "read_write_gbs": 2.0 * m * n * esz / (ms * 1e-3) / 1e9,
                     "roofline_frac": t_roof / (ms * 1e-3),
                     "roofline_note": "max(read A + write V at measured HBM, flops at derived ALU peak) / time",
                     "graph_ms_per_step": gms,
                     "graph_note": "same caqr_factor call captured once and replayed (CUDA graph); "
                                   "same prep / events protocol; excludes host launch cost",
                     "plan": caqr.caqr_plan_info(m, n, code, opts)}
        if isinstance(gms, float):
            out[name]["graph_roofline_frac"] = t_roof / (gms * 1e-3)
        del A0, A, R, ws
        torch.cuda.empty_cache()
    return out


def strong_scaling_leg(args, dev, flush, world, rank, handle, L, gather, cws):
    """Config C4' (8,000,000 x 192 fp32) split over the N ranks (strong
    scaling; N = 1: the whole matrix on one GPU).  Time per step = max over
    ranks of each rank's event time (local TSQR + all-gather + combine)."""
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_andersonbdk11_b200 import caqr
    from paper_conf_ipps_andersonbdk11_b200.dist import shard_rows

    cfg = workload("c4p_8Mx192_f32")
    m_total, n = cfg["m"], cfg["n"]
    _, rows = shard_rows(m_total, world, rank)
    A0 = make_input(cfg, 77 + rank, dev, rows=rows)
    A = caqr.colmajor_empty(rows, n, torch.float32, dev)
    R = caqr.colmajor_empty(n, n, torch.float32, dev)
    ws = torch.empty(caqr.caqr_workspace_bytes(rows, n, caqr.CAQR_F32, None), dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    def step():
        if handle is None:
            caqr.caqr_factor(A, R=R, ws=ws)
        else:
            caqr._check("caqr_dist_factor_f32", L.caqr_dist_factor_f32(
                handle, rows, n, A.data_ptr(), rows, R.data_ptr(), n, ws.data_ptr(), ws.numel(),
                gather.data_ptr(), cws.data_ptr(), cws.numel(), None, caqr.ctypes.c_void_p(stream.cuda_stream)))

    def prep():
        A.copy_(A0)
        flush.zero_()

    if world > 1:
        dist.barrier()
    steps = max(3, min(args.steps, 5))
    ms = timed_steps(step, prep, args.warmup, steps, stream)
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    fl = 2.0 * m_total * n * n - 2.0 * n ** 3 / 3.0
    del A0, A, R, ws
    torch.cuda.empty_cache()
    return {"workload": "c4p_8Mx192_f32", "scaling": "strong", "m_total": m_total, "m_per_gpu": rows,
            "n": n, "n_gpus": world, "steps": steps, "ms_per_step": ms, "value": fl / (ms * 1e-3) / 1e9,
            "unit": UNIT, "timing": "per rank CUDA events around each factor (N > 1: caqr_dist_factor incl. the "
                                    "NCCL all-gather and combine), mean over steps, max over ranks"}


# ---- the CUDA arm -------------------------------------------------------------
def main():
    args = parse()
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        relaunch_distributed(args)
    if world != args.gpus:
        sys.stderr.write(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}\n")
        raise SystemExit(1)
    if args.impl == "reference":
        run_reference(args, rank)
        return

    import torch
    import torch.distributed as dist

    from paper_conf_ipps_andersonbdk11_b200 import build as cbuild
    from paper_conf_ipps_andersonbdk11_b200 import caqr, workloads

    if rank == 0:
        cbuild.build()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
        dist.barrier()
    L = caqr.lib()
    cfg = workload(args.config)
    m, n, dt = cfg["m"], cfg["n"], cfg["dtype"]
    tdt = torch.float32 if dt == "f32" else torch.float64
    opts = caqr.make_opts(args.leaf_rows or cfg.get("leaf_rows", 0), args.panel_cols or cfg.get("nb", 0))
    code = caqr.CAQR_F32 if dt == "f32" else caqr.CAQR_F64
    esz = 4 if dt == "f32" else 8

    # synthetic input, resident in HBM (rank r draws its own shard: weak scaling)
    A0 = workloads.device_gaussian(m, n, seed=1234 + rank, dtype=tdt, device=dev).t()
    A = caqr.colmajor_empty(m, n, tdt, dev)
    R = caqr.colmajor_empty(n, n, tdt, dev)
    ws = torch.empty(caqr.caqr_workspace_bytes(m, n, code, opts), dtype=torch.uint8, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    handle = None
    if world > 1:
        import ctypes

        uid = (ctypes.c_char * 128)()
        if rank == 0:
            caqr._check("caqr_dist_unique_id", L.caqr_dist_unique_id(uid))
        obj = [bytes(uid)]
        dist.broadcast_object_list(obj, src=0)
        uid = (ctypes.c_char * 128).from_buffer_copy(obj[0])
        h = ctypes.c_void_p()
        caqr._check("caqr_dist_create", L.caqr_dist_create(ctypes.byref(h), world, rank, uid))
        handle = h
        gather = caqr.colmajor_empty(world * n, n, tdt, dev)
        cws = torch.empty(caqr.caqr_combine_workspace_bytes(world, n, code), dtype=torch.uint8, device=dev)

    def step():
        if handle is None:
            caqr.caqr_factor(A, R=R, ws=ws, opts=opts)
        else:
            suf = "f32" if dt == "f32" else "f64"
            info = getattr(L, f"caqr_dist_factor_{suf}")(
                handle, m, n, A.data_ptr(), m, R.data_ptr(), n, ws.data_ptr(), ws.numel(),
                gather.data_ptr(), cws.data_ptr(), cws.numel(), caqr._optp(opts),
                caqr.ctypes.c_void_p(stream.cuda_stream))
            caqr._check(f"caqr_dist_factor_{suf}", info)

    def prep():
        A.copy_(A0)
        flush.zero_()

    for _ in range(max(args.warmup, 3)):
        prep()
        step()
    torch.cuda.synchronize()

    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(args.steps)]
    caqr.caqr_trace_begin(1 << 17)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t_wall0 = time.perf_counter()
        for i in range(args.steps):
            prep()
            evs[i][0].record(stream)
            step()
            evs[i][1].record(stream)
        torch.cuda.synchronize()
        t_wall = time.perf_counter() - t_wall0
    trace = caqr.caqr_trace_end(1 << 17)
    if world > 1:
        dist.barrier()
    ms = [a.elapsed_time(b) for a, b in evs]
    total_ms = sum(ms)
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    m_total = m * world
    flops = 2.0 * m_total * n * n - 2.0 * n ** 3 / 3.0
    value = flops / (ms_per_step * 1e-3) / 1e9

    # correctness spot check of the timed result: column norms of R = of A
    Rn = torch.linalg.norm(R.double(), dim=0)
    An = torch.linalg.norm(A0.double(), dim=0)
    if world == 1:
        rel = float((torch.abs(Rn - An) / An).max())
        assert rel < (1e-4 if dt == "f32" else 1e-12), f"R column norms off by {rel}"

    # per-kernel roofline from the live trace (events on the launching stream)
    peaks = load_peaks()
    per = {}
    for name, kms, fl, by in trace:
        d = per.setdefault(name, [0, 0.0, 0.0, 0.0])
        d[0] += 1
        d[1] += kms
        d[2] += fl
        d[3] += by
    launches_per_step = sum(d[0] for d in per.values()) / args.steps
    dom = max(per, key=lambda k: per[k][1])
    cnt, kms, kfl, kby = per[dom]
    alu_tf = alu_peak_tflops(dt, peaks["sm_max_mhz"])
    ridge = alu_tf * 1e12 / (peaks["hbm_gbs"] * 1e9)
    if kby > 0 and kfl / kby < ridge:
        achieved = kby / (kms * 1e-3) / 1e9
        roof = {"bound": "hbm", "achieved": achieved, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": achieved / peaks["hbm_gbs"]}
    else:
        achieved = kfl / (kms * 1e-3) / 1e12
        roof = {"bound": "alu", "achieved": achieved, "peak": alu_tf, "unit": "TFLOP/s",
                "frac": achieved / alu_tf}
    roof.update({"kernel": dom, "launches_per_step": cnt / args.steps,
                 "share_of_step": kms / max(sum(d[1] for d in per.values()), 1e-9),
                 "peak_source": (peaks["source"] if roof["bound"] == "hbm" else
                                 f"derived: 148 SMs x {FP32_LANES if dt == 'f32' else FP64_LANES} FMA lanes x 2 x "
                                 f"{peaks['sm_max_mhz']:.0f} MHz"),
                 "traffic": None})
    tr_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tr_path):
        try:
            with open(tr_path) as f:
                tr = json.load(f)
            if tr.get(args.config, {}).get("kernel") == dom:
                roof["traffic"] = tr[args.config]["dram_bytes_per_launch"]
                roof["traffic_source"] = tr[args.config].get("source")
        except Exception:
            pass
    # whole-path roofline of the BASELINE metric: max(read A once / HBM, flops / ALU peak)
    t_roof = max(m_total * n * esz / world / (peaks["hbm_gbs"] * 1e9),
                 flops / world / (alu_tf * 1e12))
    path_roof = {"t_roofline_ms": t_roof * 1e3, "frac": t_roof / (ms_per_step * 1e-3),
                 "bound": "alu" if flops / world / (alu_tf * 1e12) > m * n * esz / (peaks["hbm_gbs"] * 1e9) else "hbm"}

    # e2e: the public call from pinned host memory.  caqr_factor_host streams
    # A in row chunks (H2D on a copy engine) and factors each chunk as soon as
    # it lands, then combines the chunks' R's; + D2H of R.  The serial variant
    # (whole H2D, then caqr_factor) is reported beside it for context.
    e2e = None
    Ah = None
    if not args.no_e2e and world == 1:
        Ah = torch.empty((n, m), dtype=tdt, pin_memory=True).t()
        Ah.copy_(A0)
        Rh = torch.empty((n, n), dtype=tdt, pin_memory=True)
        S = args.e2e_chunks
        hws = torch.empty(max(caqr.caqr_factor_host_workspace_bytes(m, n, S, 0 if tdt == torch.float32 else 1,
                                                                    opts), 1),
                          dtype=torch.uint8, device="cuda")
        torch.cuda.synchronize()

        def e2e_time(call):
            ee = []
            for i in range(max(3, min(args.steps, 10)) + 2):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                flush.zero_()
                a.record(stream)
                call()
                Rh.copy_(R, non_blocking=True)
                b.record(stream)
                torch.cuda.synchronize()
                if i >= 2:
                    ee.append(a.elapsed_time(b))
            return sum(ee) / len(ee)

        def serial():
            A.copy_(Ah, non_blocking=True)
            caqr.caqr_factor(A, R=R, ws=ws, opts=opts)

        serial_ms = e2e_time(serial)
        e2e_ms = e2e_time(lambda: caqr.caqr_factor_host(Ah, S, A=A, R=R, ws=hws, opts=opts))
        e2e = {"value": flops / (e2e_ms * 1e-3) / 1e9, "unit": UNIT, "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": m * n * esz, "d2h_bytes_per_step": n * n * esz,
               "api": f"paper_conf_ipps_andersonbdk11_b200.caqr.caqr_factor_host (pinned host A, {S} row chunks: "
                      "H2D overlapped with the chunk factorizations, then the combine) + D2H(R)",
               "h2d_gbs": m * n * esz / (e2e_ms * 1e-3) / 1e9,
               "serial": {"value": flops / (serial_ms * 1e-3) / 1e9, "ms_per_step": serial_ms,
                          "api": "whole pinned H2D, then caqr_factor, + D2H(R)"}}
        del hws
    elif not args.no_e2e:
        # N > 1: each rank's pinned host shard -> H2D, the distributed factor
        # (local TSQR + NCCL all-gather of the R's + combine), D2H of R; the
        # per-step time is the max over ranks.
        Ah = torch.empty((n, m), dtype=tdt, pin_memory=True).t()
        Ah.copy_(A0)
        Rh = torch.empty((n, n), dtype=tdt, pin_memory=True)
        torch.cuda.synchronize()
        ee = []
        for i in range(max(3, min(args.steps, 10)) + 2):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            flush.zero_()
            dist.barrier()
            torch.cuda.synchronize()
            a.record(stream)
            A.copy_(Ah, non_blocking=True)
            step()
            Rh.copy_(R, non_blocking=True)
            b.record(stream)
            torch.cuda.synchronize()
            if i >= 2:
                ee.append(a.elapsed_time(b))
        t = torch.tensor([sum(ee) / len(ee)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())
        e2e = {"value": flops / (e2e_ms * 1e-3) / 1e9, "unit": UNIT, "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": m_total * n * esz, "d2h_bytes_per_step": world * n * n * esz,
               "api": "per rank: pinned H2D of the row shard + caqr_dist_factor (local TSQR, NCCL all-gather "
                      "of the R's, combine) + D2H(R); max over ranks"}

    strong, extra = None, None
    if not args.no_extra:
        Ah = None  # release the e2e leg's pinned host copy
        strong = strong_scaling_leg(args, dev, flush, world, rank, handle, L,
                                    gather if world > 1 else None, cws if world > 1 else None)
        if world == 1 and rank == 0:
            extra = extra_configs_leg(args, dev, flush, peaks)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(cfg, args.cpu_sample_rows)

    if rank == 0:
        plan = caqr.caqr_plan_info(m, n, code, opts)
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": dt, "data": "synthetic",
            "config": {"workload": args.config, "m_per_gpu": m, "m_total": m_total, "n": n,
                       "input": "N(0,1) drawn on device, torch.Generator seed 1234+rank",
                       "leaf_rows": plan["leaf_rows"], "panel_cols": plan["panel_cols"],
                       "leaves": plan["leaves"], "tree_levels": plan["tree_levels"],
                       "l2": "A (>= 768 MB) exceeds the 126 MB L2; 256 MiB flush + A restore between "
                             "steps, outside the timed events",
                       "timing": "CUDA events on the launching stream around each caqr_factor; "
                                 "sum over steps; max over ranks",
                       "wall_s_timed_loop": t_wall},
            "clocks": clk.summary(),
            "gpu_launches": launches_per_step,
            "roofline": roof,
            "path_roofline": path_roof,
            "kernels": {k: {"launches_per_step": v[0] / args.steps, "ms_per_step": v[1] / args.steps}
                        for k, v in per.items()},
            "e2e": e2e,
            "cpu_baseline": cpu,
            "strong_scaling": strong,
            "configs": extra,
        }
        print(json.dumps(line), flush=True)
    if handle is not None:
        L.caqr_dist_destroy(handle)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
