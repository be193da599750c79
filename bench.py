#!/usr/bin/env python3
"""bench.py -- protected DGEMM TFLOP/s, % overhead vs unprotected, fault detection rate.

Contract (driver): ``python bench.py --gpus N --steps K --warmup W`` (N > 1 under torchrun,
one rank per GPU, NCCL).  One step = one pass of the whole A-ABFT hot path over one batch:
encode (+top-p) -> checksum-augmented GEMM -> bound/check -> correct,
plus, for N > 1, the NCCL all-reduce of the fault counters (SUM) and max |d|/eps (MAX).
Rank 0 prints ONE JSON line.

Workload at N = 1 is BASELINE.json configs[1]: 4096^3 FP64, checksum block 64, p = 2,
U[-1,1] inputs (seeds A=1, B=2).  For N > 1 each rank owns a 4096-row slab of A (weak
scaling, row sharding of SURVEY §8(e)), B is replicated by one broadcast before timing.
``--workload c4`` runs the 16384^3 row-sharded configuration instead (strong scaling).
``--impl reference`` times the CPU oracle (the only reference this paper-only task has) on a
bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

WORKLOADS = {
    # name: (M_per_rank or M_total, N, K, bs, dtype, recipe, scaling)
    "c2": dict(M=4096, N=4096, K=4096, bs=64, dtype="f64", recipe="uniform", scaling="weak",
               desc="BASELINE configs[1]: 4096^2 FP64, block 64, p=2, U[-1,1]"),
    "c1": dict(M=128, N=128, K=128, bs=32, dtype="f64", recipe="uniform", scaling="weak",
               graph=True,  # launch-latency bound: the step is one CUDA-graph replay
               desc="BASELINE configs[0]: 128^3 FP64, block 32, p=2, U[-1,1]"),
    "c3": dict(M=8192, N=8192, K=8192, bs=64, dtype="f32", recipe="wide", scaling="weak",
               desc="BASELINE configs[2]: 8192^2 FP32 FFMA, block 64, wide exponents"),
    "c4": dict(M=16384, N=16384, K=16384, bs=64, dtype="f64", recipe="uniform", scaling="strong",
               desc="BASELINE configs[3]: 16384^2 FP64 row-sharded, block 64"),
    "c5": dict(M=8192, N=8192, K=65536, bs=64, dtype="f64", recipe="uniform", scaling="strong",
               desc="BASELINE configs[4]: M=N=8192, K=65536 FP64, block 64"),
}
METRIC = "protected DGEMM TFLOP/s, % overhead vs unprotected, fault detection rate"
DMMA_PEAK_TFLOPS = 37.0   # profiles/r01_step0_pipes.jsonl: mma.sync m16n8k4 f64 issue ceiling
FFMA_PEAK_TFLOPS = 71.8   # same file, FFMA
P_TOPP = 2


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default=None, choices=sorted(WORKLOADS),
                    help="default: c2 (BASELINE configs[1]) at one GPU, c4 (configs[3], "
                         "16384^2 row-sharded, strong scaling) with several")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--campaign", type=int, default=1, help="fault-injection runs (0 = skip)")
    ap.add_argument("--no-traffic", action="store_true",
                    help="skip the ncu DRAM-traffic probe of the dominant kernel")
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def shard(wl, rank, world):
    """Rows of A owned by this rank (multiple of bs), and the global M."""
    if wl["scaling"] == "weak":
        m_local = wl["M"]
        return rank * m_local, m_local, m_local * world
    from paper_conf_dsn_braunhw14_b200.distributed import shard_rows
    row0, m_local = shard_rows(wl["M"], world, rank, wl["bs"])
    return row0, m_local, wl["M"]


# ------------------------------------------------------------------------------- clocks
class ClockSampler:
    """SM clock / throttle-reason sampling DURING the timed region (B200_PROFILING.md clocks
    line), via NVML in a background thread (nvidia-smi's start-up is slower than the region)."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "hw_power_brake_slowdown": 0x80, "sw_power_cap": 0x4}

    def __init__(self, index: int, period_s: float = 0.005):
        self.index = index
        self.period = period_s
        self.samples = []
        self.stop = threading.Event()
        self.thread = None
        self.max_mhz = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.thread = threading.Thread(target=self._run, daemon=True)
            self.thread.start()
        except Exception as e:  # no NVML: report unsampled
            self.err = repr(e)
        return self

    def _run(self):
        nv, h = self.nv, self.h
        while not self.stop.is_set():
            try:
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                try:
                    rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                except AttributeError:
                    rs = nv.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                pw = nv.nvmlDeviceGetPowerUsage(h) / 1000.0
                self.samples.append((sm, rs, pw))
            except Exception:
                pass
            time.sleep(self.period)

    def __exit__(self, *exc):
        self.stop.set()
        if self.thread:
            self.thread.join(timeout=2)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unsampled"]}
        reasons = sorted({n for _, rs, _ in self.samples for n, bit in self.REASONS.items()
                          if rs & bit})
        return {"sm_mhz": statistics.median(s for s, _, _ in self.samples),
                "sm_max_mhz": self.max_mhz, "reasons": reasons,
                "power_w_max": max(p for _, _, p in self.samples),
                "samples": len(self.samples), "source": "NVML, 5 ms period"}


# ------------------------------------------------------------------------------- oracle arms
def oracle_sample(wl, rows, nthreads):
    """The CPU oracle, as it stands, on a BS-aligned row slab of the workload: encode of A slab
    and all of B, the three products, check, correct.  Returns (useful flops, seconds)."""
    from oracle import oracle as orc
    dt = np.float64 if wl["dtype"] == "f64" else np.float32
    A = synth.generate(wl["recipe"], rows, wl["K"], seed=1, matrix_id=0, dtype=dt,
                       full_cols=wl["K"])
    B = synth.generate(wl["recipe"], wl["K"], wl["N"], seed=2, matrix_id=1, dtype=dt)
    t0 = time.perf_counter()
    orc.protected_matmul(A, B, bs=wl["bs"], p=P_TOPP, nthreads=nthreads)
    dt_s = time.perf_counter() - t0
    return 2.0 * rows * wl["N"] * wl["K"], dt_s


def cpu_rows_for(wl, budget_s, nthreads):
    """Calibrate a BS-multiple row count that takes about budget_s on this host."""
    bs = wl["bs"]
    fl, sec = oracle_sample(dict(wl, N=min(wl["N"], 512)), bs, nthreads)
    rate = fl / sec  # flop/s at N=512 (GEMM-dominated)
    rows = int(budget_s * rate / (2.0 * wl["N"] * wl["K"]) // bs * bs)
    return max(bs, min(rows, wl["M"]))


def run_reference(args, wl):
    rank, world, _ = dist_env()
    if rank != 0:
        return
    nthreads = os.cpu_count() or 1
    # each step ~2 s of oracle work so that --steps K --warmup W ends within a few minutes
    rows = cpu_rows_for(wl, 2.0, nthreads)
    for _ in range(args.warmup):
        oracle_sample(dict(wl, N=min(wl["N"], 256)), wl["bs"], nthreads)
    times, flops = [], 0.0
    for _ in range(args.steps):
        fl, sec = oracle_sample(wl, rows, nthreads)
        times.append(sec)
        flops += fl
    total = sum(times)
    value = flops / total / 1e12
    sample = (f"{rows} of {wl['M']} rows of A (x full B) per step: encode+top-p, C/Ccol/Crow, "
              f"check, correct; {nthreads} threads")
    out = {"impl": "reference", "metric": METRIC, "value": value, "unit": "TFLOP/s",
           "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
           "ms_per_step": 1e3 * total / args.steps, "higher_is_better": True,
           "scaling": wl["scaling"], "vs_baseline": None, "dtype": wl["dtype"],
           "data": "synthetic", "config": {"workload": wl["desc"], "M": wl["M"], "N": wl["N"],
                                           "K": wl["K"], "bs": wl["bs"], "p": P_TOPP},
           "cpu_baseline": {"value": value, "unit": "TFLOP/s", "cores": nthreads,
                            "kind": "oracle", "sample": sample},
           "e2e": {"value": value, "unit": "TFLOP/s", "h2d_bytes_per_step": 0,
                   "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# ------------------------------------------------------------------------------- our arm
def main():
    args = parse()
    if args.workload is None:
        args.workload = "c2" if int(os.environ.get("WORLD_SIZE", "1")) == 1 else "c4"
    wl = dict(WORKLOADS[args.workload])
    if args.impl == "reference":
        return run_reference(args, wl)

    import torch
    import torch.distributed as dist

    rank, world, local = dist_env()
    # one process per GPU; AABFT_DIST_BACKEND=gloo lets the multi-rank path be exercised with
    # several ranks sharing one GPU (tests on a 1-GPU box), NCCL otherwise
    backend = os.environ.get("AABFT_DIST_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)

    from paper_conf_dsn_braunhw14_b200 import _abi, api

    tdt = torch.float64 if wl["dtype"] == "f64" else torch.float32
    ndt = np.float64 if wl["dtype"] == "f64" else np.float32
    row0, m_local, M_glob = shard(wl, rank, world)
    N, K, bs = wl["N"], wl["K"], wl["bs"]

    # inputs: this rank's slab of A, and B broadcast from rank 0 (outside the timed region)
    A_h = synth.generate(wl["recipe"], m_local, K, seed=1, matrix_id=0, dtype=ndt, row0=row0,
                         full_cols=K)
    A = torch.from_numpy(A_h).to(dev)
    if rank == 0:
        B = torch.from_numpy(synth.generate(wl["recipe"], K, N, seed=2, matrix_id=1,
                                            dtype=ndt)).to(dev)
    else:
        B = torch.empty(K, N, dtype=tdt, device=dev)
    b_bcast_ms = None
    if world > 1:
        # B replication: one broadcast from rank 0, timed on its own (not in the step: the
        # operands are resident when the step starts)
        dist.broadcast(B, src=0)
        dist.barrier()
        torch.cuda.synchronize(dev)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        dist.broadcast(B, src=0)
        e1.record()
        torch.cuda.synchronize(dev)
        t = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        b_bcast_ms = float(t[0])
    from paper_conf_dsn_braunhw14_b200.distributed import ShardedProtectedGemm
    sharded = (ShardedProtectedGemm(m_local, N, K, world=world, rank=rank, dtype=tdt, bs=bs,
                                    p=P_TOPP, device=dev) if world > 1 else None)
    plan = sharded.plan if sharded else api.ProtectedGemm(m_local, N, K, dtype=tdt, bs=bs,
                                                          p=P_TOPP, device=dev)
    C_plain = torch.empty(m_local, N, dtype=tdt, device=dev)
    stream = torch.cuda.current_stream(dev)

    graph = plan.capture(A, B) if (wl.get("graph") and world == 1) else None

    def step():
        if graph is not None:
            graph.replay()  # encode -> gemm -> check -> correct, one launch from the host
        elif sharded is not None:
            # encode of the local A rows and of this rank's B columns, all-gather of the B
            # encoding, GEMM / check / correct of the local rows, counter all-reduce
            sharded.run(A, B)
        else:
            plan.run(A, B)

    in_bytes = (m_local * K + K * N) * (8 if wl['dtype'] == 'f64' else 4)
    flush = (torch.empty(256 << 20, dtype=torch.uint8, device=dev) if in_bytes < (126 << 20)
             else None)

    def timed(fn, steps, per_step_events=None):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        if flush is None:
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(steps):
                fn()
            e1.record(stream)
            torch.cuda.synchronize(dev)
            ms = e0.elapsed_time(e1)
        else:
            # inputs fit in L2: each step is timed alone after an (untimed) L2 flush
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                  for _ in range(steps)]
            for a, b in ev:
                flush.zero_()
                a.record(stream)
                fn()
                b.record(stream)
            torch.cuda.synchronize(dev)
            ms = sum(a.elapsed_time(b) for a, b in ev)
        if world > 1:
            dist.barrier()
        if world > 1:
            t = torch.tensor([ms], device=dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t[0])
        return ms

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize(dev)
    n0 = _abi.launch_count()
    with ClockSampler(local) as clk:
        ms = timed(step, args.steps)
    launches = _abi.launch_count() - n0
    if graph is not None:  # replays launch the captured kernels without passing the C ABI
        c0 = _abi.launch_count()
        plan.run(A, B)
        torch.cuda.synchronize(dev)
        launches = (_abi.launch_count() - c0) * args.steps
    cnt = api.counts_dict(plan.counts)
    useful = 2.0 * M_glob * N * K if wl["scaling"] == "strong" else 2.0 * m_local * world * N * K
    value = useful * args.steps / (ms * 1e-3) / 1e12

    # unprotected GEMM of the same kernel family (overhead denominator)
    for _ in range(3):
        api.gemm_plain(A, B, out=C_plain)
    ms_plain = timed(lambda: api.gemm_plain(A, B, out=C_plain), args.steps)
    value_plain = useful * args.steps / (ms_plain * 1e-3) / 1e12

    # dominant kernel (augmented GEMM): CUDA events on the launching stream around each launch
    gemm_ms = []
    for _ in range(args.steps):
        plan.encode(A, B, defer=plan.topp_in_gemm)  # as in the step: top-p rides in the GEMM
        g0 = torch.cuda.Event(enable_timing=True)
        g1 = torch.cuda.Event(enable_timing=True)
        g0.record(stream)
        plan.gemm(A, B)
        g1.record(stream)
        plan.check(correct=True)
        torch.cuda.synchronize(dev)
        gemm_ms.append(g0.elapsed_time(g1))
    gemm_avg = sum(gemm_ms) / len(gemm_ms)
    aug_flops = 2.0 * K * (m_local * N + (m_local // bs) * N + m_local * (N // bs))
    peak = DMMA_PEAK_TFLOPS if wl["dtype"] == "f64" else FFMA_PEAK_TFLOPS
    achieved = aug_flops / (gemm_avg * 1e-3) / 1e12
    traffic, traffic_src = None, "not measured (--no-traffic or N > 1)"
    if rank == 0 and world == 1 and not args.no_traffic:
        traffic, traffic_src = measure_traffic(wl, m_local, N, K, bs)

    # per-stage device times of one protected step, and Table I's comparators (NEXT-3)
    stages = stage_times(plan, A, B, stream, dev, args.steps)
    stage_roofs = stage_rooflines(stages, m_local, N, K, bs, P_TOPP,
                                  8 if wl["dtype"] == "f64" else 4, plan.fused)
    table1 = None
    unfused = None
    if world == 1:
        table1 = run_table1(plan, A, B, timed, useful, args.steps, value, value_plain)
        plan.run(A, B)
        # the same step with the unfused check (re-sums C from memory, the paper's check
        # kernel P:L372; wider fault model)
        if plan.fused:
            plan_u = api.ProtectedGemm(m_local, N, K, dtype=tdt, bs=bs, p=P_TOPP, device=dev,
                                       fused=False)
            for _ in range(3):
                plan_u.run(A, B)
            ms_u = timed(lambda: plan_u.run(A, B), args.steps)
            unfused = {"value": useful * args.steps / (ms_u * 1e-3) / 1e12, "unit": "TFLOP/s",
                       "ms_per_step": ms_u / args.steps,
                       "overhead_pct": 100.0 * (1.0 - useful * args.steps / (ms_u * 1e-3) / 1e12 / value_plain)}
            del plan_u

    # fault-injection campaign (outside the timed region): one fault per BS x BS block
    campaign = None
    # (N = 1 only: at N > 1 the other ranks would idle in the next collective meanwhile)
    if args.campaign and rank == 0 and world == 1:
        campaign = run_campaign(plan, A, B, wl, dev, ndt)

    # end-to-end through the C ABI with HOST buffers (pinned), copies inside the timed region
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(wl, m_local, N, K, bs, A, B, dev, args, world, timed)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        nthreads = os.cpu_count() or 1
        rows = cpu_rows_for(wl, 6.0, nthreads)
        fl, sec = oracle_sample(wl, rows, nthreads)
        cpu = {"value": fl / sec / 1e12, "unit": "TFLOP/s", "cores": nthreads, "kind": "oracle",
               "sample": f"{rows} of {wl['M']} rows of A x full B ({fl / 1e9:.1f} GFLOP useful): "
                         f"encode+top-p, C/Ccol/Crow, check, correct; {sec:.1f} s"}

    if rank == 0:
        out = {
            "metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": wl["scaling"], "vs_baseline": None,
            "dtype": wl["dtype"], "data": "synthetic",
            "config": {"workload": wl["desc"], "M_per_rank": m_local, "M": M_glob, "N": N,
                       "K": K, "bs": bs, "p": P_TOPP, "recipe": wl["recipe"],
                       "parallelism": f"row-sharded dp{world}" + (
                           ", B encoding sharded by columns + all-gather" if world > 1 else ""),
                       "b_broadcast_ms": b_bcast_ms,
                       "cuda_graph": graph is not None,
                       "l2": ("inputs exceed L2 (A+B = %d MiB > 126 MB); no flush" % (in_bytes >> 20)
                              if flush is None else
                              "inputs fit in L2 (A+B = %d KiB): 256 MiB L2 flush before each "
                              "step, outside its events" % (in_bytes >> 10))},
            "unprotected_tflops": value_plain,
            "overhead_pct": 100.0 * (1.0 - value / value_plain),
            "protected_over_unprotected": value / value_plain,
            "fault_detection_rate": None if campaign is None else campaign["detection_rate"],
            "fault_silent_rate_below_bound": None if campaign is None else campaign["silent_rate_below_bound"],
            "fault_model": "computational faults in the GEMM (Alg 3 sites); fused check (default) "
                           "takes the reference sums from the GEMM epilogue registers, see "
                           "campaign.memory_faults_after_gemm and DESIGN.md 6.4",
            "false_positive_checks": cnt["checks_critical"],
            "clean_max_ratio": cnt["max_ratio"],
            "campaign": campaign,
            "roofline": {"bound": "tensor" if wl["dtype"] == "f64" else "alu",
                         "kernel": "gemm_f64_kernel (DMMA)" if wl["dtype"] == "f64" else "gemm_f32_kernel (FFMA)",
                         "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "traffic_source": traffic_src,
                         "peak_source": "measured mma.sync f64 / FFMA issue ceiling, profiles/r01_step0_pipes.jsonl",
                         "algorithmic_flops_per_launch": aug_flops,
                         "avg_launch_ms": gemm_avg,
                         "share_of_step": gemm_avg / (ms / args.steps)},
            "stages_ms": stages, "stage_rooflines": stage_roofs, "table1": table1,
            "unfused_check": unfused,
            "e2e": e2e, "gpu_launches": launches, "cpu_baseline": cpu,
            "clocks": clk.summary(),
        }
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


def measure_traffic(wl, m_local, N, K, bs):
    """roofline.traffic measured in this run: ncu (dram__bytes_read.sum + dram__bytes_write.sum)
    on one launch of the dominant kernel of the same workload, in a subprocess after the timed
    region (tools/traffic_probe.py; its own process, so the bench's timings are unaffected).
    Returns (bytes per launch, source) or (None, reason)."""
    import shutil
    ncu = shutil.which("ncu") or "/usr/local/cuda/bin/ncu"
    if not os.path.exists(ncu):
        return None, "ncu not found"
    kern = "gemm_f64_kernel" if wl["dtype"] == "f64" else "gemm_f32_kernel"
    cmd = [ncu, "--metrics", "dram__bytes_read.sum,dram__bytes_write.sum", "--clock-control",
           "none", "-k", "regex:" + kern, "-s", "1", "-c", "1", "--csv", sys.executable,
           os.path.join(ROOT, "tools", "traffic_probe.py"), str(m_local), str(N), str(K), str(bs),
           wl["dtype"], wl["recipe"]]
    try:
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=240)
    except Exception as e:  # timeout / missing permissions: report, do not fail the bench
        return None, f"ncu probe failed: {e!r}"[:200]
    import csv
    total = 0.0
    seen = 0
    for row in csv.reader(l for l in r.stdout.splitlines() if l.startswith('"')):
        if len(row) > 14 and row[12] in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            unit, val = row[13], float(row[14].replace(",", ""))
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
            total += val * scale
            seen += 1
    if seen != 2:
        return None, "ncu probe: metrics not found (" + (r.stderr or r.stdout)[-160:] + ")"
    return total, f"ncu dram__bytes_read+write.sum, one {kern} launch, same shape, this run"


def hbm_peak():
    """Measured HBM GB/s of this pod (MEASURED_PEAKS.json, driver-written), else the profiling
    guide's fallback figure."""
    try:
        with open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs"
    except (OSError, KeyError, ValueError):
        return 7700.0, "nominal HBM3e fallback (no MEASURED_PEAKS.json)"


def stage_rooflines(stages, M, N, K, bs, p, w, fused):
    """HBM roofline of the encode and check stages (north_star: achieved HBM GB/s for encode
    and check).  ALGORITHMIC bytes: encode reads A and B and writes Acs, Bcs and the top-p
    tables; the fused check reads the epilogue reference sums (double), the carried checksums,
    every vector's top-p list once and writes the block reports; the unfused check also reads C."""
    peak, src = hbm_peak()
    nI, nJ = M // bs, N // bs
    vecs = M + nI + N + nJ
    enc = (M * K + K * N) * w + (nI * K + K * nJ) * w + vecs * p * 12
    chk = (nI * N + M * nJ) * (8 + w) + vecs * p * 12 + nI * nJ * 20 + (0 if fused else M * N * w)
    out = {"peak_gbs": peak, "peak_source": src}
    for name, b in (("encode", enc), ("check", chk)):
        ms = stages.get(name)
        if ms:
            gbs = b / (ms * 1e-3) / 1e9
            out[name] = {"bytes": b, "ms": ms, "achieved_gbs": gbs, "frac": gbs / peak}
    return out


def stage_times(plan, A, B, stream, dev, steps):
    """Mean device time of each C-ABI step of the protected path (CUDA events on the launching
    stream, synchronised per step, host enqueue hidden behind a preceding GEMM)."""
    import torch
    # the step's check also corrects (AABFT_FLAG_CHECK_CORRECTS: no separate correction launch)
    names = ("encode", "gemm", "check")
    fns = (lambda: plan.encode(A, B, defer=plan.topp_in_gemm), lambda: plan.gemm(A, B),
           lambda: plan.check(correct=True))
    acc = {n: 0.0 for n in names}
    for _ in range(steps):
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(len(fns) + 1)]
        # the GPU is kept busy (an untimed GEMM) while the host enqueues the stages, so each
        # event pair brackets device time, not the host's launch latency on an idle stream
        plan.gemm(A, B)
        ev[0].record(stream)
        for k, fn in enumerate(fns):
            fn()
            ev[k + 1].record(stream)
        torch.cuda.synchronize(dev)
        for k, n in enumerate(names):
            acc[n] += ev[k].elapsed_time(ev[k + 1])
    return {n: acc[n] / steps for n in names}


# Table I at n = 4096 on a Tesla K20c, GFLOPS -- context, not a target
PAPER_TABLE1_4096 = {"abft_fixed_eps": 894.14, "a_abft": 829.10, "sea_abft": 686.39,
                     "tmr": 345.26, "unprotected_8192": 1048.4}


def run_table1(plan, A, B, timed, useful, steps, v_aabft, v_plain):
    """Table I's protected variants on this workload (NEXT-3): ABFT with a fixed, manually set
    eps (checksums-only encode, GEMM, check/correct against one eps) and SEA-ABFT (norms +
    SEA bound instead of top-p), each timed as a whole step like the headline number.  'cost of
    autonomy' = 1 - A-ABFT / fixed-eps ABFT (the paper: 1 - 829.10 / 894.14 = 7.3% at 4096)."""
    eps_fixed = 1e-9
    for _ in range(3):
        plan.run_ext(A, B, mode="fixed", eps_fixed=eps_fixed)
        plan.run_ext(A, B, mode="sea")
    ms_fix = timed(lambda: plan.run_ext(A, B, mode="fixed", eps_fixed=eps_fixed), steps)
    ms_sea = timed(lambda: plan.run_ext(A, B, mode="sea"), steps)
    v_fix = useful * steps / (ms_fix * 1e-3) / 1e12
    v_sea = useful * steps / (ms_sea * 1e-3) / 1e12
    return {"unit": "TFLOP/s", "unprotected": v_plain, "abft_fixed_eps": v_fix, "a_abft": v_aabft,
            "sea_abft": v_sea, "fixed_eps": eps_fixed,
            "cost_of_autonomy_pct": 100.0 * (1.0 - v_aabft / v_fix),
            "a_abft_over_sea": v_aabft / v_sea,
            "paper_k20c_gflops_4096": PAPER_TABLE1_4096}


def _xor(v, bit, ndt):
    ut = np.uint64 if ndt == np.float64 else np.uint32
    a = np.array([v], dtype=ndt).view(ut) ^ ut(1 << bit)
    with np.errstate(all="ignore"):
        return float(a.view(ndt)[0])


def run_campaign(plan, A, B, wl, dev, ndt):
    """Fault-injection campaign outside the timed region: one fault per BS x BS block (P:L543
    injects one fault per GEMM; the partitioned encoding makes every block an independent
    trial), 4096 trials per c2 GEMM.  Faults: additive e = r * max(eps_col, eps_row),
    r = +-2^(x/2), x = -12..12, at the final value (site 2) and in the accumulator mid-k
    (site 3) -- Alg 3 errorVecAdd2 / errorVecAdd1 -- and single-bit XOR of a random bit of the
    final value (site 0).  Labels (reading R22): 'must detect' |e| > 2 max eps, 'must be
    silent' |e| < min eps / 2, else 'band'; paper-style 'critical' |e| > 3 sigma_ij
    (P:L543).  Run through both check modes: the fused check (epilogue reference sums) and the
    unfused one that re-sums C from memory (the paper's check kernel); plus faults that
    corrupt C in device memory after the GEMM, which only the unfused mode can see (fault
    model).  Verdicts are checked against the CPU oracle block by block in
    tests/test_gpu_fullsize_faults.py; here they are counted."""
    import torch
    from paper_conf_dsn_braunhw14_b200 import api
    M, N, K, bs = plan.M, plan.N, plan.K, plan.bs
    plan.run(A, B)
    b = plan.bound()
    torch.cuda.synchronize(dev)
    C0 = plan.C.detach().cpu().numpy().copy()
    eps_col = b["eps_col"].cpu().numpy()
    eps_row = b["eps_row"].cpu().numpy()
    rng = np.random.default_rng(1234)
    nI, nJ = M // bs, N // bs
    nbits = 64 if ndt == np.float64 else 32
    faults, lab, mag, site = [], [], [], []
    for I in range(nI):
        for J in range(nJ):
            i = I * bs + int(rng.integers(bs))
            j = J * bs + int(rng.integers(bs))
            lo = min(eps_col[I, j], eps_row[i, J])
            hi = max(eps_col[I, j], eps_row[i, J])
            kind = int(rng.integers(3))
            if kind < 2:
                r = 2.0 ** (int(rng.integers(-12, 13)) / 2) * (1 if rng.integers(2) else -1)
                faults.append(dict(row=i, col=j, site=2 if kind == 0 else 3, k_step=K // 2,
                                   add=float(r * hi)))
                e = abs(r * hi)
            else:
                bit = int(rng.integers(nbits))
                faults.append(dict(row=i, col=j, site=0, xor_mask=1 << bit))
                e = abs(_xor(C0[i, j], bit, ndt) - float(C0[i, j]))
            fin = bool(np.isfinite(e))
            lab.append("detect" if (not fin or e > 2 * hi) else ("silent" if e < 0.5 * lo else "band"))
            mag.append(e / hi if fin else float("inf"))
            site.append(faults[-1]["site"])
    rows = torch.tensor([f["row"] for f in faults], dtype=torch.int64)
    cols = torch.tensor([f["col"] for f in faults], dtype=torch.int64)
    sig, _ = plan.bound_elements(rows, cols)
    sig = sig.cpu().numpy()
    fb = api.make_faults(faults, dev)
    out = {"faults_per_gemm": len(faults), "one_fault_per_block": True,
           "sites": "0 = XOR final value (random bit), 2 = additive final value, "
                    "3 = additive accumulator after k = K/2", "modes": {}}
    plan_u = api.ProtectedGemm(M, N, K, dtype=plan.dtype, bs=bs, p=plan.p, device=dev, fused=False)
    for mode, pl in (("fused", plan), ("unfused", plan_u)):
        res = pl.run(A, B, faults=fb)
        torch.cuda.synchronize(dev)
        st = res.reports()["status"]
        C1 = pl.C.detach().cpu().numpy()
        det = np.array([st[f["row"] // bs, f["col"] // bs] != 0 for f in faults])
        cor = np.array([st[f["row"] // bs, f["col"] // bs] == 1 for f in faults])
        L = np.array(lab)
        m = np.array(mag)
        crit = np.array([(not np.isfinite(x)) or x * max(eps_col[f["row"] // bs, f["col"]],
                                                         eps_row[f["row"], f["col"] // bs]) > 3 * s
                         for x, f, s in zip(m, faults, sig)])
        bit = np.array(site) == 0
        nd, ns, nb = (L == "detect").sum(), (L == "silent").sum(), (L == "band").sum()
        und = ~det
        out["modes"][mode] = {
            "must_detect": int(nd), "detected": int(det[L == "detect"].sum()),
            "corrected": int(cor[L == "detect"].sum()),
            "detection_rate": float(det[L == "detect"].mean()) if nd else None,
            "correction_rate": float(cor[L == "detect"].mean()) if nd else None,
            "must_be_silent": int(ns), "silent": int(und[L == "silent"].sum()),
            "silent_rate_below_bound": float(und[L == "silent"].mean()) if ns else None,
            "band": int(nb), "band_detected": int(det[L == "band"].sum()),
            "undetected_of_all": float(und.mean()),
            "max_undetected_e_over_eps": float(m[und].max()) if und.any() else 0.0,
            "paper_critical_3sigma": int(crit.sum()),
            "paper_detected_of_critical": float(det[crit].mean()) if crit.any() else None,
            "paper_detected_of_critical_bitflips": float(det[crit & bit].mean()) if (crit & bit).any() else None,
            "max_abs_err_after_correction": float(np.max(np.abs(C1 - C0))),
            "counts": res.counts()}
    # memory faults: C corrupted in device memory between aabft_gemm and aabft_check
    mem = {}
    for mode, pl in (("fused", plan), ("unfused", plan_u)):
        pl.run(A, B)
        pl.encode(A, B)
        pl.gemm(A, B)
        hit = []
        for I in range(0, nI, max(1, nI // 16)):
            J = int(rng.integers(nJ))
            i, j = I * bs + int(rng.integers(bs)), J * bs + int(rng.integers(bs))
            pl._C[i, j] += 1.0e3 * max(eps_col[I, j], eps_row[i, J]) + 1.0
            hit.append((I, J))
        pl.check()
        pl.correct()
        torch.cuda.synchronize(dev)
        st = pl.result().reports()["status"]
        mem[mode] = {"injected": len(hit), "detected": int(sum(st[I, J] != 0 for I, J in hit))}
    out["memory_faults_after_gemm"] = mem
    out["fault_model"] = ("fused check: computational faults inside the GEMM (Alg 3 sites), "
                          "reference sums from the epilogue registers; unfused check: also "
                          "corruption of C in memory after the GEMM (the paper's re-sum, P:L372)")
    f = out["modes"]["fused"]
    out["detection_rate"] = f["detection_rate"]
    out["silent_rate_below_bound"] = f["silent_rate_below_bound"]
    plan.run(A, B)  # leave the plan clean
    del plan_u
    return out


def run_e2e(wl, m_local, N, K, bs, A, B, dev, args, world, timed):
    """aabft_protected_gemm_host: pinned host A, B in; corrected C + counts out."""
    import ctypes as C
    import torch
    from paper_conf_dsn_braunhw14_b200 import _abi
    L = _abi.lib()
    code = _abi.F64 if wl["dtype"] == "f64" else _abi.F32
    cfg = _abi.Config(code, bs, m_local, N, K, P_TOPP, 0, 3.0, 1, 0)
    nbytes = L.aabft_host_arena_bytes(C.byref(cfg))
    arena = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    Ah = A.cpu().pin_memory()
    Bh = B.cpu().pin_memory()
    Ch = torch.empty(m_local, N, dtype=A.dtype).pin_memory()
    cnt = _abi.Counts()
    stream = torch.cuda.current_stream(dev).cuda_stream

    def call():
        _abi.ok(L.aabft_protected_gemm_host(C.byref(cfg), Ah.data_ptr(), Bh.data_ptr(),
                                            Ch.data_ptr(), C.addressof(cnt), arena.data_ptr(),
                                            nbytes, stream), "aabft_protected_gemm_host")
    call()
    steps = max(1, min(args.steps, 10))
    ms = timed(call, steps)
    es = A.element_size()
    useful = 2.0 * m_local * world * N * K
    del arena
    return {"value": useful * steps / (ms * 1e-3) / 1e12, "unit": "TFLOP/s",
            "h2d_bytes_per_step": (m_local * K + K * N) * es,
            "d2h_bytes_per_step": m_local * N * es + C.sizeof(_abi.Counts),
            "ms_per_step": ms / steps, "api": "aabft_protected_gemm_host (C ABI, pinned host)"}


if __name__ == "__main__":
    main()
