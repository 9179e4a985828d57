#!/usr/bin/env python3
"""bench.py -- CUDAlign 2.0 Stage-1 hot path on B200 (BASELINE.json metric).

One step = the whole hot path of SURVEY.md 8(a) over one synthetic pair:
encode/pack (a1) -> Stage-1 matrix fill with the exact best cell (a2-a5) ->
every k-th special row (H, F) streamed to a host sink (a6) -> reverse goal
pass to the start cell (a8).  GCUPS = m n / (t 10^9).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C2] [--impl ours|reference]

N > 1 (torchrun, one process per GPU): the band-cyclic pipeline (a7, DESIGN.md
8): rank r runs bands r, r + N, ... and stores each band's bottom row and
progress into rank (r + 1) mod N's area by peer stores over NVLink (CUDA IPC);
strong scaling (the same matrix on N GPUs).  Each rank's sink gets the whole
special rows of its bands; the reverse pass runs on rank 0.  SWB_MULTI=stripes
selects the column-stripe pipeline instead (rank g owns columns
[g n / N, (g+1) n / N)).  SWB_SAME_DEVICE=1 maps every rank to cuda:0 with gloo
(a functional check of the N > 1 path on one GPU).

--impl reference: the CPU oracle (oracle/, single-threaded plain C) timed on a
bounded row-band sample of the same workload on the host cores.
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

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GCUPS at 1/2/4/8 B200 (33×47 MBP synthetic) + % of INT-pipe roofline"
SCORING = (1, -3, 3, 2)  # match +1, mismatch -3, first gap -5 (G_open 3), extension -2
# Paper Table IV 543K x 536K Stage 1 with flush (SRA 50M): 21,419 MCUPS on a GTX 285.
PAPER_GCUPS = {"C2": 21.419}
# Roofline: ALU-pipe cycles of each kernel's cell-update
# mix with the measured rates (profiles/r01_microbench_int.txt; half-rate ops
# occupy the ALU pipe 2 cycles per warp instruction, full-rate ops 1):
#   int32 kernel: 8 ALU cycles per 32 cells  -> 16.0 cells/clk/SM
#   packed 16x2 : 11 ALU cycles per 64 cells -> 23.27 cells/clk/SM
#     (SWB_FMODE 2 mix: VIMNMX3 E*, PRMT p, 3x VIADDMNMX D/t/F', 1/2 VIMNMX3 max;
#      the earlier mix with 9 ALU cycles issued 2 more instructions per slot and
#      ran 14-18 % slower)
ROOF_CELLS_PER_CLK_SM = {"int32": 16.0, "int16x2": round(4 * 64 / 11, 2)}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=3)
    p.add_argument("--warmup", type=int, default=3)
    # C4 (10M x 10M): the largest BASELINE config that fits one GPU's bench
    # window (the metric's C5 pair takes ~5 min per step; tools/c5_align.py)
    p.add_argument("--workload", default=os.environ.get("SWB_WORKLOAD", "C4"))
    p.add_argument("--e2e-steps", type=int, default=3, help="host-API steps timed for e2e (<= --steps)")
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--k", type=int, default=None, help="special_row_interval override")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-align", action="store_true", help="skip the one-off full alignment (Stages 1-5)")
    return p.parse_args()


# ---------------------------------------------------------------- clocks sampler

class ClockSampler:
    FIELDS = "clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown," \
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap"

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def __exit__(self, *exc):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------- oracle (CPU) timing

def host_cpu():
    """(logical CPUs usable by this process, CPU model string)."""
    try:
        ncpu = len(os.sched_getaffinity(0))
    except Exception:
        ncpu = os.cpu_count() or 1
    model = "unknown"
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return ncpu, model


def oracle_sample(A, B, target_s=12.0, threads=None):
    """Time the oracle's band recompute (oracle.band: the same row loop as its
    Stage 1 and as the band-induction checker) on a bounded sample of the
    workload, as it stands: `threads` concurrent bands of distinct rows (the
    band-induction driver's parallelism; ctypes releases the GIL), each a full
    sweep of all n columns.  Returns (GCUPS over all threads, sample text, s, threads)."""
    from multiprocessing.pool import ThreadPool

    import numpy as np

    import oracle

    n, m = len(B), len(A)
    ma, mi, go, ge = SCORING
    ncpu, model = host_cpu()
    # one band's working set is 4 int64 rows of n + 1 entries: cap the threads at ~16 GB
    T = threads or max(1, min(ncpu, 64, int(16e9 // (32 * (n + 1)))))
    Htop = np.zeros(n + 1, np.int64)
    Ftop = np.full(n + 1, oracle.NEG, np.int64)
    r = max(1, min(m, int(2e8 // max(n, 1))))
    t0 = time.perf_counter()
    oracle.band(A, B, ma, mi, go, ge, 0, r, Htop, Ftop)
    rate1 = r * n / max(time.perf_counter() - t0, 1e-9)
    rows = int(max(1, min(m // T, target_s * rate1 / n)))

    def job(t):
        r0 = t * rows
        oracle.band(A, B, ma, mi, go, ge, r0, r0 + rows, Htop, Ftop)

    t0 = time.perf_counter()
    with ThreadPool(T) as pool:
        pool.map(job, range(T), chunksize=1)
    dt = time.perf_counter() - t0
    cells = float(T) * rows * n
    sample = (f"oracle.band on {T} threads (of {ncpu} logical CPUs, {model}), each rows r0+1..r0+{rows} x all "
              f"{n} columns of the workload ({cells:.3g} cells, {dt:.1f} s)")
    return cells / dt / 1e9, sample, dt, T, rate1 / 1e9


def reference_arm(args, cfg, k, rank, world):
    if rank != 0:
        return 0  # rank 0 alone runs the CPU oracle
    import synth
    import oracle

    A, B = synth.make_pair(cfg)
    oracle.build()
    vals, samples, times, T = [], "", [], 1
    for _ in range(args.warmup):
        oracle_sample(A, B, target_s=1.0)
    for _ in range(args.steps):
        v, samples, dt, T, _ = oracle_sample(A, B, target_s=8.0)
        vals.append(v)
        times.append(dt)
    value = statistics.median(vals)
    line = {
        "impl": "reference", "metric": METRIC, "workload": f"{cfg.name} ({cfg.m} x {cfg.n}, k={k})",
        "value": round(value, 4), "unit": "GCUPS",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1e3 * statistics.mean(times), 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
        "config": {"workload": cfg.name, "m": cfg.m, "n": cfg.n, "k": k, "scoring": list(SCORING)},
        "cpu_baseline": {"value": round(value, 4), "unit": "GCUPS", "cores": T, "kind": "oracle", "sample": samples,
                         "nproc": host_cpu()[0], "cpu_model": host_cpu()[1]},
        "e2e": {"value": round(value, 4), "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------- main

def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))

    import numpy as np

    import synth

    cfg = synth.CONFIGS[args.workload]
    k = cfg.k if args.k is None else args.k
    if args.impl == "reference":
        return reference_arm(args, cfg, k, rank, world)

    import torch

    same_dev = bool(os.environ.get("SWB_SAME_DEVICE"))
    dev_index = 0 if same_dev else local_rank
    torch.cuda.set_device(dev_index)
    dev = torch.device("cuda", dev_index)
    dist = None
    if world > 1:
        import torch.distributed as dist

        if same_dev:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cpu" if same_dev else dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    from paper_conf_ipps_sandesm11_b200 import Context, build

    if rank == 0:
        build.build()
    if world > 1:
        dist.barrier()
    build.build()
    A, B = synth.make_pair(cfg)
    m, n = len(A), len(B)
    dA = torch.from_numpy(A).to(dev)
    dB = torch.from_numpy(B).to(dev)
    # a dedicated stream: the library launches every kernel of the step on it, so
    # the CUDA events recorded on it bracket exactly the step's device work
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)
    sptr = stream.cuda_stream
    ctx = Context(dev_index)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2
    grp = None
    multi = os.environ.get("SWB_MULTI", "cyclic")
    if world > 1:
        from paper_conf_ipps_sandesm11_b200.parallel import CyclicGroup, StripeGroup

        grp = StripeGroup(ctx, rank, world, max_rows=m) if multi == "stripes" else \
            CyclicGroup(ctx, rank, world, max_rows=m, max_cols=n)

    sink_rows = [0]

    def sink(row, H, F):
        sink_rows[0] += 1
        return False

    def step():
        """One step on this rank; returns (best, start, stage-1 stats, launches)."""
        if grp is None:
            r, _ = ctx.align_stage1_dev(dA.data_ptr(), m, dB.data_ptr(), n, *SCORING, k=k, sink=sink, stream=sptr)
            best = r.astuple()
        else:
            best = grp.align_stage1(dA.data_ptr(), m, dB.data_ptr(), n, SCORING, k=k, sink=sink, stream=sptr)[0]
        s1 = ctx.stats()
        launches = s1["kernel_launches"]
        start = None
        if rank == 0 and best[0] > 0:
            st = ctx.reverse_goal_dev(dA.data_ptr(), best[1], dB.data_ptr(), best[2], best[0], *SCORING, stream=sptr)
            start = st.astuple()
            launches += ctx.stats()["kernel_launches"]
        return best, start, s1, launches

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    fill_ms, launches, replays, sp_bytes = [], 0, 0, 0
    results = set()
    sink_rows[0] = 0
    with ClockSampler(dev_index) as clk:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t_wall0 = time.perf_counter()
        for s in range(args.steps):
            flush.fill_(s & 0xFF)  # evict L2 between timed steps (outside the events)
            ev[s][0].record(stream)
            best, start, s1, nl = step()
            ev[s][1].record(stream)
            fill_ms.append(s1["fill_ms"])
            launches += nl
            replays += s1["replays"]
            sp_bytes += s1["special_bytes_d2h"]
            results.add((best, start))
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t_wall = time.perf_counter() - t_wall0
    step_ms = [a.elapsed_time(b) for a, b in ev]
    ms_per_step = max_over_ranks(sum(step_ms) / args.steps)
    cells = float(m) * float(n)
    value = cells / (ms_per_step * 1e-3) / 1e9
    assert len(results) == 1, f"non-deterministic results {results}"
    (best, start) = results.pop()
    rows_per_step = sink_rows[0] // max(1, args.steps)

    # ---- e2e through the host API from pinned host memory
    e2e = None
    if not args.no_e2e:
        hA = torch.from_numpy(A).pin_memory()
        hB = torch.from_numpy(B).pin_memory()
        import ctypes

        def host_view(t, size):
            return np.ctypeslib.as_array((ctypes.c_uint8 * size).from_address(t.data_ptr()))

        def e2e_step():
            if grp is None:
                r, _ = ctx.align_stage1(host_view(hA, m), host_view(hB, n), *SCORING, k=k, sink=sink)
                b = r.astuple()
                st = ctx.reverse_goal(host_view(hA, m), b[1], host_view(hB, n), b[2], b[0], *SCORING).astuple() if b[0] > 0 else None
                return b, st
            # multi-GPU: copy this step's inputs host -> device, then the stripe call
            dA.copy_(hA, non_blocking=True)
            dB.copy_(hB, non_blocking=True)
            b = grp.align_stage1(dA.data_ptr(), m, dB.data_ptr(), n, SCORING, k=k, sink=sink, stream=sptr)[0]
            st = None
            if rank == 0 and b[0] > 0:
                st = ctx.reverse_goal(host_view(hA, m), b[1], host_view(hB, n), b[2], b[0], *SCORING).astuple()
            return b, st

        e2e_step()
        torch.cuda.synchronize()
        ts = []
        for s in range(max(1, min(args.steps, args.e2e_steps))):
            flush.fill_(s & 0xFF)
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            t0 = time.perf_counter()
            b, st = e2e_step()
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t0)
            assert (b, st) == (best, start)
        e2e_s = max_over_ranks(sum(ts) / len(ts))
        h2d = m + n + ((best[1] + best[2]) if rank == 0 else 0)
        d2h = sp_bytes // args.steps + 3 * 16
        e2e = {"value": round(cells / e2e_s / 1e9, 3), "unit": "GCUPS", "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h), "ms_per_step": round(1e3 * e2e_s, 3), "steps": len(ts)}

    # ---- the full alignment (Stages 1-5, sw_align) once, outside the timed region:
    # the N2/N3 rows of SURVEY 8(f) measured on the same workload
    full = None
    if not args.no_align and world == 1:
        if m * n < 1e12:
            ctx.align(A, B, *SCORING, k=k)  # warm-up: first use of the Stage 2-5 kernels and their buffers
        t0 = time.perf_counter()
        ra = ctx.align(A, B, *SCORING, k=k)
        full = {"ms": round(1e3 * (time.perf_counter() - t0), 2),
                "stages_ms": {kk: round(v, 2) for kk, v in ra["ms"].items()},
                "score": ra["score"], "start": list(ra["start"]), "end": list(ra["end"]),
                "gap_runs": [len(ra["gap1"]), len(ra["gap2"])], "partitions": ra["partitions"],
                "mm_levels": ra["mm_levels"], "note": "host API call, wall clock; not part of the timed step"}

    fill_avg = max_over_ranks(statistics.mean(fill_ms))
    if rank != 0:
        ctx.close()
        if world > 1:
            dist.destroy_process_group()
        return 0

    clocks = clk.summary()
    # ---- roofline of the dominant kernel (the fill), from live CUDA events on its stream
    achieved = cells / (fill_avg * 1e-3) / 1e9 / world  # per GPU
    sm_max = clocks.get("sm_max_mhz") or 1965.0
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        sm_max = float(peaks.get("sm_max_mhz", sm_max))
    except Exception:
        pass
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    kdtype = "int16x2" if s1["alpha"] < 0 else "int32"  # stats.alpha < 0: the packed kernel ran
    roof = ROOF_CELLS_PER_CLK_SM[kdtype]
    peak = nsm * roof * sm_max * 1e6 / 1e9
    traffic = None
    try:
        for tr in json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json"))):
            if (tr.get("workload") == cfg.name and tr.get("kernel_dtype") == kdtype and world == 1
                    and tr.get("alpha", abs(s1["alpha"])) == abs(s1["alpha"]) and tr.get("warps", s1["warps"]) == s1["warps"]):
                traffic = tr.get("fill_dram_bytes_per_launch")
    except Exception:
        pass
    roofline = {"bound": "alu", "achieved": round(achieved, 2), "peak": round(peak, 1), "unit": "GCUPS",
                "frac": round(achieved / peak, 4), "traffic": traffic,
                "peak_basis": f"{kdtype} kernel: {nsm} SM x {roof} cells/clk/SM x {sm_max:.0f} MHz (measured pipe rates, DESIGN.md 5)",
                "fill_ms": round(fill_avg, 3), "per": "GPU",
                "peak_at_measured_clock": round(nsm * roof * (clocks.get('sm_mhz') or sm_max) * 1e-3, 1)}

    cpu = None
    if not args.no_cpu_baseline and world == 1:
        v, sample, _, T, v1 = oracle_sample(A, B, target_s=10.0)
        ncpu, model = host_cpu()
        cpu = {"value": round(v, 4), "unit": "GCUPS", "cores": T, "kind": "oracle", "sample": sample,
               "nproc": ncpu, "cpu_model": model, "single_thread_value": round(v1, 4)}

    line = {
        "metric": METRIC, "workload": f"{cfg.name} ({m} x {n}, k={k})",
        "value": round(value, 2), "unit": "GCUPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3), "higher_is_better": True,
        "scaling": "strong",
        "vs_baseline": (round(value / PAPER_GCUPS[cfg.name], 2) if cfg.name in PAPER_GCUPS else None),
        "dtype": "int16x2" if s1["alpha"] < 0 else "int32", "data": "synthetic",
        "config": {"workload": cfg.name, "m": m, "n": n, "k": k, "scoring": list(SCORING),
                   "step": "encode + Stage-1 fill + special rows to host sink + reverse goal pass",
                   "l2": "flushed between timed steps (256 MiB write)",
                   "parallelism": "single" if world == 1 else (
                       f"column stripes x{world} (NVLink border hand-off)" if multi == "stripes" else
                       f"band-cyclic x{world} (rank r runs bands r, r+{world}, ...; bottom rows over NVLink)")
                   + (" [same device, functional check]" if same_dev else ""),
                   "kernel": {"alpha": abs(s1["alpha"]), "packed16x2": s1["alpha"] < 0, "warps": s1["warps"],
                              "width": s1["width"], "grid": s1["grid"]},
                   "baseline_note": "vs_baseline = value / paper Table IV 543Kx536K flush (21.419 GCUPS, GTX 285, real DNA)"},
        "result": {"best": list(best), "start": list(start) if start else None, "special_rows_per_step": rows_per_step},
        "roofline": roofline,
        "cpu_baseline": cpu,
        "full_alignment": full,
        "e2e": e2e,
        "gpu_launches": int(launches),
        "replays_per_step": replays // args.steps,
        "clocks": clocks,
        "wall_s_timed": round(t_wall, 3),
    }
    print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
