#!/usr/bin/env python3
"""Benchmark: input GB/s scanned per regex set on 1..8 B200 (and % of HBM roofline).

Metric (BASELINE.json): "input GB/s scanned per regex set at 1/2/4/8 B200; % of
HBM roofline".  A step = one pass of the whole hot path (every regex of the
set over the whole input: fused transposition, all IR instructions, the
count/digest epilogue and the carry fix-up pass).  Default workload (N=1):
the Snort-like config -- 1,000 regexes over 256 MiB of synthetic packet
payloads (BASELINE.json configs[1]).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config snort|tiny|...]
  python bench.py --impl reference ...   # the CPU oracle, timed on a bounded sample

Multi-GPU (torchrun, one rank per GPU, NCCL), DESIGN.md "Multi-GPU":
  --split chunk (default, weak scaling): the stream is N x 256 MiB; rank r
    holds chunk r (generated with its own seed) at global offset r x 256 MiB.
    Every timed step exchanges the halos (rx_max_lookback / lookahead bytes of
    the neighbour chunks, one all_gather), matches the chunk speculatively,
    resolves the boundary states (all_gather rounds + rx_rematch_chunk where
    a rank's true incoming state differs) and all-reduces the counts, so
    every rank ends with the whole stream's exact counts
    (paper_conf_micro_ge0025_b200/parallel.py).
  --split regex (strong scaling): rank r compiles its share of the regex set
    (parallel.shard_patterns) and scans the same input; each step scatters
    its counts into the full per-regex vector and all-reduces it.

Timing: CUDA events on the matching stream around exactly K steps, barrier +
synchronize on both sides, max over ranks.  The input (256 MiB) is larger
than L2 (126 MB), so no L2 flush is needed between steps.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))

HBM_FALLBACK = 6650.0  # GB/s, B200_PROFILING.md fallback


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return HBM_FALLBACK, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.rows = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.FIELDS}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=5)
                if out.returncode == 0 and out.stdout.strip():
                    self.rows.append(out.stdout.strip().split(", "))
            except Exception:
                pass
            self._stop.wait(0.2)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, nm in enumerate(names):
                if len(r) > 5 + i and r[5 + i].strip().lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


# Per-workload compile options of the timed launch configuration (the GPU
# parity tests build the same program: tests/test_gpu_fullsize.py,
# tests/test_gpu_configs.py).  Snort-like: K = 4 words per lane (4096
# positions per warp window) measured 24.4 vs 20.2 GB/s at K = 2; the
# Dotstar-like set is slower at K = 4 (4.1 vs 5.2 GB/s: coarser skipping), so
# the others keep the compiler's default.
# Round 2: max_regs 168 (12-warp pass-1 CTAs, fewer spills) measured 50.8 vs
# 47.0 GB/s at 128 (16 warps), profiles/r2_ab_regs.log.
PROGRAM_OPTS = {"snort": {"words_per_lane": 4, "max_regs": 168}}

WORKLOADS = {
    # name: (pattern builder, input builder(length, rank), default bytes per GPU, description)
    "snort": (lambda: __import__("gen").snort_patterns(1000, 2)[0],
              lambda n, r: __import__("gen").snort_input(n, seed=2 + 1000 * r), 256 << 20,
              "snort-like 1k regexes x 256 MiB payloads"),
    "clamav": (lambda: __import__("gen").clamav_brill_patterns(1000, 3)[0],
               lambda n, r: __import__("gen").text_input(n, seed=3 + 1000 * r), 1 << 30,
               "clamav/brill-like 2k regexes x 1 GiB text"),
    "dotstar": (lambda: __import__("gen").dotstar_protomata_patterns(1000, 4)[0],
                lambda n, r: __import__("gen").dotstar_input(n, seed=4 + 1000 * r), 1 << 30,
                "dotstar/protomata-like 2k regexes x 1 GiB amino/long-line text"),
    "multi": (lambda: __import__("gen").multi_patterns(2500),
              lambda n, r: __import__("gen").multi_input(n, seed=5 + 1000 * r), 8 << 30,
              "10k regexes (2.5k per family) x 8 GiB"),
}


def ncu_traffic(workload: str, kernel: str, nbytes: int):
    """DRAM bytes (read + write) per launch of `kernel` from the committed
    ncu --set full summary (profiles/ncu_traffic.json), scaled to this input
    size, or None."""
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            t = json.load(f)
        e = t[workload][kernel]
        return e["dram_bytes_per_launch"] * nbytes / e["input_bytes"]
    except Exception:
        return None


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


def int_peak():
    """Measured integer-pipe peak of this GPU (scripts/int_peak.cu, committed
    as profiles/r2_int_peak.json): LOP3 / IADD3 / SHF / PRMT all issue at the
    same rate -- the ALU pipe's -- which bounds the bitstream body."""
    try:
        with open(os.path.join(ROOT, "profiles", "r2_int_peak.json")) as f:
            d = json.load(f)
        return float(d["rates"]["lop3"]["tops"]), "profiles/r2_int_peak.json (LOP3 rate, measured on a B200 at 1965 MHz)"
    except Exception:
        return None, None


def int_block(workload, kernel, avg_ms, nbytes):
    """Integer-pipe view of the dominant kernel: executed thread instructions
    per launch (copied from the committed ncu capture named in `inst_source`,
    scaled to this input) over its live duration, against the ALU peak."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            e = json.load(f)[workload][kernel]
        ti = float(e["thread_inst_per_launch"]) * nbytes / float(e["input_bytes"])
    except Exception:
        return None
    peak, src = int_peak()
    ach = ti / (avg_ms * 1e-3) / 1e12
    return {"thread_ops_per_byte": ti / nbytes, "achieved": ach, "peak": peak, "unit": "Tops/s",
            "frac": ach / peak if peak else None, "inst_source": "copied: " + str(e.get("source", "ncu")),
            "peak_source": src}


def roofline(ktimes, nbytes, n_regex, hbm, hbm_src, workload, step_ms, steps):
    """Roofline of the dominant kernel (the one with the largest share of the
    step): achieved = its ALGORITHMIC bytes per launch (the input, read once,
    plus 8 B of counts per regex -- DESIGN.md "Roofline") / its average launch
    duration from CUDA events on the launch stream."""
    busy = {k: v for k, v in ktimes.items() if v[1] > 0}
    if not busy:
        return None
    k, (tot_ms, n) = max(busy.items(), key=lambda kv: kv[1][0])
    avg_ms = tot_ms / n
    alg = nbytes + 8 * n_regex
    ach = alg / (avg_ms * 1e-3) / 1e9
    traffic = ncu_traffic(workload, k, nbytes)
    return {"bound": "hbm", "achieved": ach, "peak": hbm, "unit": "GB/s", "frac": ach / hbm,
            "traffic": traffic, "kernel": k, "kernel_ms": avg_ms, "share_of_step": tot_ms / steps / step_ms,
            "algorithmic_bytes_per_launch": alg, "peak_source": hbm_src,
            "kernels_ms_per_step": {kk: vv[0] / steps for kk, vv in busy.items()},
            "launches_per_step": {kk: vv[1] / steps for kk, vv in busy.items()},
            "traffic_source": "copied: profiles/ncu_traffic.json (ncu --set full dram__bytes_read+write per launch)",
            "int": int_block(workload, k, avg_ms, nbytes),
            "note": "%HBM is the metric's denominator; the kernels are bound by issue / latency of integer "
                    "work (see int and DESIGN.md Roofline), not by DRAM"}


def load_workload(config: str, length=None, rank: int = 0):
    """(patterns, input u8 array, bytes, description) of a named workload."""
    import gen
    if config == "tiny":
        data = np.frombuffer(gen.tiny_input(), dtype=np.uint8)
        return gen.tiny_patterns(), data, data.size, "tiny"
    if config not in WORKLOADS:
        raise SystemExit(f"unknown config {config}")
    pb, ib, n, desc = WORKLOADS[config]
    n = int(length or n)
    return pb(), ib(n, rank), n, desc


# ---------------------------------------------------------------------------
# reference arm: the CPU oracle, as it stands, on a bounded sample
# ---------------------------------------------------------------------------
def oracle_rate(patterns, data: np.ndarray, target_s: float = 15.0, threads=None):
    import oracle
    threads = threads or (os.cpu_count() or 1)
    # calibrate on a small prefix, then size the sample to ~target_s of wall time
    probe = data[: 1 << 16]
    t0 = time.perf_counter()
    oracle.run_set(patterns, probe, threads=threads)
    dt = max(time.perf_counter() - t0, 1e-3)
    n = int(min(data.size, max(1 << 16, probe.size * target_s / dt)))
    sample = data[:n]
    t0 = time.perf_counter()
    oracle.run_set(patterns, sample, threads=threads)
    dt = time.perf_counter() - t0
    return n / dt / 1e9, n, dt, threads


def run_reference(args):
    """The CPU oracle, as it stands, on a bounded prefix of the SAME workload
    the GPU arm times (same generator, seed and length), on this box's host
    cores; rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    pats, data, nbytes, name = load_workload(args.config, (args.length_mib << 20) if args.length_mib else None, 0)
    probe = data[: 1 << 16]
    for _ in range(args.warmup):  # untimed warm-up: page in the oracle and its DFA caches
        oracle_rate(pats, probe, target_s=0.0)
    rates = []
    samples = []
    for _ in range(max(1, args.steps)):
        r, n, dt, thr = oracle_rate(pats, data, target_s=max(2.0, 30.0 / max(1, args.steps)))
        rates.append(r)
        samples.append((n, dt))
    gbs = float(np.mean(rates))
    n, dt = samples[-1]
    line = {"metric": "input GB/s scanned per regex set", "value": gbs, "unit": "GB/s", "impl": "reference",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * n / (gbs * 1e9), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": {"workload": name, "n_regex": len(pats), "input_bytes_per_gpu": int(data.size),
                       "parallelism": "host cores (rank 0 only)"},
            "cpu_baseline": {"value": gbs, "unit": "GB/s", "cores": thr, "cpu": cpu_model(), "kind": "oracle",
                             "sample": f"all {len(pats)} regexes over the first {n} bytes of the bench input "
                                       f"({dt:.1f} s per step, Thompson NFA + lazy DFA cache)"},
            "e2e": {"value": gbs, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------
# our arm
# ---------------------------------------------------------------------------
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="snort")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--length-mib", type=int, default=0, help="input bytes per GPU (default: the config's)")
    ap.add_argument("--no-prefilter", action="store_true", help="ablation: RX_F_NO_PREFILTER")
    ap.add_argument("--words-per-lane", type=int, default=0, help="experiment: minimum K (rx_options.words_per_lane)")
    ap.add_argument("--group-size", type=int, default=0, help="experiment: max regexes per group (rx_options)")
    ap.add_argument("--max-regs", type=int, default=0, help="experiment: registers per thread (rx_options; "
                    "pass-1 CTA = 64K / (32 x max_regs) warps)")
    ap.add_argument("--interval", type=int, default=0, help="experiment: zero-block guard interval (rx_options)")
    ap.add_argument("--batch", type=int, default=0, help="N3: match N independent packet-sized records (0-1460 B, "
                    "cut from the workload's input) with rx_match_batch, one launch sequence per step")
    ap.add_argument("--outputs", default="counts", choices=["counts", "list"],
                    help="counts (default) or counts + the compacted match list (rx_output.d_matches)")
    ap.add_argument("--piece-mib", type=int, default=0, help="rx_match_host piece size for e2e (0: library default)")
    ap.add_argument("--split", default="chunk", choices=["chunk", "regex"], help="multi-GPU partition (N>1)")
    ap.add_argument("--ablate", default="", help="comma list of rx flags to set (ablation ladder, DESIGN.md): "
                    "no_prefilter, modeb, no_lockstep, lockstep_round, no_guards, rebalance")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    import paper_conf_micro_ge0025_b200 as rx

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # one rank per GPU; RX_DIST_BACKEND=gloo (functional check of the N > 1
    # path on a one-GPU box: ranks share the GPU, collectives go through the
    # host, so no kernel waits on another rank's) -- never for a reported number
    local = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        backend = os.environ.get("RX_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    split_regex = world > 1 and args.split == "regex"
    # regex split: every rank scans the same input (rank 0's); chunk split:
    # rank r's own chunk of the stream
    pats, data, nbytes, name = load_workload(args.config, (args.length_mib << 20) if args.length_mib else None,
                                             0 if split_regex else rank)
    nbytes = int(data.size)
    all_pats = pats
    if split_regex:
        from paper_conf_micro_ge0025_b200 import parallel
        mine = parallel.shard_patterns(len(pats), world, rank, costs=[float(len(p)) for p in pats])
        pats = [pats[i] for i in mine]
    t0 = time.perf_counter()
    popts = dict(PROGRAM_OPTS.get(args.config, {}))
    if args.words_per_lane:
        popts["words_per_lane"] = args.words_per_lane
    if args.group_size:
        popts["group_size"] = args.group_size
    if args.interval:
        popts["interval"] = args.interval
    if args.max_regs:
        popts["max_regs"] = args.max_regs
    flags = rx.RX_F_NO_PREFILTER if args.no_prefilter else 0
    for a in filter(None, args.ablate.split(",")):
        flags |= getattr(rx, "RX_F_" + a.upper())
    prog = rx.Program(pats, flags=flags, **popts)
    compile_s = time.perf_counter() - t0

    host = torch.from_numpy(np.ascontiguousarray(data)).pin_memory()
    d_in = host.to(dev, non_blocking=False)
    stream = torch.cuda.current_stream(dev)
    # the compacted match list (one {regex, position} entry per match end) is
    # the scalable form of the match-end bitstreams (dense streams: 31 GiB here)
    list_cap = (64 << 20) if args.outputs == "list" else None
    out = prog.alloc_outputs(nbytes, dev, dense=False, digests=False, match_cap=list_cap)

    def step_device():
        prog.match(d_in, out=out, stream=stream)

    if args.batch:
        # N3: records of 0-1460 B (seeded), back to back from the input start
        rng = np.random.default_rng(1460)
        lens = rng.integers(0, 1461, size=args.batch)
        offs = np.concatenate([[0], np.cumsum(lens)]).astype(np.uint64)
        assert int(offs[-1]) <= nbytes, "input too short for that many records"
        nbytes = int(offs[-1])
        d_batch = d_in[:nbytes]
        bout = prog.match_batch(d_batch, offs, digests=False, stream=stream)
        name = f"{name}; rx_match_batch of {args.batch} records (0-1460 B)"

        def step_device():  # noqa: F811
            prog.match_batch(d_batch, offs, stream=stream, out=bout)

    def step_e2e():
        # the public API end to end: H2D of the step's input from pinned host
        # memory, the step (with its collectives at N > 1), D2H of the counts.
        # At N = 1 through rx_match_host, which overlaps the copy of piece i+1
        # with the matching of piece i (exact: pieces in order, state chained)
        if args.batch:
            d_in[:nbytes].copy_(host[:nbytes], non_blocking=True)
            step_device()
            return bout["counts"].to("cpu", non_blocking=False)
        if world == 1:
            prog.match_host(host, out=out, stream=stream, device=dev, piece_bytes=args.piece_mib << 20)
            return out["counts"].to("cpu", non_blocking=False)
        d_in.copy_(host, non_blocking=True)
        step_device()
        return (full if split_regex else out["counts"]).to("cpu", non_blocking=False)

    if world > 1 and not split_regex:
        from paper_conf_micro_ge0025_b200 import parallel
        ctx = parallel.ChunkMatcher(prog, dev)

        def step_device():  # noqa: F811
            ctx.match_stream_chunk(d_in, rank, world, out, rank * nbytes)
    elif split_regex:
        full = torch.zeros(len(all_pats), dtype=torch.int64, device=dev)
        idx = torch.tensor(mine, dtype=torch.int64, device=dev)

        def step_device():  # noqa: F811
            prog.match(d_in, out=out, stream=stream)
            parallel.combine_shard_counts(dist, full, idx, out["counts"])

    for _ in range(args.warmup):
        step_device()
    torch.cuda.synchronize(dev)

    # inputs smaller than L2 (126 MB): flush L2 before every timed step and
    # time the steps one by one (the flush stays outside the events)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev) if nbytes <= (128 << 20) else None

    def timed(fn, k):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        if flush is not None:
            tot = 0.0
            for _ in range(k):
                flush.fill_(1)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                fn()
                e1.record(stream)
                torch.cuda.synchronize(dev)
                tot += e0.elapsed_time(e1)
            ms = tot / k
            if world > 1:
                t = torch.tensor([ms], device=dev)
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                ms = float(t.item())
            return ms
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(k):
            fn()
        e1.record(stream)
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        ms = e0.elapsed_time(e1) / k
        if world > 1:
            t = torch.tensor([ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms

    # per-kernel CUDA events on the launch stream during the timed region
    # (rx_set_profiling): the dominant kernel's average launch duration
    prog.set_profiling(True)
    prog.kernel_times(reset=True)
    with ClockSampler(local) as clk:
        ms = timed(step_device, args.steps)
    clocks = clk.summary()
    ktimes = prog.kernel_times(reset=True)
    prog.set_profiling(False)
    # e2e through the public API with host buffers (H2D of the step's input,
    # D2H of the counts) -- same metric
    e2e_ms = timed(step_e2e, max(1, min(args.steps, 5)))

    total_bytes = nbytes if split_regex else nbytes * world
    gbs = total_bytes / (ms * 1e-3) / 1e9
    hbm, hbm_src = measured_peaks()
    launches_per_step = prog.kernels_per_match
    line = {
        "metric": "input GB/s scanned per regex set", "value": gbs, "unit": "GB/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "strong" if split_regex else "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": name, "n_regex": len(all_pats), "input_bytes_per_gpu": nbytes,
                   "parallelism": (f"regex-shard x{world}" if split_regex else f"input-chunk x{world}") if world > 1
                   else "1 GPU",
                   "groups": prog.n_groups, "outputs": ("per-regex counts + compacted match list" if args.outputs == "list"
                               else "per-regex counts (dense streams off: 31 GiB at this size)"),
                   "l2": f"input {nbytes >> 20} MiB per GPU" + (" > 126 MB L2: no flush needed" if nbytes > (126 << 20)
                                                                  else " < L2: L2 flushed between steps"),
                   "prefilter": not args.no_prefilter, "ablate": args.ablate or None, "compile_s": round(compile_s, 1),
                   **popts},
        "roofline": roofline(ktimes, nbytes, len(pats), hbm, hbm_src, name, ms, args.steps),
        "clocks": clocks,
        "gpu_launches": sum(v[1] for v in ktimes.values()) or launches_per_step * args.steps,
    }
    if e2e_ms is not None:
        line["e2e"] = {"value": total_bytes / (e2e_ms * 1e-3) / 1e9, "unit": "GB/s", "h2d_bytes_per_step": nbytes,
                       "d2h_bytes_per_step": 8 * len(all_pats) * (args.batch or 1),
                       "api": ("H2D copy + rx_match_batch" if args.batch else
                               "rx_match_host (pinned host input, pipelined 64 MiB pieces)") if world == 1
                       else "H2D copy + rx_match_chunk protocol"}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        r, n, dt, thr = oracle_rate(pats, data, target_s=15.0)
        line["cpu_baseline"] = {"value": r, "unit": "GB/s", "cores": thr, "cpu": cpu_model(), "kind": "oracle",
                                "sample": f"all {len(pats)} regexes over the first {n} bytes ({dt:.1f} s)"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
