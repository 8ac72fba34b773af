#!/usr/bin/env python
"""Benchmark: chunked LZSS compression throughput on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3_runs20_1g] [--scaling strong|weak]
    python bench.py --impl reference ...        # the CPU oracle as the reference arm
    torchrun --nproc-per-node N bench.py --gpus N ...

One step = one pass of the whole hot path over the
rank's input, resident in HBM: culzss_compress at N = 1; at N > 1 each rank
compresses its contiguous chunk range with culzss_compress_chunks_async (the
payload total stays on the device) and the ranks all-gather the int64 totals
over NCCL (the one exchange step), with one host sync per step.  Scaling is
"strong" by default, as BASELINE.json states the configs ("1 GB ... on 1 and
8 B200", "64 GB ... sharded across 2/4/8 B200"): the config's input is split
into N chunk ranges; "weak" gives every rank its own config-sized input.
Timing is device time from CUDA events on the call's stream; L2 is flushed
between steps; the max over ranks is reported.  The default config is the
slower 1 GiB one (c3 runs20); at N = 1 the line also carries the
other configs (c1 latency, c2, c4, the c5 slice) in `configs`.  Rank 0
prints one JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_cluster_ozsoys11_b200 import datagen, sharding  # noqa: E402

METRIC = "LZSS compress GB/s (input) at 1/2/4/8 B200 + ratio, vs CPU oracle"
UNIT = "GB/s"
PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0  # B200_PROFILING.md fallback
CONFIG_TEXT = {
    "c1_english_64k": "64 KiB English-like text (english generator, seed 1)",
    "c2_csource_128m": "128 MiB source-code-like text (csource generator, seed 2; PAPER.md:1@23843 'C files')",
    "c3_runs20_1g": "1 GiB runs of 20 identical bytes (runs20 generator, seed 3; PAPER.md:1@24662)",
    "c4_random_1g": "1 GiB random bytes (splitmix64, seed 4)",
    "c5_tarmix_64g": "64 GiB tarball-like mix (tarmix generator, seed 5) -- per-rank slices; at N=1 the "
                     "8 GiB slice of rank 0 of a dp8 split (64 GiB + its output + buckets exceed one GPU)",
}


def parse_args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["culzss", "reference"], default="culzss")
    ap.add_argument("--config", default="c3_runs20_1g", choices=sorted(datagen.CONFIGS))
    ap.add_argument("--scaling", choices=["strong", "weak"], default="strong",
                    help="strong (default): the config input split over the N ranks; weak: one config-sized "
                         "input per rank")
    ap.add_argument("--no-other-configs", action="store_true",
                    help="N = 1: skip the short runs of the other configs (the `configs` block)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-decompress", action="store_true")
    ap.add_argument("--assemble", action="store_true",
                    help="N > 1: also gather the whole stream on rank 0 (point-to-point sends of every "
                         "rank's table slice and payload; timed separately, not part of the metric)")
    ap.add_argument("--no-versions", action="store_true",
                    help="skip timing params.version = 2 (the paper's V2 all-position search) beside the default")
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


C5_N1_PARTS = 8  # c5 at N = 1: rank 0's slice of a dp8 split (64 GiB + output + buckets exceed one GPU)


def rank_range(cfg: str, rank: int, world: int, scaling: str):
    """(n_global, seed, b0, b1): this rank's byte range of the generator input.
    strong: chunk-aligned ranges [S*floor(rC/N), S*floor((r+1)C/N)) of the
    config input (c5 at N = 1: rank 0 of a dp8 split); weak: each rank its own
    config-sized input (seed offset by rank; c5: an 8 GiB input per rank)."""
    spec = datagen.CONFIGS[cfg]
    n, seed, S = spec["n"], spec["seed"], 4096
    if scaling == "weak":
        if cfg == "c5_tarmix_64g":
            n //= C5_N1_PARTS
        return n, seed + 1000 * rank, 0, n
    parts = C5_N1_PARTS if (cfg == "c5_tarmix_64g" and world == 1) else world
    b0, b1 = sharding.byte_range(rank, parts, n, S)
    return n, seed, b0, b1


def rank_input(cfg: str, rank: int, world: int, scaling: str = "strong") -> np.ndarray:
    """Host copy of this rank's input (the reference arm, the CPU baseline and
    the e2e leg; the device copy is built by datagen.generate_range_device)."""
    n, seed, b0, b1 = rank_range(cfg, rank, world, scaling)
    return datagen.generate_range(datagen.CONFIGS[cfg]["kind"], n, seed, b0, b1)


def load_int_peak(device: int = 0, live: bool = True):
    """Integer-pipe peak for the compare term: the ALU-pipe
    LOP3 rate measured by tools/micro/int_peak.cu -- live on this rank's GPU
    when the binary is built, else the committed B200 measurement (also when
    several ranks share one GPU, or under a profiler)."""
    exe = os.path.join(ROOT, "tools", "micro", "int_peak")
    if live and os.path.exists(exe) and not os.environ.get("CULZSS_BENCH_NO_LIVE_PEAK"):
        try:
            r = subprocess.run([exe, str(device)], capture_output=True, text=True, timeout=60)
            d = json.loads(r.stdout.strip().splitlines()[-1])
            if r.returncode == 0:
                return d, "measured live on this GPU (tools/micro/int_peak.cu, LOP3 / ALU pipe)"
        except Exception:
            pass
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "int_peak.json")))
        return d, "measured on a B200 of this pool (profiles/int_peak.json from tools/micro/int_peak.cu)"
    except Exception:
        return ({"lop3_tops": 148 * 64 * 1.965e9 / 1e12},
                "guide-derived fallback: 148 SM x 64 ALU lanes/clk x 1965 MHz (DESIGN.md §6)")


def load_peaks():
    try:
        p = json.load(open(PEAKS_PATH))
        return float(p["hbm_gbs"]), float(p.get("sm_max_mhz", 1965.0)), "measured"
    except Exception:
        return FALLBACK_HBM, 1965.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.proc = None
        self.gpu = gpu_index

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "50", "-i", str(self.gpu)], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL,
                text=True)
            time.sleep(0.3)  # nvidia-smi start-up: the first samples bracket the timed region
        except Exception:
            self.proc = None

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            out, _ = self.proc.communicate(timeout=5)
        except Exception:
            self.proc.kill()
            out = ""
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                smax.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[3:7]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def cpu_baseline(x: np.ndarray, stream_bytes: bytes | None, budget_s: float = 10.0):
    """The C oracle, as it stands, on the host cores over a bounded sample:
    contiguous chunk ranges in threads (ctypes releases the GIL), the paper's
    Pthread decomposition (PAPER.md:1@11659).  The sample is the config
    input's leading chunks, sized from a 1-chunk-per-thread probe to about
    budget_s of wall time."""
    import concurrent.futures as cf
    import oracle
    S = 4096
    cores = max(1, min(len(os.sched_getaffinity(0)), 64))
    C = (x.size + S - 1) // S
    t0 = time.perf_counter()
    oracle.compress_range(x, 0, min(C, 16))
    per_chunk = (time.perf_counter() - t0) / min(C, 16)
    nchunks = int(min(C, max(cores, budget_s * cores / max(per_chunk, 1e-6))))
    nchunks = max(1, nchunks)
    bounds = [(i * nchunks // cores, (i + 1) * nchunks // cores) for i in range(cores)]
    bounds = [b for b in bounds if b[1] > b[0]]
    t0 = time.perf_counter()
    with cf.ThreadPoolExecutor(len(bounds)) as ex:
        res = list(ex.map(lambda b: oracle.compress_range(x, b[0], b[1]), bounds))
    dt = time.perf_counter() - t0
    nbytes = min(x.size, nchunks * S)
    parity = None
    if stream_bytes is not None:
        sizes = np.concatenate([r[1] for r in res]).astype(np.int64)
        payload = b"".join(r[0] for r in res)
        Ctot = (x.size + S - 1) // S
        gpu_sizes = np.frombuffer(stream_bytes, dtype="<u4", count=nchunks, offset=32).astype(np.int64)
        start = 32 + 4 * Ctot
        parity = bool(np.array_equal(sizes, gpu_sizes)
                      and stream_bytes[start:start + len(payload)] == payload)
    # single-core figure beside the all-core one: one thread
    # over a ~1 s sample of the same leading chunks
    n1 = int(max(1, min(nchunks, 1.0 / max(per_chunk, 1e-6))))
    t0 = time.perf_counter()
    oracle.compress_range(x, 0, n1)
    dt1 = time.perf_counter() - t0
    cpu_model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                cpu_model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"value": nbytes / dt / 1e9, "unit": UNIT, "cores": len(bounds), "kind": "oracle",
            "sample": f"first {nchunks} chunks ({nbytes} B) of the same input, {len(bounds)} threads "
                      f"over contiguous chunk ranges, {dt:.2f} s wall",
            "single_core": {"value": min(x.size, n1 * S) / dt1 / 1e9, "unit": UNIT,
                            "sample": f"first {n1} chunks, 1 thread, {dt1:.2f} s"},
            "cpu_model": cpu_model,
            "parity_with_gpu_stream": parity}


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle (the only reference there is: the
    paper ships no code) on the host cores, same metric/config/unit."""
    if rank != 0:
        return
    import concurrent.futures as cf
    import oracle
    n_glob, seed, b0, b1 = rank_range(args.config, 0, 1, args.scaling)
    # the sample is the input's leading chunks: only a bounded prefix is made
    x = datagen.generate_range(datagen.CONFIGS[args.config]["kind"], n_glob, seed, b0, min(b1, b0 + (256 << 20)))
    S = 4096
    cores = max(1, min(len(os.sched_getaffinity(0)), 64))
    C = (x.size + S - 1) // S
    t0 = time.perf_counter()
    oracle.compress_range(x, 0, min(C, 8))
    per_chunk = (time.perf_counter() - t0) / min(C, 8)
    # each step ~ (10 s / (steps + warmup)) of wall so the run stays within minutes
    step_budget = max(0.5, 12.0 / (args.steps + args.warmup))
    nchunks = int(min(C, max(cores, step_budget * cores / max(per_chunk, 1e-6))))
    bounds = [(i * nchunks // cores, (i + 1) * nchunks // cores) for i in range(cores)]
    bounds = [b for b in bounds if b[1] > b[0]]
    times = []
    out_bytes = 0
    with cf.ThreadPoolExecutor(len(bounds)) as ex:
        for it in range(args.warmup + args.steps):
            t0 = time.perf_counter()
            res = list(ex.map(lambda b: oracle.compress_range(x, b[0], b[1]), bounds))
            dt = time.perf_counter() - t0
            if it >= args.warmup:
                times.append(dt)
            out_bytes = sum(len(r[0]) for r in res) + 4 * nchunks + 32
    nbytes = min(x.size, nchunks * S)
    ms = 1000 * statistics.mean(times)
    value = nbytes / (ms / 1000) / 1e9
    sample = (f"first {nchunks} chunks ({nbytes} B) of {args.config} per step, {len(bounds)} threads "
              f"over contiguous chunk ranges")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": f"{args.config}: {CONFIG_TEXT[args.config]}", "bytes": int(b1 - b0),
                   "sample_bytes_per_step": int(nbytes), "chunk": 4096, "window": 128,
                   "max_match": 128, "min_match": 3},
        "ratio": out_bytes / nbytes,
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": len(bounds), "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)


CONFIG_ORDER = ("c1_english_64k", "c2_csource_128m", "c3_runs20_1g", "c4_random_1g", "c5_tarmix_64g")


def chunk_pairs(n: int, S: int = 4096, W: int = 128) -> int:
    """North-star compare count: every (p, d) with 1 <= d <= min(W, p) in each
    chunk is one byte-pair test (516,032 per full 4 KiB chunk)."""
    full, tail = divmod(n, S)
    return full * (S * W - W * (W + 1) // 2) + sum(min(W, p) for p in range(tail))


def roofline(n: int, C: int, pay_bytes: int, ck_ms: float, int_peak_tops: float, hbm_peak: float):
    """The slower of (a) HBM bytes at the measured copy bandwidth and (b) the
    window-compare count at the measured ALU-pipe integer peak (BASELINE.json
    north star): 4 byte-pair tests per packed 32-bit op."""
    pairs = chunk_pairs(n)
    alg_ops = pairs / 4.0
    alg_bytes = n + pay_bytes + 4 * C
    t_cmp = alg_ops / (int_peak_tops * 1e12) * 1000
    t_hbm = alg_bytes / (hbm_peak * 1e9) * 1000
    return {"bound": "alu" if t_cmp >= t_hbm else "hbm",
            "achieved": alg_ops / (ck_ms / 1000) / 1e12, "peak": int_peak_tops, "unit": "Tops/s",
            "frac": max(t_cmp, t_hbm) / ck_ms,
            "algorithmic": {"byte_pair_tests": pairs, "int32_ops": alg_ops, "hbm_bytes": alg_bytes},
            "t_cmp_ms": t_cmp, "t_hbm_ms": t_hbm, "t_kernel_ms": ck_ms,
            "hbm": {"achieved": alg_bytes / (ck_ms / 1000) / 1e9, "peak": hbm_peak, "unit": "GB/s",
                    "frac": alg_bytes / (ck_ms / 1000) / 1e9 / hbm_peak}}


def measure_config(cfg, dev, culzss, flush, steps, int_peak_tops, hbm_peak):
    """A short N = 1 run of another config (the `configs` block): its input
    built on the device, `steps` timed compress calls (L2 flushed), the chunk
    kernel's share from profiled calls, its roofline fraction; c1 (64 KiB) is
    a latency point (report microseconds per call)."""
    import torch
    n_glob, seed, b0, b1 = rank_range(cfg, 0, 1, "strong")
    kind = datagen.CONFIGS[cfg]["kind"]
    x = datagen.generate_range_device(kind, n_glob, seed, b0, b1, dev)
    n = b1 - b0
    S = 4096
    C = (n + S - 1) // S
    out = torch.empty(culzss.max_compressed_size(n), dtype=torch.uint8, device=dev)
    culzss.set_profiling(True, call_only=True)
    if cfg == "c1_english_64k":
        for _ in range(20):
            culzss.compress_into(x, out)
        dev_us, wall_us = [], []
        for _ in range(200):
            t0 = time.perf_counter()
            on = culzss.compress_into(x, out)
            wall_us.append((time.perf_counter() - t0) * 1e6)
            dev_us.append(culzss.last_kernel_ms("call") * 1000)
        r = {"us_per_call_device": statistics.median(dev_us), "us_per_call_wall": statistics.median(wall_us),
             "calls": len(dev_us), "value": n / (statistics.median(dev_us) / 1e6) / 1e9, "unit": UNIT,
             "ratio": on / n, "what": "latency: one culzss_compress call on 64 KiB (16 chunks), median of 200; "
                                      "device = CUDA events around the call, wall = host time incl. its sync"}
    else:
        ms = []
        on = 0
        for it in range(2 + steps):
            flush.fill_(1)
            torch.cuda.synchronize()
            on = culzss.compress_into(x, out)
            if it >= 2:
                ms.append(culzss.last_kernel_ms("call"))
        culzss.set_profiling(True)
        ck = []
        for _ in range(3):
            flush.fill_(1)
            torch.cuda.synchronize()
            culzss.compress_into(x, out)
            ck.append(culzss.last_kernel_ms("chunk"))
        rf = roofline(n, C, on - 32 - 4 * C, statistics.mean(ck), int_peak_tops, hbm_peak)
        r = {"value": n / (statistics.mean(ms) / 1000) / 1e9, "unit": UNIT, "ms_per_step": statistics.mean(ms),
             "steps": steps, "bytes": n, "ratio": on / n, "chunk_kernel_ms": statistics.mean(ck),
             "roofline_frac": rf["frac"], "roofline_bound": rf["bound"]}
    r["workload"] = f"{cfg}: {CONFIG_TEXT[cfg]}"
    culzss.set_profiling(True, call_only=True)
    del x, out
    torch.cuda.empty_cache()
    return r


def main():
    args = parse_args()
    rank, world, local = dist_env()
    if world != args.gpus and world > 1:
        print(f"warning: WORLD_SIZE={world} but --gpus {args.gpus}", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_cluster_ozsoys11_b200 import culzss

    # one process per GPU; BENCH_DIST_BACKEND=gloo lets several ranks share
    # one GPU to exercise the N > 1 code path where only one GPU is visible
    backend = os.environ.get("BENCH_DIST_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cdev = dev if backend == "nccl" else None  # device of the collectives' tensors
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    kind = datagen.CONFIGS[args.config]["kind"]
    n_glob, seed, b0, b1 = rank_range(args.config, rank, world, args.scaling)
    n = b1 - b0
    # the rank's input, built on the device (tiled corpora from an uploaded base)
    x = datagen.generate_range_device(kind, n_glob, seed, b0, b1, dev)
    S = 4096
    C = (n + S - 1) // S
    out = torch.empty(culzss.max_compressed_size(n), dtype=torch.uint8, device=dev)
    payload = out[32 + 4 * C:]
    sizes = torch.empty(max(C, 1), dtype=torch.int32, device=dev)
    dev_tot = torch.zeros(1, dtype=torch.int64, device=dev)
    tots = torch.zeros(max(world, 1), dtype=torch.int64, device=cdev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2
    stream = torch.cuda.current_stream()
    # timed steps: events at the call's start and end only (nothing between its
    # kernels, so programmatic dependent launch overlaps them as in production);
    # the per-kernel split comes from separate profiled calls after the timed region
    culzss.set_profiling(True, call_only=True)
    last_totals = [None]
    exch_ms = []  # N > 1: time of the all-gather of totals per step

    def step():
        if world == 1:
            return culzss.compress_into(x, out), culzss.last_kernel_ms("call")
        # the rank's chunk range -> payload + sizes, its total left on the
        # device; the one exchange (all-gather of int64 totals) fixes every
        # rank's global offsets; one host sync per step
        ev0, ev1, ev2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        ev0.record(stream)
        culzss.compress_chunks_async(x, payload, sizes, dev_tot)
        ev1.record(stream)
        if backend == "nccl":
            dist.all_gather_into_tensor(tots, dev_tot)
            ev2.record(stream)
            ev2.synchronize()
            ex = ev1.elapsed_time(ev2)
            ms = ev0.elapsed_time(ev2)
            got = tots.tolist()
        else:  # gloo (CPU tensors; the test path): the exchange is timed on the host
            ev1.synchronize()
            t0 = time.perf_counter()
            dist.all_gather_into_tensor(tots, dev_tot.cpu())
            ex = (time.perf_counter() - t0) * 1000
            ms = ev0.elapsed_time(ev1) + ex
            got = tots.tolist()
        exch_ms.append(ex)
        last_totals[0] = [int(v) for v in got]
        return last_totals[0][rank], ms

    for _ in range(args.warmup):
        flush.fill_(1)
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = ClockSampler(local)
    clocks.start()
    launches0 = culzss.launch_count()
    step_ms, chunk_ms, scan_ms, compact_ms = [], [], [], []
    out_n = 0
    for _ in range(args.steps):
        flush.fill_(1)
        torch.cuda.synchronize()
        r, ms = step()
        out_n = r
        step_ms.append(ms)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = culzss.launch_count() - launches0
    clk = clocks.stop()
    # per-kernel device times (roofline of the chunk kernel): the same call with
    # events between its kernels, outside the timed region
    culzss.set_profiling(True)
    for _ in range(max(3, min(args.steps, 10))):
        flush.fill_(1)
        torch.cuda.synchronize()
        if world == 1:
            culzss.compress_into(x, out)
        else:
            culzss.compress_chunks(x, payload, sizes)
        chunk_ms.append(culzss.last_kernel_ms("chunk"))
        scan_ms.append(culzss.last_kernel_ms("scan"))
        compact_ms.append(culzss.last_kernel_ms("compact"))
    culzss.set_profiling(True, call_only=True)
    total_ms = sum(step_ms)
    n_total = n
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=cdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
        nt = torch.tensor([n], dtype=torch.int64, device=cdev)
        dist.all_reduce(nt, op=dist.ReduceOp.SUM)
        n_total = int(nt.item())
        dist.barrier()
    ms_per_step = total_ms / args.steps
    # whole-job throughput: the bytes all ranks compressed over the slowest rank's time
    value = n_total / (ms_per_step / 1000) / 1e9
    placed = sharding.placements(last_totals[0], n_total, S)[rank] if world > 1 else None
    stream_len = out_n if world == 1 else placed.stream_bytes
    ratio = stream_len / n_total

    # Roofline of the dominant kernel (the fused chunk kernel, rows a1-a4) as
    # BASELINE.json's north star defines it.  The kernel
    # searches only where the greedy parse lands, through hash chains with
    # exact prunes, so it can beat the compare term; HBM is the hard floor.
    hbm_peak, sm_max_mhz, peak_kind = load_peaks()
    ip, ip_src = load_int_peak(local, live=backend == "nccl" or world == 1)
    int_peak_tops = float(ip["lop3_tops"])
    pay_bytes = (out_n - 32 - 4 * C) if world == 1 else placed.payload_bytes
    ck = statistics.mean(chunk_ms)
    rf = roofline(n, C, pay_bytes, ck, int_peak_tops, hbm_peak)
    rf["traffic"] = None
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        per = tr.get("per_launch_bytes", tr)
        if isinstance(per.get(args.config), (int, float)):
            rf["traffic"] = per[args.config]
            rf["traffic_source"] = tr.get("source", tr.get("_comment"))
    except Exception:
        pass
    rf["kernel"] = "chunk_kernel (fused a1-a4)"
    rf["peak_source"] = ip_src
    rf["peak_other"] = {k: ip.get(k) for k in ("iadd3_tops", "imad_tops", "lop3_imad_mixed_tops") if k in ip}
    rf["hbm"]["peak_kind"] = peak_kind
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step,
        "ms_step_median": statistics.median(step_ms), "ms_step_min": min(step_ms),  # this rank's
        "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": f"{args.config}: {CONFIG_TEXT[args.config]}", "bytes_total": n_total,
                   "bytes_per_rank": n, "chunk": 4096, "window": 128, "max_match": 128, "min_match": 3,
                   "l2": "flushed (256 MiB write) between steps", "parallelism": f"dp{world} (chunk ranges)",
                   "input": "built on the device (datagen.generate_range_device)",
                   "exchange": f"{backend} all_gather of per-rank compressed totals (device-resident)"
                   if world > 1 else "none"},
        "ratio": ratio,
        "kernels_ms": {"chunk": ck, "scan": statistics.mean(scan_ms), "compact": statistics.mean(compact_ms)},
        "roofline": rf,
        "clocks": clk,
        "gpu_launches": launches,
    }
    if world > 1 and args.assemble:
        # optional assembly on rank 0, verified by a
        # device round trip against every rank's input
        tpay = culzss.compress_chunks(x, payload, sizes)
        pay_t, sz_t = payload[:tpay], sizes[:C]
        if backend != "nccl":
            pay_t, sz_t = pay_t.cpu(), sz_t.cpu()
        torch.cuda.synchronize()
        dist.barrier()
        t0 = time.perf_counter()
        full = sharding.assemble_on_root_tensors(pay_t, sz_t, last_totals[0], n_total, (S, 128, 128, 3))
        torch.cuda.synchronize()
        dist.barrier()
        wall = (time.perf_counter() - t0) * 1000
        if rank == 0:
            full = full.to(dev)
            y = culzss.decompress(full)
            ok, pos = True, 0
            for r in range(world):
                ng, sd, rb0, rb1 = rank_range(args.config, r, world, args.scaling)
                xr = datagen.generate_range_device(kind, ng, sd, rb0, rb1, dev)
                ok = ok and bool(torch.equal(y[pos:pos + rb1 - rb0], xr))
                pos += rb1 - rb0
                del xr
            line["assembly"] = {"wall_ms": wall, "stream_bytes": int(full.numel()),
                                "gbps_into_rank0": full.numel() / (wall / 1000) / 1e9,
                                "op": f"{backend} point-to-point sends of table slices and payloads to rank 0",
                                "roundtrip_exact": bool(ok)}
            del y
        del full
    if world > 1:
        # the one exchange step: its share of a step
        ex = statistics.mean(exch_ms[args.warmup:args.warmup + args.steps]) if exch_ms else None
        line["exchange"] = {"op": f"{backend} all_gather_into_tensor of int64 per-rank totals "
                                  f"({'device-resident, CUDA events' if backend == 'nccl' else 'host-timed'})",
                            "ms_per_step": ex, "share_of_step": ex / ms_per_step if ex else None}
    # params.version = 2 (the paper's V2 search design: every position, every
    # window offset) on the same input, same protocol, fewer
    # steps: the measured cost of the brute-force design the default replaces
    if world == 1 and not args.no_versions:
        p2 = culzss.Params.make(version=2)
        out2 = torch.empty_like(out)
        v2_ms, v2_ck = [], []
        n2 = 0
        for it in range(1 + max(1, min(3, args.steps))):
            flush.fill_(1)
            torch.cuda.synchronize()
            culzss.set_profiling(True)
            n2 = culzss.compress_into(x, out2, p2)
            if it >= 1:
                v2_ms.append(culzss.last_kernel_ms("call"))
                v2_ck.append(culzss.last_kernel_ms("chunk"))
        culzss.set_profiling(True, call_only=True)
        ck2 = statistics.mean(v2_ck)
        alg_ops = rf["algorithmic"]["int32_ops"]
        line["versions"] = {
            "0": {"what": "lazy greedy search over 3-gram hash chains with exact run-skip / chain-switch prunes "
                          "(default)", "value": value, "chunk_ms": ck, "roofline_frac": rf["frac"]},
            "2": {"what": "paper V2 design: warp-cooperative longest match at every position over all "
                          "window offsets, __reduce_max_sync argmax",
                  "value": n / (statistics.mean(v2_ms) / 1000) / 1e9, "unit": UNIT, "chunk_ms": ck2,
                  "compares_tops": alg_ops / (ck2 / 1000) / 1e12,
                  "roofline_frac": max(rf["t_cmp_ms"], rf["t_hbm_ms"]) / ck2,
                  "steps": len(v2_ms),
                  "stream_identical": bool(n2 == out_n and torch.equal(out2[:n2], out[:out_n]))},
        }
        del out2

    # a6: decompression of this rank's stream (N=1: the full stream), device
    # time of the decode kernels and of the whole culzss_decompress call
    if world == 1 and not args.no_decompress:
        culzss.compress_into(x, out)
        dec = torch.empty(n, dtype=torch.uint8, device=dev)
        sview = out[:out_n]
        dms, cms = [], []
        culzss.set_profiling(True)
        for it in range(args.warmup + args.steps):
            flush.fill_(1)
            torch.cuda.synchronize()
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            culzss.decompress(sview, dec)
            ev1.record(stream)
            ev1.synchronize()
            if it >= args.warmup:
                dms.append(culzss.last_kernel_ms("decode"))
                cms.append(ev0.elapsed_time(ev1))
        culzss.set_profiling(True, call_only=True)
        ok = bool(torch.equal(dec, x))
        # decoder roofline: HBM-bound at (r + 1) bytes per output
        # byte -- the stream read once, the output written once -- over the
        # device time of the decode kernels
        dk = statistics.mean(dms)
        dec_bytes = out_n + n
        line["decompress"] = {"value": n / (statistics.mean(cms) / 1000) / 1e9, "unit": "GB/s (output)",
                              "decode_kernel_ms": dk, "call_ms": statistics.mean(cms),
                              "roundtrip_exact": ok,
                              "roofline": {"bound": "hbm", "kernels": "decoder kernels (classify + literal + walk + decode)",
                                           "algorithmic_bytes": dec_bytes,
                                           "achieved": dec_bytes / (dk / 1000) / 1e9, "peak": hbm_peak,
                                           "unit": "GB/s", "frac": dec_bytes / (dk / 1000) / 1e9 / hbm_peak,
                                           "peak_kind": peak_kind}}
        del dec

    # NEXT-1 sharded decompression at N > 1: every rank decodes its own chunk
    # range from its compress_chunks payload + sizes (no exchange needed);
    # aggregate output GB/s over the max-over-ranks device time
    if world > 1 and not args.no_decompress:
        dec = torch.empty(n, dtype=torch.uint8, device=dev)
        tpay = culzss.compress_chunks(x, payload, sizes)
        dms = []
        for it in range(args.warmup + args.steps):
            flush.fill_(1)
            torch.cuda.synchronize()
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            culzss.decompress_chunks(payload[:tpay], sizes[:C], n, dec)
            ev1.record(stream)
            ev1.synchronize()
            if it >= args.warmup:
                dms.append(ev0.elapsed_time(ev1))
        ok = torch.tensor([1.0 if torch.equal(dec, x) else 0.0], dtype=torch.float64, device=cdev)
        tt = torch.tensor([statistics.mean(dms)], dtype=torch.float64, device=cdev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        line["decompress"] = {"value": n_total / (float(tt.item()) / 1000) / 1e9, "unit": "GB/s (output)",
                              "call_ms_max_over_ranks": float(tt.item()),
                              "api": "culzss_decompress_chunks (each rank its own chunk range)",
                              "roundtrip_exact": bool(ok.item() == 1.0)}
        del dec

    # host copy of (a bounded prefix of) the rank's input: the e2e leg and the
    # CPU baseline; c5's 8-32 GiB slices are sampled by their first 1 GiB
    e2e_n = min(n, 1 << 30)
    x_np = x[:e2e_n].cpu().numpy() if (not args.no_e2e or not args.no_cpu_baseline) else None
    if not args.no_e2e:
        hin = torch.from_numpy(x_np).pin_memory()
        hout = torch.empty(culzss.max_compressed_size(e2e_n), dtype=torch.uint8).pin_memory()
        times = []
        on = 0
        for it in range(args.warmup + max(3, args.steps // 2)):
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            ev0.record(stream)
            on = culzss.compress_host_ptr(hin.data_ptr(), e2e_n, hout.data_ptr(), hout.numel())
            ev1.record(stream)
            ev1.synchronize()
            if it >= args.warmup:
                times.append(ev0.elapsed_time(ev1))
        e2e_ms = statistics.mean(times)
        e2e_tot = e2e_n
        if world > 1:
            t = torch.tensor([e2e_ms], dtype=torch.float64, device=cdev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_ms = float(t.item())
            nt = torch.tensor([e2e_n], dtype=torch.int64, device=cdev)
            dist.all_reduce(nt, op=dist.ReduceOp.SUM)
            e2e_tot = int(nt.item())
        line["e2e"] = {"value": e2e_tot / (e2e_ms / 1000) / 1e9, "unit": UNIT,
                       "h2d_bytes_per_step": e2e_n, "d2h_bytes_per_step": int(on),
                       "api": "culzss_compress_host (pinned host in/out)",
                       "sample": "the whole rank input" if e2e_n == n else f"first {e2e_n} B of the rank input"}
        if world == 1 and "decompress" in line:
            # host-to-host decompression of the same stream (culzss_decompress_host)
            hdec = torch.empty(e2e_n, dtype=torch.uint8).pin_memory()
            dtimes = []
            for it in range(args.warmup + max(3, args.steps // 2)):
                ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize()
                ev0.record(stream)
                culzss.decompress_host_ptr(hout.data_ptr(), int(on), hdec.data_ptr(), e2e_n)
                ev1.record(stream)
                ev1.synchronize()
                if it >= args.warmup:
                    dtimes.append(ev0.elapsed_time(ev1))
            line["decompress"]["e2e"] = {"value": e2e_n / (statistics.mean(dtimes) / 1000) / 1e9,
                                         "unit": "GB/s (output)", "h2d_bytes_per_step": int(on),
                                         "d2h_bytes_per_step": e2e_n,
                                         "roundtrip_exact": bool(torch.equal(hdec, hin)),
                                         "api": "culzss_decompress_host (pinned host in/out)"}
            del hdec
        del hin, hout
    if rank == 0 and world == 1 and not args.no_cpu_baseline:  # the CPU baseline at N = 1 only
        sb = out[:out_n].cpu().numpy().tobytes()
        line["cpu_baseline"] = cpu_baseline(x_np, sb if e2e_n == n else None)
    # the other BASELINE configs, short runs at N = 1 (the headline
    # is the slower 1 GiB config; the others ride along here)
    if world == 1 and not args.no_other_configs:
        del out, payload, sizes
        torch.cuda.empty_cache()
        line["configs"] = {}
        for cfg in CONFIG_ORDER:
            if cfg != args.config:
                line["configs"][cfg] = measure_config(cfg, dev, culzss, flush, 5, int_peak_tops, hbm_peak)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    if rank == 0:
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
