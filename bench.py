#!/usr/bin/env python
"""bench.py -- MTTKRP GFLOP/s and HBM GB/s against the measured B200 roofline.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config h|c1|c2|c3|c4|c5]
                    [--scaling weak|strong] [--impl reference]

One STEP = COO MTTKRP of every mode (output zero-fill + kernel, the paper times all modes and
averages) over the synthetic tensor resident in HBM.  Rank 0 prints one JSON line.
GFLOP/s uses the nominal N*M*R flops per mode (Table I generalised; R#7).

The default workload is the north_star target: a 100M-nonzero 3rd-order power-law tensor,
regL-shaped (2^23)^3 (Table II s3), R = 16.  `--gpus N` without a torchrun
environment re-launches itself under torch.distributed.run with N ranks (127.0.0.1).  At N
ranks every rank owns the nnz-balanced row shard of every mode and the timed step has no
collective (the all-gather of the owned output rows -- needed only when the next CP-ALS step
consumes the factor -- is timed separately, `allgather`).  Scaling: weak (default; N x the
config's nonzeros) or strong (default for c5, BASELINE config 5: the config's 1B nonzeros
split over the ranks; rank 0 also times the full tensor on its GPU before sharding, T_1).

roofline.frac = SURVEY 8(d)'s compulsory bytes of the dominant kernel per launch (stream +
each distinct gathered factor row once + the output) / its mean launch time / the measured
HBM peak; the paper's upper-bound model (every gather a DRAM access, Table I) is model_frac.
roofline.traffic = DRAM bytes per launch counted by ncu on launches of this same workload in
a child process of this run (not timed).  cpu_baseline = the fp64 oracle (oracle/), as it
stands, on the full workload shape, pinned to one host core (taskset -c 0).

--impl reference times that oracle, pinned to one core, on the same config: each step is one
mode's MTTKRP over a block of the workload's nonzeros; under torchrun only rank 0 works.
"""
from __future__ import annotations

import argparse
import json
import os
import shutil
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth_inputs as si  # noqa: E402

METRIC = "MTTKRP GFLOP/s and HBM GB/s vs ~8 TB/s roofline at 1/2/4/8 B200"
FALLBACK_HBM_GBS = 6650.0


def model_flops(order, nnz, R):
    """N*M*R per mode (N-1 multiplies + 1 add per r per nonzero; Table I's 3MR at N = 3)."""
    return order * nnz * R


def model_bytes_coo(order, nnz, R):
    """Table I COO upper bound generalised (R#8): 4(N+1)M stream + 4NRM factor/output rows."""
    return 4 * (order + 1) * nnz + 4 * order * R * nnz


def model_bytes_hicoo(order, nnz, nblocks, R, B=128):
    """Table I HiCOO bound generalised (R#8): (N+4)M + (8+4N)n_b + 4NR min(n_b B, M)."""
    return (order + 4) * nnz + (8 + 4 * order) * nblocks + 4 * order * R * min(nblocks * B, nnz)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks and throttle reasons sampled DURING the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.path = None

    def start(self):
        fd, self.path = tempfile.mkstemp(prefix="clocks_", suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None
        time.sleep(0.3)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.15)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        rows = []
        with open(self.path) as f:
            for line in f:
                parts = [p.strip() for p in line.split(",")]
                if len(parts) >= 8:
                    rows.append(parts)
        os.unlink(self.path)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        smax = max(float(r[1]) for r in rows if r[1].replace(".", "").isdigit())
        loaded = [s for s in sm if s > 0.5 * smax] or sm
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[4 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": smax, "reasons": reasons,
                "samples": len(rows), "power_w_max": max(float(r[2]) for r in rows
                                                           if r[2].replace(".", "").isdigit())}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def host_workload(cfg, nnz):
    """The config's shape and law drawn on the host by synth_inputs (never by the CUDA path):
    product-form Kronecker bits with P(1) = 1/4, values U[-1, 1); no dedup pass (repeats are
    ~1e-8 of the draws at these sizes and are separate nonzeros, R#15)."""
    dims = cfg["dims"]
    if cfg["kind"] == "uniform":
        return si.uniform_coo(dims, nnz, seed=cfg["seed"])
    if all(d & (d - 1) == 0 for d in dims):
        return si.powerlaw_coo_lean(dims, nnz, seed=cfg["seed"])
    return si.powerlaw_coo(dims, nnz, seed=cfg["seed"], dedup=False, shuffle=False)


def host_cpu_info():
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count()}


def pin_to_core0():
    """Pin this process to host core 0 (the oracle is single-threaded by mandate)."""
    try:
        os.sched_setaffinity(0, {0})
    except Exception:
        pass
    return len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else 1


def cpu_oracle_child(args):
    """Child process (started under `taskset -c 0`): the fp64 oracle on the workload shape,
    timed with a steady clock per mode; prints one JSON line."""
    import oracle
    cores = pin_to_core0()
    cfg = si.CONFIGS[args.config]
    dims, R = cfg["dims"], cfg["R"]
    nnz = min(args.cpu_sample or cfg["nnz"], cfg["nnz"])
    inds, vals = host_workload(cfg, nnz)
    U = si.factors(dims, R, seed=cfg["seed"])
    modes = range(len(dims)) if args.cpu_modes == "all" else [int(m) for m in args.cpu_modes.split(",")]
    oracle.build()
    secs = []
    for n in modes:
        t0 = time.perf_counter()
        oracle.mttkrp(dims, inds, vals, n, U)
        secs.append(time.perf_counter() - t0)
    flops = sum(model_flops(len(dims), nnz, R) for _ in modes)
    print(json.dumps({"gflops": flops / sum(secs) / 1e9, "seconds_per_mode": [round(t, 3) for t in secs],
                      "modes": list(modes), "nnz": nnz, "cores": cores}), flush=True)


def cpu_omp_child(args):
    """Child process: the paper's CPU method (baselines/: COO-MTTKRP-OMP, fp32 + omp atomic,
    all host threads) on the same host-drawn workload; prints one JSON line."""
    import baselines
    cfg = si.CONFIGS[args.config]
    dims, R = cfg["dims"], cfg["R"]
    nnz = min(args.cpu_sample or cfg["nnz"], cfg["nnz"])
    inds, vals = host_workload(cfg, nnz)
    U = si.factors(dims, R, seed=cfg["seed"])
    baselines.build()
    modes = range(len(dims)) if args.cpu_modes == "all" else [int(m) for m in args.cpu_modes.split(",")]
    baselines.mttkrp(dims, inds[:, :1000], vals[:1000], 0, U)  # thread-pool warm-up
    secs = []
    for n in modes:
        t0 = time.perf_counter()
        baselines.mttkrp(dims, inds, vals, n, U)
        secs.append(time.perf_counter() - t0)
    flops = sum(model_flops(len(dims), nnz, R) for _ in modes)
    print(json.dumps({"gflops": flops / sum(secs) / 1e9, "seconds_per_mode": [round(t, 3) for t in secs],
                      "modes": list(modes), "nnz": nnz, "threads": baselines.threads()}), flush=True)


def cpu_omp(args, cfg):
    cmd = [sys.executable, os.path.abspath(__file__), "--cpu-omp-child", "--config", args.config,
           "--cpu-modes", args.cpu_modes, "--cpu-sample", str(args.cpu_sample or 0)]
    try:
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=900)
        d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    except Exception as e:
        return {"unavailable": f"omp child failed: {str(e)[:160]}"}
    return {"value": round(d["gflops"], 3), "unit": "GFLOP/s", "cores": d["threads"],
            "kind": "paper CPU method (COO-MTTKRP-OMP, fp32, omp atomic; P:157, P:282), not the oracle",
            "sample": f"the same {d['nnz']} host-drawn nonzeros as cpu_baseline, modes {d['modes']}",
            "seconds_per_mode": d["seconds_per_mode"]}


def cpu_baseline(args, cfg):
    """Run cpu_oracle_child pinned to core 0 (taskset when present) and report it."""
    cmd = [sys.executable, os.path.abspath(__file__), "--cpu-oracle-child", "--config", args.config,
           "--cpu-modes", args.cpu_modes, "--cpu-sample", str(args.cpu_sample or 0)]
    if shutil.which("taskset"):
        cmd = ["taskset", "-c", "0"] + cmd
    try:
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=1800)
        d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    except Exception as e:
        return {"unavailable": f"oracle child failed: {str(e)[:160]}"}
    info = host_cpu_info()
    full = d["nnz"] == cfg["nnz"]
    return {"value": round(d["gflops"], 4), "unit": "GFLOP/s", "cores": d["cores"], "kind": "oracle",
            "sample": (f"{'the full' if full else 'the first ' + str(d['nnz'])} {cfg['name']} "
                       f"nonzeros ({d['nnz']}, host-drawn by synth_inputs: same shape and law, R = "
                       f"{cfg['R']}), modes {d['modes']}, one run each, 1 thread pinned to core 0 "
                       f"(taskset -c 0) of {info['nproc']}"),
            "seconds_per_mode": d["seconds_per_mode"], **info}


NCU_METRICS = "dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct"
_UNITS = {"byte": 1, "kbyte": 1e3, "mbyte": 1e6, "gbyte": 1e9, "tbyte": 1e12, "%": 1}


def dram_probe_child(args):
    """Child process run under ncu: the bench workload, three warm-up steps, then one step
    whose launches ncu counts (bytes only -- nothing timed here is reported)."""
    import torch

    import paper_conf_iiswc_lilwlob20_b200 as pasta
    cfg = si.CONFIGS[args.config]
    dims, R = cfg["dims"], cfg["R"]
    x = pasta.pasta_gen_powerlaw(dims, cfg["nnz"], cfg["seed"], kind=0 if cfg["kind"] == "uniform" else 1)
    g = torch.Generator(device="cuda")
    g.manual_seed(cfg["seed"])
    U = [torch.rand((d, R), generator=g, device="cuda", dtype=torch.float32) for d in dims]
    outs = [torch.empty((d, R), dtype=torch.float32, device="cuda") for d in dims]
    for _ in range(4):
        for n in range(len(dims)):
            pasta.pasta_mttkrp_coo(x, n, U, out=outs[n])
    torch.cuda.synchronize()


def dram_counters(args, cfg):
    """DRAM bytes and L2 hit rate per MTTKRP launch, counted by ncu on the bench workload's
    last step in a child process (launches 3N .. 4N-1 of the MTTKRP kernel)."""
    ncu = shutil.which("ncu") or ("/usr/local/cuda/bin/ncu" if os.path.exists("/usr/local/cuda/bin/ncu") else None)
    if ncu is None:
        return None
    N = len(cfg["dims"])
    fd, log = tempfile.mkstemp(prefix="ncu_", suffix=".csv")
    os.close(fd)
    cmd = [ncu, "--metrics", NCU_METRICS, "--clock-control", "none", "-k",
           "regex:coo_staged_kernel|mttkrp_kernel", "--launch-skip", str(3 * N), "--launch-count", str(N),
           "--csv", "--log-file", log, sys.executable, os.path.abspath(__file__), "--dram-probe",
           "--config", args.config]
    try:
        subprocess.run(cmd, capture_output=True, text=True, timeout=900)
        import csv
        vals = {}
        with open(log) as f:
            rows = [r for r in csv.reader(l for l in f if l.startswith('"'))]
        hdr = rows[0]
        iid, iname, iunit, ival = (hdr.index("ID"), hdr.index("Metric Name"), hdr.index("Metric Unit"),
                                   hdr.index("Metric Value"))
        for r in rows[1:]:
            v = float(r[ival].replace(",", "")) * _UNITS.get(r[iunit].lower(), 1)
            vals.setdefault(r[iname], {})[r[iid]] = v
        launches = sorted(vals["dram__bytes_read.sum"])
        per = [vals["dram__bytes_read.sum"][i] + vals["dram__bytes_write.sum"][i] for i in launches]
        hit = [vals["lts__t_sector_hit_rate.pct"][i] for i in launches]
        return {"bytes_per_launch": sum(per) / len(per), "per_mode": [round(v) for v in per],
                "l2_hit_pct": round(sum(hit) / len(hit), 2),
                "how": f"ncu --metrics {NCU_METRICS} on the 4th step's {N} MTTKRP launches of this "
                       "workload in a child process (counts only; not a timed run)"}
    except Exception as e:
        return {"unavailable": str(e)[:200]}
    finally:
        try:
            os.unlink(log)
        except OSError:
            pass


def workload_name(key, cfg, world, scaling):
    if world == 1:
        return f"{key}: {cfg['name']}"
    if scaling == "strong":
        return f"{key}: {cfg['name']}, {cfg['nnz']} nonzeros split over {world} ranks (strong scaling)"
    return f"{key}x{world}: {cfg['name']} grown to {world} x {cfg['nnz']} nonzeros (weak scaling)"


def run_reference(args, cfg, world, rank, scaling):
    """The oracle as it stands, pinned to one host core, on this run's workload config: each
    step = one mode's MTTKRP over one block of the workload's nonzeros (modes and blocks taken
    round-robin), so that the steps stay bounded while the whole tensor is the input."""
    if rank != 0:
        return
    import oracle
    cores = pin_to_core0()
    oracle.build()
    dims, R = cfg["dims"], cfg["R"]
    N = len(dims)
    M_total = cfg["nnz"] * (world if scaling == "weak" else 1)
    inds, vals = host_workload(dict(cfg, nnz=M_total), M_total)
    U = si.factors(dims, R, seed=cfg["seed"])
    blk = min(args.ref_block, M_total)
    nblk = (M_total + blk - 1) // blk
    times, nz = [], []
    for it in range(args.warmup + args.steps):
        n, b = it % N, (it // N) % nblk
        lo, hi = b * blk, min(M_total, (b + 1) * blk)
        ii, vv = np.ascontiguousarray(inds[:, lo:hi]), vals[lo:hi]
        t0 = time.perf_counter()
        oracle.mttkrp(dims, ii, vv, n, U)
        if it >= args.warmup:
            times.append(time.perf_counter() - t0)
            nz.append(hi - lo)
    gflops = sum(model_flops(N, m, R) for m in nz) / sum(times) / 1e9
    info = host_cpu_info()
    sample = (f"{len(times)} steps, each one mode's oracle MTTKRP over a block of <= {blk} of the "
              f"{M_total} workload nonzeros (host-drawn by synth_inputs, same shape and law), modes "
              f"and blocks round-robin; 1 thread pinned to core 0 of {info['nproc']}")
    line = {
        "impl": "reference", "metric": METRIC, "value": round(gflops, 4), "unit": "GFLOP/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(sum(times) / len(times) * 1e3, 3), "higher_is_better": True,
        "scaling": scaling if world > 1 else "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (synth_inputs, the workload's shape and law)",
        "config": {"workload": workload_name(args.config, cfg, world, scaling), "dims": list(dims),
                   "nnz": M_total, "R": R, "format": "COO", "modes": "all (round-robin)",
                   "same_config": True},
        "cpu_baseline": {"value": round(gflops, 4), "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                         "sample": sample, **info},
        "e2e": {"value": round(gflops, 4), "unit": "GFLOP/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def spawn_ranks(args):
    """--gpus N outside torchrun: re-launch this script with N ranks (one process per GPU)."""
    import socket
    sock = socket.socket()
    sock.bind(("127.0.0.1", 0))
    port = sock.getsockname()[1]
    sock.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="h", choices=sorted(si.CONFIGS))
    ap.add_argument("--scaling", default="auto", choices=["auto", "weak", "strong"],
                    help="N > 1: weak = N x the config's nonzeros, strong = the config's nonzeros "
                         "split over the ranks (auto: strong for c5, weak otherwise)")
    ap.add_argument("--impl", default="pasta", choices=["pasta", "reference"])
    ap.add_argument("--ref-block", type=int, default=16_000_000,
                    help="reference arm: nonzeros per oracle step")
    ap.add_argument("--cpu-sample", type=int, default=0,
                    help="cpu_baseline nonzeros (0: the full workload; c5: 100M)")
    ap.add_argument("--cpu-modes", default="0", help="cpu_baseline modes: comma list or all")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-dram-counters", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--hicoo-steps", type=int, default=20)
    ap.add_argument("--cpals-iters", type=int, default=5)
    ap.add_argument("--ew-steps", type=int, default=20)
    ap.add_argument("--dram-probe", action="store_true", help=argparse.SUPPRESS)
    ap.add_argument("--cpu-oracle-child", action="store_true", help=argparse.SUPPRESS)
    ap.add_argument("--cpu-omp-child", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3  # timing rule: >= 3 warm-up steps
    cfg = si.CONFIGS[args.config]
    if cfg["nnz"] >= 500_000_000:  # C5: the extra legs' copies would not fit next to the COO copies
        args.hicoo_steps = args.cpals_iters = args.ew_steps = 0
    if args.cpu_sample == 0 and cfg["nnz"] > 200_000_000:
        args.cpu_sample = 100_000_000
    if args.dram_probe:
        return dram_probe_child(args)
    if args.cpu_oracle_child:
        return cpu_oracle_child(args)
    if args.cpu_omp_child:
        return cpu_omp_child(args)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(args))
    world, rank, local = dist_env()
    scaling = args.scaling if args.scaling != "auto" else ("strong" if args.config == "c5" else "weak")

    if args.impl == "reference":
        run_reference(args, cfg, world, rank, scaling)
        return

    import torch
    import torch.distributed as dist

    import paper_conf_iiswc_lilwlob20_b200 as pasta
    from paper_conf_iiswc_lilwlob20_b200.parallel import RowPartitionedMTTKRP, gather_rows

    # PASTA_BENCH_SHARED_GPU=1 (tests only): every rank on cuda:0 with the gloo backend, to
    # exercise the N > 1 code path on a single-GPU box; real runs use one GPU per rank + NCCL
    shared = os.environ.get("PASTA_BENCH_SHARED_GPU") == "1"
    local_dev = 0 if shared else local
    torch.cuda.set_device(local_dev)
    dev = torch.device("cuda", local_dev)
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.current_stream()

    dims, R = cfg["dims"], cfg["R"]
    M = cfg["nnz"] * (world if scaling == "weak" else 1)
    N = len(dims)
    g = torch.Generator(device=dev)
    g.manual_seed(cfg["seed"])
    U = [torch.rand((d, R), generator=g, device=dev, dtype=torch.float32) for d in dims]

    def timed(step, steps):
        """CUDA-event ms per step on the current stream, after the caller's warm-up."""
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(stream)
        for _ in range(steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / steps

    t1 = None  # strong scaling: rank 0's single-GPU time of the whole tensor
    t_gen = t_prep = 0.0
    if world == 1:
        t0 = time.perf_counter()
        x = pasta.pasta_gen_powerlaw(dims, M, cfg["seed"], kind=0 if cfg["kind"] == "uniform" else 1)
        torch.cuda.synchronize()
        t_gen = time.perf_counter() - t0
        t0 = time.perf_counter()
        for n in range(N):
            pasta.pasta_coo_prepare(x, n)
        torch.cuda.synchronize()
        t_prep = time.perf_counter() - t0
        outs = [torch.empty((d, R), dtype=torch.float32, device=dev) for d in dims]
        shards = [x] * N
        bounds = [(0, d) for d in dims]

        def step():
            for n in range(N):
                pasta.pasta_mttkrp_coo(x, n, U, out=outs[n])
    else:
        # every rank generates the same tensor (counter-based generator), keeps its row shard of
        # every mode and frees the rest; ranks sharing one GPU take turns (bounded peak memory)
        part = None
        for turn in range(world if shared else 1):
            if not shared or turn == rank:
                t0 = time.perf_counter()
                x = pasta.pasta_gen_powerlaw(dims, M, cfg["seed"], kind=0 if cfg["kind"] == "uniform" else 1)
                torch.cuda.synchronize()
                t_gen = time.perf_counter() - t0
                if scaling == "strong" and rank == 0:
                    full = [torch.empty((d, R), dtype=torch.float32, device=dev) for d in dims]

                    def step1():
                        for n in range(N):
                            pasta.pasta_mttkrp_coo(x, n, U, out=full[n])
                    for _ in range(args.warmup):
                        step1()
                    t1 = timed(step1, max(3, min(args.steps, 10)))
                    del full
                t0 = time.perf_counter()
                # shards cut mode by mode, each full sorted copy released after its shard
                part = RowPartitionedMTTKRP(x, rank, world, R, dev, release=True)
                del x
                torch.cuda.synchronize()
                t_prep = time.perf_counter() - t0
            if shared:
                dist.barrier()
        shards = part.shards
        bounds = [(int(part.bounds[n][rank]), int(part.bounds[n][rank + 1])) for n in range(N)]

        def step():
            part.step(U, gather=False)
    shard_nnz = [sh.nnz for sh in shards]

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    clocks = ClockSampler(local_dev)
    if rank == 0:
        clocks.start()
    pasta.pasta_profile_read(0, reset=True)
    pasta.pasta_profile_read(2, reset=True)
    pasta.pasta_profile_enable(True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches0 = pasta.pasta_launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for _ in range(args.steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = pasta.pasta_launch_count() - launches0
    pasta.pasta_profile_enable(False)
    elapsed_ms = ev0.elapsed_time(ev1)
    kern_ms, kern_n = pasta.pasta_profile_read(0, reset=True)
    zero_ms, zero_n = pasta.pasta_profile_read(2, reset=True)
    clk = clocks.stop() if rank == 0 else None
    if world > 1:
        t = torch.tensor([elapsed_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        elapsed_ms = float(t.item())

    ms_per_step = elapsed_ms / args.steps
    total_flops = N * model_flops(N, M, R)  # all ranks together, every mode
    value = total_flops / (ms_per_step * 1e-3) / 1e9

    # SURVEY 8(d) compulsory bytes per launch of this rank (the honest lower bound): the stream,
    # every distinct gathered factor row once, the owned output rows once
    touched = [[int(np.count_nonzero(pasta.pasta_coo_row_counts(shards[n], k))) for k in range(N)]
               for n in range(N)]
    comp = [4 * (N + 1) * shard_nnz[n] + 4 * R * sum(touched[n][k] for k in range(N) if k != n)
            + 4 * R * (bounds[n][1] - bounds[n][0]) for n in range(N)]
    comp_launch = sum(comp) / N

    # e2e: the same metric through the public API with HOST buffers (pinned)
    e2e = None
    if world == 1 and args.e2e_steps > 0:
        hf = [u.cpu().pin_memory() for u in U]
        ho = [torch.empty((d, R), dtype=torch.float32).pin_memory() for d in dims]
        ho2 = [torch.empty((d, R), dtype=torch.float32).pin_memory() for d in dims]
        for _ in range(2):
            pasta.pasta_mttkrp_coo_allmodes_host(x, hf, ho)  # warm-up (allocates staging)
        pasta.pasta_mttkrp_coo_allmodes_host_batch(x, [(hf, ho), (hf, ho2)])  # second slot
        torch.cuda.synchronize()
        t0 = time.perf_counter()  # each call returns after its results are in host memory
        for _ in range(args.e2e_steps):
            pasta.pasta_mttkrp_coo_allmodes_host(x, hf, ho)
        e1_ms = (time.perf_counter() - t0) * 1e3 / args.e2e_steps
        # the same steps as one pipelined stream of factor sets (outputs alternate between two
        # pinned host buffer sets): step i+1's uploads overlap step i's downloads
        batch = [(hf, ho if i % 2 == 0 else ho2) for i in range(args.e2e_steps)]
        t0 = time.perf_counter()
        pasta.pasta_mttkrp_coo_allmodes_host_batch(x, batch)
        e_ms = (time.perf_counter() - t0) * 1e3 / args.e2e_steps
        nbytes = sum(d * R * 4 for d in dims)
        e2e = {"value": round(total_flops / (e_ms * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
               "h2d_bytes_per_step": nbytes, "d2h_bytes_per_step": nbytes,
               "ms_per_step": round(e_ms, 3),
               "path": f"pasta_mttkrp_coo_allmodes_host_batch, {args.e2e_steps} steps in one call "
                       "(pinned host factors in, every step's results out; copies pipelined "
                       "against the kernels and step i+1's uploads against step i's downloads; "
                       "wall clock)",
               "single_call": {"value": round(total_flops / (e1_ms * 1e-3) / 1e9, 3),
                               "ms_per_step": round(e1_ms, 3),
                               "path": "pasta_mttkrp_coo_allmodes_host, one call per step"}}
        pasta.pasta_coo_release_staging(x)
        del hf, ho, ho2

    # N > 1: the exchange step, timed apart from the MTTKRP step (max over ranks)
    allgather = None
    strong = None
    if world > 1:
        def max_over_ranks(v):
            t = torch.tensor([v], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            return float(t.item())

        def gather_timing(method):
            def gstep():
                works = []
                for n in range(N):
                    works += gather_rows(part.out[n], part.bounds[n], async_op=True, method=method)
                for w in works:
                    w.wait()
            for _ in range(2):
                gstep()
            dist.barrier()
            return max_over_ranks(timed(gstep, max(3, min(args.steps, 10))))

        recv = sum((d - (bounds[n][1] - bounds[n][0])) * R * 4 for n, d in enumerate(dims))
        g_ms = gather_timing("allgather")
        b_ms = gather_timing("broadcast")
        allgather = {"ms_per_step": round(g_ms, 4), "bytes_received_per_rank": recv,
                     "gbs_per_rank": round(recv / (g_ms * 1e-3) / 1e9, 1),
                     "value_with_allgather": round(total_flops / ((ms_per_step + g_ms) * 1e-3) / 1e9, 3),
                     "how": "one padded all_gather_into_tensor per mode (NCCL) of the owned output "
                            "rows, then the peers' blocks copied into place (parallel.gather_rows)",
                     "broadcast": {"ms_per_step": round(b_ms, 4),
                                   "how": "P in-place NCCL broadcasts per mode"}}
        # the same exchange by peer stores over NVLink (CUDA IPC replicas, pasta_bcast_f32)
        try:
            from paper_conf_iiswc_lilwlob20_b200.parallel import PeerReplicas, gather_rows_p2p
            reps = PeerReplicas(dims, R)
            flag = torch.zeros(1, device=dev)

            def p2p_step():
                for n in range(N):
                    gather_rows_p2p(reps, n, part.bounds[n], rank)
                dist.all_reduce(flag)  # orders the peers' reads after the stores

            for _ in range(2):
                p2p_step()
            dist.barrier()
            p_ms = max_over_ranks(timed(p2p_step, max(3, min(args.steps, 10))))
            allgather["p2p"] = {"ms_per_step": round(p_ms, 4),
                                "gbs_per_rank": round(recv / (p_ms * 1e-3) / 1e9, 1),
                                "how": "owned rows stored into every peer's replica by one kernel "
                                       "per mode (CUDA IPC P2P stores) + a 1-element all-reduce"}
            # MTTKRP and all-gather fused in one kernel per mode (pasta_mttkrp_coo_bcast)
            for _ in range(2):
                part.step_fused(U, reps)
            dist.barrier()
            f_ms = max_over_ranks(timed(lambda: part.step_fused(U, reps), max(3, min(args.steps, 10))))
            allgather["fused"] = {"ms_per_step": round(f_ms, 4),
                                  "value": round(total_flops / (f_ms * 1e-3) / 1e9, 3),
                                  "how": "MTTKRP step with the all-gather fused into the kernel: every "
                                         "row flush also stored into the peers' replicas over P2P "
                                         "(pasta_mttkrp_coo_bcast) + a 1-element all-reduce"}
            dist.barrier()
            reps.close()
        except Exception as e:  # e.g. no IPC between the ranks' GPUs
            allgather["p2p"] = {"unavailable": str(e)[:200]}
        if scaling == "strong":
            t1 = max_over_ranks(t1 if t1 is not None else 0.0)
            strong = {"t1_ms_per_step": round(t1, 4), "tp_ms_per_step": round(ms_per_step, 4),
                      "tp_with_allgather_ms_per_step": round(ms_per_step + g_ms, 4),
                      "t1_over_p_tp": round(t1 / (world * ms_per_step), 4),
                      "t1_over_p_tp_with_allgather": round(t1 / (world * (ms_per_step + g_ms)), 4),
                      "how": "T_1 = rank 0 timing the whole tensor on its GPU before sharding "
                             "(same kernels, same step); T_P = this run's step, max over ranks"}
        if args.e2e_steps > 0:
            hf = [u.cpu().pin_memory() for u in U]
            ho = [torch.empty((hi - lo, R), dtype=torch.float32).pin_memory() for lo, hi in bounds]

            def e2e_step():
                for k in range(N):
                    U[k].copy_(hf[k], non_blocking=True)
                part.step(U, gather=False)
                for n, (lo, hi) in enumerate(bounds):
                    ho[n].copy_(part.out[n][lo:hi], non_blocking=True)
                torch.cuda.synchronize()

            e2e_step()
            dist.barrier()
            t0 = time.perf_counter()
            for _ in range(args.e2e_steps):
                e2e_step()
            e_ms = max_over_ranks((time.perf_counter() - t0) * 1e3 / args.e2e_steps)
            e2e = {"value": round(total_flops / (e_ms * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
                   "h2d_bytes_per_step": sum(d * R * 4 for d in dims),
                   "d2h_bytes_per_step": sum((hi - lo) * R * 4 for lo, hi in bounds),
                   "ms_per_step": round(e_ms, 3),
                   "path": "per rank: pinned factors H2D, pasta_mttkrp_coo on the rank's shards, owned "
                           "rows D2H (wall clock, max over ranks); bytes are rank 0's"}

    # a7: HiCOO MTTKRP (B = 128) on the same tensor, every mode per step; NEXT-2: the
    # same on the gHiCOO form with the storage-minimising mask
    def time_blocked(make, label):
        t0 = time.perf_counter()
        h = make()
        torch.cuda.synchronize()
        t_conv = time.perf_counter() - t0
        t0 = time.perf_counter()
        for n in range(N):
            pasta.pasta_hicoo_prepare(h, n)
        torch.cuda.synchronize()
        t_hprep = time.perf_counter() - t0
        houts = [torch.empty((d, R), dtype=torch.float32, device=dev) for d in dims]
        t0 = time.perf_counter()  # the first launches build the R#36 tier-block copies
        for n in range(N):
            pasta.pasta_mttkrp_hicoo(h, n, U, out=houts[n])
        torch.cuda.synchronize()
        t_first = time.perf_counter() - t0
        for _ in range(2):
            for n in range(N):
                pasta.pasta_mttkrp_hicoo(h, n, U, out=houts[n])
        torch.cuda.synchronize()
        pasta.pasta_profile_read(1, reset=True)
        pasta.pasta_profile_enable(True)
        h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        h0.record(stream)
        for _ in range(args.hicoo_steps):
            for n in range(N):
                pasta.pasta_mttkrp_hicoo(h, n, U, out=houts[n])
        h1.record(stream)
        torch.cuda.synchronize()
        pasta.pasta_profile_enable(False)
        hk_ms, hk_n = pasta.pasta_profile_read(1, reset=True)
        h_ms = h0.elapsed_time(h1) / args.hicoo_steps
        nc = bin(h.cmask).count("1")
        if nc == N:
            hb = model_bytes_hicoo(N, M, h.nblocks, R)
            stream_b = (N + 4) * M + (8 + 4 * N) * h.nblocks
            bm = "(N+4)M + (8+4N)n_b + 4NR min(n_b B, M) per launch"
        else:  # gHiCOO stream + the COO upper bound for the gathers (R#29)
            stream_b = (nc + 4 * (N - nc) + 4) * M + (8 + 4 * nc) * h.nblocks
            hb = stream_b + 4 * N * R * M
            bm = "(N_c + 4N_u + 4)M + (8+4N_c)n_b + 4NRM per launch"
        # compulsory: the format's own stream (Table I storage) + every distinct gathered row
        # once + the output, averaged over the modes
        hc = sum(stream_b + 4 * R * sum(touched[n][k] for k in range(N) if k != n) + 4 * R * dims[n]
                 for n in range(N)) / N
        peak_h, _ = load_peaks()
        hl_ms = hk_ms / max(hk_n, 1)
        ach = hc / (hl_ms * 1e-3) / 1e9
        mg = hb / (hl_ms * 1e-3) / 1e9
        res = {"value": round(total_flops / (h_ms * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
               "ms_per_step": round(h_ms, 4), "nblocks": h.nblocks, "block": 128,
               "cmask": h.cmask, "nnz_per_block": round(M / max(h.nblocks, 1), 3),
               "vs_coo_launch_time": round(hl_ms / avg_coo_launch_ms, 3),
               "roofline": {"bound": "hbm", "achieved": round(ach, 1), "peak": peak_h,
                            "unit": "GB/s", "frac": round(ach / peak_h, 4),
                            "bytes": "compulsory: format stream + 4R sum_{k!=n} touched_k + 4R I_n",
                            "bytes_per_launch": round(hc),
                            "model_bytes_per_launch": round(hb), "model_frac": round(mg / peak_h, 4),
                            "model": bm,
                            "kernel": f"coo_staged_kernel<..., WA 10 / WA 9> ({label} row slices decoded "
                                      "warp-wide into the staged kernel; WA 10 = tier blocks (R#36), used "
                                      "when every gathered factor exceeds 2x the L2)",
                            "avg_launch_ms": round(hl_ms, 4)},
               "preprocess_s": {"convert": round(t_conv, 3), "mode_copies_all": round(t_hprep, 3),
                                "first_launches_incl_tier_blocks": round(t_first, 3)}}
        del h, houts
        return res

    hicoo = ghicoo = None
    avg_coo_launch_ms = kern_ms / max(kern_n, 1)
    if world == 1 and args.hicoo_steps > 0:
        hicoo = time_blocked(lambda: pasta.pasta_coo_to_hicoo(x, 7), "hicoo")
        ghicoo = time_blocked(lambda: pasta.pasta_coo_to_ghicoo(x, 7, 0), "ghicoo")

    # NEXT-1: CP-ALS sweeps (each = MTTKRP + solve + normalise + gram for every mode)
    cpals = None
    if world == 1 and args.cpals_iters > 0:
        Uc = [u.clone() for u in U]
        pasta.pasta_cpals_coo(x, Uc, max_iters=1, tol=0.0)  # warm-up
        Uc = [u.clone() for u in U]
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        lam_c, fits_c, it_c = pasta.pasta_cpals_coo(x, Uc, max_iters=args.cpals_iters, tol=0.0)
        torch.cuda.synchronize()
        c_ms = (time.perf_counter() - t0) * 1e3 / max(it_c, 1)
        cpals = {"ms_per_sweep": round(c_ms, 3), "sweeps": it_c,
                 "fit": [round(f, 6) for f in fits_c],
                 "mttkrp_share": round(ms_per_step / c_ms, 3),
                 "note": "pasta_cpals_coo from random U[0,1) factors; wall clock incl. the "
                         "per-sweep fit read-back"}
        del Uc

    # NEXT-3: semi-sparse TTM (R) and TTV along mode 0 (Table I: TTM 4MR + 4M_F R + 16M_F + 8M,
    # TTV 12M + 12M_F bytes; 2MR / 2M flops); fibers are pre-processing
    ttm = None
    if world == 1 and args.ew_steps > 0:
        t0 = time.perf_counter()
        MF = pasta.pasta_coo_fibers(x, 0)
        torch.cuda.synchronize()
        t_fib = time.perf_counter() - t0
        Ut = torch.rand((dims[0], R), device=dev)
        vt = torch.rand(dims[0], device=dev)
        yt = torch.empty((MF, R), device=dev)
        yv = torch.empty(MF, device=dev)
        peak_t, _ = load_peaks()
        ttm = {"mode": 0, "fibers": MF, "preprocess_s": round(t_fib, 3)}
        for name, fn, nbytes, flops in (
                ("ttm", lambda: pasta.pasta_ttm_coo(x, 0, Ut, out=yt), 4 * M * R + 4 * MF * R + 16 * MF + 8 * M,
                 2 * M * R),
                ("ttv", lambda: pasta.pasta_ttv_coo(x, 0, vt, out=yv), 12 * M + 12 * MF, 2 * M)):
            for _ in range(3):
                fn()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(args.ew_steps):
                fn()
            e1.record(stream)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / args.ew_steps
            gbs = nbytes / (ms * 1e-3) / 1e9
            ttm[name] = {"ms": round(ms, 4), "GFLOP/s": round(flops / (ms * 1e-3) / 1e9, 1),
                         "model_gbs": round(gbs, 1), "frac": round(gbs / peak_t, 4)}
        del Ut, vt, yt, yv

    # NEXT-4: TS and same-pattern TEW on the tensor's value array (Table I: TS 8M bytes, TEW
    # 12M bytes, M flops) -- the streaming kernels that bound the HBM roofline
    ew = None
    if world == 1 and args.ew_steps > 0:
        vals = torch.empty(M, dtype=torch.float32, device=dev)
        vals.uniform_(-1.0, 1.0)
        other = torch.empty_like(vals)
        dst = torch.empty_like(vals)
        peak_e, _ = load_peaks()
        ew = {}
        for name, fn, nbytes in (
                ("ts_mul", lambda: pasta.pasta_ts(vals, "mul", 0.5, out=dst), 8 * M),
                ("tew_add", lambda: pasta.pasta_tew(vals, other, "add", out=dst), 12 * M)):
            for _ in range(3):
                fn()
            torch.cuda.synchronize()
            pasta.pasta_profile_read(3, reset=True)
            pasta.pasta_profile_enable(True)
            for _ in range(args.ew_steps):
                fn()
            torch.cuda.synchronize()
            pasta.pasta_profile_enable(False)
            e_ms, e_n = pasta.pasta_profile_read(3, reset=True)
            avg = e_ms / max(e_n, 1)
            gbs = nbytes / (avg * 1e-3) / 1e9
            ew[name] = {"ms": round(avg, 4), "GFLOP/s": round(M / (avg * 1e-3) / 1e9, 1),
                        "roofline": {"bound": "hbm", "achieved": round(gbs, 1), "peak": peak_e,
                                     "unit": "GB/s", "frac": round(gbs / peak_e, 4),
                                     "bytes_model": "TS 8M / TEW 12M per launch (Table I, P:117)"}}
        del vals, other, dst

    balance = None
    if world > 1:  # max / mean nonzeros per rank, per mode (every rank joins)
        allsh = [None] * world
        dist.all_gather_object(allsh, [int(v) for v in shard_nnz])
        balance = [round(max(r[n] for r in allsh) / (sum(r[n] for r in allsh) / world), 4)
                   for n in range(N)]

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    peak, peak_src = load_peaks()
    avg_launch_ms = kern_ms / max(kern_n, 1)
    achieved = comp_launch / (avg_launch_ms * 1e-3) / 1e9
    model_launch = sum(model_bytes_coo(N, m, R) for m in shard_nnz) / N
    model_gbs = model_launch / (avg_launch_ms * 1e-3) / 1e9
    counters = None
    if world == 1 and not args.no_dram_counters:
        counters = dram_counters(args, cfg)
    traffic = counters.get("bytes_per_launch") if counters else None

    cpu = comp_omp = None
    if not args.no_cpu_baseline and world == 1:
        cpu = cpu_baseline(args, cfg)
        comp_omp = cpu_omp(args, cfg)

    line = {
        "metric": METRIC, "value": round(value, 3), "unit": "GFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4),
        "higher_is_better": True, "scaling": scaling if world > 1 else "strong",
        "vs_baseline": None, "dtype": "f32",
        "data": f"synthetic: GPU Stochastic Kronecker generator (q=0.75), seed {cfg['seed']}",
        "config": {"workload": workload_name(args.config, cfg, world, scaling), "dims": list(dims), "nnz": M,
                   "R": R, "format": "COO", "modes": f"all {N} per step",
                   "parallelism": f"row-partitioned x{world}, no collective in the step" +
                                  (" (NCCL all-gather timed separately)" if world > 1 else ""),
                   "l2": "no flush: per-step working set (COO copies + factors + outputs) "
                         "> 126 MB L2"},
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "traffic": round(traffic) if traffic else None,
                     "kernel": "coo_staged_kernel (a6, csrc/mttkrp.cu)",
                     "bytes": "compulsory (SURVEY 8(d)): 4(N+1)M + 4R sum_{k!=n} touched_k + 4R I_n "
                              "per launch, averaged over the modes",
                     "bytes_per_launch": round(comp_launch),
                     "avg_launch_ms": round(avg_launch_ms, 4), "launches": kern_n,
                     "peak_source": peak_src,
                     "model_bytes_per_launch": round(model_launch),
                     "model_gbs": round(model_gbs, 1), "model_frac": round(model_gbs / peak, 4),
                     "model": "paper upper bound 4(N+1)M + 4NRM (Table I, P:117): every gather a "
                              "DRAM access; exceeds 1 when gathers hit L2 (P:330)",
                     "dram_gbs": round(traffic / (avg_launch_ms * 1e-3) / 1e9, 1) if traffic else None,
                     "dram_frac": round(traffic / (avg_launch_ms * 1e-3) / 1e9 / peak, 4) if traffic else None,
                     "traffic_over_compulsory": round(traffic / comp_launch, 3) if traffic else None,
                     "l2_hit_pct": counters.get("l2_hit_pct") if counters else None,
                     "counters": counters},
        "touched_rows": touched[0] if world == 1 else None,
        "zero_fill_ms_per_step": round(zero_ms / args.steps, 4),
        "preprocess_s": {"generate": round(t_gen, 3), "mode_sort_all" if world == 1 else "shard_all": round(t_prep, 3)},
        "clocks": clk,
        "e2e": e2e,
        "allgather": allgather,
        "strong_scaling": strong,
        "hicoo": hicoo,
        "ghicoo": ghicoo,
        "cpals": cpals,
        "ew": ew,
        "ttm": ttm,
        "gpu_launches": launches,
        "cpu_baseline": cpu,
        "cpu_omp": comp_omp,
        "max_shard_nnz": max(shard_nnz),
        "shard_max_over_mean": balance,
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
