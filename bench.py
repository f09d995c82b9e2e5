#!/usr/bin/env python
"""bench.py -- MTTKRP GFLOP/s and HBM GB/s against the measured B200 roofline.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config h|c2|c3|c4|c1] [--impl reference]

One STEP = COO MTTKRP of every mode (output zero-fill + kernel, the paper times all modes and
averages) over the synthetic tensor resident in HBM.  Rank 0 prints one JSON line.
GFLOP/s uses the nominal N*M*R flops per mode (Table I generalised; R#7).

The default workload is the north_star target: a 100M-nonzero 3rd-order power-law tensor,
regL-shaped (2^23)^3 (Table II s3), R = 16.  At N GPUs (torchrun) the tensor has
N x 100M nonzeros of the same draw sequence and shape (weak scaling, cf. BASELINE config 5:
1B nonzeros at 8 GPUs); every rank owns the nnz-balanced row shard of every mode and the
timed step has no collective.  The all-gather of the owned output rows over NCCL -- needed
only when the next CP-ALS step consumes the factor (north_star) -- is timed separately
(`allgather` object).

--impl reference times the fp64 CPU oracle (oracle/, the slow correctness reference) on a
bounded sample of the same workload on the host cores; under torchrun only rank 0 works.
"""
from __future__ import annotations

import argparse
import json
import os
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


def cpu_baseline(cfg, R, sample_nnz, steps=1, warmup=0):
    """The fp64 oracle (as it stands, single thread) on a bounded sample of the workload:
    the first `sample_nnz` distinct coordinates of the SAME counter-based draw sequence
    (the oracle's own generator), all modes.  Returns (GFLOP/s, seconds per step)."""
    import oracle
    dims = cfg["dims"]
    inds, vals = oracle.gen_powerlaw(dims, sample_nnz, cfg["seed"], q=0.5 if cfg["kind"] ==
                                     "uniform" else 0.75)
    U = si.factors(dims, R, seed=cfg["seed"])
    times = []
    for it in range(warmup + steps):
        t0 = time.perf_counter()
        for n in range(len(dims)):
            oracle.mttkrp(dims, inds, vals, n, U)
        if it >= warmup:
            times.append(time.perf_counter() - t0)
    t = sum(times) / len(times)
    flops = len(dims) * model_flops(len(dims), sample_nnz, R)
    return flops / t / 1e9, t


def ncu_traffic(config_key, family="coo_mttkrp"):
    """DRAM bytes per MTTKRP launch from the committed ncu --set full summary, if any."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        e = d.get(config_key, {}).get(family)
        return float(e["dram_bytes_per_launch"]) if e else None
    except Exception:
        return None


def workload_name(key, cfg, world):
    if world == 1:
        return f"{key}: {cfg['name']}"
    return f"{key}x{world}: {cfg['name']} grown to {world} x {cfg['nnz']} nonzeros (weak scaling)"


def run_reference(args, cfg, world, rank):
    if rank != 0:
        return
    R = cfg["R"]
    M_total = cfg["nnz"] * world
    sample = args.ref_sample
    gflops, t = cpu_baseline(cfg, R, sample, steps=args.steps, warmup=args.warmup)
    cores = 1
    line = {
        "impl": "reference", "metric": METRIC, "value": round(gflops, 4), "unit": "GFLOP/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(t * 1e3, 3), "higher_is_better": True,
        "scaling": "weak" if world > 1 else "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic (oracle generator, same draws)",
        "config": {"workload": workload_name(args.config, cfg, world), "dims": list(cfg["dims"]),
                   "nnz": M_total, "R": R, "format": "COO", "modes": "all"},
        "cpu_baseline": {"value": round(gflops, 4), "unit": "GFLOP/s", "cores": cores,
                         "kind": "oracle",
                         "sample": f"first {sample} distinct nonzeros of the workload's draw "
                                   f"sequence, all {len(cfg['dims'])} modes per step"},
        "e2e": {"value": round(gflops, 4), "unit": "GFLOP/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="h", choices=sorted(si.CONFIGS))
    ap.add_argument("--impl", default="pasta", choices=["pasta", "reference"])
    ap.add_argument("--ref-sample", type=int, default=1_000_000)
    ap.add_argument("--cpu-sample", type=int, default=4_000_000)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--hicoo-steps", type=int, default=20)
    ap.add_argument("--cpals-iters", type=int, default=5)
    ap.add_argument("--ew-steps", type=int, default=20)
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3  # timing rule: >= 3 warm-up steps
    cfg = si.CONFIGS[args.config]
    world, rank, local = dist_env()

    if args.impl == "reference":
        run_reference(args, cfg, world, rank)
        return

    import torch
    import torch.distributed as dist

    import paper_conf_iiswc_lilwlob20_b200 as pasta
    from paper_conf_iiswc_lilwlob20_b200.parallel import RowPartitionedMTTKRP

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
    M = cfg["nnz"] * world  # weak scaling: cfg["nnz"] nonzeros per GPU
    N = len(dims)
    t0 = time.perf_counter()
    x = pasta.pasta_gen_powerlaw(dims, M, cfg["seed"], kind=0 if cfg["kind"] == "uniform" else 1)
    torch.cuda.synchronize()
    t_gen = time.perf_counter() - t0
    t0 = time.perf_counter()
    for n in range(N):
        pasta.pasta_coo_prepare(x, n)
    torch.cuda.synchronize()
    t_prep = time.perf_counter() - t0
    g = torch.Generator(device=dev)
    g.manual_seed(cfg["seed"])
    U = [torch.rand((d, R), generator=g, device=dev, dtype=torch.float32) for d in dims]

    if world > 1:
        part = RowPartitionedMTTKRP(x, rank, world, R, dev)
        shard_nnz = part.shard_nnz()
        del x
        torch.cuda.synchronize()

        def step():
            part.step(U, gather=False)
    else:
        outs = [torch.empty((d, R), dtype=torch.float32, device=dev) for d in dims]
        shard_nnz = [M] * N

        def step():
            for n in range(N):
                pasta.pasta_mttkrp_coo(x, n, U, out=outs[n])

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
        del hf, ho, ho2

    # N > 1: the exchange step, timed apart from the MTTKRP step (max over ranks)
    allgather = None
    if world > 1:
        from paper_conf_iiswc_lilwlob20_b200.parallel import gather_rows

        def gather_step():
            works = []
            for n in range(N):
                works += gather_rows(part.out[n], part.bounds[n], async_op=True)
            for w in works:
                w.wait()

        for _ in range(2):
            gather_step()
        torch.cuda.synchronize()
        dist.barrier()
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        gsteps = max(3, min(args.steps, 10))
        g0.record(stream)
        for _ in range(gsteps):
            gather_step()
        g1.record(stream)
        torch.cuda.synchronize()
        dist.barrier()
        t = torch.tensor([g0.elapsed_time(g1) / gsteps], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        g_ms = float(t.item())
        recv = sum((d - (int(part.bounds[n][rank + 1]) - int(part.bounds[n][rank]))) * R * 4
                   for n, d in enumerate(dims))
        allgather = {"ms_per_step": round(g_ms, 4), "bytes_received_per_rank": recv,
                     "gbs_per_rank": round(recv / (g_ms * 1e-3) / 1e9, 1),
                     "value_with_allgather": round(N * model_flops(N, M, R) /
                                                   ((elapsed_ms / args.steps + g_ms) * 1e-3) / 1e9, 3),
                     "how": "in-place uneven all-gather of owned output rows: one NCCL broadcast "
                            "per rank per mode (parallel.gather_rows)"}
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
            torch.cuda.synchronize()
            dist.barrier()
            g0.record(stream)
            for _ in range(gsteps):
                p2p_step()
            g1.record(stream)
            torch.cuda.synchronize()
            dist.barrier()
            t = torch.tensor([g0.elapsed_time(g1) / gsteps], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            p_ms = float(t.item())
            allgather["p2p"] = {"ms_per_step": round(p_ms, 4),
                                "gbs_per_rank": round(recv / (p_ms * 1e-3) / 1e9, 1),
                                "how": "owned rows stored into every peer's replica by one kernel "
                                       "per mode (CUDA IPC P2P stores) + a 1-element all-reduce"}
            dist.barrier()
            reps.close()
        except Exception as e:  # e.g. no IPC between the ranks' GPUs
            allgather["p2p"] = {"unavailable": str(e)[:200]}
    if world > 1 and args.e2e_steps > 0:
        hf = [u.cpu().pin_memory() for u in U]
        own = [(int(part.bounds[n][rank]), int(part.bounds[n][rank + 1])) for n in range(N)]
        ho = [torch.empty((hi - lo, R), dtype=torch.float32).pin_memory() for lo, hi in own]

        def e2e_step():
            for k in range(N):
                U[k].copy_(hf[k], non_blocking=True)
            part.step(U, gather=False)
            for n, (lo, hi) in enumerate(own):
                ho[n].copy_(part.out[n][lo:hi], non_blocking=True)
            torch.cuda.synchronize()

        e2e_step()
        dist.barrier()
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            e2e_step()
        t = torch.tensor([(time.perf_counter() - t0) * 1e3 / args.e2e_steps], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e_ms = float(t.item())
        e2e = {"value": round(N * model_flops(N, M, R) / (e_ms * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
               "h2d_bytes_per_step": sum(d * R * 4 for d in dims),
               "d2h_bytes_per_step": sum((hi - lo) * R * 4 for lo, hi in own),
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
        for _ in range(3):
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
            bm = "(N+4)M + (8+4N)n_b + 4NR min(n_b B, M) per launch"
        else:  # gHiCOO stream + the COO upper bound for the gathers (R#29)
            hb = (nc + 4 * (N - nc) + 4) * M + (8 + 4 * nc) * h.nblocks + 4 * N * R * M
            bm = "(N_c + 4N_u + 4)M + (8+4N_c)n_b + 4NRM per launch"
        peak_h, _ = load_peaks()
        ach = hb / (hk_ms / max(hk_n, 1) * 1e-3) / 1e9
        res = {"value": round(total_flops / (h_ms * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
               "ms_per_step": round(h_ms, 4), "nblocks": h.nblocks, "block": 128,
               "cmask": h.cmask, "nnz_per_block": round(M / max(h.nblocks, 1), 3),
               "roofline": {"bound": "hbm", "achieved": round(ach, 1), "peak": peak_h,
                            "unit": "GB/s", "frac": round(ach / peak_h, 4),
                            "traffic": ncu_traffic(args.config, label + "_mttkrp"),
                            "kernel": f"coo_staged_kernel<..., WA 9> ({label} row slices decoded "
                                      "warp-wide into the staged kernel)",
                            "bytes_model": bm,
                            "avg_launch_ms": round(hk_ms / max(hk_n, 1), 4)},
               "preprocess_s": {"convert": round(t_conv, 3), "mode_copies_all": round(t_hprep, 3)}}
        del h, houts
        return res

    hicoo = ghicoo = None
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
    per_launch_nnz = max(shard_nnz)  # rank 0's launches cover its shard
    my_launch_nnz = [shard_nnz[n] for n in range(N)]
    avg_launch_ms = kern_ms / max(kern_n, 1)
    launch_bytes = sum(model_bytes_coo(N, m, R) for m in my_launch_nnz) / N
    achieved = launch_bytes / (avg_launch_ms * 1e-3) / 1e9
    traffic = ncu_traffic(args.config) if world == 1 else None
    # SURVEY 8(d) compulsory bytes per launch (the honest lower bound): the stream, every
    # distinct gathered factor row once, the output rows once
    compulsory = None
    if world == 1:
        touched = [int(np.count_nonzero(pasta.pasta_coo_row_counts(x, k))) for k in range(N)]
        cb = sum(4 * (N + 1) * M + 4 * R * sum(touched[k] for k in range(N) if k != n) + 4 * R * dims[n]
                 for n in range(N)) / N
        cg = cb / (avg_launch_ms * 1e-3) / 1e9
        compulsory = {"bytes_per_launch": round(cb), "gbs": round(cg, 1), "frac": round(cg / peak, 4),
                      "touched_rows": touched,
                      "def": "4(N+1)M + 4R sum_{k!=n} touched_k + 4R I_n, averaged over modes"}

    cpu = None
    if not args.no_cpu_baseline and world == 1:
        sample = min(args.cpu_sample, M)
        gf, t = cpu_baseline(cfg, R, sample)
        cpu = {"value": round(gf, 4), "unit": "GFLOP/s", "cores": 1, "kind": "oracle",
               "sample": f"first {sample} distinct nonzeros of the same draw sequence (oracle "
                         f"generator), all {N} modes, 1 run, 1 host thread"}

    line = {
        "metric": METRIC, "value": round(value, 3), "unit": "GFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4),
        "higher_is_better": True, "scaling": "weak" if world > 1 else "strong",
        "vs_baseline": None, "dtype": "f32",
        "data": f"synthetic: GPU Stochastic Kronecker generator (q=0.75), seed {cfg['seed']}",
        "config": {"workload": workload_name(args.config, cfg, world), "dims": list(dims), "nnz": M,
                   "R": R, "format": "COO", "modes": f"all {N} per step",
                   "parallelism": f"row-partitioned x{world}, no collective in the step" +
                                  (" (NCCL all-gather timed separately)" if world > 1 else ""),
                   "l2": "no flush: per-step working set (COO copies + factors + outputs) "
                         "> 126 MB L2"},
        "model_gbs": round(model_bytes_coo(N, M, R) * N / (ms_per_step * 1e-3) / 1e9, 1),
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "traffic": traffic,
                     "kernel": "coo_staged_kernel (a6, csrc/mttkrp.cu)",
                     "bytes_model": "4(N+1)M + 4NRM per launch (Table I, P:117)",
                     "avg_launch_ms": round(avg_launch_ms, 4), "launches": kern_n,
                     "peak_source": peak_src,
                     "dram_gbs": round(traffic / (avg_launch_ms * 1e-3) / 1e9, 1) if traffic else None,
                     "dram_frac": round(traffic / (avg_launch_ms * 1e-3) / 1e9 / peak, 4)
                     if traffic else None,
                     "note": "frac uses the paper's byte model, which counts every factor gather as a "
                             "DRAM access (P:117); dram_* use the ncu-measured traffic"},
        "compulsory": compulsory,
        "zero_fill_ms_per_step": round(zero_ms / args.steps, 4),
        "preprocess_s": {"generate": round(t_gen, 3), "mode_sort_all": round(t_prep, 3)},
        "clocks": clk,
        "e2e": e2e,
        "allgather": allgather,
        "hicoo": hicoo,
        "ghicoo": ghicoo,
        "cpals": cpals,
        "ew": ew,
        "ttm": ttm,
        "gpu_launches": launches,
        "cpu_baseline": cpu,
        "max_shard_nnz": per_launch_nnz,
        "shard_max_over_mean": balance,
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
