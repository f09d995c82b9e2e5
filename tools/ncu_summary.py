#!/usr/bin/env python
"""Summarise ncu outputs into profiles/ (committed evidence).

  launches <launches.csv> <out.md>            per-kernel device time from a
                                              `--metrics gpu__time_duration.sum` launch list
  full <prof.ncu-rep> <config> <out.md>       key counters of a `--set full` capture; also
                                              merges dram bytes/launch into profiles/ncu_summary.json
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0,
         "s": 1e3, "second": 1e3}


def short(name):
    for key in ("mttkrp_kernel", "zero_rows_kernel", "Onesweep", "RadixSort", "gather_kernel",
                "pack_keys", "valid_flag", "coords_kernel", "emit_kernel", "Select", "Compact"):
        if key in name:
            break
    return name.split("(")[0][:90]


def launches(path, out):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr, data = rows[h], rows[h + 1:]
    ki, mi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = collections.OrderedDict()
    seq = []
    for r in data:
        ms = float(r[mi].replace(",", "")) * SCALE.get(r[ui].strip(), 1.0)
        name = short(r[ki])
        agg.setdefault(name, [0, 0.0])
        agg[name][0] += 1
        agg[name][1] += ms
        seq.append((name, ms))
    lines = [f"# ncu launch list: {os.path.basename(path)}", "",
             "Cold-cache, serialised replay (`--metrics gpu__time_duration.sum --clock-control none`):",
             "compare SHARES with the bench, not absolute times.", "",
             "| launches | total ms | mean ms | kernel |", "|---:|---:|---:|---|"]
    for k, (n, t) in agg.items():
        lines.append(f"| {n} | {t:.3f} | {t / n:.4f} | `{k}` |")
    # the last bench steps: mttkrp vs zero-fill share
    mt = [t for n, t in seq if ("mttkrp_kernel" in n and "CooSrc" in n) or "coo_staged_kernel" in n]
    ht = [t for n, t in seq if "mttkrp_kernel" in n and "Hicoo" in n]
    zf = [t for n, t in seq if "zero_rows_kernel" in n]
    zc = zf[: len(mt)]  # bench order: every COO launch is preceded by its zero-fill
    if mt:
        lines += ["", f"COO MTTKRP kernel: {len(mt)} launches, mean {sum(mt) / len(mt):.4f} ms; "
                  f"zero-fill mean {sum(zc) / max(len(zc), 1):.4f} ms; COO MTTKRP share of a bench "
                  f"step (MTTKRP + zero-fill) = {sum(mt) / (sum(mt) + sum(zc)):.3f}"]
    if ht:
        lines += [f"HiCOO MTTKRP kernel: {len(ht)} launches, mean {sum(ht) / len(ht):.4f} ms"]
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__grid_size", "launch__block_size",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
        "lts__t_sectors_srcunit_tex_op_read.sum", "lts__t_sectors_srcunit_tex_op_red.sum",
        "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "smsp__warps_eligible.avg.per_cycle_active",
        "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum"]


def full(path, config, out, family=None):
    txt = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    idx = {h: i for i, h in enumerate(hdr)}
    lines = [f"# ncu --set full: {os.path.basename(path)} ({config})", ""]
    per = collections.defaultdict(list)
    for d in data:
        kname = short(d[idx["Kernel Name"]])
        lines.append(f"## `{kname}`")
        lines.append("")
        lines.append("| metric | value | unit |")
        lines.append("|---|---:|---|")
        vals = {}
        for w in WANT:
            if w in idx:
                lines.append(f"| {w} | {d[idx[w]]} | {units[idx[w]]} |")
                vals[w] = (d[idx[w]], units[idx[w]])
        lines.append("")
        per[kname].append(vals)

    def to_bytes(v):
        num, unit = float(v[0].replace(",", "")), v[1].strip()
        return num * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)

    summ_path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    summ = json.load(open(summ_path)) if os.path.exists(summ_path) else {}
    for kname, lst in per.items():
        fam = "hicoo_mttkrp" if "Hicoo" in kname else (
            "coo_mttkrp" if ("CooSrc" in kname or "coo_staged" in kname) else (
                "ew" if "ew_kernel" in kname else None))
        if family:
            fam = family
        if not fam:
            continue
        db = [to_bytes(v["dram__bytes_read.sum"]) + to_bytes(v["dram__bytes_write.sum"]) for v in lst]
        summ.setdefault(config, {})[fam] = {
            "dram_bytes_per_launch": sum(db) / len(db), "launches_captured": len(db),
            "source": os.path.basename(path)}
    json.dump(summ, open(summ_path, "w"), indent=1)
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines[:40]))


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        full(sys.argv[2], sys.argv[3], sys.argv[4], sys.argv[5] if len(sys.argv) > 5 else None)
