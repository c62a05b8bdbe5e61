"""Summarise ncu outputs into profiles/ (run here, on the CPU box).

  python scripts/ncu_summary.py launches gpurun_out/launches.csv  > profiles/rNN_launches.md
  python scripts/ncu_summary.py full gpurun_out/prof_fold.ncu-rep  > profiles/rNN_fold_full.md

`launches`: per-kernel count, total and mean device time from an
`ncu --metrics gpu__time_duration.sum` launch list, and each kernel's share of
the profiled time (cold-cache, serialised -- compare shares, not absolutes).
`full`: the key `--set full` metrics per profiled launch (duration, DRAM
bytes read/written, DRAM throughput, occupancy, registers, stall summary).
`traffic`: python scripts/ncu_summary.py traffic <config> [G]  reads
gpurun_out/full_{fold,stash}_<config>.ncu-rep and writes
profiles/traffic_<config>_g<G>.json (dram read + write bytes per launch), which
bench.py reports as roofline.traffic.
`steady`: python scripts/ncu_summary.py steady <csv> <config> [G]  reads an
`ncu --cache-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum` list of the default command's graph replays and merges the
per-launch mean DRAM bytes (dirty L2 lines of the previous kernel written back
under this one, as in the timed step) into profiles/traffic_<config>_g<G>.json
as <kernel>_dram_bytes_per_launch_steady; bench.py reports roofline.traffic_steady
and frac_steady from them.
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("dram__bytes.sum.per_second", "dram_rate"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct_peak"),
    ("lts__t_bytes.sum", "l2_bytes"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved_occupancy_pct"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_pct"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall_long_sb"),
]


def _csv_after_header(text):
    lines = text.splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    return list(csv.DictReader(lines[start:]))


def launches(path):
    rows = _csv_after_header(open(path).read())
    agg = collections.OrderedDict()
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"]
        short = name.split("(")[0].replace("void ", "")
        for k in ("k_fold", "k_stash", "k_swap"):
            if k in short:
                short = k + ("<bf16>" if "BF16T" in name and k != "k_swap" else "")
        ns = float(r["Metric Value"]) * (1000.0 if r.get("Metric Unit") == "us" else 1.0)
        a = agg.setdefault(short, [0, 0.0])
        a[0] += 1
        a[1] += ns
    total = sum(v[1] for v in agg.values()) or 1.0
    print(f"# ncu launch list: {path}\n")
    print("| kernel | launches | total us | mean us | share of profiled time |")
    print("|---|---|---|---|---|")
    for k, (n, ns) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"| {k} | {n} | {ns / 1e3:.1f} | {ns / n / 1e3:.2f} | {100 * ns / total:.1f} % |")


def full(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    print(f"# ncu --set full summary: {path}\n")
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")][:90]}
        for key, nice in KEYS:
            if key in hdr:
                i = hdr.index(key)
                d[nice] = f"{r[i]} {units[i]}".strip()
        print("```json\n" + json.dumps(d, indent=1) + "\n```")


def _raw(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def _bytes(v, unit):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[unit]
    return int(round(float(v.replace(",", "")) * scale))


def traffic(config, G="1", rnd="r01"):
    path = f"profiles/traffic_{config}_g{G}.json"
    d = json.load(open(path)) if os.path.exists(path) else {}     # keeps the *_steady entries
    for kname, tag in (("k_fold", "fold"), ("k_stash", "stash")):
        rep = f"gpurun_out/full_{tag}_{config}.ncu-rep"
        hdr, units, rows = _raw(rep)
        r = rows[0]
        rd, wr = hdr.index("dram__bytes_read.sum"), hdr.index("dram__bytes_write.sum")
        d[f"{kname}_dram_bytes_per_launch"] = _bytes(r[rd], units[rd]) + _bytes(r[wr], units[wr])
    d["source"] = (f"ncu --set full (profiles/{rnd}_k_fold_full_{config}.md, {rnd}_k_stash_full_{config}.md): "
                   "dram__bytes_read.sum + dram__bytes_write.sum per launch, cold cache; writes still dirty "
                   "in L2 at kernel end are not counted")
    with open(path, "w") as f:
        json.dump(d, f, indent=1)
        f.write("\n")
    print(path, d)


def steady(path, config, G="1"):
    rows = _csv_after_header(open(path).read())
    per = collections.defaultdict(lambda: collections.defaultdict(float))   # (kernel, launch id) -> metric
    for r in rows:
        name = r["Kernel Name"]
        k = next((k for k in ("k_fold", "k_stash") if k in name), None)
        if k is None:
            continue
        m, v, u = r["Metric Name"], float(r["Metric Value"].replace(",", "")), r.get("Metric Unit", "")
        if m.startswith("dram__bytes"):
            v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
        elif u == "us":
            v *= 1e3
        elif u == "ms":
            v *= 1e6
        per[(k, r["ID"])][m] += v
    tfile = f"profiles/traffic_{config}_g{G}.json"
    d = json.load(open(tfile)) if os.path.exists(tfile) else {}
    for k in ("k_fold", "k_stash"):
        ls = [v for (kk, _), v in per.items() if kk == k]
        if not ls:
            continue
        byt = sum(v["dram__bytes_read.sum"] + v["dram__bytes_write.sum"] for v in ls) / len(ls)
        ns = sum(v["gpu__time_duration.sum"] for v in ls) / len(ls)
        d[f"{k}_dram_bytes_per_launch_steady"] = int(round(byt))
        d[f"{k}_steady_launches"] = len(ls)
        d[f"{k}_steady_mean_us"] = round(ns / 1e3, 2)
    d["source_steady"] = (f"{path}: ncu --cache-control none over the default command's CUDA-graph replays "
                          "(after the eager warm-up), mean dram__bytes_read + write per launch: dirty L2 lines a "
                          "kernel leaves are written back (and counted) under the next, as in the timed step")
    with open(tfile, "w") as f:
        json.dump(d, f, indent=1)
        f.write("\n")
    print(tfile, d)


if __name__ == "__main__":
    {"launches": launches, "full": full, "traffic": traffic, "steady": steady}[sys.argv[1]](*sys.argv[2:])
