"""Summarise ncu outputs into profiles/ (committed evidence).

    python tools/ncu_summary.py --rep gpurun_out/prof.ncu-rep --launches gpurun_out/launches.csv \
        --name r01_netflix_fp16_hogwild --key netflix/hogwild/fp16/k128 --updates 99072112 \
        --bytes-per-update 1036

Writes profiles/<name>.md (launch-list shares + the top kernel's key metrics) and merges the
per-launch DRAM traffic into profiles/ncu_traffic.json (read by bench.py's roofline.traffic).
"""
import argparse
import collections
import csv
import io
import json
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput % of peak"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_active", "L1 throughput %"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock"),
]


def raw_metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2:]
    return hdr, units, vals


def to_bytes(v, unit):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


def to_ms(v, unit):
    f = float(v.replace(",", ""))
    return f * {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1, "msecond": 1,
                "s": 1e3, "second": 1e3}.get(unit, 1)


def launches(path):
    rows = [r for r in csv.reader(open(path)) if r]
    start = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[start]
    ki, mi, vi, ui = (hdr.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    agg = collections.OrderedDict()
    for r in rows[start + 1:]:
        if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
            continue
        name = re.sub(r"\(.*", "", r[ki]).replace("void ", "")
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += to_ms(r[vi], r[ui])
    return agg


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rep")
    ap.add_argument("--launches")
    ap.add_argument("--name", required=True)
    ap.add_argument("--key", required=True)
    ap.add_argument("--updates", type=float, required=True, help="updates per launch")
    ap.add_argument("--bytes-per-update", type=float, required=True)
    ap.add_argument("--note", default="")
    a = ap.parse_args()
    lines = [f"# ncu summary: {a.name}", "", f"config key `{a.key}`. {a.note}", ""]
    traffic = None
    if a.rep:
        hdr, units, vals = raw_metrics(a.rep)
        v = vals[0]
        lines += [f"## top kernel (`ncu --set full`, {os.path.basename(a.rep)})", "",
                  f"kernel: `{v[hdr.index('Kernel Name')]}`", "", "| metric | value |", "|---|---|"]
        got = {}
        for k, label in KEYS:
            if k in hdr:
                i = hdr.index(k)
                got[k] = (v[i], units[i])
                lines.append(f"| {label} (`{k}`) | {v[i]} {units[i]} |")
        rd = to_bytes(*got["dram__bytes_read.sum"])
        wr = to_bytes(*got["dram__bytes_write.sum"])
        ms = to_ms(*got["gpu__time_duration.sum"])
        alg = a.updates * a.bytes_per_update
        traffic = rd + wr
        stalls = []
        for i, h in enumerate(hdr):
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                try:
                    stalls.append((float(v[i]), h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
                except ValueError:
                    pass
        stalls.sort(reverse=True)
        lines += ["", f"- DRAM traffic per launch: {traffic/1e9:.2f} GB "
                  f"(read {rd/1e9:.2f} + write {wr/1e9:.2f}); algorithmic {alg/1e9:.2f} GB "
                  f"({a.updates:.0f} updates x {a.bytes_per_update:.0f} B) -> traffic/algorithmic "
                  f"{traffic/alg:.3f}",
                  f"- algorithmic bandwidth under ncu (cold, serialised): {alg/ms/1e6:.1f} GB/s; "
                  f"DRAM bandwidth {traffic/ms/1e6:.1f} GB/s",
                  "- top stall reasons (warp cycles per issued instruction): " +
                  ", ".join(f"{n} {x:.2f}" for x, n in stalls[:6]), ""]
    if a.launches:
        agg = launches(a.launches)
        tot = sum(x[1] for x in agg.values())
        lines += [f"## launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`, "
                  f"{os.path.basename(a.launches)})", "",
                  "cold-cache, serialised per-launch times of the whole bench command (data "
                  "generation, one-time preprocessing, warm-up and timed epochs): compare SHARES.",
                  "", "| launches | total ms | share | kernel |", "|---|---|---|---|"]
        for k, (c, ms) in sorted(agg.items(), key=lambda x: -x[1][1])[:20]:
            lines.append(f"| {c} | {ms:.3f} | {100*ms/tot:.1f}% | `{k[:100]}` |")
        lines.append("")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", a.name + ".md"), "w") as f:
        f.write("\n".join(lines))
    if traffic is not None:
        path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        d = json.load(open(path)) if os.path.exists(path) else {}
        d[a.key] = {"dram_bytes_per_launch": traffic, "source": a.name,
                    "algorithmic_bytes_per_launch": a.updates * a.bytes_per_update}
        with open(path, "w") as f:
            json.dump(d, f, indent=1, sort_keys=True)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
