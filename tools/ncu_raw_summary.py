"""Summarise `ncu --page raw --csv` exports (and a launch list) into a markdown table.

    python tools/ncu_raw_summary.py --raw name=gpurun_out/x_raw.csv [--raw ...] \
        [--launches gpurun_out/launches.csv] [--updates N --bpu 1036]
"""
import argparse
import collections
import csv
import re

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput % of peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall long_scoreboard / issue"),
    ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "stall short_scoreboard / issue"),
    ("smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio", "stall lg_throttle / issue"),
    ("smsp__average_warps_issue_stalled_membar_per_issue_active.ratio", "stall membar / issue"),
]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def raw(path):
    rows = list(csv.reader(open(path)))
    h, u, v = rows[0], rows[1], rows[2]
    return {h[i]: (v[i], u[i]) for i in range(len(h))}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--raw", action="append", default=[])
    ap.add_argument("--launches")
    ap.add_argument("--updates", type=float, default=0)
    ap.add_argument("--bpu", type=float, default=0)
    a = ap.parse_args()
    cols = [(x.rsplit("=", 1)[0], raw(x.rsplit("=", 1)[1])) for x in a.raw]
    print("| metric | " + " | ".join(n for n, _ in cols) + " |")
    print("|---|" + "---|" * len(cols))
    for k, name in KEYS:
        print(f"| {name} (`{k}`) | " + " | ".join(f"{d.get(k, ('-', ''))[0]} {d.get(k, ('', ''))[1]}" for _, d in cols) + " |")
    for n, d in cols:
        try:
            rb = float(d["dram__bytes_read.sum"][0].replace(",", "")) * SCALE[d["dram__bytes_read.sum"][1]]
            wb = float(d["dram__bytes_write.sum"][0].replace(",", "")) * SCALE[d["dram__bytes_write.sum"][1]]
            print(f"\n- {n}: DRAM {(rb + wb) / 1e9:.2f} GB per launch", end="")
            if a.updates and a.bpu:
                print(f" = {(rb + wb) / (a.updates * a.bpu):.3f} of the algorithmic {a.updates * a.bpu / 1e9:.1f} GB", end="")
            print(f"; kernel `{d.get('Kernel Name', ('?',))[0][:90]}`")
        except (KeyError, ValueError):
            pass
    if a.launches:
        rows = [r for r in csv.reader(open(a.launches)) if r]
        start = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        hdr = rows[start]
        ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
        tot = collections.Counter()
        cnt = collections.Counter()
        for r in rows[start + 1:]:
            if len(r) > vi and r[mi] == "gpu__time_duration.sum":
                name = re.sub(r"\(.*", "", r[ki])[:70]
                tot[name] += float(r[vi].replace(",", ""))
                cnt[name] += 1
        allt = sum(tot.values())
        print("\n| launches | total ms | share | kernel |\n|---|---|---|---|")
        for name, t in tot.most_common(12):
            print(f"| {cnt[name]} | {t / 1e6:.3f} | {100 * t / allt:.1f}% | `{name}` |")


if __name__ == "__main__":
    main()
