#!/usr/bin/env python
"""Summarise ncu evidence for profiles/ (run here, on the CPU box).

    python scripts/ncu_summary.py launches <launches.csv>          # per-kernel device time (launch list)
    python scripts/ncu_summary.py full <report.ncu-rep> [regex]    # key counters + hottest source lines
    python scripts/ncu_summary.py longest <report.ncu-rep> [regex] # the same for the longest matching launch only

The launch list is the `--metrics gpu__time_duration.sum --clock-control none`
pass (cold-cache, serialised: compare SHARES of the step, not absolutes).
"""

import collections
import gzip
import csv
import io
import re
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads per warp-inst (warp efficiency x32)"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("sass__inst_executed_local_loads", "local-memory loads (spills)"),
    ("sass__inst_executed_local_stores", "local-memory stores (spills)"),
]


def launches(path):
    rows = list(csv.reader(gzip.open(path, 'rt') if path.endswith('.gz') else open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.OrderedDict()
    total = 0.0
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        unit = r[ui]
        us = v / 1e3 if unit in ("ns", "nsecond") else (v * 1e3 if unit in ("ms", "msecond") else v)
        name = re.sub(r"\(.*", "", r[ki])[:70]
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += us
        total += us
    print(f"| kernel | launches | total us | share |\n|---|---|---|---|")
    for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"| `{k}` | {c} | {t:.1f} | {100 * t / total:.1f}% |")
    print(f"\n{sum(c for c, _ in agg.values())} launches, {total:.1f} us total")


def full(path, regex=None, longest=False):
    raw = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], stderr=subprocess.DEVNULL).decode()
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    body = rows[2:]
    if longest:  # only the longest launch (of the kernels matching regex)
        di = h.index("gpu__time_duration.sum")
        cand = [r for r in body if not regex or re.search(regex, r[h.index("Kernel Name")])]
        body = [max(cand, key=lambda r: float(r[di].replace(",", "")))] if cand else []
        print(f"(longest of {len(cand)} captured launches)\n")
    for r in body:
        name = r[h.index("Kernel Name")]
        if regex and not re.search(regex, name):
            continue
        print(f"### `{re.sub(r'[(].*', '', name)}`\n")
        print("| counter | value |\n|---|---|")
        for key, label in KEYS:
            if key in h:
                i = h.index(key)
                print(f"| {label} (`{key}`) | {r[i]} {units[i]} |")
        print()
    src = subprocess.check_output(["ncu", "-i", path, "--page", "source", "--csv"] + (["-k", f"regex:{regex}"] if regex else []),
                                  stderr=subprocess.DEVNULL).decode()
    srows = [r for r in csv.reader(io.StringIO(src))]
    hdr = next((r for r in srows if "Source" in r and "Address" in r), None)
    if hdr:
        si, ii, ci = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed"), hdr.index("Source")
        data = [r for r in srows if len(r) > ci and r[0].startswith("0x")]
        seen, out = set(), []
        for r in sorted(data, key=lambda r: -int(r[si] or 0)):
            if r[0] in seen:
                continue
            seen.add(r[0])
            out.append(r)
            if len(out) >= 12:
                break
        tot = sum(int(r[si] or 0) for r in data) or 1
        print("hottest SASS (stall samples, share, executions):\n")
        for r in out:
            print(f"    {int(r[si] or 0):7d} {100 * int(r[si] or 0) / tot:5.1f}% {r[ii]:>10}  {r[ci].strip()[:90]}")
        print()


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2])
    else:
        full(sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else None, longest=sys.argv[1] == "longest")
