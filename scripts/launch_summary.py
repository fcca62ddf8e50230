"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per
kernel: launches, total ms, share, median us.  Usage: launch_summary.py CSV..."""
import csv
import io
import statistics
import sys
from collections import defaultdict


def summarise(path):
    txt = open(path).read()
    i = txt.find('"ID"')
    rows = list(csv.DictReader(io.StringIO(txt[i:])))
    t = defaultdict(list)
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "")
        us = v / 1e3 if unit in ("ns", "nsecond") else v * 1e3 if unit in ("ms", "msecond") else v
        t[r["Kernel Name"].split("(")[0]].append(us)
    tot = sum(sum(v) for v in t.values())
    print(f"{len(rows)} launches, {tot / 1e3:.2f} ms of kernel time\n")
    print("| kernel | launches | total ms | share | median us |\n|---|---|---|---|---|")
    for k, v in sorted(t.items(), key=lambda kv: -sum(kv[1])):
        print(f"| `{k}` | {len(v)} | {sum(v) / 1e3:.3f} | {100 * sum(v) / tot:.1f} % | {statistics.median(v):.1f} |")


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(f"## {p.split('/')[-1]}\n")
        summarise(p)
        print()
