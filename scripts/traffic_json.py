"""profiles/r02_traffic.json from the raw ncu exports of scripts/capture_r02.sh:
DRAM bytes per launch (dram__bytes_read.sum + dram__bytes_write.sum), keyed by
bench config and the bench's kernel name ("<kind> (prefill|decode)"), which
bench.py reads for roofline.traffic.

  python scripts/traffic_json.py profiles/r02b/ncu/*.raw.csv > profiles/r02b_traffic.json
"""
import csv
import io
import json
import os
import re
import sys

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
NAME = {"qkv": "qkv", "oproj": "o_proj", "gateup": "gate_up", "down": "down", "attn": "attn"}
CFG = {"c2": "sharegpt-8b", "c3": "arxiv-8b"}


def main():
    out = {}
    for p in sys.argv[1:]:
        m = re.match(r"r02b?_(c\d)_(\w+?)_(dec|pre)_p\d+\.raw\.csv", os.path.basename(p))
        if not m:
            continue
        r = list(csv.reader(io.StringIO(open(p).read())))
        d = dict(zip(r[0], r[2])); u = dict(zip(r[0], r[1]))
        b = sum(float(d[k]) * UNIT[u[k]] for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
        out.setdefault(CFG[m.group(1)], {})[f"{NAME[m.group(2)]} ({'prefill' if m.group(3) == 'pre' else 'decode'})"] = b
    print(json.dumps({"source": "ncu --set full --clock-control none captures, scripts/capture_r02.sh at the "
                      "bench splits (final round-2 kernels); bytes per launch = dram__bytes_read.sum + "
                      "dram__bytes_write.sum; keyed by bench config then kernel", "bytes": out}, indent=1))


if __name__ == "__main__":
    main()
