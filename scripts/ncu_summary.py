"""Summarise ncu reports (.ncu-rep, or their `--page raw --csv` exports) into
a markdown table: duration, SM clock, tensor-pipe %, DRAM bytes read/written,
DRAM %, achieved occupancy."""
import csv, io, subprocess, sys

KEYS = [("gpu__time_duration.sum", "us"), ("sm__cycles_elapsed.avg.per_second", "GHz"),
        ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor %"),
        ("dram__bytes_read.sum", "DRAM read"), ("dram__bytes_write.sum", "DRAM write"),
        ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM %"),
        ("sm__warps_active.avg.pct_of_peak_sustained_active", "occupancy %"),
        ("launch__registers_per_thread", "regs"), ("launch__grid_size", "grid")]


def rows(path):
    """Rows of a report (.ncu-rep, read through ncu) or of its exported raw page (.csv)."""
    if path.endswith(".csv"):
        out = open(path).read()
    else:
        out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units = r[0], r[1]
    for row in r[2:]:
        d = dict(zip(hdr, row)); u = dict(zip(hdr, units))
        yield d, u


def main():
    print("| report | kernel | " + " | ".join(k[1] for k in KEYS) + " |")
    print("|---" * (len(KEYS) + 2) + "|")
    for p in sys.argv[1:]:
        for d, u in rows(p):
            name = d.get("Kernel Name", "")[:40]
            vals = []
            for k, _ in KEYS:
                v = d.get(k, "")
                vals.append(f"{v} {u.get(k, '')}".strip())
            print(f"| {p.split('/')[-1]} | {name} | " + " | ".join(vals) + " |")


if __name__ == "__main__":
    main()
