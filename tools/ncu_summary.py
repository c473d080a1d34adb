"""Summarise ncu --set full reports (key metrics per kernel) into a text table.

    python tools/ncu_summary.py report.ncu-rep [...]
    python tools/ncu_summary.py --traffic OUT.json KEY=report.ncu-rep [...]
        writes {KEY: dram__bytes_read.sum + dram__bytes_write.sum} (bytes, first kernel of the
        report) into OUT.json, merged with what is there (the bench's roofline `traffic`)
"""
import json
import os
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "launch__grid_size", "launch__block_size",
        "launch__registers_per_thread", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__m_xbar2l1tex_read_bytes.sum", "lts__t_sectors.sum.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]


def raw(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def to_bytes(v, unit):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(unit, 1)
    return float(v.replace(",", "")) * scale


def traffic(out_path, pairs):
    d = json.load(open(out_path)) if os.path.exists(out_path) else {}
    for pr in pairs:
        key, path = pr.split("=", 1)
        rows = raw(path)
        if len(rows) < 3:
            print(path, "no data")
            continue
        h, u, v = rows[0], rows[1], rows[2]
        rd, wr = h.index("dram__bytes_read.sum"), h.index("dram__bytes_write.sum")
        d[key] = int(to_bytes(v[rd], u[rd]) + to_bytes(v[wr], u[wr]))
        d[key.replace("_dram_bytes", "_kernel")] = v[h.index("Kernel Name")][:120]
        print(key, d[key])
    json.dump(d, open(out_path, "w"), indent=1)


def main():
    if sys.argv[1] == "--traffic":
        return traffic(sys.argv[2], sys.argv[3:])
    for path in sys.argv[1:]:
        rows = raw(path)
        if len(rows) < 3:
            print(path, "no data")
            continue
        h, u = rows[0], rows[1]
        for v in rows[2:]:
            print(f"== {path}: {v[h.index('Kernel Name')][:100]}")
            for k in KEYS:
                if k in h:
                    i = h.index(k)
                    print(f"  {k:70s} {v[i]:>14s} {u[i]}")


if __name__ == "__main__":
    main()
