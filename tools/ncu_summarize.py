"""Summarise an ncu --set full report into profiles/ (profiling aid).

    python tools/ncu_summarize.py REPORT.ncu-rep OUT.csv [--traffic KEY1,KEY2,...]

Writes one row per captured kernel with duration, DRAM bytes, DRAM / L2 / tensor / issue
utilisation, registers, smem and SM clock.  With --traffic, the i-th kernel's
dram__bytes_read.sum + dram__bytes_write.sum is recorded in profiles/traffic.json under
the i-th key (the per-launch `traffic` bench.py reports).
"""
import csv
import io
import json
import os
import subprocess
import sys

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
           "lts__throughput.avg.pct_of_peak_sustained_elapsed",
           "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
           "sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
           "smsp__issue_active.avg.pct_of_peak_sustained_active",
           "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic", "sm__cycles_elapsed.avg.per_second"]


def main():
    rep, out = sys.argv[1], sys.argv[2]
    keys = sys.argv[sys.argv.index("--traffic") + 1].split(",") if "--traffic" in sys.argv else []
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units, data = rows[0], rows[1], rows[2:]
    cols = ["Kernel Name", "Grid Size", "Block Size"] + [m for m in METRICS if m in h]
    with open(out, "w", newline="") as f:
        wtr = csv.writer(f)
        wtr.writerow(cols)
        wtr.writerow([units[h.index(c)] for c in cols])
        for r in data:
            wtr.writerow([r[h.index(c)] for c in cols])
    print(open(out).read())
    if keys:
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        path = os.path.join(root, "profiles", "traffic.json")
        tj = json.load(open(path)) if os.path.exists(path) else {}
        mb = lambda r, c: float(r[h.index(c)].replace(",", "")) * (1e6 if units[h.index(c)] == "Mbyte" else 1e9 if units[h.index(c)] == "Gbyte" else 1e3 if units[h.index(c)] == "Kbyte" else 1)  # noqa: E731
        for k, r in zip(keys, data):
            if k:
                tj[k] = {"bytes_per_launch": mb(r, "dram__bytes_read.sum") + mb(r, "dram__bytes_write.sum"),
                         "source": f"{os.path.relpath(out, root)} (ncu --set full, dram__bytes_read.sum + dram__bytes_write.sum)"}
        json.dump(tj, open(path, "w"), indent=1)


if __name__ == "__main__":
    main()
