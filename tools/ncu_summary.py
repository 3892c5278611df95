#!/usr/bin/env python
"""Per-launch summary of an ncu report (--page raw): kernel, duration, DRAM bytes, L2 hit
rate, L2 throughput, issue activity, warps active -- the numbers profiles/r02_*.md quote.

    python tools/ncu_summary.py gpurun_out/l2split_c5.ncu-rep [--json out.json]
"""
import csv
import io
import json
import subprocess
import sys

METRICS = {
    "gpu__time_duration.sum": "duration_ms",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum": "l2_read_hit_sectors",
    "lts__t_sectors_srcunit_tex_op_read.sum": "l2_read_sectors",
    "lts__t_bytes.sum": "l2_bytes",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_throughput_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct",
    "smsp__inst_executed.sum": "warp_instructions",
}
UNITS = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1.0, "Tbyte": 1e12, "msecond": 1.0, "usecond": 1e-3,
         "nsecond": 1e-6, "second": 1e3}


def main():
    rep = sys.argv[1]
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    out = []
    for row in rows[2:]:
        d = {"kernel": row[h.index("Kernel Name")][:90], "id": row[h.index("ID")]}
        for m, k in METRICS.items():
            if m in h:
                i = h.index(m)
                try:
                    val = float(row[i].replace(",", ""))
                except ValueError:
                    continue
                d[k] = val * UNITS.get(units[i], 1.0)
        out.append(d)
    for d in out:
        print(json.dumps(d))
    if "--json" in sys.argv:
        with open(sys.argv[sys.argv.index("--json") + 1], "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
