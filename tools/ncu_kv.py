"""Print selected metrics of ncu raw CSV captures side by side:
    python tools/ncu_kv.py a.raw.csv b.raw.csv ... [-g regex]"""
import csv
import re
import sys

files = [a for a in sys.argv[1:] if a.endswith(".csv")]
pat = None
if "-g" in sys.argv:
    pat = re.compile(sys.argv[sys.argv.index("-g") + 1])
DEFAULT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
           "launch__registers_per_thread", "launch__grid_size", "launch__occupancy_limit_shared_mem",
           "sm__maximum_warps_per_active_cycle_pct"]
cols = []
for f in files:
    rows = list(csv.reader(open(f)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    cols.append(dict(zip(hdr, zip(vals, units))))
keys = [k for k in cols[0] if pat.search(k)] if pat else DEFAULT
for k in keys:
    print(f"{k[:80]:80s}", "  ".join(f"{c.get(k, ('-', ''))[0]:>14s}" for c in cols), cols[0].get(k, ("", ""))[1])
