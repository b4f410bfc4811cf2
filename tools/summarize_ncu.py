"""Summarise gpurun_out/ncu/ into profiles/ (launch-list shares, per-kernel
DRAM traffic vs algorithmic bytes, key full-set metrics)."""
import csv
import glob
import json
import os
import sys
from collections import defaultdict

src = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ncu"
tag = sys.argv[2] if len(sys.argv) > 2 else "r01"
os.makedirs("profiles", exist_ok=True)

# ---- launch list
rows = []
with open(os.path.join(src, "launches.csv")) as fp:
    lines = [l for l in fp if l.startswith('"')]
rd = csv.reader(lines)
hdr = next(rd)
ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
agg = defaultdict(lambda: [0, 0.0])
for r in rd:
    if r[mi] != "gpu__time_duration.sum":
        continue
    name = r[ki].split("(")[0].replace("void ", "").strip()
    v = float(r[vi].replace(",", ""))
    unit = hdr[vi]
    agg[name][0] += 1
    agg[name][1] += v
tot = sum(v[1] for v in agg.values())
with open(f"profiles/{tag}_ncu_launches_summary.csv", "w") as fp:
    fp.write("kernel,launches,total_time,share\n")
    for k, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        fp.write(f"{k},{c},{t:.1f},{t / tot:.4f}\n")

# ---- full captures
ALG = {  # algorithmic bytes of the captured launch
    "segscan_flat_n1": 8 * 2**26, "segscan_flat_n4096": 8 * 2**26, "segscan_flat_n65536": 8 * 2**26, "segred_flat_n1": 4 * (2**26 + 1),
    "segred_middle_n2e16": 4 * (2**26 + 65536), "segscan_middle_n2e18": 8 * 2**26,
    "segred_top_n2e24": 4 * (2**26 + 2**24), "segscan_top_n2e23": 8 * 2**26,
    "redomap2_tc_8192": 2 * (2 * 8192 * 8192) + 4 * 8192 * 8192, "redomap2_flat_n1": 2 * (2 * 2**30) + 4,
    "redomap2_flat_n8": 2 * (16 * 2**24) + 4 * 64, "segred_flat_n4096": 4 * (2**26 + 4096),
    "segred_cluster_n16": 4 * (2**26 + 16),
    "tridag_middle_large": 8 * 65536 * 256, "tridag_flat_large": 8 * 65536 * 256,
    "lvc_outer_large": 2 * 8 * 256 * 256 * 256,  # one read + one write per element for the whole loop
    "colred_flat_n2e20": 4 * 2**26, "colscan_top_n4": 8 * 2**26, "colscan_flat_n2e26": 8 * 2**26,
}
GROUP = {"segscan_flat_n1": "segscan_flat", "segscan_flat_n65536": "segscan_flat_dlb", "segred_flat_n1": "segred_flat", "segred_middle_n2e16": "segred_middle",
         "segscan_middle_n2e18": "segscan_middle", "segred_top_n2e24": "segred_top", "segscan_top_n2e23": "segscan_top",
         "redomap2_tc_8192": "redomap2_tc", "redomap2_flat_n1": "redomap2_flat", "redomap2_flat_n8": "redomap2_flat",
         "segred_cluster_n16": "segred_cluster", "tridag_middle_large": "tridag_middle",
         "tridag_flat_large": "tridag_flat", "lvc_outer_large": "lvc_outer", "colred_flat_n2e20": "colred_flat",
         "colscan_top_n4": "colscan_top", "colscan_flat_n2e26": "colscan_flat",
         "segred_irr_flat_m1k": "segred_irr_flat", "segscan_irr_flat_m1k": "segscan_irr_flat"}
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio"]
traffic = {}
md = [f"# ncu summary ({tag})\n", "Full-set captures (`--set full --clock-control none`, one launch each, "
      "cold cache), from `tools/profile_round.sh`.  traffic = dram read + write; alg = algorithmic bytes "
      "(SURVEY 8(d)).  DRAM % = gpu__dram_throughput (of ncu's DRAM peak); tensor % = "
      "sm__pipe_tensor_cycles_active (of active cycles) / bf16 dense op rate (of peak, elapsed).\n",
      "| capture | kernel | time | DRAM read | DRAM write | traffic / alg | DRAM % peak | "
      "L2 hit % | warps active % | issue active % | tensor pipe % | bf16 MMA % |",
      "|---|---|---|---|---|---|---|---|---|---|---|---|"]
for f in sorted(glob.glob(os.path.join(src, "*.raw.csv"))):
    name = os.path.basename(f).replace(".raw.csv", "")
    with open(f) as fp:
        rr = list(csv.reader(fp))
    h, units, data = rr[0], rr[1], rr[2:]
    if not data:
        continue
    d = dict(zip(h, data[-1]))
    u = dict(zip(h, units))

    def num(k, scale_to=None):
        v = float(d.get(k, "nan").replace(",", ""))
        un = u.get(k, "")
        if scale_to == "B":
            v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(un, 1)
        if scale_to == "us":
            v *= {"nsecond": 1e-3, "usecond": 1, "msecond": 1e3}.get(un, 1)
        return v
    t_us = num("gpu__time_duration.sum", "us")
    rdb, wrb = num("dram__bytes_read.sum", "B"), num("dram__bytes_write.sum", "B")
    alg = ALG.get(name)
    ratio = (rdb + wrb) / alg if alg else float("nan")
    kern = d.get("Kernel Name", "?").split("(")[0].replace("void ", "")
    md.append(f"| {name} | `{kern}` | {t_us:.1f} us | {rdb / 1e6:.1f} MB | {wrb / 1e6:.1f} MB | {ratio:.3f} | "
              f"{num('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed'):.1f} | "
              f"{num('lts__t_sector_hit_rate.pct'):.1f} | "
              f"{num('sm__warps_active.avg.pct_of_peak_sustained_active'):.1f} | "
              f"{num('smsp__issue_active.avg.pct_of_peak_sustained_active'):.1f} | "
              f"{num('sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active'):.1f} | "
              f"{num('sm__ops_path_tensor_op_hmma_src_bf16_dst_fp32_sparsity_off.avg.pct_of_peak_sustained_elapsed'):.1f} |")
    if name in GROUP:
        traffic[GROUP[name]] = {"capture": name, "dram_bytes_per_launch": rdb + wrb, "algorithmic_bytes": alg,
                                "ratio": round(ratio, 4), "ncu_time_us": round(t_us, 2)}
md.append("\nLaunch-list shares (`--metrics gpu__time_duration.sum`, bench command with "
          "`--steps 2 --warmup 3 --no-e2e --no-cpu --no-forced`): `profiles/%s_ncu_launches_summary.csv`." % tag)
open(f"profiles/{tag}_ncu_summary.md", "w").write("\n".join(md) + "\n")
json.dump(traffic, open("profiles/ncu_traffic.json", "w"), indent=1)
print("\n".join(md))
print(json.dumps(traffic, indent=1))
