"""Write profiles/<tag>_summary.md from the round's bench and suite lines
(headline, per-row results) plus the hand-written change / gap notes below."""
import json
import sys

tag = sys.argv[1] if len(sys.argv) > 1 else "r02"
b = json.load(open(f"profiles/{tag}_bench.json"))
L = ["# Round 2 summary (B200, sm_100a)", "",
     "Evidence files are in this directory (`" + tag + "_*`); design, readings and measured alternatives in `DESIGN.md`.",
     "", "## Headline (`bench.py`, configs[1] sweep, N = 1)", ""]
r = b["roofline"]
L.append(f"* {b['value']} GB/s = {b['frac_of_8TBps'] * 100:.1f} % of 8 TB/s, {b['frac_of_measured_hbm'] * 100:.1f} % of the "
         f"measured {r['peak']} GB/s copy peak; {b['ms_per_step']} ms per step (54 calls); "
         f"{b['speedup_vs_best_single_version']}x the best single version; every shape within "
         f"{100 - b['min_shape_best_over_auto'] * 100:.1f} % of its best version.")
L.append(f"* Dominant kernel `{r['kernel']}`: {r['achieved']} GB/s = {r['frac']} of the measured peak "
         f"(ncu DRAM traffic / algorithmic bytes {r['traffic']['ratio']}).")
L.append(f"* e2e through the C ABI from pinned host memory: {b['e2e']['value']} GB/s (PCIe-bound). Parity of every "
         f"timed call: {b['parity']['calls_checked']} checked, {b['parity']['failed']} failed. Clocks "
         f"{b['clocks']['sm_mhz']} MHz, reasons {b['clocks']['reasons']}.")
L.append(f"* CPU oracle baseline: {b['cpu_baseline']['value']} GB/s on {b['cpu_baseline']['cores']} core.")
L += ["", "## Rows (suites, `bench.py --suite X`)", "", "| suite | value | roofline frac | min best/auto |",
      "|---|---|---|---|"]
for s in ["config0", "redomap2", "tridag", "dist", "lvc", "col", "irr", "arg", "mmtree", "seg2"]:
    d = json.load(open(f"profiles/{tag}_suite_{s}.json"))
    rr = d.get("roofline") or {}
    mb = [v for k, v in d.items() if k.startswith("min_shape_best_over_auto")]
    L.append(f"| {s} | {d['value']} {d['unit']} | {rr.get('frac', '-')} | {min(mb) if mb else '-'} |")
L += ["", "Per-shape minima under 0.90 are on 7-12 µs calls (tridag small, redomap2 k = 25 n = 128..512, seg2) "
      "and move run to run; mmtree's is structural (see gaps).", "", "## What changed this round (second session)", ""]
for t in [
    "Irregular segments V_FLAT rebuilt on a merge path over segment ends and elements: equal work per tile for any "
    "length mix, thread starts claimed by the ends, a walk chosen per tile density, lead elements scanned in a second "
    "pass, cp.async element staging, parallel two-kernel tile scan; sweep 1.49 -> 2.99 TB/s (designs measured: "
    "`DESIGN.md` section 5, launch lists `" + tag + "_irr_designs.md`).",
    "redomap2 reads B given as yss [m][p] in place everywhere it matters: SIMT tile kernels, the skinny engine "
    "(XOR-swizzled cooperative slice copies) and the tcgen05 kernel (MN-major UMMA descriptors, 0.986x the k-major "
    "time at 8192^3).",
    "Skinny V_FLAT engine is one kernel (last CTA per output tile sums the k-splits deterministically); finer "
    "k-chunks on small problems (k = 25 n = p = 1: 88 -> 65 us).",
    "V_MIDDLE of redomap2: groups of 1-8 warps per output when few outputs reduce a long k.",
    "bench.py: native stdout writes (NCCL banner) go to stderr, stdout carries the JSON line only.",
    "Tests: merge-path edge descriptors, full-size (2^26) irregular parity at means 1 / 64 / 65536 for both "
    "operations, irregular segments past 2^31 elements, row-major B over every SIMT tile config and the tcgen05 kernel "
    "(1024^3, ragged p, 8192^3 first/last tiles), skinny finalize determinism and counter re-arming; smoke covers "
    "the irregular engine and the MN-major operand.",
    "Job-ring parameter sweep (chunk tiles, lag, slots x CTAs): the shipped point is the local optimum.",
]:
    L.append("* " + t)
L += ["", "## Known gaps", ""]
for t in [
    "Matmul tree on the Fig 2 family (train k = 20, test k = 25): min best/auto ~0.45 -- the guard's Par_mid is "
    "constant along the family (`DESIGN.md` section 8).",
    "Flat segscan on long rows (job ring) at 0.855 of the copy peak; segscan rows of 2048-4096 elements.",
    "Irregular V_FLAT at 0.46 of the copy peak: one tile per CTA is bounded by CTA launches and per-tile round trips.",
    "Multi-GPU paths are tested with gloo world 2 and NCCL world 1 only (one GPU per gpurun call).",
    "compute-sanitizer is closed on this pool since the first session: the merge-path and skinny-finalize kernels "
    "have no sanitizer logs (parity and determinism tests only).",
]:
    L.append("* " + t)
open(f"profiles/{tag}_summary.md", "w").write("\n".join(L) + "\n")
print("\n".join(L[:12]))
