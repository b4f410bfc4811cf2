"""Per-row measurement suites for bench.py (``python bench.py --suite X``).
Each prints ONE JSON line for its BASELINE.json config.  All device times
are CUDA-graph replays timed with CUDA events on the launching stream."""
from __future__ import annotations

import json
import os
import statistics
import time

import numpy as np
import torch

import ifl_inputs as gen
import paper_conf_ppopp_henriksenteo19_b200 as ifl

ROOT = os.path.dirname(os.path.abspath(__file__))


def gtime(fn, R=4, reps=3):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    fn()
    e1.record()
    torch.cuda.synchronize()
    one = e0.elapsed_time(e1)
    if one > 50.0:
        return one
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(R):
            fn()
    g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / R)
    return statistics.median(ts)


NOMINAL_HBM = 8000.0  # GB/s (north_star "~8 TB/s")
# f32 FMA (CUDA cores) peak: 148 SMs x 128 FMA/clk x 2 flop x 1.965 GHz
FMA_TFLOPS = 148 * 128 * 2 * 1.965e9 / 1e12


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), float(d["bf16_tflops"]), "measured (MEASURED_PEAKS.json)"
    return 6650.0, 1590.0, "fallback (B200_PROFILING.md)"


def base_line(metric, value, unit, cfg, hib=True, dtype="f32"):
    return {"metric": metric, "value": value, "unit": unit, "n_gpus": 1, "higher_is_better": hib,
            "vs_baseline": None, "dtype": dtype, "data": "synthetic", "config": cfg}


# ------------------------------------------------------------------ config 0


def suite_config0():
    import oracle
    n = m = 1024
    x = gen.matrix("I32_FULL", 1, n, m)
    xd = x.cuda()
    out = torch.empty(n, dtype=torch.int32, device="cuda")
    ws = ifl.workspace(ifl.workspace_bytes("segred", n, m, dt="i32"))
    res = {}
    for v in ("top", "middle", "flat", "auto"):
        res[v] = gtime(lambda: ifl.segred(xd, out=out, ws=ws, version=v)) * 1e3
        assert np.array_equal(out.cpu().numpy(), oracle.segred(x.numpy(), "sum"))
    t0 = time.perf_counter()
    for _ in range(5):
        oracle.segred(x.numpy(), "sum")
    cpu_s = (time.perf_counter() - t0) / 5
    line = base_line("int32 segmented sum latency, 1024x1024 (configs[0])", round(res["auto"], 3), "us",
                     {"workload": "configs[0] int32 segred sum 1024x1024", "per_version_us": res}, hib=False,
                     dtype="int32")
    line["cpu_baseline"] = {"value": round(cpu_s * 1e6, 1), "unit": "us", "cores": 1, "kind": "oracle",
                            "sample": "full 1024x1024"}
    line["note"] = "4.2 MB is L2-resident and below launch latency: latency, not a bandwidth roofline"
    return line


# ------------------------------------------------------------------ redomap2


def mm_shapes(k):
    return [(1 << a, 1 << (k - 2 * a), 1 << a) for a in range(0, k // 2 + 1)]


def suite_redomap2():
    hbm, tc_peak, src = peaks()
    rows = []
    tuned = {}
    for dt, tdt, site, ktrain, ks in (("bf16", torch.bfloat16, "redomap2.bf16", (28, 31), (30,)),
                                      ("f32", torch.float32, "redomap2.f32", (23, 27), (25,))):
        # P:138 protocol (tune on other constant-work families than the test
        # one): training families bracket the test size, as for the sweep --
        # k = 28 and 31 (bf16) / 23 and 27 (f32), testing k = 30 / 25
        train = [s for kt in ktrain for s in mm_shapes(kt)]
        need = ifl.lib().ifl_tune_scratch_bytes(site.encode(), np.asarray(train, np.int64).ctypes.data, len(train))
        scratch = torch.zeros(need, dtype=torch.uint8, device="cuda")
        a, b, tbl = ifl.tune(site, train, reps=7, cost=1, scratch=scratch)
        tuned[site] = {"t_top": a, "t_intra": b}
        del scratch
        for k in ks:
            for (n, m, p) in mm_shapes(k):
                A = gen.generate("BF16_SIGNED", 6, n * m, device="cuda").view(n, m).to(tdt)
                Bt = gen.generate("BF16_SIGNED", 7, p * m, device="cuda").view(p, m).to(tdt)
                C = torch.empty(n, p, device="cuda")
                ws = ifl.workspace(ifl.workspace_bytes("redomap2", n, m, p, dt), "cuda", "mm")
                r = {"dt": dt, "k": k, "n": n, "m": m, "p": p}
                for v in ("top", "middle", "flat", "auto"):
                    hopeless = (v == "middle" and (n * p > (1 << 22) or m >= (1 << 24))) or \
                               (v == "top" and dt == "f32" and n * p < 64 and m >= (1 << 22)) or \
                               (v == "flat" and n * p > (1 << 24))
                    r[v] = None if hopeless else gtime(lambda: ifl.redomap2(A, Bt, out=C, ws=ws, version=v)) * 1e3
                r["chosen"] = ifl.redomap2(A, Bt, out=C, ws=ws, return_choice=True)[1].version
                best = min(t for t in (r["top"], r["middle"], r["flat"]) if t is not None)
                r["best_over_auto"] = best / r["auto"]
                r["flops"] = 2.0 * n * m * p
                r["bytes"] = (2 if dt == "bf16" else 4) * (n * m + m * p) + 4 * n * p
                # per-shape roofline: max(bytes / HBM, flops / tensor or FMA peak)
                fpeak = tc_peak if dt == "bf16" else FMA_TFLOPS
                r["auto_GBps"] = r["bytes"] / (r["auto"] * 1e-6) / 1e9
                r["frac_of_8TBps"] = r["auto_GBps"] / NOMINAL_HBM
                r["frac_of_measured_hbm"] = r["auto_GBps"] / hbm
                r["roofline_us"] = max(r["bytes"] / (hbm * 1e9), r["flops"] / (fpeak * 1e12)) * 1e6
                r["frac_of_roofline"] = r["roofline_us"] / r["auto"]
                # B given as yss [m][p] (b_kmajor = 0), AUTO: read in place by V_FLAT
                if r["chosen"] == "flat":
                    Bm = Bt.t().contiguous()
                    r["auto_rowmajor_B"] = gtime(lambda: ifl.redomap2(A, Bm, b_kmajor=False, out=C, ws=ws)) * 1e3
                    r["rowmajor_over_kmajor"] = r["auto_rowmajor_B"] / r["auto"]
                    del Bm
                rows.append(r)
                del A, Bt, C
    # dense bf16 square (tensor-core roofline)
    sq = {}
    for q in (2048, 4096, 8192):
        A = gen.generate("BF16_SIGNED", 6, q * q, device="cuda").view(q, q).to(torch.bfloat16)
        Bt = gen.generate("BF16_SIGNED", 7, q * q, device="cuda").view(q, q).to(torch.bfloat16)
        C = torch.empty(q, q, device="cuda")
        t = gtime(lambda: ifl.redomap2(A, Bt, out=C, version="top"), R=2)
        sq[q] = {"us": t * 1e3, "TFLOPs": 2.0 * q ** 3 / (t * 1e-3) / 1e12}
        del A, Bt, C
    tot_t = sum(r["auto"] for r in rows if r["dt"] == "bf16" and r["k"] == 30)
    tot_b = sum(r["bytes"] for r in rows if r["dt"] == "bf16" and r["k"] == 30)
    line = base_line("map-map-redomap (matmul-shaped) sweep throughput, configs[2] k=30 bf16",
                     round(tot_b / (tot_t * 1e-6) / 1e9, 1), "GB/s",
                     {"workload": "configs[2]: A[2^a][2^(k-2a)] x B[2^(k-2a)][2^a], test k=30 (bf16) / 25 (f32), "
                                  "tuned on k=28+31 / 23+27 (P:138 protocol)", "thresholds": tuned}, dtype="bf16")
    line["min_shape_best_over_auto"] = round(min(r["best_over_auto"] for r in rows), 4)
    k30 = [r for r in rows if r["dt"] == "bf16" and r["k"] == 30]
    line["k30_per_shape"] = [{"n": r["n"], "m": r["m"], "chosen": r["chosen"], "auto_us": round(r["auto"], 1),
                              "GBps": round(r["auto_GBps"]), "frac_of_8TBps": round(r["frac_of_8TBps"], 3),
                              "frac_of_roofline": round(r["frac_of_roofline"], 3),
                              "rowmajor_over_kmajor": round(r.get("rowmajor_over_kmajor", float("nan")), 3)}
                             for r in k30]
    top = sq[8192]
    line["roofline"] = {"bound": "tensor", "kernel": "mm_top_tc_kernel (8192^3 bf16)",
                        "achieved": round(top["TFLOPs"], 1), "peak": tc_peak, "unit": "TFLOP/s",
                        "frac": round(top["TFLOPs"] / tc_peak, 4), "traffic": None, "peak_source": src}
    line["dense_square"] = sq
    line["shapes"] = rows
    return line


# -------------------------------------------------------------------- tridag

LVC = {"small": (16, 256, 32, 256), "medium": (128, 64, 256, 32), "large": (256, 64, 256, 256)}


def sites(ds):
    numS, numT, numX, numY = LVC[ds]
    return [(numS * numX, numY, numX), (numS * numY, numX, numY)], numT


def suite_tridag():
    hbm, _, src = peaks()
    # tune on other data (seed 9) over the small and large datasets' sites
    train = [s for ds in ("small", "large") for s in sites(ds)[0]]
    need = ifl.lib().ifl_tune_scratch_bytes(b"tridag", np.asarray(train, np.int64).ctypes.data, len(train))
    scratch = torch.zeros(need, dtype=torch.uint8, device="cuda")
    a_, b_, tbl = ifl.tune("tridag", train, reps=7, cost=1, scratch=scratch)
    del scratch
    rows = []
    for ds in ("small", "medium", "large"):
        shp, numT = sites(ds)
        for (S, L, R) in shp:
            a, b, c, y = (t.cuda() for t in gen.tridag_system(7, S, L, R))
            x = torch.empty_like(y)
            ws = ifl.workspace(ifl.workspace_bytes("tridag", S, L, R), "cuda", "tri")
            r = {"dataset": ds, "S": S, "L": L, "R": R, "numT": numT}
            for v in ("top", "middle", "flat", "auto"):
                if v == "middle" and L > 4096:
                    r[v] = None
                    continue
                r[v] = gtime(lambda: ifl.tridag(a, b, c, y, out=x, ws=ws, version=v)) * 1e3
            r["chosen"] = ifl.tridag(a, b, c, y, out=x, ws=ws, return_choice=True)[1].version
            best = min(t for t in (r["top"], r["middle"], r["flat"]) if t is not None)
            r["best_over_auto"] = best / r["auto"]
            r["GBps"] = 8.0 * S * L / (r["auto"] * 1e-6) / 1e9
            rows.append(r)
    # whole-run time per dataset: numT steps x both sites (P:400 structure)
    per_ds = {}
    for ds in ("small", "medium", "large"):
        rr = [r for r in rows if r["dataset"] == ds]
        per_ds[ds] = {"ms_numT_steps": sum(r["auto"] for r in rr) * rr[0]["numT"] / 1e3,
                      "GBps": sum(8.0 * r["S"] * r["L"] for r in rr) / (sum(r["auto"] for r in rr) * 1e-6) / 1e9}
    large = [r for r in rows if r["dataset"] == "large"]
    ach = sum(8.0 * r["S"] * r["L"] for r in large) / (sum(r["auto"] for r in large) * 1e-6) / 1e9
    line = base_line("batched tridiagonal solves via three scans (LocVolCalib sites), large dataset",
                     round(ach, 1), "GB/s",
                     {"workload": "configs[3]: LocVolCalib small/medium/large per-site tridag (P:402), "
                                  "tuned on small+large with other data", "thresholds": {"t_top": a_, "t_intra": b_}})
    line["per_dataset"] = per_ds
    line["min_shape_best_over_auto"] = round(min(r["best_over_auto"] for r in rows), 4)
    line["roofline"] = {"bound": "hbm", "kernel": "tridag (large, both sites, AUTO)", "achieved": round(ach, 1),
                        "peak": hbm, "unit": "GB/s", "frac": round(ach / hbm, 4), "traffic": None,
                        "peak_source": src}
    line["sites"] = rows
    return line


# ----------------------------------------------------------------------- lvc

# FP32 lanes x SMs: the ALU roof for V_OUTER, which keeps every system in
# registers for all numT steps (no HBM traffic inside the loop).  Algorithmic
# work per element and step = the Thomas recurrences with the loop-invariant
# elimination hoisted: 1 FMA (forward), 1 MUL (1/beta), 1 FMA (backward).
LVC_OPS_PER_ELEM_STEP = 3


def alu_peak_ops(sm_mhz=1965.0):
    return 148 * 128 * sm_mhz * 1e6


def suite_lvc():
    """NEXT-1: the whole LocVolCalib loop of Fig 6a
    dataset, every version of Fig 6c plus the outermost branch (V_OUTER), the
    per-site G3 tuned as in the tridag suite and the outermost t0 tuned on
    reduced-numT copies of the datasets (the tuner sees other data)."""
    hbm, _, src = peaks()
    ifl.reset_thresholds()
    train = [s for ds in ("small", "large") for s in sites(ds)[0]]
    need = ifl.lib().ifl_tune_scratch_bytes(b"tridag", np.asarray(train, np.int64).ctypes.data, len(train))
    scratch = torch.zeros(need, dtype=torch.uint8, device="cuda")
    ifl.tune("tridag", train, reps=7, cost=1, scratch=scratch)
    del scratch
    ltrain = [(S, 8, X, Y) for (S, T, X, Y) in gen.LVC_DATASETS.values()]
    t0, _, ltbl = ifl.tune("lvc", ltrain, reps=7, cost=1)
    rows = []
    for ds, (S, T, X, Y) in gen.LVC_DATASETS.items():
        (ax, bx, cx), (ay, by, cy), xs, ys = gen.lvc_problem(17, S, X, Y, "cuda")
        xc, yc = (ax, bx, cx), (ay, by, cy)
        E = S * X * Y
        r = {"dataset": ds, "numS": S, "numT": T, "numX": X, "numY": Y}
        for v in ("outer", "top", "middle", "flat", "auto"):
            r[v + "_ms"] = gtime(lambda: ifl.lvc(xs, ys, xc, yc, T, version=v), R=2)
        r["chosen"] = ifl.lvc(xs, ys, xc, yc, T, return_choice=True).version
        best = min(r[v + "_ms"] for v in ("outer", "top", "middle", "flat"))
        best_step = min(r[v + "_ms"] for v in ("top", "middle", "flat"))
        r["best_over_auto"] = round(best / r["auto_ms"], 4)
        r["speedup_outer_vs_best_per_step"] = round(best_step / r["outer_ms"], 3)
        # per-step traffic the stepwise versions must move (read y + write x per
        # element, both sites); V_OUTER moves it once for the whole loop
        r["per_step_equiv_GBps"] = round(8.0 * 2 * E * T / (r["auto_ms"] * 1e-3) / 1e9, 1)
        r["alu_Gops"] = round(LVC_OPS_PER_ELEM_STEP * 2 * E * T / (r["outer_ms"] * 1e-3) / 1e9, 1)
        rows.append(r)
    peak = alu_peak_ops()
    large = [r for r in rows if r["dataset"] == "large"][0]
    ach = LVC_OPS_PER_ELEM_STEP * 2 * (256 * 256 * 256) * 64 / (large["outer_ms"] * 1e-3)
    line = base_line("LocVolCalib loop (Fig 6a): numT steps of tridag on both sites, large dataset",
                     round(large["auto_ms"], 4), "ms", {"workload": "SURVEY 8(f) NEXT-1: whole LocVolCalib-shaped "
                     "program, P:402 datasets, coefficients loop-invariant", "t0": t0}, hib=False)
    line["per_dataset"] = rows
    line["lvc_tune_table_ms"] = ltbl.tolist()
    line["min_shape_best_over_auto"] = min(r["best_over_auto"] for r in rows)
    line["roofline"] = {"bound": "alu", "kernel": "lvc_outer_kernel (large)", "achieved": round(ach / 1e12, 3),
                        "peak": round(peak / 1e12, 2), "unit": "Tops/s (FP32 lanes x SMs x 1965 MHz)",
                        "frac": round(ach / peak, 4), "traffic": None,
                        "note": f"{LVC_OPS_PER_ELEM_STEP} Thomas ops per element and step; HBM peak {hbm} GB/s ({src})"}
    return line


# ----------------------------------------------------------------------- col


def suite_col():
    """NEXT-3: column (axis-0) segred / segscan, G4,
    over the same constant-work sweep as configs[1]: [n][m] f32 with
    n*m = 2^26, n = 2^k.  Thresholds tuned on the 2^25 and 2^27 sweeps
    (bracketing, other data); every forced version timed where it can occupy the GPU
    (TOP needs >= 4096 column threads, MIDDLE >= 64 column tiles -- the
    others run a few threads for seconds and are reported as null)."""
    hbm, _, src = peaks()
    ifl.reset_thresholds()
    L2N = 26
    sh = [(1 << k, 1 << (L2N - k)) for k in range(L2N + 1)]
    tuned = {}
    for site in ("colred.b4", "colscan.b4"):
        train = [(1 << k, 1 << (lg - k)) for lg in (25, 27) for k in range(lg + 1)]
        need = ifl.lib().ifl_tune_scratch_bytes(site.encode(), np.asarray(train, np.int64).ctypes.data, len(train))
        scratch = torch.empty(need, dtype=torch.uint8, device="cuda")
        scratch.view(-1)[: (need // 4) * 4].view(torch.float32).copy_(gen.generate("F32_UNIT", 4, need // 4, "cuda"))
        a, b, _ = ifl.tune(site, train, reps=7, cost=1, scratch=scratch)
        del scratch
        tuned[site] = {"t_top": a, "t_intra": b}
    N = 1 << L2N
    xs = gen.generate("F32_UNIT", 2, N, device="cuda")
    out = torch.empty(N, dtype=torch.float32, device="cuda")
    ws = ifl.workspace(max(ifl.workspace_bytes("colscan", n, m) for n, m in sh), "cuda", "colsuite")
    rows = []
    for kind in ("colred", "colscan"):
        fn = ifl.colscan if kind == "colscan" else ifl.colred
        for (n, m) in sh:
            x = xs.view(n, m)
            o = out.view(n, m) if kind == "colscan" else out[:m]
            r = {"op": kind, "n": n, "m": m}
            for v in ("top", "middle", "flat", "auto"):
                if (v == "top" and m < 4096 * (4 if m % 4 == 0 else 1)) or (v == "middle" and (m + 127) // 128 < 64):
                    r[v] = None
                    continue
                r[v] = gtime(lambda: fn(x, out=o, ws=ws, version=v)) * 1e3
            r["chosen"] = fn(x, out=o, ws=ws, return_choice=True)[1].version
            best = min(t for t in (r["top"], r["middle"], r["flat"]) if t is not None)
            r["best_over_auto"] = round(best / r["auto"], 4)
            byt = (8 * n * m) if kind == "colscan" else 4 * (n * m + m)
            r["GBps"] = round(byt / (r["auto"] * 1e-6) / 1e9, 1)
            rows.append(r)
    tot_b = sum((8 * r["n"] * r["m"]) if r["op"] == "colscan" else 4 * (r["n"] * r["m"] + r["m"]) for r in rows)
    tot_t = sum(r["auto"] for r in rows)
    agg = tot_b / (tot_t * 1e-6) / 1e9
    line = base_line("colred/colscan GB/s over the n x m sweep (G4 axis-0 reductions)", round(agg, 1), "GB/s",
                     {"workload": "SURVEY 8(f) NEXT-3: column segred + segscan, f32 sum, n*m = 2^26, n = 2^0..2^26, "
                                  "AUTO with tuned thresholds", "thresholds": tuned})
    line["min_shape_best_over_auto"] = min(r["best_over_auto"] for r in rows)
    line["roofline"] = {"bound": "hbm", "kernel": "colred+colscan sweep (AUTO)", "achieved": round(agg, 1),
                        "peak": hbm, "unit": "GB/s", "frac": round(agg / hbm, 4), "traffic": None,
                        "peak_source": src}
    line["shapes"] = rows
    return line


# -------------------------------------------------------------------- segred2


def seg2_shapes(lg):
    out = []
    for a in range(0, lg + 1, 2):  # n = 2^a, the rest split between m and k
        r = lg - a
        out.append((1 << a, 1 << (r // 2), 1 << (r - r // 2)))
    return out


def suite_seg2():
    """NEXT-2 (ii): the nested reduce (G9's e_rec),
    sum of per-segment maxima over [n][m][k] f32 with n*m*k = 2^26; thresholds
    from ifl_tune_search over forced-version timings of the 2^25 / 2^27 sets."""
    hbm, _, src = peaks()
    ifl.reset_thresholds()

    def run(lg, seed, versions):
        x = gen.generate("F32_SIGNED", seed, 1 << lg, "cuda")
        out = torch.empty(1 << lg, device="cuda")
        res = []
        for (n, m, k) in seg2_shapes(lg):
            xv = x.view(n, m, k)
            ws = ifl.workspace(ifl.workspace_bytes("segred2", n, m, k), "cuda", "seg2")
            r = {"n": n, "m": m, "k": k}
            for v in versions:
                if v == "top" and n < 4096:
                    r[v] = None  # a few threads walking 2^14+ elements each: cannot win
                    continue
                r[v] = gtime(lambda: ifl.segred2(xv, "sum", "max", version=v, out=out[:n], ws=ws)) * 1e3
            if "auto" in versions:
                r["chosen"] = ifl.segred2(xv, "sum", "max", out=out[:n], ws=ws, return_choice=True)[1].version
            res.append(r)
        return res

    pt, pm, tbl = [], [], []
    for lg in (25, 27):
        for r in run(lg, 30 + lg, ("top", "middle", "flat")):
            c = ifl.select("segred2.b4", r["n"], r["m"])
            pt.append(c.par_top)
            pm.append(c.par_mid)
            tbl.append([float("inf") if r[v] is None else r[v] for v in ("top", "middle", "flat")])
    a, b, npaths = ifl.tune_search(pt, pm, tbl, cost=1)
    ifl.set_thresholds("segred2.b4", a, b)
    rows = run(26, 2, ("top", "middle", "flat", "auto"))
    for r in rows:
        best = min(r[v] for v in ("top", "middle", "flat") if r[v] is not None)
        r["best_over_auto"] = round(best / r["auto"], 4)
        r["GBps"] = round((4 * r["n"] * r["m"] * r["k"] + 4 * r["n"]) / (r["auto"] * 1e-6) / 1e9, 1)
    tot = sum(4 * r["n"] * r["m"] * r["k"] + 4 * r["n"] for r in rows) / (sum(r["auto"] for r in rows) * 1e-6) / 1e9
    line = base_line("nested reduce (sum of per-segment max) GB/s over [n][m][k] shapes", round(tot, 1), "GB/s",
                     {"workload": "SURVEY 8(f) NEXT-2 (ii): f32, n*m*k = 2^26, n = 4^0..4^13", "thresholds":
                      {"t_top": a, "t_intra": b, "paths": npaths}})
    line["min_shape_best_over_auto"] = min(r["best_over_auto"] for r in rows)
    line["roofline"] = {"bound": "hbm", "kernel": "segred2 sweep (AUTO)", "achieved": round(tot, 1), "peak": hbm,
                        "unit": "GB/s", "frac": round(tot / hbm, 4), "traffic": None, "peak_source": src}
    line["shapes"] = rows
    return line


# -------------------------------------------------------------------- mmtree


def suite_mmtree():
    """NEXT-2: the 5-leaf branching tree of matrix
    multiplication (row-level G3 leaves ROW_TOP / ROW_MIDDLE, then TOP /
    MIDDLE / FLAT over the two-map context), f32, on the paper's Fig 2 family
    A[2^a][2^(k-2a)] x B[2^(k-2a)][2^a]: thresholds tuned on k = 20
    and applied to k = 25 (the paper's protocol), by the chain search over
    every distinct tree path (Fig 5); the 3-leaf tuning of the same
    training set is timed beside it."""
    ifl.reset_thresholds()
    train, test = mm_shapes(20), mm_shapes(25)
    # 3-leaf tuning (the row level off), then the 5-leaf tree
    # the k = 20 shapes run for microseconds: 9 repetitions (median) per leaf
    a3, b3, _ = ifl.tune("redomap2.f32", train, reps=9, cost=1)
    t_top, t_intra, tbl = ifl.tune("redomap2.f32.tree", train, reps=9, cost=1)
    rt, ri = ifl.get_thresholds("redomap2.f32.row")
    rows = []
    for (n, m, p) in test:
        A = gen.generate("F32_SIGNED", 6, n * m, "cuda").view(n, m)
        Bt = gen.generate("F32_SIGNED", 7, p * m, "cuda").view(p, m)
        C = torch.empty(n, p, device="cuda")
        ws = ifl.workspace(ifl.workspace_bytes("redomap2", n, m, p, "f32"), "cuda", "mmtree")
        r = {"n": n, "m": m, "p": p}
        for v in ("row_top", "row_middle", "top", "middle", "flat"):
            if v == "row_middle" and m > 8192:
                r[v] = None
                continue
            r[v] = gtime(lambda: ifl.redomap2(A, Bt, out=C, ws=ws, version=v)) * 1e3
        r["auto5"] = gtime(lambda: ifl.redomap2(A, Bt, out=C, ws=ws)) * 1e3
        r["chosen5"] = ifl.redomap2(A, Bt, out=C, ws=ws, return_choice=True)[1].version
        ifl.set_thresholds("redomap2.f32.row", 2**63 - 1, 2**63 - 1)
        ifl.set_thresholds("redomap2.f32", a3, b3)
        r["auto3"] = gtime(lambda: ifl.redomap2(A, Bt, out=C, ws=ws)) * 1e3
        r["chosen3"] = ifl.redomap2(A, Bt, out=C, ws=ws, return_choice=True)[1].version
        ifl.set_thresholds("redomap2.f32.row", rt, ri)
        ifl.set_thresholds("redomap2.f32", t_top, t_intra)
        best = min(r[v] for v in ("row_top", "row_middle", "top", "middle", "flat") if r[v] is not None)
        r["best_over_auto5"] = round(best / r["auto5"], 4)
        r["best_over_auto3"] = round(best / r["auto3"], 4)
        rows.append(r)
    t5, t3 = sum(r["auto5"] for r in rows), sum(r["auto3"] for r in rows)
    line = base_line("matmul branching tree (5 leaves) on the Fig 2 family, k = 25, f32: total us", round(t5, 2),
                     "us", {"workload": "SURVEY 8(f) NEXT-2: A[2^a][2^(25-2a)] x B, a = 0..12, tuned on k = 20",
                            "thresholds": {"row": [rt, ri], "two_map": [t_top, t_intra], "three_leaf_only": [a3, b3]}},
                     hib=False)
    line["total_us_3leaf"] = round(t3, 2)
    line["speedup_5leaf_vs_3leaf"] = round(t3 / t5, 4)
    line["min_shape_best_over_auto5"] = min(r["best_over_auto5"] for r in rows)
    line["min_shape_best_over_auto3"] = min(r["best_over_auto3"] for r in rows)
    line["train_cost_table_ms"] = tbl.tolist()
    line["shapes"] = rows
    return line


# -------------------------------------------------------------------- segarg


def suite_arg():
    """NEXT-3: the tuple-valued per-row argmin (NN's
    argmin P:474) over the configs[1] constant-work sweep, f32, n*m = 2^26.
    Thresholds from ifl_tune_search over forced-version timings of the 2^25
    and 2^27 sweeps (other data, bracketing the test size as in bench.py); a thread-per-row TOP on fewer than 4096 rows
    runs for seconds and is reported as null (cannot win)."""
    hbm, _, src = peaks()
    ifl.reset_thresholds()

    def sweep(lg, seed, versions):
        x = gen.generate("F32_SIGNED", seed, 1 << lg, "cuda")
        out = (torch.empty(1 << lg, device="cuda"), torch.empty(1 << lg, dtype=torch.int32, device="cuda"))
        ws = ifl.workspace(max(ifl.workspace_bytes("segarg", 1 << k, 1 << (lg - k)) for k in range(lg + 1)) + 16,
                           "cuda", "argsuite")
        res = []
        for k in range(lg + 1):
            n, m = 1 << k, 1 << (lg - k)
            xv = x.view(n, m)
            o = (out[0][:n], out[1][:n])
            r = {"n": n, "m": m}
            for v in versions:
                if v == "top" and n < 4096:
                    r[v] = None
                    continue
                r[v] = gtime(lambda: ifl.segarg(xv, "min", version=v, out=o, ws=ws)) * 1e3
            if "auto" in versions:
                r["chosen"] = ifl.segarg(xv, "min", out=o, ws=ws, return_choice=True)[1].version
            res.append(r)
        return res

    pt, pm, tbl = [], [], []
    for lg in (25, 27):
        for r in sweep(lg, 5 + lg, ("top", "middle", "flat")):
            c = ifl.select("segarg.b4", r["n"], r["m"])
            pt.append(c.par_top)
            pm.append(c.par_mid)
            tbl.append([float("inf") if r[v] is None else r[v] for v in ("top", "middle", "flat")])
    a, b, npaths = ifl.tune_search(pt, pm, tbl, cost=1)
    ifl.set_thresholds("segarg.b4", a, b)
    rows = sweep(26, 2, ("top", "middle", "flat", "auto"))
    for r in rows:
        best = min(r[v] for v in ("top", "middle", "flat") if r[v] is not None)
        r["best_over_auto"] = round(best / r["auto"], 4)
        r["GBps"] = round((4 * r["n"] * r["m"] + 8 * r["n"]) / (r["auto"] * 1e-6) / 1e9, 1)
    tot = sum(4 * r["n"] * r["m"] + 8 * r["n"] for r in rows) / (sum(r["auto"] for r in rows) * 1e-6) / 1e9
    line = base_line("per-row argmin (tuple-valued reduce) GB/s over the n x m sweep", round(tot, 1), "GB/s",
                     {"workload": "SURVEY 8(f) NEXT-3: f32 argmin, n*m = 2^26, n = 2^0..2^26, AUTO tuned on the "
                                  "2^25 / 2^27 sweeps", "thresholds": {"t_top": a, "t_intra": b, "paths": npaths}})
    line["min_shape_best_over_auto"] = min(r["best_over_auto"] for r in rows)
    line["roofline"] = {"bound": "hbm", "kernel": "segarg sweep (AUTO)", "achieved": round(tot, 1), "peak": hbm,
                        "unit": "GB/s", "frac": round(tot / hbm, 4), "traffic": None, "peak_source": src}
    line["shapes"] = rows
    return line


# ----------------------------------------------------------------------- irr


def _irr_case(seed, total_log2, mean):
    n = max(1, (1 << total_log2) // int(mean))
    off = gen.irregular_offsets(seed, n, float(mean))
    return off


def suite_irr():
    """NEXT-4: irregular segments -- segred + segscan
    over Pareto(1.5)-distributed segment lengths (the heavy-tailed degree
    distributions of graph / sparse workloads), ~2^26 f32 elements, mean
    length 2^0..2^16.  The inspector (ifl_irr_inspect, timed separately)
    supplies max_len for the guard's imbalance measure; thresholds come from
    the exact search (ifl_tune_search) over forced-version timings of the same
    sweep at 2^24 and 2^27 elements with other seeds."""
    hbm, _, src = peaks()
    ifl.reset_thresholds()
    means = [1 << k for k in range(0, 17, 2)]

    def run_case(off, seed, versions, R=4):
        offd = torch.from_numpy(off).cuda()
        total = int(off[-1])
        x = gen.generate("F32_UNIT", seed, total, "cuda")
        ob = torch.empty(max(total, off.size - 1), device="cuda")
        t0 = time.perf_counter()
        mx = ifl.irr_inspect(offd, total)
        t_insp = (time.perf_counter() - t0) * 1e3
        ws = ifl.workspace(ifl.workspace_bytes("segscan_irr", off.size - 1, total), "cuda", "irrsuite")
        r = {}
        for kind in ("segred", "segscan"):
            fn = ifl.segscan_irr if kind == "segscan" else ifl.segred_irr
            o = ob[:total] if kind == "segscan" else ob[: off.size - 1]
            for v in versions:
                r[(kind, v)] = gtime(lambda: fn(x, offd, out=o, ws=ws, version=v, max_len=mx), R=R) * 1e3
            r[(kind, "choice")] = fn(x, offd, out=o, ws=ws, max_len=mx, return_choice=True)[1]
        return r, mx, total, t_insp

    # ---- tune (other seeds, bracketing sizes)
    thr = {}
    tabs = {"segred": ([], [], []), "segscan": ([], [], [])}
    for lg in (24, 27):
        for k, mean in enumerate(means):
            off = _irr_case(200 + k + lg, lg, mean)
            r, mx, total, _ = run_case(off, 300 + k, ("top", "middle", "flat"), R=2)
            for kind in ("segred", "segscan"):
                c = ifl.select(kind + ".irr", off.size - 1, total, mx)
                tabs[kind][0].append(c.par_top)
                tabs[kind][1].append(c.par_mid)
                tabs[kind][2].append([r[(kind, "top")], r[(kind, "middle")], r[(kind, "flat")]])
    for kind in ("segred", "segscan"):
        a, b, npaths = ifl.tune_search(tabs[kind][0], tabs[kind][1], tabs[kind][2], cost=1)
        ifl.set_thresholds(kind + ".irr", a, b)
        thr[kind + ".irr"] = {"t_top": a, "t_intra": b, "paths": npaths}
    # ---- test sweep (2^26)
    rows = []
    for k, mean in enumerate(means):
        off = _irr_case(100 + k, 26, mean)
        r, mx, total, t_insp = run_case(off, 2, ("top", "middle", "flat", "auto"))
        n = off.size - 1
        for kind in ("segred", "segscan"):
            byt = (8 * total + 8 * (n + 1)) if kind == "segscan" else (4 * total + 4 * n + 8 * (n + 1))
            row = {"op": kind, "mean": mean, "n": n, "total": total, "max_len": mx, "inspect_ms": round(t_insp, 3),
                   "chosen": r[(kind, "choice")].version}
            for v in ("top", "middle", "flat", "auto"):
                row[v] = round(r[(kind, v)], 2)
            best = min(row["top"], row["middle"], row["flat"])
            row["best_over_auto"] = round(best / row["auto"], 4)
            row["GBps"] = round(byt / (row["auto"] * 1e-6) / 1e9, 1)
            row["bytes"] = byt
            rows.append(row)
    agg = sum(r["bytes"] for r in rows) / (sum(r["auto"] for r in rows) * 1e-6) / 1e9
    line = base_line("irregular segred/segscan GB/s over a Pareto segment-length sweep (P:532)", round(agg, 1),
                     "GB/s", {"workload": "SURVEY 8(f) NEXT-4: f32 sum, ~2^26 elements, Pareto(1.5) lengths, mean "
                                          "2^0..2^16, AUTO with the inspector's max_len and tuned thresholds",
                              "thresholds": thr})
    line["min_shape_best_over_auto"] = min(r["best_over_auto"] for r in rows)
    line["roofline"] = {"bound": "hbm", "kernel": "irregular sweep (AUTO, data + offsets bytes)",
                        "achieved": round(agg, 1), "peak": hbm, "unit": "GB/s", "frac": round(agg / hbm, 4),
                        "traffic": None, "peak_source": src}
    line["shapes"] = rows
    return line


# ---------------------------------------------------------------------- dist


def suite_dist():
    """configs[4]: 2^30-element f32 segred on this GPU through dist.py with a
    world-1 NCCL communicator: outer (no collective) and inner (one
    all_reduce) splits, n in {1, 2^4, 2^10, 2^16, 2^20, 2^24}."""
    import socket

    import torch.distributed as td

    from paper_conf_ppopp_henriksenteo19_b200 import dist
    hbm, _, src = peaks()
    if not td.is_initialized():
        s = socket.socket()
        s.bind(("127.0.0.1", 0))
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(s.getsockname()[1]))
        s.close()
        td.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    # the local segreds run AUTO with thresholds tuned as the bench tunes them
    # (V_MIDDLE group size, then the 4-leaf chain on the 2^25 / 2^27 sweeps)
    train = [(1 << k, 1 << (lg - k)) for lg in (25, 27) for k in range(lg + 1)]
    g, _, _ = ifl.tune("segred.b4.midg", [s for s in train if s[1] <= 8192], reps=7, cost=1)
    nb = ifl.lib().ifl_tune_scratch_bytes(b"segred.b4.tree", np.asarray(train, np.int64).ctypes.data, len(train))
    scratch = torch.empty(nb, dtype=torch.uint8, device="cuda")
    scratch.view(-1)[: (nb // 4) * 4].view(torch.float32).copy_(gen.generate("F32_UNIT", 4, nb // 4, device="cuda"))
    ifl.tune("segred.b4.tree", train, reps=7, cost=1, scratch=scratch)
    del scratch
    N = 1 << 30
    x = gen.generate("F32_UNIT", 8, N, device="cuda")
    rows = []
    for lg in (0, 4, 10, 16, 20, 24):
        n, m = 1 << lg, N >> lg
        xv = x.view(n, m)
        r = {"n": n, "m": m}
        for mode, t_dev in (("outer", 1), ("inner", 2), ("auto", None)):
            plan = dist.plan_segred(n, m, 1, 0, t_dev)
            t = gtime(lambda: dist.segred_dist(xv, n, m, "sum", plan=plan), R=2)
            r[mode + "_us"] = t * 1e3
            r[mode + "_GBps"] = 4.0 * (N + n) / (t * 1e-3) / 1e9
        rows.append(r)
    # the line's value: the whole n sweep through the default device-level
    # guard (bytes of all shapes / their total time); the best shape beside it
    sweep = sum(4.0 * (N + r["n"]) for r in rows) / (sum(r["auto_us"] for r in rows) * 1e-6) / 1e9
    best = max(max(r["outer_GBps"], r["inner_GBps"]) for r in rows)
    line = base_line("2^30-element segmented reduce, GB/s per GPU (configs[4])", round(sweep, 1), "GB/s",
                     {"workload": "configs[4]: 2^30 f32 segred via dist.py over n in {1, 2^4, 2^10, 2^16, 2^20, "
                                  "2^24}, world size 1 on this box (default device-level guard)"})
    line["scaling"] = "weak"
    line["thresholds"] = {"segred.b4": list(ifl.get_thresholds("segred.b4")),
                          "segred.b4.cl": list(ifl.get_thresholds("segred.b4.cl")), "group_shift": g - 8}
    line["best_shape_GBps"] = round(best, 1)
    line["rows"] = rows
    line["roofline"] = {"bound": "hbm", "kernel": "segred sweep (read-only stream: the copy peak counts a read "
                                                "and a write)", "achieved": round(sweep, 1), "peak": hbm,
                        "unit": "GB/s", "frac": round(sweep / hbm, 4), "traffic": None, "peak_source": src}
    return line


SUITES = {"config0": suite_config0, "redomap2": suite_redomap2, "tridag": suite_tridag, "dist": suite_dist,
          "lvc": suite_lvc, "col": suite_col, "irr": suite_irr, "arg": suite_arg, "mmtree": suite_mmtree,
          "seg2": suite_seg2}
