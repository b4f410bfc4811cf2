"""Host-side tests of the C ABI (no GPU needed): the library loads, exports
every entry point include/ifl.h declares, validates arguments before any
launch, and the G3 selector / threshold table / tuner search behave as the
paper's rules say."""
import ctypes
import math
import os
import re

import numpy as np
import pytest

import paper_conf_ppopp_henriksenteo19_b200 as ifl

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_ppopp_henriksenteo19_b200 import build
    build.build()
    lib = ifl.lib()
    ifl.reset_thresholds()
    yield lib
    ifl.reset_thresholds()


def header_functions():
    src = open(os.path.join(ROOT, "include", "ifl.h")).read()
    return sorted(set(re.findall(r"^\s*(?:int|size_t|const char\*)\s+(ifl_\w+)\s*\(", src, re.M)))


def test_exports_every_declared_symbol(L):
    names = header_functions()
    assert len(names) >= 19
    for n in names:
        assert hasattr(L, n), n
        assert n in ifl.EXPORTED, f"binding lacks {n}"


def test_binary_is_sm100a():
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", ifl.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_build_info(L):
    assert "sm_100a" in ifl.build_info()


# ----------------------------------------------------------- validation


def _segred(L, inp, out, n, m, dt=1, op=0, f=0, version=-1):
    return L.ifl_segred(inp, out, n, m, dt, op, f, None, version, None, 0, None, None)


def test_validation_errors(L):
    E = ifl.IFL_EINVAL
    assert _segred(L, 256, 512, -1, 4) == E
    assert _segred(L, 256, 512, 4, -1) == E
    assert _segred(L, 0, 512, 4, 4) == E                 # NULL input
    assert _segred(L, 256, 0, 4, 4) == E                 # NULL output
    assert _segred(L, 256, 1 << 40, 1 << 40, 1 << 40) == E  # n*m overflows
    assert _segred(L, 258, 512, 4, 4) == E               # misaligned element pointer
    assert _segred(L, 256, 512, 4, 4, dt=2) == ifl.IFL_EUNSUPPORTED  # bf16 segred
    assert _segred(L, 256, 512, 4, 4, dt=1, op=4) == ifl.IFL_EUNSUPPORTED  # AND on f32
    assert _segred(L, 256, 512, 4, 4, op=9) == E
    assert _segred(L, 256, 512, 4, 4, f=5) == E
    assert _segred(L, 256, 512, 4, 4, version=7) == E
    assert _segred(L, 4096, 4096 + 8, 4, 4) == E         # out overlaps in
    # segscan: in place is fine (validated only), partial overlap is not
    assert L.ifl_segscan(4096, 4096 + 4, 4, 4, 1, 0, 0, None, 0, -1, None, 0, None, None) == E
    assert L.ifl_segscan(4096, 4096, 4, 4, 1, 0, 0, None, 2, -1, None, 0, None, None) == E  # reverse is 0 or 1
    assert "reverse" in L.ifl_last_error().decode()
    assert L.ifl_segscan(4096, 4096, 0, 4, 1, 0, 0, None, 1, -1, None, 0, None, None) == 0   # reverse, n = 0: no-op


def test_empty_n_is_noop(L):
    c = ifl.ifl_choice()
    assert L.ifl_segred(256, 512, 0, 100, 1, 0, 0, None, -1, None, 0, None, ctypes.byref(c)) == 0
    assert L.ifl_segscan(256, 512, 0, 100, 0, 0, 0, None, 0, -1, None, 0, None, None) == 0


def test_flat_requires_workspace(L):
    # forced V_FLAT with no workspace is refused before launching anything
    assert _segred(L, 256, 1 << 30, 4, 1 << 16, version=2) == ifl.IFL_EWORKSPACE
    assert ifl.workspace_bytes("segred", 4, 1 << 16, version="flat") > 0
    assert ifl.workspace_bytes("segred", 4, 1 << 16, version="top") == 0
    assert ifl.workspace_bytes("segred", 4, 1 << 16, version="auto") == ifl.workspace_bytes(
        "segred", 4, 1 << 16, version="flat")


def test_redomap2_tridag_validation(L):
    assert L.ifl_redomap2(256, 512, 1024, -1, 2, 2, 1, 1, -1, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_redomap2(256, 512, 1024, 2, 2, 2, 0, 1, -1, None, 0, None, None) == ifl.IFL_EUNSUPPORTED
    assert L.ifl_redomap2(256, 512, 0, 2, 2, 2, 1, 1, -1, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_tridag(256, 256, 256, 256, 256, 4, 4, 0, -1, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_tridag(256, 256, 256, 256, 0, 4, 4, 1, -1, None, 0, None, None) == ifl.IFL_EINVAL
    # forced V_MIDDLE on a system too long for shared memory: the A-fit clause
    assert L.ifl_tridag(256, 256, 256, 256, 512, 4, 1 << 20, 1, 1, None, 0, None, None) == ifl.IFL_ENOTFIT


# ------------------------------------------------------------- selector


def test_default_thresholds_are_2_pow_15(L):
    ifl.reset_thresholds()
    for s in ifl.SITES:
        if s.endswith((".row", ".cl")):  # the matmul row level / the cluster level are off until tuned (R17, R18)
            assert ifl.get_thresholds(s) == (2**63 - 1, 2**63 - 1)
        elif s.endswith(".midg"):  # V_MIDDLE group-size exponent 0, biased by 8 (R19)
            assert ifl.get_thresholds(s) == (8, 0)
        else:
            assert ifl.get_thresholds(s) == (2**15, 2**15)


@pytest.mark.parametrize("site", ["segred.b4", "segscan.b4"])
def test_cluster_level_guard_chain(L, site):
    """Reading R18: TOP -> MIDDLE -> CLUSTER -> FLAT; Par_cl = n*min(m, 8192);
    the cluster level is off by default (the paper's three versions), and a
    segscan row that does not fit 16 shared-memory pieces never takes it."""
    ifl.reset_thresholds()
    assert ifl.select(site, 4, 1 << 20).version == "flat"               # default: no cluster leaf
    ifl.set_thresholds(site, 1 << 20, 1 << 30)                           # TOP / MIDDLE guards fail below
    ifl.set_thresholds(site + ".cl", 1 << 15, 0)
    assert ifl.select(site, 4, 1 << 19).version == "cluster"             # Par_cl = 4 * 8192 >= 2^15
    assert ifl.select(site, 3, 1 << 19).version == "flat"                # 3 * 8192 < 2^15
    assert ifl.select(site, 64, 100).version == "flat"                   # 64 * 100 < 2^15
    assert ifl.select(site, 1 << 20, 4).version == "top"                 # the outer guard still first
    if site == "segscan.b4":
        assert ifl.select(site, 4, 16 * 40960 + 4).version == "flat"     # does not fit: never CLUSTER
        assert ifl.select(site, 4, 16 * 40960).version == "cluster"
    ifl.reset_thresholds()


@pytest.mark.parametrize("site", ["segred.b4", "segscan.b4"])
def test_g3_guard_truth_table(L, site):
    """if Par(Sigma') >= t_top then e_top else if Par(e_middle) >=
    t_intra then e_middle else e_flat; Par(Sigma') = n, Par(e_middle) =
    n*min(m, 1024) (R3) or n*m (R2); ties go to the outer version (R1)."""
    ifl.set_thresholds(site, 1000, 50000)
    for mode in (1, 0):
        ifl.set_par_mode(mode)
        for n in (1, 7, 48, 49, 999, 1000, 1001, 100000):
            for m in (1, 16, 1024, 1025, 1 << 20):
                c = ifl.select(site, n, m)
                pm = n * min(m, 1024) if mode == 1 else n * m
                want = "top" if n >= 1000 else ("middle" if pm >= 50000 else "flat")
                assert (c.version, c.par_top, c.par_mid) == (want, n, pm), (mode, n, m)
                assert (c.t_top, c.t_intra) == (1000, 50000)
    ifl.set_par_mode(1)
    ifl.reset_thresholds()


def test_fig6c_guards_on_locvolcalib(L):
    # Fig 6c: numS*numX > t1 -> version 1, numS*numX*numY > t2 -> version 2.
    ifl.set_par_mode(0)
    # Y-site of the small dataset: numS*numY = 4096 systems of length numX = 32
    ifl.set_thresholds("tridag", 4097, 131073)
    assert ifl.select("tridag", 16 * 256, 32).version == "flat"     # 4096 < t1, 131072 < t2
    ifl.set_thresholds("tridag", 4097, 131072)
    assert ifl.select("tridag", 16 * 256, 32).version == "middle"   # 131072 >= t2
    assert ifl.select("tridag", 256 * 256, 256).version == "top"    # large: 65536 >= t1
    ifl.set_par_mode(1)
    ifl.reset_thresholds()


def test_monotone_single_crossover(L):
    """Along a constant-work sweep n*m = 2^26 the chosen version moves
    outward monotonically: FLAT -> MIDDLE -> TOP as n grows."""
    rank = {"flat": 0, "middle": 1, "top": 2}
    for tt, ti in [(2**15, 2**15), (2**20, 2**18), (16, 2**30), (2**27, 1)]:
        ifl.set_thresholds("segred.b4", tt, ti)
        seq = [rank[ifl.select("segred.b4", 1 << k, 1 << (26 - k)).version] for k in range(27)]
        assert seq == sorted(seq)
    ifl.reset_thresholds()


def test_threshold_file_roundtrip(L, tmp_path):
    ifl.set_thresholds("segred.b4", 123, 456)
    ifl.set_thresholds("tridag", 7, 8)
    p = str(tmp_path / "thr.txt")
    ifl.save_thresholds(p)
    ifl.reset_thresholds()
    assert ifl.get_thresholds("segred.b4") == (2**15, 2**15)
    ifl.load_thresholds(p)
    assert ifl.get_thresholds("segred.b4") == (123, 456)
    assert ifl.get_thresholds("tridag") == (7, 8)
    with pytest.raises(ifl.IflError):
        ifl.set_thresholds("nope", 1, 1)
    ifl.reset_thresholds()


# ---------------------------------------------------------------- tuner


def _path_cost(pt, pm, table, a, b):
    s = 0.0
    for i in range(len(pt)):
        v = 0 if pt[i] >= a else (1 if pm[i] >= b else 2)
        s += table[i][v]
    return s


@pytest.mark.parametrize("seed", range(6))
def test_tune_search_matches_brute_force(L, seed):
    """Exact search over distinct tree paths == brute force over a dense
    grid of threshold pairs (the paper's LogIntegerParameter space)."""
    rng = np.random.default_rng(seed)
    ks = np.arange(0, 21)
    pt = (1 << ks).astype(np.int64)
    pm = (pt * np.minimum(1 << (20 - ks), 1024)).astype(np.int64)
    table = rng.uniform(1, 10, size=(len(ks), 3))
    a, b, npaths = ifl.tune_search(pt, pm, table, cost=0)
    got = _path_cost(pt, pm, table, a, b)
    grid = [0] + [1 << e for e in range(0, 41)] + [2**63 - 1]
    brute = min(_path_cost(pt, pm, table, x, y) for x in grid for y in grid)
    assert got == pytest.approx(brute)
    # every distinct path evaluated once: no more than (#t_top cands)*(#t_intra cands)
    assert npaths <= (len(set(pt)) + 1) * (len(set(pm)) + 1)


def test_tune_search_recovers_planted_crossover(L):
    """Cost table where TOP wins for n >= 2^12, MIDDLE for 2^5 <= n < 2^12,
    FLAT below: the tuned thresholds reproduce the per-shape best version
    and generalise to unseen shapes in between (geometric midpoints)."""
    ks = np.arange(0, 27, 2)
    pt = (1 << ks).astype(np.int64)
    pm = pt * np.minimum(1 << (26 - ks), 1024)
    table = np.full((len(ks), 3), 5.0)
    for i, k in enumerate(ks):
        best = 0 if k >= 12 else (1 if k >= 5 else 2)
        table[i, best] = 1.0
    for cost in (0, 1):
        a, b, _ = ifl.tune_search(pt, pm, table, cost=cost)
        ifl.set_thresholds("segred.b4", a, b)
        for k in range(27):
            want = "top" if k >= 12 else ("middle" if k >= 6 else "flat")
            if k in (5, 11):  # untrained, between two trained shapes with different best versions
                continue
            assert ifl.select("segred.b4", 1 << k, 1 << (26 - k)).version == want, k
    ifl.reset_thresholds()


def test_fig5_duplicate_paths_memoised(L):
    """(n1,n2,n3)=(10,20,30) with (p1,p2,p3)=(5,15,25) takes the first
    branch, and so does p1=6 -- the same path.  A one-dataset table has at
    most 3 distinct paths however many threshold pairs are tried."""
    ifl.set_thresholds("segred.b4", 5, 15)
    v1 = ifl.select("segred.b4", 10, 2).version
    ifl.set_thresholds("segred.b4", 6, 15)
    assert ifl.select("segred.b4", 10, 2).version == v1 == "top"
    a, b, npaths = ifl.tune_search([10], [20], [[3.0, 2.0, 1.0]], cost=0)
    assert npaths <= 3
    ifl.set_thresholds("segred.b4", a, b)
    assert ifl.select("segred.b4", 10, 2).version == "flat"
    ifl.reset_thresholds()


def test_tune_search_minimax_tie_tolerance(L):
    """cost = 1: a path whose worst slowdown is within 1 % of the optimum is a
    tie and the smaller sum of runtimes wins; beyond 1 % the minimax decides.
    Two shapes with the same Par share a version: FLAT for both costs a worst
    slowdown of 1.001 (sum 11.0), MIDDLE for both 1.005 (sum 10.995)."""
    pt = pm = [5, 5]
    table = [[9.0, 1.005, 1.0], [99.0, 9.99, 10.0]]
    a, b, _ = ifl.tune_search(pt, pm, table, cost=1)
    ifl.set_thresholds("segred.b4", a, b)
    assert ifl.select("segred.b4", 5, 1).version == "middle"
    table2 = [[9.0, 1.05, 1.0], [99.0, 9.99, 10.0]]  # MIDDLE's worst is now 5 % off: not a tie
    a, b, _ = ifl.tune_search(pt, pm, table2, cost=1)
    ifl.set_thresholds("segred.b4", a, b)
    assert ifl.select("segred.b4", 5, 1).version == "flat"
    ifl.reset_thresholds()


def test_tune_search_minimax_cost(L):
    # cost 1 = max slowdown vs best; cost 0 = sum -- can disagree.
    pt = [1, 100]
    pm = [1, 100]
    table = [[10.0, 9.0, 1.0], [100.0, 50.0, 95.0]]
    a0, b0, _ = ifl.tune_search(pt, pm, table, cost=0)
    a1, b1, _ = ifl.tune_search(pt, pm, table, cost=1)
    assert _path_cost(pt, pm, table, a0, b0) <= _path_cost(pt, pm, table, a1, b1)


def test_lvc_validation_and_guard(L):
    P = [256] * 8
    # negative size / bad version / NULL pointers / overlapping arrays (no launch)
    assert L.ifl_lvc(*P, -1, 2, 4, 4, -1, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_lvc(*P[:7], 256, 2, 2, 4, 4, 7, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_lvc(0, *P[1:], 2, 2, 4, 4, -1, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_lvc(*P, 2, 2, 4, 4, -1, None, 0, None, None) == ifl.IFL_EINVAL  # xsss == ysss
    # V_OUTER keeps systems in registers: lengths > 512 do not fit (P:358 fit clause)
    xs, ys = 1 << 20, 1 << 24
    assert L.ifl_lvc(xs, ys, *P[2:], 2, 2, 4, 600, 3, None, 0, None, None) == ifl.IFL_ENOTFIT
    # no workspace
    assert L.ifl_lvc(xs, ys, *P[2:], 2, 2, 4, 8, 3, None, 0, None, None) == ifl.IFL_EWORKSPACE
    # empty problem and zero steps are no-ops
    assert L.ifl_lvc(xs, ys, *P[2:], 0, 2, 4, 8, -1, None, 0, None, None) == 0
    assert L.ifl_lvc(xs, ys, *P[2:], 2, 0, 4, 8, -1, None, 0, None, None) == 0
    assert ifl.workspace_bytes("lvc", 32, 256) == 6 * 32 * 256 * 4
    # outermost guard of Fig 6c: numS >= t0 (R1) and fit
    try:
        ifl.set_thresholds("lvc", 100, 0)
        assert ifl.select("lvc", 100, 32, 256).version == "outer"
        assert ifl.select("lvc", 99, 32, 256).version == "auto"
        assert ifl.select("lvc", 100, 32, 513).version == "auto"
        c = ifl.select("lvc", 128, 256, 32)
        assert (c.par_top, c.t_top) == (128, 100)
    finally:
        ifl.reset_thresholds()


def test_col_selector_g4(L):
    ifl.set_thresholds("colred.b4", 4096, 1024)
    try:
        assert ifl.select("colred.b4", 10, 4096).version == "top"      # Par_top = m
        c = ifl.select("colred.b4", 100, 200)
        assert c.version == "middle" and c.par_mid == 200 * 8           # m * min(n, 8)
        assert ifl.select("colred.b4", 100000, 100).version == "flat"
    finally:
        ifl.reset_thresholds()


def test_irr_guard_and_validation(L):
    # the inspector's imbalance measure in G3 -- Par_top = total / max_len
    ifl.set_thresholds("segscan.irr", 1000, 5000)
    try:
        assert ifl.select("segscan.irr", 4000, 64000, 16).version == "top"
        c = ifl.select("segscan.irr", 4000, 64000, 6400)
        assert (c.version, c.par_top, c.par_mid) == ("middle", 10, 4000 * 16)
        assert ifl.select("segscan.irr", 100, 64000, 6400).version == "flat"   # 100 * min(640, 32) < 5000
        assert ifl.select("segscan.irr", 4000, 64000, 0).par_top == 4000      # max_len unknown: n
    finally:
        ifl.reset_thresholds()
    sig = (256, 512, 1024)
    assert L.ifl_segred_irr(*sig, -1, 0, 0, 1, 0, 0, None, -1, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_segred_irr(256, 512, None, 4, 8, 0, 1, 0, 0, None, -1, None, 0, None, None) == ifl.IFL_EINVAL
    # forced V_FLAT without workspace
    assert L.ifl_segred_irr(*sig, 4, 8, 0, 1, 0, 0, None, 2, None, 0, None, None) == ifl.IFL_EWORKSPACE
    assert ifl.workspace_bytes("segred_irr", 4, 1 << 20, version="flat") > 0
    assert ifl.workspace_bytes("segred_irr", 4, 1 << 20, version="top") == 0


def test_segarg_validation(L):
    assert L.ifl_segarg(256, 512, 1024, -1, 4, 1, 0, -1, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_segarg(256, 512, 1024, 4, 4, 1, 2, -1, None, 0, None, None) == ifl.IFL_EINVAL   # which
    assert L.ifl_segarg(256, 512, None, 4, 4, 1, 0, -1, None, 0, None, None) == ifl.IFL_EINVAL   # idx NULL
    assert L.ifl_segarg(1 << 20, 512, 1024, 4, 1 << 16, 1, 0, 2, None, 0, None, None) == ifl.IFL_EWORKSPACE
    assert L.ifl_segarg(256, 512, 1024, 0, 4, 1, 0, -1, None, 0, None, None) == 0                # n == 0
    assert ifl.workspace_bytes("segarg", 4, 1 << 16, version="flat") > 0



def _chain_brute(par, cost, kind):
    """Every combination of candidate thresholds, evaluated directly."""
    import itertools
    ns, G = par.shape

    def cands(v):
        v = sorted(set(int(x) for x in v))
        return [v[0]] + [v[i] + 1 for i in range(len(v) - 1)] + [2**63 - 1]
    best = cost.min(axis=1)
    keys = []
    for th in itertools.product(*[cands(par[:, k]) for k in range(G)]):
        leaf = []
        for s in range(ns):
            lf = G
            for k in range(G):
                if par[s, k] >= th[k]:
                    lf = k
                    break
            leaf.append(lf)
        c = [cost[s, leaf[s]] for s in range(ns)]
        keys.append((sum(c) if kind == 0 else max(ci / bi for ci, bi in zip(c, best)), sum(c)))
    if kind == 0:
        return min(keys)
    # minimax with the 1 % tie rule of tune.cpp: the smallest sum among paths
    # whose worst slowdown is within 1 % of the optimum
    opt = min(k[0] for k in keys)
    return min((k for k in keys if k[0] <= opt * 1.01), key=lambda k: k[1])


@pytest.mark.parametrize("G", [1, 2, 3, 4])
def test_chain_search_matches_brute_force(L, G):
    # Fig 5: the chain search reaches the brute-force optimum over all
    # threshold combinations, evaluating each distinct path once
    rng = np.random.default_rng(G)
    for trial in range(4):
        ns = 7
        par = rng.integers(1, 40, size=(ns, G)).astype(np.int64)
        cost = rng.uniform(1, 10, size=(ns, G + 1))
        for kind in (0, 1):
            th, npaths = ifl.tune_search_chain(par, cost, kind)
            leaf = [next((k for k in range(G) if par[s, k] >= th[k]), G) for s in range(ns)]
            c = [cost[s, leaf[s]] for s in range(ns)]
            got = (sum(c) if kind == 0 else max(ci / bi for ci, bi in zip(c, cost.min(axis=1))), sum(c))
            want = _chain_brute(par, cost, kind)
            assert abs(got[0] - want[0]) < 1e-9 and abs(got[1] - want[1]) < 1e-9, (G, trial, kind)
            assert 1 <= npaths <= (G + 1) ** ns


def test_chain_search_g2_equals_pair_search(L):
    rng = np.random.default_rng(11)
    pt = rng.integers(1, 1000, 12).astype(np.int64)
    pm = (pt * rng.integers(1, 50, 12)).astype(np.int64)
    cost = rng.uniform(1, 5, size=(12, 3))
    a, b, _ = ifl.tune_search(pt, pm, cost, cost=1)
    th, _ = ifl.tune_search_chain(np.stack([pt, pm], 1), cost, 1)
    leaf2 = lambda t0, t1: [0 if pt[s] >= t0 else (1 if pm[s] >= t1 else 2) for s in range(12)]
    assert leaf2(a, b) == leaf2(*th) or max(cost[s, l] / cost[s].min() for s, l in enumerate(leaf2(a, b))) == \
        max(cost[s, l] / cost[s].min() for s, l in enumerate(leaf2(*th)))


def test_mm_tree_guard(L):
    # the 5-leaf matmul chain: row guards first, then the two-map G3
    ifl.reset_thresholds()
    assert ifl.select("redomap2.f32", 4096, 64, 64).version in ("top", "middle", "flat")
    ifl.set_thresholds("redomap2.f32.row", 4096, 1 << 19)
    try:
        # B as yss [m][p] without a workspace: the choice is reported, then
        # IFL_EWORKSPACE (the transposition buffer) -- nothing is launched
        c = ifl.ifl_choice()
        assert L.ifl_redomap2(256, 512, 1024, 4096, 64, 16, 1, 0, -1, None, 0, None, ctypes.byref(c)) == \
            ifl.IFL_EWORKSPACE
        assert c.version == 4                                                    # ROW_TOP: n >= t_rt
        assert L.ifl_redomap2(256, 512, 1024, 4095, 64, 16, 1, 0, -1, None, 0, None, ctypes.byref(c)) != 0
        assert c.version == 5                                                    # ROW_MIDDLE: 4095*8*32 >= 2^19
        assert L.ifl_redomap2(256, 512, 1024, 64, 64, 4, 1, 0, -1, None, 0, None, ctypes.byref(c)) != 0
        assert c.version in (0, 1, 2)                                            # 64*4*32 < 2^19
        assert L.ifl_redomap2(256, 512, 1024, 64, 10000, 4, 1, 1, 5, None, 0, None, None) == ifl.IFL_ENOTFIT
    finally:
        ifl.reset_thresholds()


def test_segred2_validation(L):
    assert L.ifl_segred2(256, 512, -1, 2, 2, 1, 0, 3, 0, None, None, -1, None, 0, None, None) == ifl.IFL_EINVAL
    assert L.ifl_segred2(256, 512, 2, 2, 2, 1, 4, 0, 0, None, None, -1, None, 0, None, None) == ifl.IFL_EUNSUPPORTED
    assert L.ifl_segred2(1 << 20, 1 << 30, 4, 64, 64, 1, 0, 3, 0, None, None, 2, None, 0, None, None) == ifl.IFL_EWORKSPACE
    assert L.ifl_segred2(256, 512, 0, 4, 4, 1, 0, 3, 0, None, None, -1, None, 0, None, None) == 0
    assert ifl.workspace_bytes("segred2", 4, 64, 64, version="flat") >= 4 * 64 * 4
