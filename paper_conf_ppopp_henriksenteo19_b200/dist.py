"""Multi-GPU layer: rule G3 lifted to a third hardware level,
l = 2 = devices.  The paper is single-GPU; it notes the rules apply to
other heterogeneous hardware.

One process per GPU, ``torch.distributed`` for the plumbing (NCCL over
NVLink on B200, gloo for the CPU tests).  For segred over an [n][m] array
the device-level guard is ``n >= t_dev`` (Par over devices = n):

  * outer split (n >= t_dev): rank r owns rows [r*ceil(n/G), ...) and runs
    the single-GPU selector on its block -- independent units, NO collective
    on the data path (``all_gather`` only if the caller wants the full
    result replicated);
  * inner split (n < t_dev): rank r owns columns [r*m/G, (r+1)*m/G) of every
    row; the local segred runs WITHOUT d (canonical neutral element), one
    ``all_reduce``/``reduce`` of the n partials combines them -- the one real
    exchange step -- and d is applied once, after the collective.

Bitwise operators have no NCCL reduction: partials are all-gathered and
combined with the library's own segred over the [n][G] partial matrix.

segscan uses the same guard.  Outer split: independent rows, no collective.
Inner split: (1) local segred of the rank's column block without d -> n
totals; (2) one ``all_gather`` of the [G][n] totals -- the exchange step;
(3) carry-in of rank r = d (+) tot_0 (+) ... (+) tot_{r-1}, an ordered
segred over the [n][r] matrix of lower ranks' totals; (4) the local scan
seeded row by row with that carry (ifl_segscan_seeded).  Three global
accesses per element (read, read + write), as SURVEY 8(e) plans.
redomap2 splits the rows of A (B replicated) and tridag the systems: both
are outer splits without a collective.

The local computation is injectable (``local_segred``) so the host logic
(plans, collectives, d handling) is tested with world size 2 on gloo/CPU.
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as td

_REDUCE = {"sum": td.ReduceOp.SUM, "prod": td.ReduceOp.PRODUCT, "min": td.ReduceOp.MIN, "max": td.ReduceOp.MAX,
           "and": td.ReduceOp.BAND, "or": td.ReduceOp.BOR, "xor": td.ReduceOp.BXOR}
_BITWISE = ("and", "or", "xor")


@dataclass
class Plan:
    mode: str        # "outer" or "inner"
    lo: int          # first owned row (outer) or column (inner)
    hi: int          # one past the last owned row / column


def plan_segred(n: int, m: int, world: int, rank: int, t_dev: int | None = None) -> Plan:
    """Device-level G3 guard: split rows when there are >= t_dev of them
    (default: the number of devices), else split every row's columns."""
    t_dev = world if t_dev is None else t_dev
    if n >= t_dev:
        per = -(-n // world)
        lo = min(n, rank * per)
        return Plan("outer", lo, min(n, lo + per))
    lo = (m * rank) // world
    return Plan("inner", lo, (m * (rank + 1)) // world)


def _default_local(x: torch.Tensor, op: str, f: str, ne):
    import paper_conf_ppopp_henriksenteo19_b200 as ifl
    return ifl.segred(x, op, f, ne=ne)


def _apply_ne(partial: torch.Tensor, op: str, ne, local_segred):
    """out[i] = d (+) partial[i]: a segred over [n][1] with neutral element d."""
    if ne is None:
        return partial
    return local_segred(partial.reshape(-1, 1).contiguous(), op, "id", ne)


def segred_dist(x_block: torch.Tensor, n: int, m: int, op: str = "sum", f: str = "id", ne=None,
                plan: Plan | None = None, group=None, gather: bool = False, local_segred=None,
                gather_partials: bool | None = None) -> torch.Tensor:
    """Distributed segred.  ``x_block`` is this rank's block: rows
    [plan.lo, plan.hi) x all m columns (outer) or all n rows x columns
    [plan.lo, plan.hi) (inner).  Returns this rank's rows of the result
    (outer; all rows if ``gather``) or the full [n] result on every rank
    (inner)."""
    local = local_segred or _default_local
    world = td.get_world_size(group)
    rank = td.get_rank(group)
    plan = plan or plan_segred(n, m, world, rank)
    if plan.mode == "outer":
        out = local(x_block, op, f, ne)
        if not gather:
            return out
        per = -(-n // world)
        buf = torch.empty(per * world, dtype=out.dtype, device=out.device)
        padded = torch.empty(per, dtype=out.dtype, device=out.device)
        padded[: out.numel()] = out
        td.all_gather_into_tensor(buf, padded, group=group)
        return buf[:n]
    # inner split: partials without d, one exchange, then d once
    part = local(x_block, op, f, None)
    if gather_partials is None:
        gather_partials = op in _BITWISE and td.get_backend(group) == "nccl"
    if gather_partials:
        allp = torch.empty(world * n, dtype=part.dtype, device=part.device)
        td.all_gather_into_tensor(allp, part.contiguous(), group=group)
        stacked = allp.view(world, n).t().contiguous()  # [n][G] partials, rank order
        total = local(stacked, op, "id", None)
    else:
        total = part.clone()
        td.all_reduce(total, op=_REDUCE[op], group=group)
    return _apply_ne(total, op, ne, local)


def _default_local_scan(x: torch.Tensor, op: str, f: str, ne, seed):
    import paper_conf_ppopp_henriksenteo19_b200 as ifl
    return ifl.segscan(x, op, f, ne=ne, seed=seed)


def segscan_dist(x_block: torch.Tensor, n: int, m: int, op: str = "sum", f: str = "id", ne=None,
                 plan: Plan | None = None, group=None, local_segred=None, local_segscan=None) -> torch.Tensor:
    """Distributed segscan.  ``x_block`` as for segred_dist; returns this
    rank's block of the [n][m] result (its rows for the outer split, its
    columns of every row for the inner split)."""
    red = local_segred or _default_local
    scan = local_segscan or _default_local_scan
    world = td.get_world_size(group)
    rank = td.get_rank(group)
    plan = plan or plan_segred(n, m, world, rank)
    if plan.mode == "outer" or world == 1:
        return scan(x_block, op, f, ne, None)
    # (1) block totals without d (canonical neutral element)
    if x_block.shape[1] > 0:
        tot = red(x_block, op, f, None).contiguous()
    else:
        tot = red(x_block.new_empty((n, 0)), op, f, None).contiguous()
    # (2) the exchange step: every rank's totals
    allt = torch.empty(world * n, dtype=tot.dtype, device=tot.device)
    td.all_gather_into_tensor(allt, tot, group=group)
    if x_block.shape[1] == 0:
        return x_block.new_empty((n, 0))
    # (3) carry-in = d (+) totals of ranks 0..r-1, in rank order
    if rank == 0:
        return scan(x_block, op, f, ne, None)
    lower = allt.view(world, n)[:rank].t().contiguous()  # [n][rank]
    seed = red(lower, op, "id", ne).contiguous()
    # (4) local scan continued from the carry
    return scan(x_block, op, f, None, seed)


def rows_of(n: int, world: int, rank: int):
    per = -(-n // world)
    lo = min(n, rank * per)
    return lo, min(n, lo + per)


def plan_redomap2(n: int, m: int, p: int, world: int, rank: int, t_dev: int | None = None) -> Plan:
    """Device-level guard for redomap2 (Par_dev = n, rows of C): split the
    rows of A when n >= t_dev (B replicated, no collective), else split k
    (columns of A / rows of yss) and sum the [n][p] partials with one
    all_reduce ("split-K, then ncclReduce")."""
    t_dev = world if t_dev is None else t_dev
    if n >= t_dev:
        lo, hi = rows_of(n, world, rank)
        return Plan("outer", lo, hi)
    return Plan("inner", (m * rank) // world, (m * (rank + 1)) // world)


def _default_local_mm(A, B, b_kmajor):
    import paper_conf_ppopp_henriksenteo19_b200 as ifl
    return ifl.redomap2(A, B, b_kmajor=b_kmajor)


def redomap2_dist(A_block: torch.Tensor, B_block: torch.Tensor, n: int, m: int, p: int, plan: Plan | None = None,
                  group=None, b_kmajor: bool = True, gather: bool = False, local_redomap2=None) -> torch.Tensor:
    """Distributed C = xss x yss.  Outer plan: A_block = rows
    [lo, hi) of A, B_block = all of B; returns those rows of C (all rows if
    ``gather``).  Inner plan: A_block = A[:, lo:hi], B_block = the matching
    k-block of B (Bt[:, lo:hi] when b_kmajor, else B[lo:hi]); returns the
    full C on every rank after one all_reduce of the fp32 partials."""
    local = local_redomap2 or _default_local_mm
    world = td.get_world_size(group)
    rank = td.get_rank(group)
    plan = plan or plan_redomap2(n, m, p, world, rank)
    if plan.mode == "outer":
        C = local(A_block, B_block, b_kmajor)
        if not gather:
            return C
        per = -(-n // world)
        buf = torch.empty(per * world * p, dtype=C.dtype, device=C.device)
        padded = torch.zeros(per * p, dtype=C.dtype, device=C.device)
        padded[: C.numel()] = C.reshape(-1)
        td.all_gather_into_tensor(buf, padded, group=group)
        return buf.view(per * world, p)[:n]
    if A_block.shape[1] == 0:
        C = torch.zeros(n, p, dtype=torch.float32, device=A_block.device)
    else:
        C = local(A_block, B_block, b_kmajor).contiguous()
    td.all_reduce(C, op=td.ReduceOp.SUM, group=group)
    return C


def tridag_dist(a: torch.Tensor, b: torch.Tensor, c: torch.Tensor, y_rows: torch.Tensor, lo: int,
                local_tridag=None, **kw) -> torch.Tensor:
    """System split (independent units, no collective).  y_rows holds the
    systems s in [lo, lo + len); coefficients are the full [R][L] arrays and
    system s uses row s % R (R9), so when lo % R != 0 the rows are rotated
    to keep that mapping for the local call (R * L elements, tiny)."""
    R = a.shape[0]
    sh = lo % R
    if sh:
        a, b, c = (torch.roll(t, -sh, dims=0).contiguous() for t in (a, b, c))
    if local_tridag is not None:
        return local_tridag(a, b, c, y_rows)
    import paper_conf_ppopp_henriksenteo19_b200 as ifl
    return ifl.tridag(a, b, c, y_rows, **kw)


# ------------------------------------------------------------- colred (G4)


def plan_colred(n: int, m: int, world: int, rank: int, t_dev: int | None = None) -> Plan:
    """Device-level guard of the column reduction (the segments are the m
    columns, Par over devices = m): split the columns when m >= t_dev (outer,
    no collective), else split the rows (inner: one all_reduce of the m
    partials)."""
    t_dev = world if t_dev is None else t_dev
    if m >= t_dev:
        lo = (m * rank) // world
        return Plan("outer", lo, (m * (rank + 1)) // world)
    per = -(-n // world)
    lo = min(n, rank * per)
    return Plan("inner", lo, min(n, lo + per))


def _default_local_col(x: torch.Tensor, op: str, f: str, ne):
    import paper_conf_ppopp_henriksenteo19_b200 as ifl
    return ifl.colred(x, op, f, ne=ne)


def colred_dist(x_block: torch.Tensor, n: int, m: int, op: str = "sum", f: str = "id", ne=None,
                plan: Plan | None = None, group=None, gather: bool = False, local_colred=None) -> torch.Tensor:
    """Distributed column reduction (G4).  ``x_block``: all n rows x
    columns [plan.lo, plan.hi) (outer; contiguous copy of the column block)
    or rows [plan.lo, plan.hi) x all m columns (inner).  Returns this rank's
    columns (outer; all m if ``gather``) or the full [m] result (inner)."""
    local = local_colred or _default_local_col
    world = td.get_world_size(group)
    rank = td.get_rank(group)
    plan = plan or plan_colred(n, m, world, rank)
    if plan.mode == "outer":
        out = local(x_block, op, f, ne)
        if not gather:
            return out
        parts = [None] * world
        td.all_gather_object(parts, out.cpu(), group=group)
        return torch.cat(parts).to(out.device)
    part = local(x_block, op, f, None)  # partials without d
    if op in _BITWISE and td.get_backend(group) == "nccl":
        allp = torch.empty(world * m, dtype=part.dtype, device=part.device)
        td.all_gather_into_tensor(allp, part.contiguous(), group=group)
        total = local(allp.view(world, m).contiguous(), op, "id", None)
    else:
        total = part.clone()
        td.all_reduce(total, op=_REDUCE[op], group=group)
    if ne is None:
        return total
    return local(total.view(1, m).contiguous(), op, "id", ne)  # d (+) total, once


# ------------------------------------------------------- LocVolCalib loop


def lvc_dist(xsss_block: torch.Tensor, ysss_block: torch.Tensor, xcoef, ycoef, numT: int, local_lvc=None,
             **kw):
    """The LocVolCalib loop split over numS (its outermost map, Fig 6a):
    every s is an independent unit and the coefficients do not depend on s,
    so each rank runs its block [numS_r][numX][numY] / [numS_r][numY][numX]
    with no collective (weak scaling).  In place, like ifl_lvc."""
    if local_lvc is not None:
        return local_lvc(xsss_block, ysss_block, xcoef, ycoef, numT)
    import paper_conf_ppopp_henriksenteo19_b200 as ifl
    return ifl.lvc(xsss_block, ysss_block, xcoef, ycoef, numT, **kw)


# ------------------------------------------------------ irregular segments


def plan_irr(offsets, world: int, rank: int):
    """Split n irregular segments (host int64 offsets [n+1]) into contiguous
    segment ranges of about total/G elements each, cut at segment boundaries
    (independent units, no collective).  Returns (seg_lo, seg_hi)."""
    import numpy as np
    off = np.asarray(offsets, dtype=np.int64)
    n, total = off.size - 1, int(off[-1])
    cuts = [0] + [int(np.searchsorted(off, (total * r) // world, side="left")) for r in range(1, world)] + [n]
    cuts = [min(max(c, 0), n) for c in cuts]
    for r in range(1, len(cuts)):  # monotone
        cuts[r] = max(cuts[r], cuts[r - 1])
    return cuts[rank], cuts[rank + 1]


def segred_irr_dist(x: torch.Tensor, offsets, seg_lo: int, seg_hi: int, op: str = "sum", f: str = "id", ne=None,
                    local=None, **kw) -> torch.Tensor:
    """This rank's segments [seg_lo, seg_hi): the element range
    x[off[seg_lo]:off[seg_hi]] with rebased offsets; no collective."""
    import numpy as np
    off = np.asarray(offsets, dtype=np.int64)
    e0, e1 = int(off[seg_lo]), int(off[seg_hi])
    loc_off = torch.from_numpy(off[seg_lo:seg_hi + 1] - e0)
    xb = x[e0:e1]
    if local is not None:
        return local(xb, loc_off, op, f, ne)
    import paper_conf_ppopp_henriksenteo19_b200 as ifl
    return ifl.segred_irr(xb.contiguous(), loc_off.to(x.device), op, f, ne=ne, **kw)
