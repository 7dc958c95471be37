"""ORACLE (test infrastructure only): CRSD construction written step by step
in the order and notation of PAPER.md §II-§III (Sun et al., ICPP 2011).

Pure-Python loops; meant for small matrices (<= ~1e5 nonzeros). Every step
cites the passage it follows; where the paper is silent or garbled the
DESIGN.md reading (R#) is named. The product builder (C++) is NOT consulted.

Steps
  1. canonical()         -- input canonicalisation (DESIGN R10: duplicates,
                            explicit zeros)
  2. offset()            -- diagonal identification, offset = col - row
                            (§II-A)
  3. present_sets()      -- row segments of mrows rows (§II-C);
                            scatter points and idle sections with the
                            bridged-piece reading (DESIGN R1/R2)
  4. groups()            -- AD / NAD grouping = the diagonal pattern
                            (§II-B)
  5. build()             -- patterns as row-contiguous runs of segments with
                            Table II quantities NRS, NNzRS, SR, NDias, Colv
                            (P:L581-611), arrays `matrix` and
                            `crsd_dia_index` (Fig. 4), and
                            `crsd_dia_val` filled through the address formula
                            of P:L613-623 (DESIGN R4); scatter points in the
                            paper's whole-row ELL (R6) and in the
                            per-segment list of the B200 layout (R5).
"""
from __future__ import annotations

from collections import Counter, defaultdict
from dataclasses import dataclass, field
from typing import Dict, List, Tuple

import numpy as np


class DuplicateEntry(ValueError):
    pass


def _is_zero(v) -> bool:
    return float(v) == 0.0


# -- step 1 -----------------------------------------------------------------
def canonical(nrows, ncols, row, col, val, sum_duplicates=False):
    """Sort entries by (row, col). Duplicates raise DuplicateEntry unless
    ``sum_duplicates`` (then values are summed in input order). Explicit
    zeros are kept (DESIGN R10). Returns a list of (r, c, v)."""
    acc: Dict[Tuple[int, int], object] = {}
    order: List[Tuple[int, int]] = []
    for r, c, v in zip(np.asarray(row).tolist(), np.asarray(col).tolist(), np.asarray(val)):
        if not (0 <= r < nrows and 0 <= c < ncols):
            raise IndexError((r, c))
        k = (r, c)
        if k in acc:
            if not sum_duplicates:
                raise DuplicateEntry(k)
            acc[k] = acc[k] + v
        else:
            acc[k] = v
            order.append(k)
    return [(r, c, acc[(r, c)]) for (r, c) in sorted(acc)]


# -- step 2 -----------------------------------------------------------------
def offset(r: int, c: int) -> int:
    """a diagonal is identified by its offset from the main
    diagonal, positive above and negative below."""
    return c - r


# -- step 3 -----------------------------------------------------------------
def present_sets(nrows: int, entries, mrows: int, idle_max: int) -> List[frozenset]:
    """Diagonals present in each row segment.

    P:L351-361: the matrix is split into row segments of ``mrows`` rows.
    P:L361-369: "if only one nonzero is on a diagonal within one row segment,
    the nonzero is viewed as scatter point".
    P:L369-389: an idle section (zero run along a diagonal) of few zeros is
    filled and the pattern is unchanged; a long one breaks the diagonal.
    Reading R1/R2: along each diagonal the nonzeros are split into
    *pieces* wherever a zero run is longer than ``idle_max``; diagonal d is
    present in segment s iff s holds >= 2 nonzeros of d, or s intersects the
    row span of a piece holding >= 2 nonzeros. This reproduces Fig. 4 (fill at
    v43, scatter v55) for idle_max in {1, 2} at mrows = 2.
    Explicit zeros are not nonzeros (R10).
    """
    nseg = -(-nrows // mrows)
    rows_on: Dict[int, List[int]] = defaultdict(list)
    for r, c, v in entries:
        if not _is_zero(v):
            rows_on[offset(r, c)].append(r)
    present = [set() for _ in range(nseg)]
    for d, rows in rows_on.items():
        rows = sorted(rows)
        cnt = Counter(r // mrows for r in rows)
        for s, k in cnt.items():
            if k >= 2:
                present[s].add(d)
        piece = [rows[0]]
        pieces = []
        for a, b in zip(rows, rows[1:]):
            if b - a - 1 <= idle_max:
                piece.append(b)
            else:
                pieces.append(piece)
                piece = [b]
        pieces.append(piece)
        for pc in pieces:
            if len(pc) >= 2:
                for s in range(pc[0] // mrows, pc[-1] // mrows + 1):
                    present[s].add(d)
    return [frozenset(p) for p in present]


# -- step 4 -----------------------------------------------------------------
def groups(offsets) -> List[Tuple[str, List[int]]]:
    """two diagonals are adjacent if their offsets differ by 1;
    adjacent diagonals go into an adjacent (AD) group; removing them breaks
    the remaining sequence into pieces, each piece is a nonadjacent (NAD)
    group. Groups are listed in ascending offset order (Fig. 4, R13)."""
    offs = sorted(offsets)
    n = len(offs)
    in_ad = [False] * n
    for i in range(n - 1):
        if offs[i + 1] - offs[i] == 1:
            in_ad[i] = in_ad[i + 1] = True
    out = []
    i = 0
    while i < n:
        j = i
        if in_ad[i]:
            while j + 1 < n and offs[j + 1] - offs[j] == 1:
                j += 1
            out.append(("AD", offs[i : j + 1]))
        else:
            while j + 1 < n and not in_ad[j + 1]:
                j += 1
            out.append(("NAD", offs[i : j + 1]))
        i = j + 1
    return out


def pattern_repr(offsets) -> List[Tuple[str, int]]:
    """group = (group type, number of diagonals)."""
    return [(t, len(g)) for t, g in groups(offsets)]


# -- step 5 -----------------------------------------------------------------
@dataclass
class CRSDRef:
    nrows: int
    ncols: int
    mrows: int
    idle_max: int
    seg_present: List[frozenset]
    # paper's patterns (row-contiguous runs of segments)
    offsets: List[List[int]] = field(default_factory=list)  # per pattern, ascending
    SR: List[int] = field(default_factory=list)
    NRS: List[int] = field(default_factory=list)
    NNzRS: List[int] = field(default_factory=list)
    NDias: List[int] = field(default_factory=list)
    Colv: List[List[int]] = field(default_factory=list)
    matrix: List[List[Tuple[str, int]]] = field(default_factory=list)
    crsd_dia_index: List[int] = field(default_factory=list)
    crsd_dia_val: np.ndarray = None
    fill: np.ndarray = None  # bool per slot: slot holds a filled zero
    # B200 layout scatter: per segment (row_in_seg, col, val), sorted by (row, col)
    seg_scatter: List[List[Tuple[int, int, object]]] = field(default_factory=list)
    # paper layout scatter (whole rows in ELL, column-major, -1/0 padded; R6)
    num_scatter_rows: int = 0
    scatter_rowno: List[int] = field(default_factory=list)
    num_scatter_width: int = 0
    scatter_colval: List[int] = field(default_factory=list)
    scatter_val: List[object] = field(default_factory=list)

    @property
    def num_dia_patterns(self) -> int:
        return len(self.SR)


def build(nrows, ncols, row, col, val, mrows, idle_max=None, sum_duplicates=False, dtype=np.float64) -> CRSDRef:
    if idle_max is None or idle_max < 0:
        idle_max = mrows - 1  # DESIGN R2 default
    entries = canonical(nrows, ncols, row, col, val, sum_duplicates)
    seg_present = present_sets(nrows, entries, mrows, idle_max)
    nseg = len(seg_present)
    R = CRSDRef(nrows, ncols, mrows, idle_max, seg_present)

    # Patterns: maximal runs of consecutive segments with the same diagonals;
    # one work-group per row segment, pattern p owns groups
    # sum_{i<p} NRS_i <= group_id < sum_{i<=p} NRS_i.
    s = 0
    while s < nseg:
        t = s
        while t + 1 < nseg and seg_present[t + 1] == seg_present[s]:
            t += 1
        offs = sorted(seg_present[s])
        R.offsets.append(offs)
        R.SR.append(s * mrows)  # start row (Table II)
        R.NRS.append(t - s + 1)  # number of row segments (Table II)
        R.NDias.append(len(offs))  # number of diagonals (Table II)
        R.NNzRS.append(len(offs) * mrows)  # nonzeros in one row segment (Table II)
        R.Colv.append([s * mrows + o for o in offs])  # column index of d-th diagonal at SR
        s = t + 1

    # `matrix` and `crsd_dia_index` (Fig. 4): per pattern SR, NRS,
    # then the column of every diagonal of an NAD group and only the first
    # column of an AD group.
    for p, offs in enumerate(R.offsets):
        R.matrix.append(pattern_repr(offs))
        R.crsd_dia_index += [R.SR[p], R.NRS[p]]
        for t, g in groups(offs):
            cols = [R.SR[p] + o for o in g]
            R.crsd_dia_index += cols if t == "NAD" else cols[:1]

    # crsd_dia_val through the address formulas of P:L613-629 (R4: the
    # garbled "x NNzRS_i" reads NNzRS_p).
    where = {(r, c): v for r, c, v in entries}
    total = sum(R.NRS[p] * R.NNzRS[p] for p in range(len(R.NRS)))
    vals = np.zeros(total, dtype=dtype)
    fill = np.ones(total, dtype=bool)
    stored = set()
    prefix_nrs = 0
    prefix_val = 0
    for p in range(len(R.NRS)):
        for group_id in range(prefix_nrs, prefix_nrs + R.NRS[p]):
            for d in range(R.NDias[p]):
                for local_id in range(mrows):
                    loc = prefix_val + (group_id - prefix_nrs) * R.NNzRS[p] + d * mrows + local_id
                    xcol = R.Colv[p][d] + (group_id - prefix_nrs) * mrows + local_id
                    yrow = R.SR[p] + (group_id - prefix_nrs) * mrows + local_id
                    v = where.get((yrow, xcol))
                    # explicit zeros are never stored on a diagonal (R10)
                    if v is not None and not _is_zero(v):
                        vals[loc] = v
                        fill[loc] = False
                        stored.add((yrow, xcol))
        prefix_nrs += R.NRS[p]
        prefix_val += R.NRS[p] * R.NNzRS[p]
    R.crsd_dia_val = vals
    R.fill = fill

    # Scatter points: everything not stored on a diagonal.
    R.seg_scatter = [[] for _ in range(nseg)]
    scatter_rows = set()
    for r, c, v in entries:
        if (r, c) not in stored:
            R.seg_scatter[r // mrows].append((r % mrows, c, v))
            scatter_rows.add(r)
    # Paper layout: whole rows with a scatter point in ELL, R6.
    R.scatter_rowno = sorted(scatter_rows)
    R.num_scatter_rows = len(R.scatter_rowno)
    rows_entries = {r: [(c, v) for rr, c, v in entries if rr == r] for r in R.scatter_rowno}
    R.num_scatter_width = max((len(e) for e in rows_entries.values()), default=0)
    W, N = R.num_scatter_width, R.num_scatter_rows
    R.scatter_colval = [-1] * (W * N)
    R.scatter_val = [0.0] * (W * N)
    for i, r in enumerate(R.scatter_rowno):
        for k, (c, v) in enumerate(rows_entries[r]):
            R.scatter_colval[k * N + i] = c
            R.scatter_val[k * N + i] = v
    return R


def to_layout(R: CRSDRef) -> dict:
    """The B200 layout as numpy arrays (same keys as the product's export),
    derived from the paper-order construction above."""
    nseg = len(R.seg_present)
    ptr = np.zeros(nseg + 1, dtype=np.int64)
    rs, cs, vs = [], [], []
    for s, lst in enumerate(R.seg_scatter):
        ptr[s + 1] = ptr[s] + len(lst)
        for (lr, c, v) in lst:
            rs.append(lr)
            cs.append(c)
            vs.append(v)
    return dict(
        nrows=R.nrows,
        ncols=R.ncols,
        mrows=R.mrows,
        inst_first_seg=np.array([sr // R.mrows for sr in R.SR], dtype=np.int64),
        inst_nseg=np.array(R.NRS, dtype=np.int64),
        inst_offsets=[list(o) for o in R.offsets],
        vals=R.crsd_dia_val,
        scat_ptr=ptr,
        scat_row=np.array(rs, dtype=np.int64),
        scat_col=np.array(cs, dtype=np.int64),
        scat_val=np.array(vs, dtype=R.crsd_dia_val.dtype),
    )


def paper_ell_rows(R: CRSDRef, x, alpha=1.0, dtype=np.float64):
    """Second part of the paper's SpMV kernel ("the final kernel is
    composed of two parts"; the ELL part computes the scatter rows, stored
    whole): for every stored row i, y[scatter_rowno[i]] =
    alpha * (((0 + v_0 x_0) + v_1 x_1) + ...), entries in stored (ascending
    column) order, each product and sum rounded to `dtype` separately (the
    CSR evaluation order). Returns {row: value} in `dtype`."""
    dt = np.dtype(dtype).type
    N, W = R.num_scatter_rows, R.num_scatter_width
    x = np.asarray(x, dtype=dt)
    out = {}
    for i, r in enumerate(R.scatter_rowno):
        s = dt(0)
        for k in range(W):
            c = R.scatter_colval[k * N + i]
            if c < 0:
                break
            s = dt(s + dt(dt(R.scatter_val[k * N + i]) * x[c]))
        out[r] = dt(dt(alpha) * s)
    return out
