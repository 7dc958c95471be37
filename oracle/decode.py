"""ORACLE (test infrastructure only): independent CRSD decoder and structural
invariant checker, written from the documented layout (DESIGN.md "Data
layout") -- never from the product builder's code.

Layout dict keys (what ``crsd_export`` returns, and what
``oracle.crsd_ref.to_layout`` derives from the paper-order construction):
  nrows, ncols, mrows
  inst_first_seg[i], inst_nseg[i], inst_offsets[i] (ascending offsets)
  vals      flat; instance i, local segment g, diagonal d, local row l at
            base_i + g*NDias_i*mrows + d*mrows + l, base_i = sum_{j<i}
            nseg_j*NDias_j*mrows   (P:L613-623 address formula)
  scat_ptr[nseg+1], scat_row (row within segment), scat_col, scat_val

Vectorised numpy so it handles the full-size configurations.
"""
from __future__ import annotations

import numpy as np

from . import crsd_ref


def canonical_arrays(nrows, ncols, row, col, val):
    """Canonical COO as sorted arrays; raises on duplicates / out-of-range."""
    row = np.asarray(row, dtype=np.int64)
    col = np.asarray(col, dtype=np.int64)
    if row.size and (row.min() < 0 or row.max() >= nrows or col.min() < 0 or col.max() >= ncols):
        raise IndexError("entry out of range")
    key = row * np.int64(ncols) + col
    order = np.argsort(key, kind="stable")
    k = key[order]
    if k.size > 1 and np.any(k[1:] == k[:-1]):
        raise crsd_ref.DuplicateEntry("duplicate entry")
    return row[order], col[order], np.asarray(val)[order]


def _bits(a):
    a = np.ascontiguousarray(a)
    return a.view(np.uint64 if a.dtype == np.float64 else np.uint32)


def decode(L):
    """Return (row, col, val) of every stored nonzero, sorted by (row, col).
    Diagonal slots holding the bit pattern +0.0 are fills and are skipped;
    scatter entries are always emitted (explicit zeros live there, R10)."""
    mrows = int(L["mrows"])
    nrows, ncols = int(L["nrows"]), int(L["ncols"])
    vals = np.asarray(L["vals"])
    R, C, V = [], [], []
    base = 0
    for i in range(len(L["inst_first_seg"])):
        offs = np.asarray(L["inst_offsets"][i], dtype=np.int64)
        nd = offs.shape[0]
        nseg = int(L["inst_nseg"][i])
        sr = int(L["inst_first_seg"][i]) * mrows
        n = nseg * nd * mrows
        blk = vals[base : base + n].reshape(nseg, nd, mrows)
        base += n
        if nd == 0:
            continue
        g = np.arange(nseg, dtype=np.int64)[:, None, None]
        l = np.arange(mrows, dtype=np.int64)[None, None, :]
        rows = np.broadcast_to(sr + g * mrows + l, blk.shape)
        cols = rows + offs[None, :, None]
        keep = _bits(blk) != 0
        R.append(rows[keep])
        C.append(cols[keep])
        V.append(blk[keep])
    ptr = np.asarray(L["scat_ptr"], dtype=np.int64)
    seg_of = np.repeat(np.arange(ptr.shape[0] - 1, dtype=np.int64), np.diff(ptr))
    R.append(seg_of * mrows + np.asarray(L["scat_row"], dtype=np.int64))
    C.append(np.asarray(L["scat_col"], dtype=np.int64))
    V.append(np.asarray(L["scat_val"], dtype=vals.dtype))
    row = np.concatenate(R) if R else np.empty(0, np.int64)
    col = np.concatenate(C) if C else np.empty(0, np.int64)
    val = np.concatenate(V) if V else np.empty(0, vals.dtype)
    if row.size and (row.min() < 0 or row.max() >= nrows or col.min() < 0 or col.max() >= ncols):
        raise AssertionError("decoded entry outside the matrix (I4: out-of-range slot is not a fill)")
    order = np.lexsort((col, row))
    return row[order], col[order], val[order]


def roundtrip_equal(L, nrows, ncols, row, col, val) -> bool:
    """I3: decode(export(build(coo))) == canonical(coo), compared as bytes."""
    r0, c0, v0 = canonical_arrays(nrows, ncols, row, col, np.asarray(val, dtype=np.asarray(L["vals"]).dtype))
    r1, c1, v1 = decode(L)
    return (
        r0.shape == r1.shape
        and np.array_equal(r0, r1)
        and np.array_equal(c0, c1)
        and np.array_equal(_bits(v0), _bits(v1))
    )


def check_invariants(L, idle_max, nrows=None, ncols=None, row=None, col=None, val=None, check_rule=True):
    """Structural invariants I1-I8 of SURVEY.md §8(c). Raises AssertionError.
    The rule checks (I5/I6) need the canonical COO and use the oracle's
    paper-order presence rule (crsd_ref.present_sets)."""
    mrows = int(L["mrows"])
    nr = int(L["nrows"])
    nseg = -(-nr // mrows)
    first = np.asarray(L["inst_first_seg"], dtype=np.int64)
    cnt = np.asarray(L["inst_nseg"], dtype=np.int64)
    # I1: instances sorted, contiguous, covering every segment
    assert first.size == cnt.size
    if nseg:
        assert first[0] == 0 and np.all(cnt > 0)
        assert np.array_equal(first[1:], first[:-1] + cnt[:-1]), "I1: instances not contiguous"
        assert first[-1] + cnt[-1] == nseg, "I1: instances do not cover all segments"
    # I2: offsets strictly increasing within a pattern
    for offs in L["inst_offsets"]:
        o = np.asarray(offs, dtype=np.int64)
        assert np.all(o[1:] > o[:-1]), "I2: offsets not strictly increasing"
    # I7: adjacent instances differ
    for a, b in zip(L["inst_offsets"], L["inst_offsets"][1:]):
        assert list(a) != list(b), "I7: adjacent instances with equal offset sets"
    # value array size
    nd = np.array([len(o) for o in L["inst_offsets"]], dtype=np.int64)
    total = int(np.sum(nd * cnt * mrows))
    vals = np.asarray(L["vals"])
    assert vals.shape[0] == total, "value array size != sum NRS*NNzRS"
    ptr = np.asarray(L["scat_ptr"], dtype=np.int64)
    assert ptr.shape[0] == nseg + 1 and ptr[0] == 0 and np.all(np.diff(ptr) >= 0)
    srow = np.asarray(L["scat_row"], dtype=np.int64)
    assert srow.size == 0 or (srow.min() >= 0 and srow.max() < mrows)
    if row is None:
        return True
    r0, c0, v0 = canonical_arrays(nrows, ncols, row, col, np.asarray(val, dtype=vals.dtype))
    # I3/I4: round trip (every nonzero exactly once; every other slot +0.0)
    assert roundtrip_equal(L, nrows, ncols, row, col, val), "I3/I4: round trip differs"
    # I8: fills = stored slots - diagonal-stored nonzeros
    n_diag_nz = int(np.count_nonzero(_bits(vals)))
    n_scat = int(ptr[-1])
    assert n_diag_nz + n_scat == r0.shape[0], "I8: fill count inconsistent"
    if check_rule:
        # I5/I6: the present sets are exactly the rule's
        entries = list(zip(r0.tolist(), c0.tolist(), v0))
        rule = crsd_ref.present_sets(nrows, entries, mrows, idle_max)
        seg_sets = []
        for i in range(first.size):
            seg_sets += [frozenset(L["inst_offsets"][i])] * int(cnt[i])
        assert seg_sets == rule, "I5/I6: present sets differ from the presence rule"
    return True
