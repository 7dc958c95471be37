"""Row-partitioned path, host side, over real processes (gloo, CPU).

Each rank builds its row block with libcrsd (host-only handle), reads its x
layout, allgathers (row_begin, row_end, halo_lo_valid, halo_hi_valid), asks
crsd_dist_plan what to send/receive, exchanges the x halos with gloo
send/recv per that plan into its padded x buffer, and multiplies its local
rows with the oracle using padded-buffer column indices. The result must
equal the same rows of the global oracle product bit for bit (same entries,
same order, long double). This checks the partition, the halo widths, the
multi-hop plan and the x_padded index arithmetic without a GPU.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
from oracle import coo


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _matrix(case):
    if case == "7pt":
        return gen.stencil((16, 16, 16), "7pt", values="random", seed=4), 256
    if case == "scatter":
        a = gen.stencil((16, 16, 12), "7pt", values="random", seed=5)
        return gen.inject_scatter(a, 40, 2, 600, [0, 1, -1, 16, -16, 256, -256], seed=6), 256
    if case == "multihop":  # offsets wider than a rank's block
        n = 4096
        return gen.band(n, [(0, n, [-1500, -3, -1, 0, 1, 700, 1300])], seed=7), 256
    raise ValueError(case)


def _worker(rank, world, port, case, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import torch

        from paper_conf_icpp_sunzwzyr11_b200 import CRSDMatrix, dist_plan, partition_rows

        a, mrows = _matrix(case)
        n = a.nrows
        w = np.bincount(a.row, minlength=n).astype(np.float64)
        bounds = partition_rows(n, mrows, world, w)
        rb, re = int(bounds[rank]), int(bounds[rank + 1])
        m = (a.row >= rb) & (a.row < re)
        A = CRSDMatrix.from_coo(n, n, a.row[m], a.col[m], a.val[m], mrows=mrows, row_range=(rb, re), host_only=True)
        inf = A.info()
        lo, nloc, hi = A.x_layout()
        assert nloc == re - rb and lo % 4 == 0 and lo >= inf["halo_lo_valid"] and hi >= inf["halo_hi_valid"]
        mine = torch.tensor([rb, re, inf["halo_lo_valid"], inf["halo_hi_valid"]], dtype=torch.int64)
        allr = [torch.zeros(4, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allr, mine)
        ranges = torch.stack(allr).numpy()
        recv, send = dist_plan(world, rank, ranges)
        x = gen.vectors(n, "random", seed=11)
        xp = np.full(lo + nloc + hi, np.nan)
        xp[lo : lo + nloc] = x[rb:re]
        origin = rb - lo
        reqs, bufs = [], []
        for peer, b, cnt in send:
            reqs.append(dist.isend(torch.from_numpy(xp[b - origin : b - origin + cnt].copy()), peer))
        for peer, b, cnt in recv:
            t = torch.empty(cnt, dtype=torch.float64)
            reqs.append(dist.irecv(t, peer))
            bufs.append((b, cnt, t))
        for r in reqs:
            r.wait()
        for b, cnt, t in bufs:
            xp[b - origin : b - origin + cnt] = t.numpy()
        # every entry's column must fall inside the received/owned window
        cl = a.col[m] - origin
        assert cl.min() >= lo - inf["halo_lo_valid"] and cl.max() < lo + nloc + inf["halo_hi_valid"]
        y, _ = coo.coo_spmv(nloc, xp.shape[0], a.row[m] - rb, cl, a.val[m], np.nan_to_num(xp, nan=np.inf))
        yg, _ = coo.coo_spmv(n, n, a.row, a.col, a.val, x)
        ok = bool(np.array_equal(y, yg[rb:re]))
        q.put((rank, ok, len(recv), len(send)))
    except Exception as e:  # pragma: no cover - surfaced through the queue
        q.put((rank, repr(e), 0, 0))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case,world", [("7pt", 2), ("scatter", 2), ("7pt", 3), ("multihop", 4)])
def test_halo_plan_gloo(case, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=180) for _ in range(world)]
    for p in ps:
        p.join(timeout=60)
    for rank, ok, nr, ns in res:
        assert ok is True, (rank, ok)
    if case == "multihop":
        assert max(r[2] for r in res) >= 3  # some rank receives from more than its two neighbours


def test_plan_pure_host():
    from paper_conf_icpp_sunzwzyr11_b200 import dist_plan, CRSDError

    rg = np.array([[0, 100, 0, 10], [100, 200, 10, 10], [200, 300, 10, 0]])
    recv, send = dist_plan(3, 1, rg)
    assert sorted(recv) == [(0, 90, 10), (2, 200, 10)]
    assert sorted(send) == [(0, 100, 10), (2, 190, 10)]
    bad = np.array([[0, 100, 0, 0], [120, 200, 0, 0]])
    with pytest.raises(CRSDError):
        dist_plan(2, 0, bad)


def test_partition_rows_balanced():
    from paper_conf_icpp_sunzwzyr11_b200 import partition_rows

    b = partition_rows(100_000, 512, 8)
    assert b[0] == 0 and b[-1] == 100_000 and np.all(np.diff(b) > 0)
    assert np.all(b[1:-1] % 512 == 0)
    w = np.ones(100_000)
    w[:50_000] = 3.0  # heavier first half
    b = partition_rows(100_000, 512, 4, w)
    loads = [w[b[i] : b[i + 1]].sum() for i in range(4)]
    assert max(loads) / (sum(loads) / 4) < 1.02


def test_partition_rows_never_empty():
    """Every rank gets at least one segment, also when the weights are
    concentrated or the ranks barely fit; more ranks than segments is an
    error at the cause (not an 'empty row range' later)."""
    from paper_conf_icpp_sunzwzyr11_b200 import CRSDError, partition_rows

    b = partition_rows(1000, 256, 4)  # 4 segments, 4 ranks
    assert list(b) == [0, 256, 512, 768, 1000]
    w = np.zeros(10_000)
    w[:10] = 1.0  # all the weight in the first segment
    b = partition_rows(10_000, 256, 8, w)
    assert np.all(np.diff(b) > 0) and b[0] == 0 and b[-1] == 10_000
    assert np.all(b[1:-1] % 256 == 0)
    w = np.zeros(10_000)
    w[-10:] = 1.0  # all the weight in the last segment
    b = partition_rows(10_000, 256, 8, w)
    assert np.all(np.diff(b) > 0)
    with pytest.raises(CRSDError, match="INVALID_ARG"):
        partition_rows(1000, 256, 8)
