"""Multi-rank row-partitioned SpMV and CG through the peer-memory transport
(csrc/p2p.cu, crsd_comm_init_p2p): REAL separate processes, one rank each,
bootstrapped over gloo, exchanging x halos and CG dots through CUDA-IPC-mapped
device memory with the library's own kernels (BASELINE.json north_star (3),
SURVEY.md §8(a) a7 / §8(e)).

The gpurun boxes have one GPU, so all ranks share cuda:0 here (NCCL refuses
that: profiles/r01_nccl_shared_gpu_probe.txt); the IPC mappings, flag
handshakes, mailbox parities, multi-hop plans and the interior/boundary
overlap run exactly as they would across GPUs, only the bytes travel through
one HBM instead of NVLink. Each rank's y must match the same rows of the
global oracle product (oracle/coo.py) within the north-star tolerance, over
several consecutive exchanges (both mailbox parities, epochs > 2) with a new
x every call; the distributed CG must match the CG oracle (oracle/cg_ref.py)
step by step with the tolerances of tests/test_gpu_cg.py; the scalar
allreduce must be bit-identical on every rank and equal the rank-order sum.
"""
import os
import socket

import numpy as np
import pytest

import gen
from oracle import cg_ref, coo

pytestmark = pytest.mark.gpu

TOL = {np.float64: 1e-12, np.float32: 1e-5}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _matrix(case):
    if case == "c2":
        return gen.config2(n=40), np.float64, 256
    if case == "c3":
        return gen.config3(n=36), np.float64, 256
    if case == "c4":
        return gen.config4(n=300_000), np.float32, 512
    if case == "multihop":  # offsets wider than a rank's block: halos from 2+ owners per side
        n = 4096
        return gen.band(n, [(0, n, [-1500, -3, -1, 0, 1, 700, 1300])], seed=7), np.float64, 256
    if case == "cg7pt":
        return gen.spd_stencil_scatter((24, 24, 24), "7pt", n_pairs=200, seed=3), np.float64, 256
    if case == "cg7pt32":
        return gen.spd_stencil_scatter((24, 24, 24), "7pt", n_pairs=200, seed=3), np.float32, 256
    raise ValueError(case)


def _worker(rank, world, port, case, variant, q, mode="mailbox", distinct=False, transport="p2p"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch
    import torch.distributed as dist

    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = {"rank": rank}
    try:
        from paper_conf_icpp_sunzwzyr11_b200 import Comm, CRSDMatrix, P2PComm, partition_rows

        dev = rank if distinct else 0  # distinct: one GPU per rank (halos over NVLink)
        torch.cuda.set_device(dev)
        a, dt, mrows = _matrix(case)
        a = a.astype(dt)
        n = a.nrows
        tdt = torch.float64 if dt == np.float64 else torch.float32
        bounds = partition_rows(n, mrows, world, np.bincount(a.row, minlength=n).astype(np.float64))
        rb, re = int(bounds[rank]), int(bounds[rank + 1])
        m = (a.row >= rb) & (a.row < re)
        from paper_conf_icpp_sunzwzyr11_b200 import TUNE_HALO_UNFUSED

        tune = TUNE_HALO_UNFUSED if mode == "direct-unfused" else 0
        A = CRSDMatrix.from_coo(n, n, a.row[m], a.col[m], a.val[m], mrows=mrows, row_range=(rb, re),
                                variant=0 if variant == "timeout" else variant, device=dev, tune=tune)
        if variant == "timeout":
            os.environ["CRSD_P2P_TIMEOUT_S"] = "2"
        # capacities differ per rank on purpose: a receiver must address the
        # sender's parity-1 mailbox with the sender's capacity, not its own
        if transport == "nccl":
            comm = Comm(rank, world, dev)
        else:
            comm = P2PComm(rank, world, dev, mailbox_bytes=(1 << 20) * (rank + 1))
        A.dist_bind(comm)
        lo, nloc, hi = A.x_layout()
        if variant == "timeout":
            # rank 1 never joins the exchange: rank 0's receive must give up
            # after 2 s and report it instead of hanging the GPU
            if rank == 0:
                xd = torch.zeros(lo + nloc + hi, device=f"cuda:{dev}", dtype=tdt)
                yd = torch.empty(nloc, device=f"cuda:{dev}", dtype=tdt)
                A.spmv_dist(xd, yd, 1.0, 0.0, comm)
                torch.cuda.synchronize()
            dist.barrier()
            out["err"] = comm.error()
            comm.close()
            return
        if case.startswith("cg"):
            rng = np.random.default_rng(11)
            b = rng.uniform(-1, 1, n)
            x0 = np.zeros(n)
            iters = 40
            bd = torch.from_numpy(b[rb:re].astype(dt)).to(f"cuda:{dev}")
            xd = torch.from_numpy(x0[rb:re].astype(dt)).to(f"cuda:{dev}")
            res = A.cg(bd, xd, iters, 0.0, check_every=7, comm=comm, history=True)
            torch.cuda.synchronize()
            xr, _, hr = cg_ref.cg(a, b.astype(dt).astype(np.float64), x0, res["iterations"])
            h = res["rr_history"]
            floor = 1e-20 if dt == np.float64 else 1e-8
            live = hr / hr[0] >= floor
            out["rr_rel"] = float((np.abs(h[live] - hr[live]) / hr[live]).max())
            out["x_rel"] = float(np.max(np.abs(xd.cpu().numpy() - xr[rb:re])) / np.max(np.abs(xr)))
            out["iterations"] = res["iterations"]
            out["rr_bits"] = h.tobytes().hex()
        else:
            errs = []
            stream = torch.cuda.Stream()
            if mode.startswith("direct"):
                # the library-owned padded x, mapped by every peer: the halo
                # arrives as one-sided puts. NaN pads once, before any rank
                # can put (barrier): every call must overwrite them.
                xdir = A.dist_x_alloc(comm)
                xdir.fill_(float("nan"))
                torch.cuda.synchronize()
                dist.barrier()
            for call in range(5):  # epochs 1..5: both mailbox parities, reuse after consumed
                x = np.random.default_rng(100 + call).uniform(-1, 1, n).astype(dt)
                yref, scale = coo.coo_spmv(n, n, a.row, a.col, a.val, x)
                if mode.startswith("direct"):
                    # only the owned part is ours to write; peers write the pads
                    xdir[lo : lo + nloc].copy_(torch.from_numpy(x[rb:re]).to(f"cuda:{dev}", tdt))
                    xd = xdir
                else:
                    xp = np.full(lo + nloc + hi, np.nan, dt)  # pads must be written by the exchange
                    xp[lo : lo + nloc] = x[rb:re]
                    xd = torch.from_numpy(xp).to(f"cuda:{dev}", tdt)
                yd = torch.full((nloc,), float("nan"), device=f"cuda:{dev}", dtype=tdt)
                # xd / yd were written on the default stream; the side stream
                # (non-blocking) must not start before those writes land, or
                # the NaN pads of xd could overwrite the received halo
                stream.wait_stream(torch.cuda.current_stream())
                with torch.cuda.stream(stream):
                    A.spmv_dist(xd, yd, 1.0, 0.0, comm, stream=stream)
                stream.synchronize()
                errs.append(coo.parity_error(yd.cpu().numpy(), yref[rb:re], scale[rb:re]))
            out["errs"] = errs
            out["launches"] = A.last_launch_count()
            if mode.startswith("direct") and case == "c2":
                # a CG on the same handle uses a direct buffer of its own for
                # p: the caller's x_padded (owned part and halo) must survive
                keep = xdir.clone()
                y_before = yd.clone()
                bd = torch.ones(nloc, dtype=tdt, device=f"cuda:{dev}")
                xc = torch.zeros(nloc, dtype=tdt, device=f"cuda:{dev}")
                A.cg(bd, xc, 3, 0.0, check_every=3, comm=comm)
                torch.cuda.synchronize()
                out["x_kept"] = bool(torch.equal(xdir[lo : lo + nloc], keep[lo : lo + nloc]))
                y2 = torch.full((nloc,), float("nan"), device=f"cuda:{dev}", dtype=tdt)
                stream.wait_stream(torch.cuda.current_stream())
                with torch.cuda.stream(stream):
                    A.spmv_dist(xdir, y2, 1.0, 0.0, comm, stream=stream)
                stream.synchronize()
                out["y_same_after_cg"] = bool(torch.equal(y2, y_before))
            # scalar allreduce: every rank contributes distinct values; results bit-identical
            v = torch.tensor([0.1 * (rank + 1), 1e16 * (-1) ** rank, 3.0 + rank / 7.0], dtype=torch.float64, device=f"cuda:{dev}")
            comm.allreduce_f64(v)
            torch.cuda.synchronize()
            out["red"] = v.cpu().numpy().tobytes().hex()
        out["err"] = comm.error()
        comm.close()
        A.close() if hasattr(A, "close") else None
    except Exception as e:  # pragma: no cover - surfaced through the queue
        import traceback

        out["exc"] = repr(e) + traceback.format_exc()
    finally:
        q.put(out)
        dist.destroy_process_group()


def _run(case, world, variant=0, check_err=True, mode="mailbox", distinct=False, transport="p2p"):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, case, variant, q, mode, distinct, transport)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=400) for _ in range(world)]
    for p in ps:
        p.join(timeout=60)
    res.sort(key=lambda r: r["rank"])
    for r in res:
        assert "exc" not in r, r["exc"]
        assert not check_err or r["err"] == 0, f"rank {r['rank']}: a peer-memory wait timed out (code {r['err']})"
    return res


@pytest.fixture(scope="module")
def torch_cuda():
    import torch

    if not torch.cuda.is_available():
        pytest.fail("no CUDA device: -m gpu tests need a B200")
    return torch


@pytest.mark.parametrize(
    "case,world,variant,mode",
    [("c2", 2, 0, "mailbox"), ("c3", 2, 0, "mailbox"), ("c4", 2, 0, "mailbox"), ("c2", 3, 4, "mailbox"),
     ("c3", 3, 3, "mailbox"), ("multihop", 4, 0, "mailbox"), ("c4", 4, 1, "mailbox"),
     ("c2", 2, 0, "direct"), ("c3", 3, 0, "direct"), ("c4", 2, 0, "direct"), ("multihop", 4, 0, "direct"),
     ("c3", 2, 0, "direct-unfused"), ("multihop", 4, 0, "direct-unfused"), ("c3", 2, 3, "direct")],
)
def test_p2p_spmv_dist(torch_cuda, case, world, variant, mode):
    """mailbox: caller-owned x_padded, two-stage exchange; direct: the
    crsd_dist_x_alloc buffer, one-sided puts into the neighbours' pads, the
    receive fused into the boundary kernel (JIT variant; separate wait /
    release kernels with CRSD_TUNE_HALO_UNFUSED or a table-driven variant)."""
    _, dt, _ = _matrix(case)
    res = _run(case, world, variant, mode=mode)
    for r in res:
        assert max(r["errs"]) <= TOL[dt], (r["rank"], r["errs"])
        if "x_kept" in r:
            assert r["x_kept"] and r["y_same_after_cg"], r
    # bit-identical allreduce on every rank, equal to the rank-order sum
    vals = [np.array([0.1 * (q + 1), 1e16 * (-1) ** q, 3.0 + q / 7.0]) for q in range(world)]
    expect = np.zeros(3)
    for v in vals:
        expect = expect + v
    for r in res:
        got = np.frombuffer(bytes.fromhex(r["red"]), np.float64)
        assert got.tobytes() == expect.tobytes(), (r["rank"], got, expect)


@pytest.mark.parametrize("case,world", [("cg7pt", 2), ("cg7pt", 3), ("cg7pt32", 2)])
def test_p2p_cg(torch_cuda, case, world):
    """Distributed CG (halo exchange + allreduced dots through peer memory,
    graph-captured batches) against the CG oracle; every rank must see the
    same residual history bit for bit (deterministic allreduce)."""
    _, dt, _ = _matrix(case)
    res = _run(case, world)
    rr_tol = 1e-11 if dt == np.float64 else 1e-3
    x_tol = 1e-12 if dt == np.float64 else 1e-4
    for r in res:
        assert r["rr_rel"] <= rr_tol, r
        assert r["x_rel"] <= x_tol, r
    assert len({r["rr_bits"] for r in res}) == 1


def test_p2p_wait_is_bounded(torch_cuda):
    """A peer that never arrives: the waiting kernel gives up after
    CRSD_P2P_TIMEOUT_S (2 s here) and crsd_comm_error reports the receive
    timeout (2) on that rank; the other rank saw nothing wrong."""
    res = _run("c2", 2, "timeout", check_err=False)
    assert res[0]["err"] == 2 and res[1]["err"] == 0, res


def _ngpus():
    import torch

    return torch.cuda.device_count() if torch.cuda.is_available() else 0


@pytest.mark.parametrize("transport,mode", [("p2p", "mailbox"), ("p2p", "direct"), ("nccl", "mailbox")])
@pytest.mark.parametrize("case", ["c2", "c4", "multihop"])
def test_distinct_devices_spmv_dist(torch_cuda, case, transport, mode):
    """Ranks on DISTINCT GPUs (runs whenever >= 2 are visible; the gpurun
    boxes have one): the halo crosses NVLink -- NCCL send/recv, or the
    library's peer-memory kernels (mailbox pull or one-sided puts) -- and each
    rank's rows match the oracle over 5 consecutive exchanges."""
    world = min(_ngpus(), 4 if case == "multihop" else 2)
    if world < 2:
        pytest.skip("needs >= 2 visible GPUs")
    _, dt, _ = _matrix(case)
    res = _run(case, world, 0, mode=mode, distinct=True, transport=transport)
    for r in res:
        assert max(r["errs"]) <= TOL[dt], (r["rank"], r["errs"])


@pytest.mark.parametrize("transport", ["p2p", "nccl"])
def test_distinct_devices_cg(torch_cuda, transport):
    """Distributed CG with one GPU per rank (>= 2 visible GPUs) against the CG oracle."""
    if _ngpus() < 2:
        pytest.skip("needs >= 2 visible GPUs")
    res = _run("cg7pt", 2, distinct=True, transport=transport)
    for r in res:
        assert r["rr_rel"] <= 1e-11 and r["x_rel"] <= 1e-12, r
    if transport == "p2p":
        assert len({r["rr_bits"] for r in res}) == 1
