"""World-size-2 CPU tests (gloo) of the tile-row sharding and the y
all-gather assembly used for N > 1 (paper_conf_ipps_niuldj0t21_b200/sharded.py).
Each rank's "SpMV" is the CPU oracle on its row slice (a CPU fake of the GPU
kernel), so the partition/assembly logic is tested without GPUs: the gathered
vector must equal the unsharded oracle y bitwise."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_niuldj0t21_b200.sharded import ShardedSpMV, partition_tile_rows


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, weighted, iters, q):
    try:
        from oracle import oracle as O
        from synthetic import gen
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        A, x = gen.make(name)
        w = None
        if weighted:
            idx = np.minimum(np.arange(0, A.m + 16, 16), A.m)
            w = np.diff(A.rowptr[idx].astype(np.int64))
        b = partition_tile_rows(A.m, world, w)
        S = A.row_slice(b[rank], b[rank + 1])

        def spmv(xf, yout):
            y, _ = O.spmv(S, xf.numpy())
            yout.copy_(torch.from_numpy(y))

        sh = ShardedSpMV(spmv, b, rank, world, device="cpu")
        xk = torch.from_numpy(x.copy())
        outs = []
        for _ in range(iters):
            xk = sh.step(xk).clone()
            outs.append(xk.numpy().copy())
        q.put((rank, b, outs))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, None, repr(e)))


@pytest.mark.parametrize("name,weighted", [("stencil27_21", False), ("rmat12", True),
                                           ("lap2d_37x29", True)])
def test_sharded_allgather_equals_unsharded(name, weighted):
    from oracle import oracle as O
    from synthetic import gen
    world, iters = 2, 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, weighted, iters, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for r, b, outs in res:
        assert b is not None, outs
    A, x = gen.make(name)
    # reference: the unsharded oracle iterate x_{k+1} = A x_k
    ref = []
    xk = x.copy()
    for _ in range(iters):
        xk, _ = O.spmv(A, xk)
        ref.append(xk.copy())
    for r, b, outs in res:
        assert b[0] == 0 and b[-1] == A.m and all(v % 16 == 0 for v in b[:-1])
        for k in range(iters):
            assert np.array_equal(outs[k].view(np.uint64), ref[k].view(np.uint64)), (name, r, k)


def test_partition_properties():
    for m, P in [(8_000_000, 8), (100, 3), (17, 4), (16, 2), (1, 2), (0, 2)]:
        b = partition_tile_rows(m, P)
        assert len(b) == P + 1 and b[0] == 0 and b[-1] == m
        assert all(b[i] <= b[i + 1] for i in range(P))
        assert all(v % 16 == 0 for v in b[:-1])
    b = partition_tile_rows(8_000_000, 8)
    assert b == [1_000_000 * i for i in range(9)]   # C5: 62,500 tile rows per rank
    w = np.ones(100)
    w[:10] = 50
    b = partition_tile_rows(1600, 4, w)
    loads = [w[b[i] // 16:b[i + 1] // 16].sum() for i in range(4)]
    assert max(loads) <= 1.5 * (w.sum() / 4) + 50


# ---------------------------------------------------------------------------
# halo exchange: neighbour-only x exchange + overlap
# ---------------------------------------------------------------------------

def _halo_worker(rank, world, port, name, iters, q):
    try:
        from oracle import oracle as O
        from paper_conf_ipps_niuldj0t21_b200.sharded import HaloSpMV, plan_halo
        from synthetic import gen
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        A, x = gen.make(name)
        b = partition_tile_rows(A.m, world)
        S = A.row_slice(b[rank], b[rank + 1])
        plan = plan_halo(S.rowptr, S.colidx, b, rank, world)

        def part_spmv(r0, r1):
            P = A.row_slice(r0, r1)

            def f(xf, yout):
                y, _ = O.spmv(P, xf.numpy())
                yout.copy_(torch.from_numpy(y))
            return f

        h = HaloSpMV(plan, [part_spmv(r0, r1) for r0, r1, _ in plan.parts])
        # x_0 is replicated; afterwards only own rows + halo are valid: poison
        # the rest so that a missing halo entry shows up as NaN
        xa = torch.from_numpy(x.copy())
        xb = torch.full((A.n,), float("nan"), dtype=torch.float64)
        outs = []
        for k in range(iters):
            h.step(xa, xb)
            outs.append(xb[b[rank]:b[rank + 1]].numpy().copy())
            xa, xb = xb, xa
            xb.fill_(float("nan"))
        q.put((rank, b, plan.as_dict(), outs))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, None, traceback.format_exc(), None))


@pytest.mark.parametrize("name,world", [("stencil27_40", 2), ("stencil27_21", 3), ("lap2d_37x29", 2),
                                        ("rmat12", 2)])
def test_halo_exchange_equals_unsharded(name, world):
    """Each rank's rows of x_k equal the unsharded oracle iterate bitwise,
    although only the halo (not the whole x) crossed ranks."""
    from oracle import oracle as O
    from synthetic import gen
    iters = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_halo_worker, args=(r, world, port, name, iters, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for r, b, plan, outs in res:
        assert b is not None, plan
    A, x = gen.make(name)
    ref, xk = [], x.copy()
    for _ in range(iters):
        xk, _ = O.spmv(A, xk)
        ref.append(xk.copy())
    for r, b, plan, outs in res:
        for k in range(iters):
            assert np.array_equal(outs[k].view(np.uint64), ref[k][b[r]:b[r + 1]].view(np.uint64)), (name, r, k)
        # parts tile the rank's rows on tile-row boundaries
        parts = plan["parts"]
        assert parts[0][0] == b[r] and parts[-1][1] == b[r + 1]
        assert all(parts[i][1] == parts[i + 1][0] for i in range(len(parts) - 1))
        assert all(p0 % 16 == 0 for p0, _, _ in parts)
    # send lists mirror recv lists
    sends = {(r, q, lo, hi) for r, b, plan, _ in res for q, lo, hi in plan["send"]}
    recvs = {(q, r, lo, hi) for r, b, plan, _ in res for q, lo, hi in plan["recv"]}
    assert sends == recvs


def test_halo_needs_stencil_closed_form():
    """27-point stencil nx^3 (nx = 40, so a rank boundary falls on a z-plane
    boundary), 2 ranks: each rank needs exactly the neighbouring z-plane
    (nx^2 rows) of the other, and exactly its own plane next to the boundary
    is boundary rows; everything else is interior."""
    from paper_conf_ipps_niuldj0t21_b200.sharded import halo_needs
    from synthetic import gen
    nx = 40
    A = gen.stencil27(nx)
    b = partition_tile_rows(A.m, 2)
    pl = nx * nx
    assert b[1] % pl == 0
    S0 = A.row_slice(b[0], b[1])
    recv0, parts0 = halo_needs(S0.rowptr, S0.colidx, b, 0)
    assert recv0 == [(1, b[1], b[1] + pl)]
    assert parts0 == [(0, b[1] - pl, True), (b[1] - pl, b[1], False)]
    S1 = A.row_slice(b[1], b[2])
    recv1, parts1 = halo_needs(S1.rowptr, S1.colidx, b, 1)
    assert recv1 == [(0, b[1] - pl, b[1])]
    assert parts1 == [(b[1], b[1] + pl, False), (b[1] + pl, b[2], True)]


# ---------------------------------------------------------------------------
# build_shard_handles: AUTO resolved on the global totals (host logic)
# ---------------------------------------------------------------------------

class _FakeHandle:
    """Stands in for TiledMatrix: info() of a shard, records the mode/kernel."""

    def __init__(self, sl, md, kn, stats):
        self.sl, self.md, self.kn = sl, md, kn
        self.stats = stats
        self.closed = False

    def info(self):
        return dict(self.stats)

    def close(self):
        self.closed = True


def _shard_worker(rank, world, port, q):
    try:
        from paper_conf_ipps_niuldj0t21_b200.sharded import build_shard_handles
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        # rank 0: 1.0M nnz, remainder-heavy; rank 1: 0.9M nnz, no remainder.
        # Each alone would resolve AUTO to ADPT (< 1.8M) and its own kernel;
        # together: 1.9M nnz -> DEFERRED, and the remainder's 12 B/entry are
        # 12 * 1.2M = 14.4 MB of 27 MB -> GATHER
        stats = [dict(payload_bytes=1_000_000, tilem=1000, rem_nnz=1_200_000, alg_bytes=16_000_000, nnz=1_000_000),
                 dict(payload_bytes=9_000_000, tilem=1000, rem_nnz=0, alg_bytes=11_000_000, nnz=900_000)][rank]
        made = []

        def create(sl, md, kn):
            h = _FakeHandle(sl, md, kn, stats)
            made.append(h)
            return h

        hs, md, kn = build_shard_handles(create, [(0, 16), (16, 32)], stats["nnz"], mode="AUTO", kernel="AUTO")
        q.put((rank, md, kn, [(h.md, h.kn) for h in hs], sum(h.closed for h in made)))
        dist.destroy_process_group()
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, None, traceback.format_exc(), None, None))


def test_build_shard_handles_resolves_auto_globally():
    """Every rank resolves AUTO mode (reading R18 on the global nnz) and the
    AUTO kernel (tilespmv_auto_kernel on the global totals) identically, so
    shards run the unsharded matrix's kernel and summation order; handles
    built with a provisional kernel are closed and rebuilt."""
    from paper_conf_ipps_niuldj0t21_b200.tilespmv import KERNELS, MODES
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_shard_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, md, kn, hs, closed in res:
        assert md == MODES["DEFERRED"], (rank, md, kn)
        assert kn == KERNELS["GATHER"], (rank, kn)
        assert hs == [(MODES["DEFERRED"], KERNELS["GATHER"])] * 2
        assert closed == 2  # the two provisional SM_QUEUE handles


# ---------------------------------------------------------------------------
# chunked all-gather overlapped with the SpMV (SURVEY §8(e) improvement 1)
# ---------------------------------------------------------------------------

def _chunked_worker(rank, world, port, name, chunks, iters, q):
    try:
        from oracle import oracle as O
        from paper_conf_ipps_niuldj0t21_b200.sharded import ChunkedAllGatherSpMV, chunk_bounds
        from synthetic import gen
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        A, x = gen.make(name)
        b = partition_tile_rows(A.m, world)
        cb = chunk_bounds(b, chunks)[rank]

        def part_spmv(r0, r1):
            P = A.row_slice(r0, r1)

            def f(xf, yout):
                y, _ = O.spmv(P, xf.numpy())
                yout.copy_(torch.from_numpy(y))
            return f

        C = ChunkedAllGatherSpMV([part_spmv(cb[i], cb[i + 1]) for i in range(chunks)], b, rank, world)
        xa = torch.from_numpy(x.copy())
        xb = torch.full((A.n,), float("nan"), dtype=torch.float64)  # every row must be written or received
        outs = []
        for k in range(iters):
            C.step(xa, xb)
            outs.append(xb.numpy().copy())
            xa, xb = xb, xa
            xb.fill_(float("nan"))
        q.put((rank, b, outs))
        dist.destroy_process_group()
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, None, traceback.format_exc()))


@pytest.mark.parametrize("name,world,chunks", [("stencil27_21", 2, 3), ("rmat12", 3, 4), ("lap2d_37x29", 2, 5)])
def test_chunked_allgather_equals_unsharded(name, world, chunks):
    """Every rank holds the full x_{k+1}, bitwise equal to the unsharded
    oracle iterate (x_{k+1} starts as NaN: a row neither computed nor received
    would show)."""
    from oracle import oracle as O
    from synthetic import gen
    iters = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_chunked_worker, args=(r, world, port, name, chunks, iters, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for r, b, outs in res:
        assert b is not None, outs
    A, x = gen.make(name)
    ref, xk = [], x.copy()
    for _ in range(iters):
        xk, _ = O.spmv(A, xk)
        ref.append(xk.copy())
    for r, b, outs in res:
        for k in range(iters):
            assert np.array_equal(outs[k].view(np.uint64), ref[k].view(np.uint64)), (name, r, k)


def test_chunk_bounds():
    from paper_conf_ipps_niuldj0t21_b200.sharded import chunk_bounds
    b = partition_tile_rows(8_000_000, 8)
    cb = chunk_bounds(b, 4)
    assert cb[0] == [0, 250_000, 500_000, 750_000, 1_000_000]   # C5 at N = 8: 15,625 tile rows per chunk
    for bounds, C in [([0, 37, 100], 3), ([0, 16, 17], 4), ([0, 0, 48], 2), (partition_tile_rows(1000, 3), 7)]:
        for r, c in enumerate(chunk_bounds(bounds, C)):
            assert len(c) == C + 1 and c[0] == bounds[r] and c[-1] == bounds[r + 1]
            assert all(c[i] <= c[i + 1] for i in range(C))
            assert all((v - bounds[r]) % 16 == 0 for v in c[:-1])
