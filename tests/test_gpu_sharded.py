"""Multi-GPU readiness on one GPU (north_star item 4, §8(f)
f1): two ranks share cuda:0 over gloo (host-staged exchange, since gloo
cannot move device tensors) and run the sharded iterated SpMV
x_{k+1} = A x_k with the CUDA kernel as every part's SpMV -- the all-gather
step (ShardedSpMV) and the halo step (HaloSpMV, non-halo x poisoned with
NaN).  Every iterate must equal the 1-GPU CUDA iterate bit for bit (tile-row
sharding keeps each row's summation order) and each step must stay
within the north_star bound of the oracle applied to the same input.  A
world-size-1 NCCL group checks the NCCL collective path on the device."""
import os
import socket

import numpy as np
import pytest

from test_gpu_parity import assert_spmv_close

pytestmark = pytest.mark.gpu

ITERS = 3


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _make(name):
    from synthetic import gen
    A, x = gen.make(name)
    # iterate a scaled A so that x_k stays O(1) over ITERS steps
    return A, x


def _rank_worker(rank, world, port, name, exchange, q):
    try:
        import torch
        import torch.distributed as dist
        from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
        from paper_conf_ipps_niuldj0t21_b200.sharded import (ChunkedAllGatherSpMV, FusedScatterSpMV, HaloSpMV,
                                                             ShardedSpMV, build_shard_handles, chunk_bounds,
                                                             partition_tile_rows, plan_halo)
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        dev = torch.device("cuda", 0)
        torch.cuda.set_device(dev)
        A, x = _make(name)
        w = np.diff(A.rowptr[np.minimum(np.arange(0, A.m + 16, 16), A.m)].astype(np.int64))
        b = partition_tile_rows(A.m, world, w)
        a0, a1 = b[rank], b[rank + 1]
        S = A.row_slice(a0, a1)

        def create(sl, md, kn):
            r0, r1 = sl
            P = A.row_slice(r0, r1)
            return TiledMatrix.from_csr(torch.from_numpy(P.rowptr).to(dev), torch.from_numpy(P.colidx).to(dev),
                                        torch.from_numpy(P.val).to(dev), P.m, P.n, mode=md, kernel=kn)

        outs = []
        if exchange == "allgather":
            (M,), md, kn = build_shard_handles(create, [(a0, a1)], S.nnz)
            sh = ShardedSpMV(lambda xf, yo: M.run(xf, yo), b, rank, world, device=dev, host_staging=True)
            xk = torch.from_numpy(x).to(dev)
            for _ in range(ITERS):
                xk = sh.step(xk).clone()
                torch.cuda.synchronize()
                outs.append(xk.cpu().numpy())
            M.close()
        elif exchange == "fused":  # the kernel stores y into every rank's x_{k+1} over CUDA IPC
            (M,), md, kn = build_shard_handles(create, [(a0, a1)], S.nnz)
            F = FusedScatterSpMV(M, b, rank, world, torch.from_numpy(x).to(dev))
            for _ in range(ITERS):
                outs.append(F.step().cpu().numpy())
            F.close()
            M.close()
        elif exchange == "chunked":  # all-gather overlapped with the SpMV, 3 chunks per rank
            cb = chunk_bounds(b, 3)[rank]
            hs, md, kn = build_shard_handles(create, [(cb[i], cb[i + 1]) for i in range(3)], S.nnz)
            C = ChunkedAllGatherSpMV([lambda xf, yo, M=M: M.run(xf, yo) for M in hs], b, rank, world,
                                     host_staging=True)
            xa = torch.from_numpy(x.copy()).to(dev)
            xb = torch.full((A.n,), float("nan"), dtype=torch.float64, device=dev)
            for _ in range(ITERS):
                C.step(xa, xb)
                torch.cuda.synchronize()
                outs.append(xb.cpu().numpy())
                xa, xb = xb, xa
                xb.fill_(float("nan"))  # every row must be computed or received
            for M in hs:
                M.close()
        else:
            plan = plan_halo(S.rowptr, S.colidx, b, rank, world)
            hs, md, kn = build_shard_handles(create, [(r0, r1) for r0, r1, _ in plan.parts], S.nnz)
            H = HaloSpMV(plan, [lambda xf, yo, M=M: M.run(xf, yo) for M in hs], host_staging=True)
            xa = torch.from_numpy(x.copy()).to(dev)
            xb = torch.full((A.n,), float("nan"), dtype=torch.float64, device=dev)
            for _ in range(ITERS):
                H.step(xa, xb)
                torch.cuda.synchronize()
                outs.append(xb[a0:a1].cpu().numpy())
                xa, xb = xb, xa
                xb.fill_(float("nan"))  # only own rows + the halo may be read
            for M in hs:
                M.close()
        q.put((rank, b, (md, kn), outs))
        dist.destroy_process_group()
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, None, traceback.format_exc(), None))


@pytest.mark.parametrize("exchange", ["allgather", "halo", "chunked", "fused"])
@pytest.mark.parametrize("name", ["stencil27_40", "rmat12", "lap2d_37x29", "mixed_small"])
def test_sharded_cuda_iterates_bitwise_equal_one_gpu(cuda_device, name, exchange):
    import torch
    import torch.multiprocessing as mp
    from oracle import oracle as O
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_rank_worker, args=(r, world, port, name, exchange, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
    for r, b, info, outs in res:
        assert b is not None, info
    A, x = _make(name)
    # the 1-GPU CUDA iterate (kernel AUTO on the whole matrix) and the oracle
    ref, xk = [], torch.from_numpy(x).to(cuda_device)
    with TiledMatrix.from_host_csr(A, device=cuda_device) as M:
        kn1 = M.info()["kernel"]
        for _ in range(ITERS):
            xprev = xk.cpu().numpy()
            xk = M.run(xk).clone()
            y = xk.cpu().numpy()
            yref, absy = O.spmv(A, xprev)
            assert_spmv_close(y, yref, absy, f"{name} one-GPU step")
            ref.append(y)
    for r, b, (md, kn), outs in res:
        assert kn == kn1, (name, r, kn, kn1)
        for k in range(ITERS):
            got = outs[k] if exchange == "halo" else outs[k][b[r]:b[r + 1]]
            assert np.array_equal(got.view(np.uint64), ref[k][b[r]:b[r + 1]].view(np.uint64)), (name, exchange, r, k)
            if exchange in ("allgather", "chunked", "fused"):  # every rank holds the whole iterate
                assert np.array_equal(outs[k].view(np.uint64), ref[k].view(np.uint64))


def _nccl_worker(port, q):
    try:
        import torch
        import torch.distributed as dist
        from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
        from paper_conf_ipps_niuldj0t21_b200.sharded import ShardedSpMV, build_shard_handles
        from synthetic import gen
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dev = torch.device("cuda", 0)
        torch.cuda.set_device(dev)
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
        t = torch.arange(10, dtype=torch.float64, device=dev)
        out = torch.empty(10, dtype=torch.float64, device=dev)
        dist.all_gather_into_tensor(out, t)
        ok_ag = bool(torch.equal(out, t))
        A, x = gen.make("stencil27_21")

        def create(sl, md, kn):
            return TiledMatrix.from_host_csr(A, mode=md, kernel=kn, device=dev)

        (M,), _, _ = build_shard_handles(create, [(0, A.m)], A.nnz, device=dev)
        sh = ShardedSpMV(lambda xf, yo: M.run(xf, yo), [0, A.m], 0, 1, device=dev)
        xd = torch.from_numpy(x).to(dev)
        y_sh = sh.step(xd).clone()
        y_1 = M.run(xd)
        torch.cuda.synchronize()
        q.put((ok_ag, bool(torch.equal(y_sh, y_1))))
        M.close()
        dist.destroy_process_group()
    except Exception:  # pragma: no cover
        import traceback
        q.put((traceback.format_exc(), None))


def test_nccl_world_size_one_smoke(cuda_device):
    """NCCL on the device: init a world-size-1 group, all-gather a device
    tensor, and run one ShardedSpMV step whose exchange is the NCCL
    all_gather_into_tensor; y equals the plain run bit for bit."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_nccl_worker, args=(_port(), q))
    p.start()
    ok_ag, ok_step = q.get(timeout=600)
    p.join(timeout=120)
    assert ok_ag is True, ok_ag
    assert ok_step is True
