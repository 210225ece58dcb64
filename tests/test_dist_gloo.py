"""World-size-2 (gloo, CPU) test of the multi-GPU decomposition (reading R18):
the library's shard bounds (fp_shard_rows_*), per-rank local evaluation with beta*z on rank 0
only, and ONE sum-allreduce of w reproduce the single-process result -- exactly on integer
twins.  The local evaluation here is the oracle (test infrastructure); on GPUs the same
bounds feed fp_*_dist, whose NCCL path is exercised by test_drivers_gpu."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, fmt, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import oracle
    import paper_conf_ppopp_asharitbrcks15_b200 as fp
    import synth

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        m, n = 3001, 57
        y = synth.vector(n, "f64", kind="int_small", seed=1, stream=synth.S_Y)
        z = synth.vector(n, "f64", kind="int_small", seed=1, stream=synth.S_Z)
        v = synth.vector(m, "f64", kind="int_pos", seed=1, stream=synth.S_V)
        if fmt == "dense":
            X = synth.dense(m, n, "f64", kind="int_pm12", seed=1)
            b = fp.shard_rows_dense(m, world)
            r0, r1 = b[rank], b[rank + 1]
            Xl = synth.dense(r1 - r0, n, "f64", kind="int_pm12", seed=1, row0=r0)   # generated shard
            assert torch.equal(Xl, X[r0:r1])
            wl, _ = oracle.dense(Xl, y, v[r0:r1], z if rank == 0 else None, 2.0, -1.5 if rank == 0 else 0.0)
            full, _ = oracle.dense(X, y, v, z, 2.0, -1.5)
        else:
            rp, ci, va = synth.csr(m, n, "f64", ("powerlaw", 2.0, 3.0), kind="int_pm12", seed=1)
            b = fp.shard_rows_csr(rp, world)
            lrp, lci, lva, lv = fp.shard_slice_csr(rp, ci, va, v, b, rank)
            g = synth.csr(b[rank + 1] - b[rank], n, "f64", ("powerlaw", 2.0, 3.0), kind="int_pm12", seed=1,
                          row0=b[rank])                                               # generated shard
            assert all(torch.equal(x, y_) for x, y_ in zip(g, (lrp, lci, lva)))
            wl, _ = oracle.csr(b[rank + 1] - b[rank], n, lrp, lci, lva, y, lv, z if rank == 0 else None, 2.0,
                               -1.5 if rank == 0 else 0.0)
            full, _ = oracle.csr(m, n, rp, ci, va, y, v, z, 2.0, -1.5)
            nnz_local = torch.tensor([int(lrp[-1])])
            dist.all_reduce(nnz_local)
            assert int(nnz_local) == int(rp[-1])
        t = torch.from_numpy(wl)
        dist.all_reduce(t)                                   # the one exchange step
        q.put((rank, bool(np.array_equal(t.numpy(), full))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("fmt", ["dense", "csr"])
def test_two_rank_decomposition_exact(fmt):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, fmt, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    res = dict(q.get(timeout=5) for _ in range(2))
    assert all(p.exitcode == 0 for p in procs)
    assert res == {0: True, 1: True}
