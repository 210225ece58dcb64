"""The multi-GPU exchange step on real NCCL communicators.

* ``test_nccl_allreduce_runs_one_rank`` -- a child process with NCCL_DEBUG=INFO /
  NCCL_DEBUG_SUBSYS=COLL calls fp_dense_dist / fp_csr_dist through a one-rank libfusedpat
  communicator and the test asserts that NCCL logged the AllReduce launches (the collective
  is never short-cut at one rank) and that w still matches the oracle.
* ``test_two_rank_nccl_*`` -- world size 2 (one process per GPU, torch.distributed bootstrap
  of the NCCL unique id, exactly what bench.py does under torchrun): the row shards of
  fp_shard_rows_* evaluated by fp_*_dist with beta*z on rank 0 only (reading R18), checked
  bit for bit against the oracle on integer twins (every summation order is exact there)
  and within the north_star tolerance on U[-1,1) data; plus the CG and TRON drivers with a
  communicator against their single-GPU runs.  Skipped on a box with fewer than 2 GPUs.
"""
import os
import socket
import subprocess
import sys
import textwrap

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_nccl_allreduce_runs_one_rank(cuda_dev):
    code = textwrap.dedent(f"""
        import ctypes, sys
        sys.path.insert(0, {ROOT!r}); sys.path.insert(0, {os.path.join(ROOT, 'tests')!r})
        import torch, numpy as np
        import oracle, synth
        import paper_conf_ppopp_asharitbrcks15_b200 as fp
        from _util import assert_bitexact
        uid = (ctypes.c_ubyte * 128)()
        fp.fp_comm_get_unique_id(ctypes.cast(uid, ctypes.c_void_p))
        h = ctypes.c_void_p()
        fp.fp_comm_init(ctypes.byref(h), 1, 0, ctypes.cast(uid, ctypes.c_void_p), 0)
        class C:
            handle = h
        d = torch.device("cuda:0")
        X = synth.dense(2000, 70, "f64", kind="int_pm12", seed=3)
        y = synth.vector(70, "f64", kind="int_small", seed=3)
        z = synth.vector(70, "f64", kind="int_small", seed=3, stream=synth.S_Z)
        ref, _ = oracle.dense(X, y, None, z, 2.0, -1.5)
        w = fp.dense_dist(C, X.to(d), y.to(d), None, z.to(d), 2.0, -1.5)
        torch.cuda.synchronize()
        assert_bitexact(w, ref, "dense_dist")
        rp, ci, va = synth.csr(3000, 70, "f64", ("binomial", 0.1), kind="int_pm12", seed=4)
        ref, _ = oracle.csr(3000, 70, rp, ci, va, y, None, z, 2.0, -1.5)
        w = fp.csr_dist(C, rp.to(d), ci.to(d), va.to(d), 70, y.to(d), None, z.to(d), 2.0, -1.5)
        torch.cuda.synchronize()
        assert_bitexact(w, ref, "csr_dist")
        fp.fp_comm_destroy(h)
        print("CHILD_OK")
    """)
    env = dict(os.environ, NCCL_DEBUG="INFO", NCCL_DEBUG_SUBSYS="COLL")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
    out = r.stdout + r.stderr
    assert r.returncode == 0 and "CHILD_OK" in out, out[-4000:]
    n_ar = sum(1 for ln in out.splitlines() if "AllReduce" in ln)
    assert n_ar >= 2, "NCCL logged no AllReduce launch:\n" + out[-4000:]


def test_nvls_one_rank(cuda_dev):
    """FP_COMM_NVLS on a one-rank communicator: the multicast object, the multimem.red
    barrier and the multimem.ld_reduce sum run on the hardware (with one device the switch
    sums one copy); integer twins bit-exact, three calls (both buffer parities), allreduce."""
    import ctypes

    import oracle
    import paper_conf_ppopp_asharitbrcks15_b200 as fp
    import synth
    from _util import assert_bitexact

    uid = (ctypes.c_ubyte * 128)()
    fp.fp_comm_get_unique_id(ctypes.cast(uid, ctypes.c_void_p))
    h = ctypes.c_void_p()
    fp.fp_comm_init(ctypes.byref(h), 1, 0, ctypes.cast(uid, ctypes.c_void_p), 0)
    c = fp.Comm.__new__(fp.Comm)
    c.rank, c.size, c.device, c.handle = 0, 1, 0, h
    try:
        try:
            c.enable_nvls(1 << 20)
        except fp.FusedPatError as e:
            pytest.skip(f"no NVLS here: {e}")
        assert c.mode == fp.FP_COMM_NVLS
        n = 3000
        rp, ci, va = synth.csr(40_000, n, "f32", ("powerlaw", 2.5, 13.64), kind="int_pm12", seed=31)
        y = synth.vector(n, "f32", kind="int_small", seed=31, stream=synth.S_Y)
        z = synth.vector(n, "f32", kind="int_small", seed=31, stream=synth.S_Z)
        v = synth.vector(40_000, "f32", kind="int_pos", seed=31, stream=synth.S_V)
        ref, _ = oracle.csr(40_000, n, rp, ci, va, y, v, z, 1.0, 3.0)
        d = cuda_dev
        for _ in range(3):
            w = fp.csr_dist(c, rp.to(d), ci.to(d), va.to(d), n, y.to(d), v.to(d), z.to(d), 1.0, 3.0)
            torch.cuda.synchronize()
            assert_bitexact(w, ref, "nvls csr_dist")
        X = synth.dense(5000, 64, "f64", kind="int_pm12", seed=32)
        y2 = synth.vector(64, "f64", kind="int_small", seed=32)
        ref, _ = oracle.dense(X, y2, None, None, 2.0, 0.0)
        w = fp.dense_dist(c, X.to(d), y2.to(d), None, None, 2.0, 0.0)
        torch.cuda.synchronize()
        assert_bitexact(w, ref, "nvls dense_dist")
        t = torch.arange(1000, dtype=torch.float64, device=d)
        c.allreduce(t)
        torch.cuda.synchronize()
        assert torch.equal(t.cpu(), torch.arange(1000, dtype=torch.float64))
        assert fp.lib().fp_comm_timed_out(h) == 0
    finally:
        fp.fp_comm_destroy(h)


def _worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import torch.distributed as dist

    import oracle
    import paper_conf_ppopp_asharitbrcks15_b200 as fp
    import synth
    from _util import assert_bitexact, assert_parity

    torch.cuda.set_device(rank)
    dev = torch.device("cuda", rank)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
    comm = fp.Comm(device=rank)
    msgs = []
    try:
        # ---- dense, integer twin: bit-exact against the full-matrix oracle
        m, n = 20011, 131
        y = synth.vector(n, "f64", kind="int_small", seed=11, stream=synth.S_Y)
        z = synth.vector(n, "f64", kind="int_small", seed=11, stream=synth.S_Z)
        v = synth.vector(m, "f64", kind="int_pos", seed=11, stream=synth.S_V)
        X = synth.dense(m, n, "f64", kind="int_pm12", seed=11)
        full, _ = oracle.dense(X, y, v, z, 2.0, -1.5)
        b = fp.shard_rows_dense(m, world)
        r0, r1 = b[rank], b[rank + 1]
        w = fp.dense_dist(comm, X[r0:r1].contiguous().to(dev), y.to(dev), v[r0:r1].to(dev), z.to(dev), 2.0, -1.5)
        torch.cuda.synchronize()
        assert_bitexact(w, full, f"dense_dist rank {rank}")
        msgs.append("dense-int")

        # ---- CSR (C3/C4-shaped rows), integer twin fp64 and fp32, nnz-quantile shards
        for dt, lengths, nn in (("f64", ("binomial", 0.01), 1000), ("f32", ("powerlaw", 2.5, 13.64), 20000)):
            mm = 60000
            rp, ci, va = synth.csr(mm, nn, dt, lengths, kind="int_pm12", seed=12)
            yy = synth.vector(nn, dt, kind="int_small", seed=12, stream=synth.S_Y)
            zz = synth.vector(nn, dt, kind="int_small", seed=12, stream=synth.S_Z)
            vv = synth.vector(mm, dt, kind="int_pos", seed=12, stream=synth.S_V)
            full, _ = oracle.csr(mm, nn, rp, ci, va, yy, vv, zz, 1.0, 1.0)
            bb = fp.shard_rows_csr(rp, world)
            lrp, lci, lva, lv = fp.shard_slice_csr(rp, ci, va, vv, bb, rank)
            w = fp.csr_dist(comm, lrp.contiguous().to(dev), lci.contiguous().to(dev), lva.contiguous().to(dev), nn,
                            yy.to(dev), lv.contiguous().to(dev), zz.to(dev), 1.0, 1.0)
            torch.cuda.synchronize()
            assert_bitexact(w, full, f"csr_dist {dt} rank {rank}")
            if dt == "f32":  # the packed plan of the shard through NCCL
                plan = fp.CsrPlan(lrp.contiguous().to(dev), lci.contiguous().to(dev), nn, torch.float32)
                plan.pack(lva.contiguous().to(dev))
                w = plan.dist(comm, None, yy.to(dev), lv.contiguous().to(dev), zz.to(dev), 1.0, 1.0)
                torch.cuda.synchronize()
                assert_bitexact(w, full, f"packed plan dist (NCCL) rank {rank}")
                plan.close()
            msgs.append(f"csr-int-{dt}")

        # ---- the same exchange over peer memory (CUDA IPC) and over NVLS multicast
        mm, nn = 60000, 20000
        rp, ci, va = synth.csr(mm, nn, "f32", ("powerlaw", 2.5, 13.64), kind="int_pm12", seed=12)
        yy = synth.vector(nn, "f32", kind="int_small", seed=12, stream=synth.S_Y)
        zz = synth.vector(nn, "f32", kind="int_small", seed=12, stream=synth.S_Z)
        vv = synth.vector(mm, "f32", kind="int_pos", seed=12, stream=synth.S_V)
        full, _ = oracle.csr(mm, nn, rp, ci, va, yy, vv, zz, 1.0, 1.0)
        bb = fp.shard_rows_csr(rp, world)
        lrp, lci, lva, lv = (t.contiguous().to(dev) for t in fp.shard_slice_csr(rp, ci, va, vv, bb, rank))
        for mode, enable in ((fp.FP_COMM_PEER, comm.enable_peer), (fp.FP_COMM_NVLS, comm.enable_nvls)):
            cm = fp.Comm(device=rank)  # a fresh communicator per mode
            try:
                try:
                    (cm.enable_peer if mode == fp.FP_COMM_PEER else cm.enable_nvls)(nn * 8)
                except fp.FusedPatError:
                    if mode == fp.FP_COMM_NVLS:
                        msgs.append("nvls-unsupported")
                        continue
                    raise
                for _ in range(3):
                    w = fp.csr_dist(cm, lrp, lci, lva, nn, yy.to(dev), lv, zz.to(dev), 1.0, 1.0)
                    torch.cuda.synchronize()
                    assert_bitexact(w, full, f"csr_dist mode {mode} rank {rank}")
                # the packed plan of the shard (variant 19) through the same exchange
                plan = fp.CsrPlan(lrp, lci, nn, torch.float32)
                plan.pack(lva)
                for _ in range(3):
                    w = plan.dist(cm, None, yy.to(dev), lv, zz.to(dev), 1.0, 1.0)
                    torch.cuda.synchronize()
                    assert_bitexact(w, full, f"packed plan dist mode {mode} rank {rank}")
                plan.close()
                msgs.append(f"mode-{mode}")
            finally:
                cm.close()

        # ---- CSR fp32 U[-1,1): north_star tolerance
        mm, nn = 80000, 3000
        rp, ci, va = synth.csr(mm, nn, "f32", ("powerlaw", 2.5, 13.64), seed=13)
        yy = synth.vector(nn, "f32", seed=13, stream=synth.S_Y)
        zz = synth.vector(nn, "f32", seed=13, stream=synth.S_Z)
        vv = synth.vector(mm, "f32", kind="pos", seed=13, stream=synth.S_V)
        ref, mag = oracle.csr(mm, nn, rp, ci, va, yy, vv, zz, 1.0, 1.0)
        bb = fp.shard_rows_csr(rp, world)
        lrp, lci, lva, lv = fp.shard_slice_csr(rp, ci, va, vv, bb, rank)
        w = fp.csr_dist(comm, lrp.contiguous().to(dev), lci.contiguous().to(dev), lva.contiguous().to(dev), nn,
                        yy.to(dev), lv.contiguous().to(dev), zz.to(dev), 1.0, 1.0)
        torch.cuda.synchronize()
        assert_parity(w, ref, mag, torch.float32, f"csr_dist f32 rank {rank}")
        msgs.append("csr-f32")

        # ---- CG (Listing 1) with a communicator: every rank holds the same w as one GPU
        m, n = 20000, 50
        X = synth.dense(m, n, "f64", kind="colscaled", seed=14)
        lab = synth.vector(m, "f64", seed=14, stream=synth.S_LABEL)
        w1, it1, h1 = fp.cg_linreg_dense(X.to(dev), lab.to(dev), eps=1e-3, max_iter=10, tol=0.0)
        b = fp.shard_rows_dense(m, world)
        r0, r1 = b[rank], b[rank + 1]
        wd, itd, hd = fp.cg_linreg_dense(X[r0:r1].contiguous().to(dev), lab[r0:r1].to(dev), eps=1e-3, max_iter=10,
                                         tol=0.0, comm=comm)
        assert itd == it1 == 10
        np.testing.assert_allclose(hd.numpy(), h1.numpy(), rtol=1e-8)
        assert float((wd - w1).norm() / w1.norm()) < 1e-8
        ws = [torch.empty_like(wd) for _ in range(world)]
        dist.all_gather(ws, wd)
        assert all(torch.equal(ws[0], t) for t in ws), "ranks disagree on the CG iterate"
        msgs.append("cg")

        # ---- TRON logistic regression with a communicator
        lab = torch.where(synth.vector(m, "f64", seed=15, stream=synth.S_LABEL) >= 0, 1.0, -1.0).double()
        w1, it1, f1 = fp.logreg_tron_dense(X.to(dev), lab.to(dev), C=1.0, eps=1e-3, max_iter=8)
        wd, itd, fd = fp.logreg_tron_dense(X[r0:r1].contiguous().to(dev), lab[r0:r1].to(dev), C=1.0, eps=1e-3,
                                           max_iter=8, comm=comm)
        assert abs(itd - it1) <= 1
        assert float((wd - w1).norm() / w1.norm()) < 1e-6
        msgs.append("tron")
        q.put((rank, "ok", msgs))
    except Exception as e:  # report, do not hang the peer
        import traceback

        q.put((rank, "fail", msgs + [traceback.format_exc()]))
    finally:
        comm.close()
        dist.destroy_process_group()


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2,
                    reason="needs 2 GPUs (gpurun boxes have 1; the round-end 8-GPU node runs it)")
def test_two_rank_nccl_dist_parity():
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(2):
        r, st, msgs = q.get(timeout=600)
        res[r] = (st, msgs)
    for p in procs:
        p.join(60)
    assert all(st == "ok" for st, _ in res.values()), res
