#!/usr/bin/env python
"""bench.py -- throughput of the fused pattern w = alpha X^T (v (.) (X y)) + beta z
(Eq. 1) on B200, per BASELINE.json:

  metric: "fused-pattern GB/s of X streamed and % of B200 HBM peak; evals/s at 1/2/4/8 GPU"

A step is one pattern evaluation over the whole configured matrix (all SURVEY 8(a) rows:
plan, w init, stage y, stream X once, dot, reduce+scale, scale-back, aggregation, and at
N > 1 the NCCL allreduce of w).  Default workload: C4 (BASELINE.json configs[3]), CSR fp32
50M x 100K with power-law rows, ~2e9 nonzeros, the full pattern with v -- the largest config
that fits one GPU, the one north_star's large-sparse >= 75 % target and its >= 6x 8-GPU
scaling target both name.  (BASELINE.json does not say which config the metric is quoted
on; --config C2 / C3 / C5 time the others.)  Every config but C1 streams far more than the
126 MB L2 per step, so no L2 flush is needed between steps (C1, which fits in L2, is timed
with an explicit flush).  Inputs are synthetic (synth/, seeded), generated directly in HBM.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl reference]
  torchrun --nproc-per-node N bench.py --gpus N ...     (row-sharded, strong scaling)

`--impl reference` times the fp64 CPU oracle (oracle/, the only reference this tier has) on
a bounded sample of the same workload on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

# stdout carries exactly one JSON line.  Native libraries (NCCL's version banner with any
# NCCL_DEBUG level) write to fd 1 directly, so when bench.py runs as the program, fd 1 is
# pointed at stderr for the whole run and the JSON line goes to a duplicate of the original
# stdout (emit()); tools that import bench keep their stdout.
_JSON_OUT = None


def _stdout_to_stderr():
    global _JSON_OUT
    sys.stdout.flush()
    _JSON_OUT = os.fdopen(os.dup(1), "w")
    os.dup2(2, 1)


def emit(obj):
    line = json.dumps(obj)
    if _JSON_OUT is None:
        print(line, flush=True)
    else:
        _JSON_OUT.write(line + "\n")
        _JSON_OUT.flush()


import numpy as np
import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

COLS = "strat"  # --cols
METRIC = "fused-pattern GB/s of X streamed and % of B200 HBM peak; evals/s at 1/2/4/8 GPU"
FALLBACK_HBM_GBS = 6650.0


# ------------------------------------------------------------------------------ helpers


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs: copy, read+write bytes)"
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md 6.65 TB/s)"


def traffic_for(config, variant):
    """dram__bytes_read.sum + dram__bytes_write.sum of one step (every kernel of the fp_* call),
    from the committed ncu --set full captures (profiles/ncu_traffic.json, tools/ncu_summary.py).
    ncu cannot run inside the timed region, so this is the capture of the same build and plan
    variant; a capture of another variant is reported as stale (value None)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None, "no capture"
    e = json.load(open(p)).get(config)
    if e is None:
        return None, "no capture"
    src = f"ncu --set full capture {e.get('round', '?')} ({e.get('file', '?')})"
    if e.get("variant") is not None and variant is not None and int(e["variant"]) != int(variant):
        return None, f"stale: {src} is of plan variant {e['variant']}, this run uses {variant}"
    return e.get("dram_bytes_per_step", e.get("dram_bytes_per_launch")), src


def second_ceiling(cfg, plan, nnz, kern_ms, dev, detail=None):
    """SURVEY 8(d) C4 'second ceiling': the random on-chip accesses of the CSR paths (y gathers
    that miss the shared-memory copy of y, w updates) at the rates the device sustains, measured
    live by fp_probe_rates in this run.  floor_ms = the time those accesses alone need;
    frac = floor_ms / the measured step.  Uniform columns assumed for the prefix hit share."""
    import paper_conf_ppopp_asharitbrcks15_b200 as fp

    if cfg["fmt"] != "csr" or plan is None:
        return None
    n = cfg["n"]
    s = 8 if cfg["dtype"] == "f64" else 4
    v = int(plan.variant)
    # the random accesses hit an n-element array -- variant 20: one L2-sized column block
    n_probe = -(-n // max(1, int(plan.cluster))) if v == 20 else n
    r = fp.probe_rates(min(n_probe, 1 << 30), smem_elems=min(max(n, 1), 25600), device=dev.index)
    ops, floor = {}, 0.0
    if v in (3, 5, 6, 8):  # y and the partial w in shared memory
        ops = {"smem_gathers": nnz, "smem_fp_atomics": nnz}
        floor = nnz / r["gather_smem_f64"] + nnz / r["atom_smem_f64"]
        what = "y gathers from shared memory + shared-memory fp atomics (a CAS loop) per nonzero"
    elif v == 19:  # packed: y and the partial w of a column block in shared memory
        ops = {"smem_gathers": nnz, "smem_int_atomics": nnz}
        floor = nnz / r["gather_smem_f64"] + nnz / r["atom_smem_u32"]
        what = ("y gathers from shared memory (rate measured on fp64 words, an upper bound for fp32) + one "
                "native int32 shared atomic per nonzero")
    elif v == 20:  # L2-sized column blocks: every y gather and w red of a block pass hits L2
        hot = int((detail or {}).get("hot_entries", 0))
        ops = {"l2_gathers": nnz - hot, "l2_reds": nnz - hot, "hot_entries_by_column": hot}
        floor = (nnz - hot) / r["gather_l2"] + (nnz - hot) / r["red_l2"]
        what = ("one y gather + one fp red.global per nonzero into the L2-resident column block (the blocks "
                "run one after the other); the hot columns' nonzeros are summed by column (one red per 256) "
                "and their y words are L1 hits, so they are left out; reds measured on fp32 words")
    elif v in (4, 7, 16, 17):
        prefix = min(n, int(plan.smem_bytes) // s) if v in (16, 17) else 0
        g = int(nnz * (1.0 - prefix / n))
        if v == 17:
            ops = {"l2_gathers": g, "smem_int_atomics": nnz}
            floor = g / r["gather_l2"] + nnz / r["atom_smem_u32"]
            what = ("producer: y gathers beyond the shared-memory prefix (L1/L2); consumer: one native "
                    "int32 shared atomic per nonzero")
        else:
            ops = {"l2_gathers": g, "l2_reds": nnz}
            floor = g / r["gather_l2"] + nnz / r["red_l2"]
            what = "y gathers beyond the shared-memory prefix + one fp red.global per nonzero (L1/L2)"
    else:
        return None
    return {"what": what, "ops_per_step": ops, "rates_ops_per_s": {k: round(x / 1e9, 2) for k, x in r.items()},
            "rates_unit": "G ops/s (fp_probe_rates, live)", "floor_ms": round(floor * 1e3, 4),
            "frac": round(floor * 1e3 / kern_ms, 4)}


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax.append(float(f[2]))
            except ValueError:
                continue
            for nm, val in zip(names, f[5:9]):
                if val.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def dist_info():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ------------------------------------------------------------------------------ workloads
def algorithmic_bytes(cfg, m, nnz):
    """X once + rowptr + v + y + [beta] z + w (bytes per evaluation)."""
    s = 8 if cfg["dtype"] == "f64" else 4
    n = cfg["n"]
    vec = (m * s if cfg["use_v"] else 0) + n * s + (n * s if cfg["use_z"] else 0) + n * s
    if cfg["fmt"] == "dense":
        xb = m * n * s
        return xb, xb + vec
    xb = nnz * (s + 4) + (m + 1) * 8
    return xb, xb + vec


def build_inputs(name, rank, world, dev):
    """This rank's row shard of config `name`, generated in HBM (bit-identical to the slice of
    the full matrix, synth/ is counter-based)."""
    cfg = dict(synth.CONFIGS[name])
    if COLS == "iid" and cfg["fmt"] == "csr" and cfg.get("col_skew", 0) == 0:
        cfg["col_skew"] = -1
    seed = synth.config_seed(name)
    m, n, dt = cfg["m"], cfg["n"], cfg["dtype"]
    import paper_conf_ppopp_asharitbrcks15_b200 as fp

    if cfg["fmt"] == "dense":
        b = fp.shard_rows_dense(m, world)
        r0, r1 = b[rank], b[rank + 1]
        X = _dense_shard(r0, r1, n, dt, cfg["xkind"], seed, dev)
        inp = dict(X=X, m_local=r1 - r0, nnz_local=0, row0=r0)
    else:
        rp_full = None
        if world > 1:
            # shard bounds need the global rowptr (host); row lengths are cheap to regenerate
            thr = synth.length_table(cfg["lengths"], n)
            rp_full = _host_rowptr(m, thr, seed)
            b = fp.shard_rows_csr(rp_full, world)
        else:
            b = [0, m]
        r0, r1 = b[rank], b[rank + 1]
        rp, ci, va = synth.csr(r1 - r0, n, dt, cfg["lengths"], kind=cfg["xkind"], seed=seed, row0=r0, device=dev,
                               col_skew=cfg.get("col_skew", 0))
        inp = dict(rowptr=rp, colidx=ci, val=va, m_local=r1 - r0, nnz_local=int(va.numel()), row0=r0)
    inp["y"] = synth.vector(n, dt, seed=seed, stream=synth.S_Y, device=dev)
    inp["v"] = synth.vector(inp["m_local"], dt, kind="pos", seed=seed, stream=synth.S_V, i0=inp["row0"],
                            device=dev) if cfg["use_v"] else None
    inp["z"] = synth.vector(n, dt, seed=seed, stream=synth.S_Z, device=dev) if cfg["use_z"] else None
    inp["w"] = torch.empty(n, dtype=inp["y"].dtype, device=dev)
    return cfg, inp


def _dense_shard(r0, r1, n, dt, kind, seed, dev):
    """Rows [r0, r1) of the seeded dense matrix (bit-identical to the slice of the full one)."""
    return synth.dense(r1 - r0, n, dt, kind=kind, seed=seed, device=dev, row0=r0)


def _host_rowptr(m, thr, seed):
    lens = np.empty(m, np.int64)
    import ctypes

    lib = synth._host()
    lib.synth_row_lengths(m, 0, thr.ctypes.data_as(ctypes.c_void_p), len(thr) - 1, seed,
                          lens.ctypes.data_as(ctypes.c_void_p))
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    return torch.from_numpy(rp)


# ------------------------------------------------------------------------------ main arm
def run_gpu(args):
    world, rank, local = dist_info()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    import paper_conf_ppopp_asharitbrcks15_b200 as fp

    comm = None
    if world > 1 or args.force_dist:
        import torch.distributed as dist

        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29531")
        os.environ.setdefault("RANK", "0")
        os.environ.setdefault("WORLD_SIZE", "1")
        dist.init_process_group("nccl", device_id=dev)
        comm = fp.Comm(device=local)
    name = args.config
    cfg, inp = build_inputs(name, rank, world, dev)
    exchange = "none"
    if comm is not None:
        # the exchange of the partial w: the fused peer-memory path (FP_COMM_PEER, the product),
        # NVSwitch multicast (FP_COMM_NVLS) or ncclAllReduce (the baseline), --exchange
        exchange = args.exchange
        vec_bytes = cfg["n"] * (8 if cfg["dtype"] == "f64" else 4)
        ok = 1
        try:
            if exchange == "peer":
                comm.enable_peer(vec_bytes)
            elif exchange == "nvls":
                comm.enable_nvls(vec_bytes)
        except fp.FusedPatError as e:
            print(f"[bench] rank {rank}: {exchange} exchange unavailable ({e})", file=sys.stderr)
            ok = 0
        # the exchange checks itself once (an allreduce of rank + 1 everywhere: every element must
        # be N (N + 1) / 2 and no barrier may have timed out) before anything is timed
        if ok and exchange != "nccl":
            try:
                chk = torch.full((4096,), float(rank + 1), dtype=torch.float64, device=dev)
                comm.allreduce(chk)
                torch.cuda.synchronize()
                ok = int(bool((chk == world * (world + 1) / 2).all()) and not comm.timed_out())
            except fp.FusedPatError as e:
                print(f"[bench] rank {rank}: {exchange} exchange self-check failed ({e})", file=sys.stderr)
                ok = 0
            if not ok:
                print(f"[bench] rank {rank}: {exchange} exchange self-check failed", file=sys.stderr)
        # every rank must use the same exchange: fall back to NCCL together if any rank failed
        import torch.distributed as dist

        flag = torch.tensor([ok], dtype=torch.int32, device=dev)
        dist.all_reduce(flag, op=dist.ReduceOp.MIN)
        if exchange != "nccl" and int(flag.item()) == 0:
            if comm.mode != fp.FP_COMM_NCCL:
                comm.set_mode(fp.FP_COMM_NCCL)
            exchange = "nccl (fallback)"
    torch.cuda.synchronize()
    alpha, beta = cfg["alpha"], cfg["beta"]
    stream = torch.cuda.current_stream(dev)
    n = cfg["n"]

    plan = None
    plan_ms = None
    pack_info = None
    pack_detail = None
    if name == "C5":
        iters = args.cg_iters

        def step():
            fp.cg_linreg_dense(inp["X"], inp["labels"], eps=1e-3, max_iter=iters, tol=0.0, comm=comm)
        inp["labels"] = synth.vector(inp["m_local"], cfg["dtype"], seed=synth.config_seed(name),
                                     stream=synth.S_LABEL, i0=inp["row0"], device=dev)
        launches_per_step = 2 * iters + 2
        passes_per_step = iters + 1
    elif cfg["fmt"] == "dense":
        def step():
            if comm is None:
                fp.dense(inp["X"], inp["y"], inp["v"], inp["z"], alpha, beta, w=inp["w"])
            else:
                fp.dense_dist(comm, inp["X"], inp["y"], inp["v"], inp["z"], alpha, beta, w=inp["w"])
        plan = fp.choose(False, fp.row_stats_dense(inp["m_local"], n),
                         fp.FP_F64 if cfg["dtype"] == "f64" else fp.FP_F32, local)
        launches_per_step = 1
        passes_per_step = 1
    else:
        forced = None
        if args.launch:  # explicit plan (profiling / sweeps): variant,vs,k,grid (variant 13: k = cluster)
            var, vs, k, g = (int(t) for t in args.launch.split(","))
            forced = fp.fp_launch()
            forced.variant, forced.vs, forced.tl, forced.bs, forced.grid = var, vs, k, 256, g
            if var == 13:
                forced.cluster = k
            if var == 16:
                forced.bs = 1024
        # the once-per-matrix analysis (fp_csr_plan_create: launch parameters, column split) is
        # outside the timed region, like the paper's amortised transpose; timed here
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        cplan = None
        packed = False
        # the rank's plan (its row shard when N > 1: fp_csr_plan_dist)
        cplan = fp.CsrPlan(inp["rowptr"], inp["colidx"], n, inp["val"].dtype, launch=forced)
        torch.cuda.synchronize()
        plan_ms = (time.perf_counter() - t0) * 1e3
        if forced is None and args.pack:
            # the column-blocked copy (fp_csr_plan_pack, variant 19): once per matrix, timed here
            t0 = time.perf_counter()
            try:
                cplan.pack(inp["val"])
                packed = True
            except fp.FusedPatError as e:
                print(f"[bench] no packed plan: {e}", file=sys.stderr)
            torch.cuda.synchronize()
            pack_ms = (time.perf_counter() - t0) * 1e3
            if packed:
                pack_info = dict(cplan.pack_info, pack_ms=round(pack_ms, 1))
                pack_detail = cplan.pack_detail
                pack_info["detail"] = pack_detail

        def step():
            if comm is None:
                cplan(None if packed else inp["val"], inp["y"], inp["v"], inp["z"], alpha, beta, w=inp["w"])
            else:
                cplan.dist(comm, None if packed else inp["val"], inp["y"], inp["v"], inp["z"], alpha, beta,
                           w=inp["w"])
        plan = cplan.launch
        passes_per_step = 1
        # the L2 variants write beta*z (k_scale_z) before the main kernel and, when w is
        # replicated over L2 (csr.cu l2_replicas: 8 copies while they take <= 16 MB), fold the
        # copies after it
        launches_per_step = 1
        if plan.variant == 17:  # producer, consumer, finalize (+ a 16-byte memset)
            launches_per_step = 3
        elif plan.variant == 19:  # the packed pass + the finalize
            launches_per_step = 2
        elif plan.variant == 20:  # w init, a dot launch per other block, fused, q, a scatter launch per
            # other block, the fused block's partial chunks, hot columns (+ a memset): the library's count
            launches_per_step = int(pack_detail["launches"])
            if os.environ.get("FP_L2B_MERGE", "0") not in ("", "0"):
                launches_per_step = 9
        elif plan.variant in (4, 7, 16):
            s_b = 8 if cfg["dtype"] == "f64" else 4
            nrep = int(os.environ.get("FP_L2_REPLICAS", "0")) or (8 if 8 * n * s_b <= (16 << 20) else 1)
            launches_per_step = 2 + (1 if nrep > 1 else 0)

    flush = None
    if name == "C1":  # X fits in L2: flush between timed iterations
        flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    graphed = False
    # (the peer / NVLS exchange advances an epoch per call and is not capturable)
    if args.graph and name != "C5" and exchange in ("none", "nccl", "nccl (fallback)"):
        # Capture one step (the fp_* call; its plan is cached and its workspace exists for the
        # capture stream after the warm-up below) in a CUDA graph, so host-side marshalling is
        # off the timed path -- it matters for the latency config C1.
        gs = torch.cuda.Stream(device=dev)
        gs.wait_stream(torch.cuda.current_stream(dev))
        with torch.cuda.stream(gs):
            step()
            step()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=gs):
            step()
        torch.cuda.synchronize()
        step = g.replay
        step()
        torch.cuda.synchronize()
        graphed = True

    # global algorithmic bytes per evaluation (all ranks)
    m_all, nnz_all = cfg["m"], None
    if cfg["fmt"] == "csr":
        t = torch.tensor([inp["nnz_local"]], dtype=torch.int64, device=dev)
        if world > 1:
            import torch.distributed as dist

            dist.all_reduce(t)
        nnz_all = int(t.item())
    x_bytes, alg_bytes = algorithmic_bytes(cfg, m_all, nnz_all or 0)
    x_local, alg_local = algorithmic_bytes(cfg, inp["m_local"], inp["nnz_local"])

    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    if comm is not None:
        import torch.distributed as dist

        dist.barrier()
    torch.cuda.synchronize()
    t_begin = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_begin.record(stream)
    for i in range(args.steps):
        if flush is not None:
            flush.zero_()
        starts[i].record(stream)
        step()
        ends[i].record(stream)
    t_end.record(stream)
    torch.cuda.synchronize()
    if comm is not None:
        dist.barrier()
    clk = clocks.stop()
    step_ms = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    total_ms = t_begin.elapsed_time(t_end)
    kern_ms = float(np.mean(step_ms))
    if flush is None:
        ms_per_step = total_ms / args.steps
    else:
        ms_per_step = float(np.sum(step_ms)) / args.steps  # flush excluded
    if world > 1:
        t = torch.tensor([ms_per_step, kern_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_per_step, kern_ms = float(t[0]), float(t[1])

    evals_per_s = 1e3 / ms_per_step
    value = x_bytes * passes_per_step * evals_per_s / 1e9
    peak, peak_src = peaks()
    achieved = alg_local * passes_per_step / (kern_ms / 1e3) / 1e9   # per-GPU kernel bytes / kernel time
    variant = None if plan is None else int(plan.variant)
    traffic, traffic_src = traffic_for(name, variant)
    sc = None if world > 1 else second_ceiling(cfg, plan, nnz_all or 0, kern_ms, dev, pack_detail)
    frac = achieved / peak
    # what binds: HBM when the step runs near the copy peak; else the random on-chip accesses
    # when they alone account for most of the step; else latency / issue (profiles/)
    binding = ("hbm" if frac >= 0.8 else
               ("on-chip random access (second_ceiling)" if sc and sc["frac"] >= 0.5 else
                "latency / instruction issue (see profiles/ and DESIGN.md section 5)"))
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(frac, 4), "traffic": traffic, "traffic_source": traffic_src,
            "peak_source": peak_src, "binding": binding, "second_ceiling": sc,
            "note": ("bound = the roofline axis (the path moves ~1 flop per byte: memory); achieved = algorithmic "
                     "bytes of one fp_* call (SURVEY 8(d): X once + rowptr + v + y + z + w) / mean CUDA-event "
                     "duration of that call (all its kernels) on its launch stream; binding = what the "
                     "measurements say limits it")}

    e2e = None
    if not args.no_e2e and name != "C5":
        e2e = run_e2e(args, cfg, inp, comm, world, rank, dev, x_bytes)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(name, args.cpu_seconds)

    if rank == 0:
        out = {
            "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": cfg["dtype"],
            "data": "synthetic (counter-based seeded generator synth/, generated in HBM)",
            "config": {"workload": f"{name}: {cfg['desc']}", "m": cfg["m"], "n": cfg["n"],
                       "format": cfg["fmt"], "nnz": nnz_all,
                       "columns": (None if cfg["fmt"] != "csr" else
                                   {0: "stratified-uniform distinct, sorted", -1: "i.i.d. uniform (unsorted)"}.get(
                                       cfg.get("col_skew", 0), f"Zipf-like u^(2^{cfg.get('col_skew')})")), "alpha": alpha, "beta": beta, "v": cfg["use_v"],
                       "z": cfg["use_z"],
                       "parallelism": (f"row-sharded x{world}, one exchange of the partial w ({exchange})"
                                       if comm is not None else "1 GPU"),
                       "l2": ("flushed (256 MiB memset) between timed steps" if flush is not None else
                              f"inputs larger than L2 (X = {x_bytes / 1e9:.2f} GB >> 126 MB)"),
                       "passes_per_step": passes_per_step, "cuda_graph": graphed,
                       "plan": None if plan is None else {
                           k: int(getattr(plan, k)) for k in ("variant", "vs", "tl", "bs", "grid", "cluster",
                                                              "blocks_per_sm", "smem_bytes", "regs_per_thread")},
                       "plan_create_ms": None if plan_ms is None else round(plan_ms, 2),
                       "packed_copy": pack_info},
            "evals_per_s": round(evals_per_s * (1 if name != "C5" else 1), 3),
            "pct_hbm_peak": round(100 * value / world / peak, 2),
            "x_bytes_per_eval": x_bytes, "algorithmic_bytes_per_eval": alg_bytes,
            "kernel_ms": round(kern_ms, 4),
            "roofline": roof,
            "gpu_launches": launches_per_step * args.steps,
            "clocks": clk,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        emit(out)
    if comm is not None:
        comm.close()
        import torch.distributed as dist

        dist.destroy_process_group()


def run_e2e(args, cfg, inp, comm, world, rank, dev, x_bytes):
    """Same metric through the host-buffer C-ABI entry (fp_dense_host / fp_csr_host): inputs in
    pinned host memory, H2D of the whole shard and D2H of w inside every timed step."""
    import paper_conf_ppopp_asharitbrcks15_b200 as fp

    host = {k: (t.cpu().pin_memory() if isinstance(t, torch.Tensor) else t) for k, t in inp.items()
            if k in ("X", "rowptr", "colidx", "val", "y", "v", "z")}
    n = cfg["n"]
    z, beta = (host.get("z"), cfg["beta"]) if rank == 0 else (None, 0.0)
    wh = torch.empty(n, dtype=host["y"].dtype).pin_memory()

    def step():
        if cfg["fmt"] == "dense":
            fp.dense_host(host["X"], host["y"], host.get("v"), z, cfg["alpha"], beta, w=wh, device=dev.index)
        else:
            fp.csr_host(host["rowptr"], host["colidx"], host["val"], n, host["y"], host.get("v"), z, cfg["alpha"],
                        beta, w=wh, device=dev.index)
        if comm is not None:
            wd = wh.to(dev, non_blocking=False)
            comm.allreduce(wd)
            wh.copy_(wd.cpu())

    step()  # warm-up (allocates staging buffers)
    steps = max(1, args.e2e_steps)
    if world > 1:
        import torch.distributed as dist

        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(steps):
        step()
    dt = (time.perf_counter() - t0) / steps
    if world > 1:
        t = torch.tensor([dt], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dt = float(t[0])
    h2d = sum(t.numel() * t.element_size() for k, t in host.items() if t is not None)
    return {"value": round(x_bytes / dt / 1e9, 2), "unit": "GB/s", "h2d_bytes_per_step": int(h2d),
            "d2h_bytes_per_step": int(wh.numel() * wh.element_size()), "steps": steps,
            "ms_per_step": round(dt * 1e3, 3),
            "api": "fp_dense_host / fp_csr_host (row chunks streamed through HBM, copy/compute overlapped)"}


# ------------------------------------------------------------------------------ CPU oracle
def _oracle_sample(name, rows):
    """The first `rows` rows of config `name` (the generator is counter-based, so they are the
    matrix's actual first rows), with the matching slices of v and the full y, z."""
    cfg = synth.CONFIGS[name]
    seed = synth.config_seed(name)
    m, n, dt = cfg["m"], cfg["n"], cfg["dtype"]
    rows = max(1, min(m, int(rows)))
    if cfg["fmt"] == "dense":
        data = dict(X=synth.dense(rows, n, dt, kind=cfg["xkind"], seed=seed))
        entries = rows * n
    else:
        rp, ci, va = synth.csr(rows, n, dt, cfg["lengths"], kind=cfg["xkind"], seed=seed,
                               col_skew=cfg.get("col_skew", 0))
        data = dict(rp=rp, ci=ci, va=va)
        entries = int(va.numel())
    y = synth.vector(n, dt, seed=seed, stream=synth.S_Y)
    v = synth.vector(rows, dt, kind="pos", seed=seed, stream=synth.S_V) if cfg["use_v"] else None
    z = synth.vector(n, dt, seed=seed, stream=synth.S_Z) if cfg["use_z"] else None
    return cfg, rows, entries, data, y, v, z


def _calibrated_sample(name, target_s, threads):
    """A sample sized for ~target_s seconds of oracle work per evaluation (capped at the whole
    matrix): time a small leading block first, then scale the row count."""
    cfg = synth.CONFIGS[name]
    per_row = cfg["n"] if cfg["fmt"] == "dense" else {"C3": 10.0, "C4": 40.0}.get(name, 10.0)
    rows0 = max(1, min(cfg["m"], int(2e7 / per_row)))
    smp = _oracle_sample(name, rows0)
    t0 = time.perf_counter()
    _oracle_eval(*smp[:1], smp[1], *smp[3:], threads)
    dt0 = max(time.perf_counter() - t0, 1e-4)
    rows1 = min(cfg["m"], int(rows0 * target_s / dt0))
    if rows1 > 1.3 * rows0:
        smp = _oracle_sample(name, rows1)
    return smp


def _oracle_eval(cfg, rows, data, y, v, z, threads):
    import oracle

    if cfg["fmt"] == "dense":
        return oracle.dense(data["X"], y, v, z, cfg["alpha"], cfg["beta"], threads=threads)
    return oracle.csr(rows, cfg["n"], data["rp"], data["ci"], data["va"], y, v, z, cfg["alpha"], cfg["beta"],
                      threads=threads)


def cpu_baseline(name, target_s=15.0):
    threads = os.cpu_count() or 1
    cfg, rows, entries, data, y, v, z = _calibrated_sample(name, target_s, threads)
    t0 = time.perf_counter()
    _oracle_eval(cfg, rows, data, y, v, z, threads)
    dt = time.perf_counter() - t0
    xb, _ = algorithmic_bytes(cfg, rows, entries)
    return {"value": round(xb / dt / 1e9, 4), "unit": "GB/s", "cores": threads, "kind": "oracle",
            "sample": f"first {rows:,} of {cfg['m']:,} rows of {name} (same generator), 1 evaluation, "
                      f"{dt:.1f} s, fp64 Neumaier oracle (oracle/oracle.c, OpenMP)"}


def run_reference(args):
    """--impl reference: the CPU oracle as the reference arm (this tier has no reference code)."""
    world, rank, _ = dist_info()
    if rank != 0:
        return
    name = args.config
    threads = os.cpu_count() or 1
    cfg, rows, entries, data, y, v, z = _calibrated_sample(name, args.ref_seconds, threads)
    for _ in range(args.warmup):
        _oracle_eval(cfg, rows, data, y, v, z, threads)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        _oracle_eval(cfg, rows, data, y, v, z, threads)
    dt = (time.perf_counter() - t0) / args.steps
    xb, _ = algorithmic_bytes(cfg, rows, entries)
    val = xb / dt / 1e9
    sample = (f"first {rows:,} of {cfg['m']:,} rows of {name} per step (same generator, whole matrix when the "
              f"oracle finishes it within --ref-seconds); "
              f"GB/s of X streamed by the fp64 oracle")
    out = {"impl": "reference", "metric": METRIC, "value": round(val, 4), "unit": "GB/s", "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 3), "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f64 (oracle arithmetic; inputs " + cfg["dtype"] + ")",
           "data": "synthetic", "config": {"workload": f"{name}: {cfg['desc']}", "m": cfg["m"], "n": cfg["n"]},
           "cpu_baseline": {"value": round(val, 4), "unit": "GB/s", "kind": "oracle", "cores": threads,
                            "sample": sample},
           "e2e": {"value": round(val, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(out)


def run_unfused(args):
    """--impl unfused: the multi-kernel library chain the paper compares against (P:81-109,
    P:417): cuBLAS gemv X y, elementwise v, cuBLAS gemv X^T q (+ beta z) for dense; cuSPARSE SpMV
    X y and X^T q (torch sparse CSR, transpose via a CSC view) for CSR -- two passes over X.
    A second GPU reference (north_star), NOT the product path."""
    world, rank, local = dist_info()
    if world > 1 and rank != 0:
        return
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    name = args.config
    cfg, inp = build_inputs(name, 0, 1, dev)
    alpha, beta, n = cfg["alpha"], cfg["beta"], cfg["n"]
    if cfg["fmt"] == "dense":
        X = inp["X"]

        def step():
            p = torch.mv(X, inp["y"])
            if inp["v"] is not None:
                p = p * inp["v"]
            w = torch.mv(X.t(), p)
            w = alpha * w + (beta * inp["z"] if beta != 0.0 else 0.0)
            return w
    else:
        # torch/cuSPARSE need one index dtype: int32 when nnz fits (C3, C4), else int64 columns
        if inp["nnz_local"] < 2**31 - 1:
            crow, col = inp["rowptr"].to(torch.int32), inp["colidx"]
        else:
            crow, col = inp["rowptr"], inp["colidx"].to(torch.int64)
        del inp["rowptr"]
        torch.cuda.empty_cache()
        A = torch.sparse_csr_tensor(crow, col, inp["val"], size=(cfg["m"], n))
        At = A.t()  # CSC view of X: X^T q is a transposed SpMV

        def step():
            p = torch.mv(A, inp["y"])
            if inp["v"] is not None:
                p = p * inp["v"]
            w = torch.mv(At, p)
            return alpha * w + (beta * inp["z"] if beta != 0.0 else 0.0)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(args.steps):
        step()
    e.record()
    torch.cuda.synchronize()
    ms = s.elapsed_time(e) / args.steps
    x_bytes, _ = algorithmic_bytes(cfg, cfg["m"], inp["nnz_local"])
    out = {"impl": "unfused", "metric": METRIC, "value": round(x_bytes / ms / 1e6, 2), "unit": "GB/s", "n_gpus": 1,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": cfg["dtype"], "data": "synthetic",
           "config": {"workload": f"{name}: {cfg['desc']}", "m": cfg["m"], "n": n,
                      "chain": "torch.mv (cuBLAS gemv / cuSPARSE SpMV) x2 + elementwise"}}
    emit(out)


def main():
    _stdout_to_stderr()
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C4", choices=sorted(synth.CONFIGS))
    ap.add_argument("--impl", default="fusedpat", choices=["fusedpat", "reference", "unfused"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--cols", default="strat", choices=["strat", "iid"],
                    help="CSR column pattern: stratified-uniform distinct (default) or i.i.d. uniform")
    ap.add_argument("--ref-seconds", type=float, default=4.0)
    ap.add_argument("--cg-iters", type=int, default=20)
    ap.add_argument("--graph", dest="graph", action="store_true", default=True,
                    help="replay each step from a captured CUDA graph (default)")
    ap.add_argument("--no-graph", dest="graph", action="store_false")
    ap.add_argument("--no-pack", dest="pack", action="store_false", default=True,
                    help="CSR fp32: run the unpacked plan instead of the column-blocked copy (variant 19)")
    ap.add_argument("--launch", default=None, help="CSR only: force the plan 'variant,vs,k,grid' (profiling)")
    ap.add_argument("--exchange", default="peer", choices=["peer", "nvls", "nccl"],
                    help="N > 1: exchange of the partial w (fused peer memory, NVLS multicast, or NCCL)")
    ap.add_argument("--force-dist", action="store_true",
                    help="use the NCCL row-sharded path (fp_*_dist + allreduce) even with one rank")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    global COLS
    COLS = args.cols
    if args.impl == "reference":
        run_reference(args)
    elif args.impl == "unfused":
        run_unfused(args)
    else:
        run_gpu(args)


if __name__ == "__main__":
    main()
