"""Per-warp timing of the packed pass (variant 19) on a bench config: where the warps end.
python tools/pk_trace.py [C4]  (sets FP_PK_TRACE; prints the spread of warp end times)."""
import ctypes
import os
import sys

import numpy as np
import torch

os.environ["FP_PK_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_ppopp_asharitbrcks15_b200 as fp  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C4"
dev = torch.device("cuda", 0)
cfg, inp = bench.build_inputs(name, 0, 1, dev)
plan = fp.CsrPlan(inp["rowptr"], inp["colidx"], cfg["n"], inp["val"].dtype)
plan.pack(inp["val"])
for _ in range(3):
    plan(None, inp["y"], inp["v"], inp["z"], cfg["alpha"], cfg["beta"], w=inp["w"])
torch.cuda.synchronize()
info = plan.pack_info
nw = info["groups"] * info["blocks"] * 32
buf = (ctypes.c_ulonglong * (8 * nw))()
k = fp.lib().fpx_pack_trace(plan._h, buf, ctypes.c_int64(8 * nw))
t = np.frombuffer(buf, dtype=np.uint64).reshape(-1, 8).astype(np.float64)
t0 = t[:, 0].min()
start, end, tiles, pro = (t[:, 0] - t0) / 1e3, (t[:, 1] - t0) / 1e3, t[:, 2], (t[:, 3] - t0) / 1e3
print(f"warps {len(t)}  start us: max {start.max():.1f}  prologue end us: median {np.median(pro):.1f} max {pro.max():.1f}")
print("end us percentiles 0/10/50/90/99/100:", np.percentile(end, [0, 10, 50, 90, 99, 100]).round(1))
print("tiles per warp min/median/max:", tiles.min(), np.median(tiles), tiles.max())
cta = end.reshape(-1, 32)  # 32 warps per CTA
print("per CTA: spread (max - min) of warp ends, median/max us:", np.median(cta.max(1) - cta.min(1)).round(1),
      (cta.max(1) - cta.min(1)).max().round(1))
grp = end.reshape(info["groups"], -1)
print("per group: max end, min/median/max us:", grp.max(1).min().round(1), np.median(grp.max(1)).round(1),
      grp.max(1).max().round(1))
slow = np.argsort(end)[-5:]
print("slowest warps (cta, warp, end us, tiles):", [(int(i // 32), int(i % 32), round(end[i], 1), int(tiles[i])) for i in slow])
w = end.reshape(-1, 32)
print("mean end by warp index:", w.mean(0).round(0).astype(int).tolist())
print("corr(end, tiles):", np.corrcoef(end, tiles)[0, 1].round(3))
c = end.reshape(-1, 32).mean(1)
print("mean end by CTA (first 16):", c[:16].round(0).astype(int).tolist())
print("by block k (cta % blocks):", [round(float(c[k::info['blocks']].mean()), 1) for k in range(info['blocks'])])
