#!/usr/bin/env python
"""Per-program breakdown of one instrumented step (host-loop ms, kernel ms, wall ms)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl  # noqa: E402
from xplgen import rodinia  # noqa: E402

ctx = xpl.Context(pool_words=1 << 27, max_rows=256)
us = torch.cuda.Stream()
specs = {"hotspot": rodinia.hotspot_spec(*bench.HOT[:2]), "backprop": rodinia.backprop_spec(*bench.BACKPROP),
         "bfs": rodinia.bfs_spec(*bench.BFS), "nw": rodinia.nw_spec(bench.NW[0])}
ar = {k: apps.Arena(v) for k, v in specs.items()}
edges = rodinia.bfs_graph(*bench.BFS, 0x58504C02)
nw_in = rodinia.nw_inputs(*bench.NW, 0x58504C03)
hc = torch.zeros(1, dtype=torch.int64, device="cuda")
for rep in range(2):
    for name in ("hotspot", "backprop", "bfs", "nw"):
        for c in (ctx, None):
            apps.bfs_prepare(ar["bfs"], *bench.BFS, edges, resident=True)
            rodinia.nw_fill_host(ar["nw"].host_views(), specs["nw"], nw_in, bench.NW[0])
            torch.cuda.synchronize()
            run = apps.Run(c, us.cuda_stream, do_copies=False, diag_each=True, params=bench.PARAMS, time_kernels=True)
            t0 = time.perf_counter()
            if name == "hotspot":
                apps.hotspot(run, ar[name], *bench.HOT)
            elif name == "backprop":
                apps.backprop(run, ar[name], *bench.BACKPROP)
            elif name == "bfs":
                apps.bfs(run, ar[name], *bench.BFS, hc)
            else:
                apps.nw(run, ar[name], *bench.NW, nw_in["blosum"])
            torch.cuda.synchronize()
            wall = (time.perf_counter() - t0) * 1e3
            if rep == 1:
                print(f"{name:9s} {'instr' if c else 'twin ':5s} wall {wall:8.2f} ms  host {run.r.host_ms:8.2f} ms  "
                      f"kernels {run.r.kernel_ms:7.2f} ms  host_acc {run.r.host_accesses/1e6:7.2f} M  "
                      f"epochs {run.r.epochs}")
st = ctx.stats()
print(st)
