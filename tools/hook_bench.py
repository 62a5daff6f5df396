#!/usr/bin/env python
"""Device-hook (a3) cost on B200: instrumented kernels against their
uninstrumented twins, CUDA events on the launching stream.

  stream<T>: y[i] = 2 x[i] over n elements (real data), traceR + traceW per
             element -- the bandwidth-bound case; algorithmic bytes per element
             = 2 sizeof(T) of data + per shadow word 1 B read + 1 B written
             (shadow bytes on first touch).
  lulesh:    the cfg4 program (LULESH-shaped 100^3), `steps` timesteps, sum of
             the kernels' event times (instrumented vs twin) -> hook cost/step.

  python tools/hook_bench.py [--lulesh-steps 10] [--n 268435456]
Prints one JSON object.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1 << 28)
    ap.add_argument("--lulesh-steps", type=int, default=10)
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    import torch
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    out = {"nproc": os.cpu_count()}
    st = torch.cuda.Stream()
    s = st.cuda_stream

    def ev_time(fn, reps):
        best = None
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            fn()
            e1.record(st)
            e1.synchronize()
            t = e0.elapsed_time(e1)
            best = t if best is None else min(best, t)
        return best

    for elem, mode in ((4, 1), (8, 1), (4, 2), (8, 2)):  # mode 1: xpl_read/xpl_write, 2: array handles
        n = a.n if elem == 4 else a.n // 2
        x = torch.ones(n * elem // 4, dtype=torch.int32, device="cuda")
        y = torch.empty_like(x)
        twin = ev_time(lambda: xpl.stream_kernel(x.data_ptr(), y.data_ptr(), n, elem, 0, s), a.reps)
        words = n * elem // 4
        with xpl.Context(pool_words=2 * words + (1 << 20), max_rows=16) as ctx:
            ctx.register(x.data_ptr(), n * elem, xpl.ALLOC_DEVICE)
            ctx.register(y.data_ptr(), n * elem, xpl.ALLOC_DEVICE)
            ctx.sync()
            first = []

            def run_instr():
                ctx.kernel_begin(s)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(st)
                xpl.stream_kernel(x.data_ptr(), y.data_ptr(), n, elem, mode, s)
                e1.record(st)
                ctx.kernel_end(s)
                ctx.join(s)
                e1.synchronize()
                first.append(e0.elapsed_time(e1))
            # first epoch of an interval: every shadow word gets its bits (REDs)
            ctx.diagnose(50, 0, 256, reset=True)
            torch.cuda.synchronize()
            run_instr()
            ms_first = first[-1]
            # later epochs of the same interval: bits already set (test-before-set)
            for _ in range(a.reps):
                run_instr()
            ms_again = min(first[1:])
            torch.cuda.synchronize()
        data = 2 * n * elem
        shadow = 2 * 2 * words  # two arrays, 1 B read + 1 B written per word
        out[f"stream{elem * 8}" + ("_handles" if mode == 2 else "")] = {
            "n": n, "elem_bytes": elem, "twin_ms": twin, "instr_ms_first_touch": ms_first,
            "instr_ms_retouch": ms_again,
            "slowdown_first": ms_first / twin, "slowdown_retouch": ms_again / twin,
            "twin_gbs": data / (twin / 1e3) / 1e9,
            "instr_gbs_first": (data + shadow) / (ms_first / 1e3) / 1e9,
            "frac_first": (data + shadow) / (ms_first / 1e3) / 1e9 / peak,
            "accesses_per_s_first": 2 * n / (ms_first / 1e3),
            "slowdown_floor": (data + shadow) / data}
        del x, y
        torch.cuda.empty_cache()

    if a.lulesh_steps:
        from xplgen import lulesh as L
        S = 100
        spec = L.lulesh_spec(S)
        ar = apps.Arena(spec)
        topo = L.topology(S, 0x58504C05)
        hc = torch.zeros(1, dtype=torch.int64, device="cuda")
        res, each = {}, {}
        with xpl.Context(pool_words=1 << 28, max_rows=64) as ctx:
            for c in (ctx, None, ctx, None):
                apps.lulesh_prepare(ar, S, topo)
                hc.zero_()
                run = apps.Run(c, s, params=(50, 0, 256), out_cap=64 * (a.lulesh_steps + 1), time_kernels=True)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                rs = torch.cuda.ExternalStream(ctx.runtime_stream())
                e0.record(rs if c is not None else st)
                apps.lulesh(run, ar, S, a.lulesh_steps, hc)
                if c is not None:
                    ctx.join(rs.cuda_stream)
                e1.record(rs if c is not None else st)
                e1.synchronize()
                torch.cuda.synchronize()
                each["instr" if c is not None else "twin"] = list(run.kernel_each[:19 * a.lulesh_steps])
                res["instr" if c is not None else "twin"] = {
                    "kernel_ms": run.r.kernel_ms, "total_ms": e0.elapsed_time(e1), "host_ms": run.r.host_ms,
                    "hooks": int(hc.item()), "epochs": run.r.epochs}
        st_ = a.lulesh_steps
        import numpy as np
        med = {k: np.median(np.array(v).reshape(st_, 19), axis=0) for k, v in each.items()}
        out["lulesh100"] = dict(res, steps=st_,
                                hook_cost_ms_per_step=(res["instr"]["kernel_ms"] - res["twin"]["kernel_ms"]) / st_,
                                hook_cost_ms_per_step_median=float(np.sum(med["instr"] - med["twin"])),
                                kernel_slowdown=res["instr"]["kernel_ms"] / res["twin"]["kernel_ms"],
                                hooks_per_step=res["instr"]["hooks"] / st_)
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
