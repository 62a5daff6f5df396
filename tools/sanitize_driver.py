#!/usr/bin/env python
"""A small run of every kernel of the hot path for compute-sanitizer
(memcheck / synccheck / racecheck; tools/gpu_job.sh step `sanitize`):
host records (merge), transfers (range), device hooks with per-lane and
compile-time kinds (contiguous, one-address and grouped paths, multi-word),
epoch closes (fold), device-side epoch splits (xpl_grid_epoch), diagnoses with
and without reset / blocks (diag tile + stitch), the page view, the LULESH-shaped
program and the streaming kernel -- each checked against the oracle, so a
sanitizer-clean run is also a correct one."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import torch
    from oracle import run_trace
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, replay, xpl
    from xplgen import lulesh as L
    from xplgen.trace import parse_text, random_trace

    def same(a, b, what):
        assert a == b, what
        print("ok", what, flush=True)

    ops = parse_text(open(os.path.join(ROOT, "tests", "golden", "T01dom_fig4.trace")).read())
    same(replay.run_trace(ops), run_trace(ops), "golden T01")
    for seed in range(2):
        ops = random_trace(0x58504C01 + seed, n_allocs=5, n_steps=30, max_words=3000)
        exp = run_trace(ops)
        same(replay.run_trace(ops), exp, f"random {seed} per-lane kinds")
        same(replay.run_trace(ops, uniform=True), exp, f"random {seed} compile-time kinds")
        same(replay.run_trace(ops, uniform=True, grid=3, block=96, seed=seed), exp, f"random {seed} shuffled")
        same(replay.run_trace(ops, split_epochs=True), exp, f"random {seed} device-side splits")
    ops = random_trace(0x58504C09, n_allocs=4, n_steps=20, max_words=2000)
    ops = ops + [("PAGES", 64)]
    same(replay.run_trace(ops), run_trace(ops), "page view")
    s = 5
    spec = L.lulesh_spec(s)
    ar = apps.Arena(spec)
    topo = L.topology(s, 0x58504C05)
    apps.lulesh_prepare(ar, s, topo)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    st = torch.cuda.Stream()
    with xpl.Context(pool_words=1 << 22) as ctx:
        run = apps.Run(ctx, st.cuda_stream, params=(30, 64, 8))
        tmps = apps.lulesh(run, ar, s, 2, hc)
        got = run.reports()
    ops, _ = L.lulesh_trace(ar.addrs, spec, s, 2, topo, (30, 64, 8), tmps)
    same(got, run_trace(ops), "lulesh 5^3 x 2")
    n = 1000
    x = torch.arange(n, dtype=torch.int32, device="cuda")
    y = torch.zeros_like(x)
    with xpl.Context(pool_words=1 << 20) as ctx:
        ctx.register(x.data_ptr(), 4 * n, 0)
        ctx.register(y.data_ptr(), 4 * n, 0)
        sm = torch.cuda.current_stream().cuda_stream
        ctx.kernel_begin(sm)
        xpl.stream_kernel(x.data_ptr(), y.data_ptr(), n, 4, True, sm)
        ctx.kernel_end(sm)
        rep = ctx.diagnose(50, 0, 256, True)
    assert rep[0]["r_cg"] == n and rep[1]["w_g"] == n
    print("ok stream", flush=True)
    torch.cuda.synchronize()
    print("SANITIZE_DRIVER_DONE", flush=True)


if __name__ == "__main__":
    main()
