#!/usr/bin/env python
"""Per-kernel hook cost of the cfg4 program (LULESH-shaped 100^3): a paired
measurement run (every instrumented launch also runs its twin right before or
after it, alternating, L2 flushed before each; work_lulesh.cu time_kernels=2).
Prints, per launch position (19 per timestep), the median instrumented and twin
times and the hook cost (mean over the two orders of the median difference).

  python tools/hook_pairs.py [--steps 20]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

NAMES = ["zero_forces", "integrate_stress", "hourglass", "corner_sum", "accel", "symm", "velocity",
         "position", "kinematics", "lagrange", "monoq_grad", "monoq_region", "eos0", "eos1", "eos2", "eos3",
         "update_volumes", "dt_courant", "dt_hydro"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=20)
    a = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    from xplgen import lulesh as L
    S, T = 100, a.steps
    spec = L.lulesh_spec(S)
    ar = apps.Arena(spec)
    topo = L.topology(S, 0x58504C05)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    st = torch.cuda.Stream()
    out = {}
    with xpl.Context(pool_words=1 << 28, max_rows=64) as ctx:
        for rep in range(2):
            apps.lulesh_prepare(ar, S, topo)
            run = apps.Run(ctx, st.cuda_stream, params=(50, 0, 256), out_cap=64 * (T + 2), time_kernels=2)
            apps.lulesh(run, ar, S, T, hc)
            torch.cuda.synchronize()
        nl = 19 * T
        e = np.array(run.kernel_each[:2 * nl]).reshape(T, 19, 2)
        tf = (np.arange(nl).reshape(T, 19) & 1).astype(bool)
        ins = np.where(tf, e[:, :, 1], e[:, :, 0])
        tw = np.where(tf, e[:, :, 0], e[:, :, 1])
        tot = 0.0
        for p in range(19):
            m = tf[:, p]
            h = 0.5 * (np.median(ins[m, p] - tw[m, p]) + np.median(ins[~m, p] - tw[~m, p]))
            tot += h
            out[NAMES[p]] = {"instr_ms": float(np.median(ins[:, p])), "twin_ms": float(np.median(tw[:, p])),
                             "hook_ms": float(h)}
        out["total_hook_ms_per_timestep"] = tot
    print(json.dumps(out))


if __name__ == "__main__":
    main()
