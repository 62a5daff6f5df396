"""Parity stress sweep (GPU): for a time budget, random traces with fresh seeds
through the CUDA path -- plain, shuffled device events with split host batches,
odd launch shapes, the kernel-launch wrapper, device-side epoch splits, page
views of several page sizes -- each compared with the oracle.  Prints a summary
line per variant and exits 1 on the first mismatch.  Usage:
python tools/stress_parity.py [seconds]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from oracle import run_trace as oracle_run  # noqa: E402
from paper_conf_ipps_pirkelbauerlvl20_b200 import replay  # noqa: E402
from xplgen.trace import random_trace, with_pages  # noqa: E402


def main(budget=300.0):
    torch.cuda.set_device(0)
    variants = {
        "plain": lambda ops, s: replay.run_trace(ops),
        "shuffled": lambda ops, s: replay.run_trace(ops, seed=s, host_split=5),
        "grid3x96": lambda ops, s: replay.run_trace(ops, grid=3, block=96),
        "traced": lambda ops, s: replay.run_trace([o for o in ops], traced=True),
        "split": lambda ops, s: replay.run_trace(ops, split_epochs=True),
    }
    counts = {k: 0 for k in variants}
    counts["pages"] = 0
    t0 = time.time()
    seed = 0x5350_0000
    while time.time() - t0 < budget:
        seed += 1
        ops = random_trace(seed, n_allocs=1 + seed % 7, n_steps=40 + seed % 90, max_words=200 + (seed * 7919) % 9000,
                           p_device=(seed % 10) / 10)
        exp = oracle_run(ops)
        for name, fn in variants.items():
            got = fn(ops, seed)
            if got != exp:
                print(f"MISMATCH variant={name} seed={seed:#x}")
                return 1
            counts[name] += 1
        pops = with_pages(ops, (1, 7, 16, 256, 1024, 1 << 40), seed)
        if replay.run_trace(pops) != oracle_run(pops):
            print(f"MISMATCH variant=pages seed={seed:#x}")
            return 1
        counts["pages"] += 1
    print(f"stress parity ok: {seed - 0x5350_0000} seeds in {time.time() - t0:.0f} s, traces per variant {counts}")
    return 0


if __name__ == "__main__":
    sys.exit(main(float(sys.argv[1]) if len(sys.argv) > 1 else 300.0))
