"""Per-epoch overhead of the runtime (kernel_begin / kernel_end / fold): E epochs
of one tiny instrumented kernel each, against the same launches without the
epoch wrapper.  Wall-clock over the whole loop (host submission + GPU), and the
fold's live per-launch time.  Usage: python tools/epoch_bench.py [E]"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl  # noqa: E402


def main(E=2000, n=512):
    torch.cuda.set_device(0)
    ctx = xpl.Context(pool_words=1 << 26, max_rows=16)
    base, words = 1 << 44, 1 << 20
    ctx.register(base, 4 * words, xpl.ALLOC_DEVICE)
    addr = (base + 4 * torch.arange(n, dtype=torch.int64) * 37 % (4 * words)).cuda()
    size = torch.full((n,), 4, dtype=torch.int32, device="cuda")
    acc = torch.full((n,), 3, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    out = {}
    for name, wrap in (("launch_only", False), ("epoch", True), ("launch_only2", False), ("epoch2", True)):
        for rep in range(2):
            ctx.sync()
            torch.cuda.synchronize()
            if wrap and rep == 1:
                ctx.profile(True)
            t0 = time.perf_counter()
            for _ in range(E):
                if wrap:
                    ctx.kernel_begin(s.cuda_stream)
                ctx.replay(addr.data_ptr(), size.data_ptr(), acc.data_ptr(), n, grid=2, block=256,
                           stream=s.cuda_stream)
                if wrap:
                    ctx.kernel_end(s.cuda_stream)
            t1 = time.perf_counter()
            ctx.sync()
            torch.cuda.synchronize()
            t2 = time.perf_counter()
            if wrap and rep == 1:
                p = ctx.profile_read(reset=True)
                ctx.profile(False)
                out[name + "_fold_us"] = p["fold"]["ms"] / max(1, p["fold"]["launches"]) * 1e3
            out[name] = {"us_per_epoch": (t2 - t0) / E * 1e6, "host_us_per_epoch": (t1 - t0) / E * 1e6}
    ctx.close()
    print(json.dumps(out))


if __name__ == "__main__":
    main(int(sys.argv[1]) if len(sys.argv) > 1 else 2000)
