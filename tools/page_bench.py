"""The UM page view (NEXT-3) at cfg5 scale, standalone: 2^31-word shadow filled by
the synthetic touch kernel + a CPU-written half, then xpl_page_summary with 4 KiB
(1024-word) and 64 KiB (16384-word) pages, page_kernel timed by CUDA events
(xpl_profile).  Prints one JSON object."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl  # noqa: E402


def main(words=1 << 31, reps=3):
    torch.cuda.set_device(0)
    ctx = xpl.Context(pool_words=words + (1 << 16), max_rows=16)
    base = 1 << 44
    ctx.register(base, 4 * words, xpl.ALLOC_MANAGED)
    ctx.record_copy(base, 0x1000, 2 * words, xpl.COPY_H2D)
    s = torch.cuda.current_stream().cuda_stream
    ctx.kernel_begin(s)
    ctx.touch(base, words, 7, s, 0)
    ctx.kernel_end(s)
    ctx.sync()
    torch.cuda.synchronize()
    out = {"words": words}
    for P in (1024, 16384):
        ctx.page_summary(P)
        ctx.profile(True)
        for _ in range(reps):
            rep = ctx.page_summary(P)
        p = ctx.profile_read(reset=True)["pages"]
        ctx.profile(False)
        ms = p["ms"] / p["launches"]
        out[f"P{P}"] = {"kernel_ms": ms, "gbs": words / (ms / 1e3) / 1e9,
                        "report": {k: rep[0][k] for k in ("pages", "cpu_pages", "gpu_pages", "shared_pages",
                                                          "false_shared_pages", "alternating_pages", "flags")}}
    ctx.close()
    print(json.dumps(out))


if __name__ == "__main__":
    main()
