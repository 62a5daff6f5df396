"""The diagnose pass at cfg5 scale (bench.py's diag_at_scale), standalone."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl  # noqa: E402

if __name__ == "__main__":
    torch.cuda.set_device(0)
    words = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 31
    r = bench.diag_at_scale(xpl, torch, words=words)
    peak, _ = bench.peaks()
    for k in ("no_reset", "reset"):
        r[k]["frac"] = r[k]["gbs"] / peak
    print(json.dumps(r))
