"""The Smith-Waterman configs of bench.py's other_configs alone (cfg1 SW-128, its
device-split variant, cfg3 SW-16K), instrumented and twin.  Prints one JSON object."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl  # noqa: E402

if __name__ == "__main__":
    torch.cuda.set_device(0)
    out = bench.other_configs(xpl, apps, torch, lulesh_steps=0, lulesh250_steps=0)
    print(json.dumps({k: {"ms": v["ms"], "twin_ms": v["twin_ms"], "slowdown": v["slowdown"]} for k, v in out.items()}))
