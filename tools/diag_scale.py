#!/usr/bin/env python
"""Run only bench.py's diagnose-at-scale measurement (for ncu captures)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl  # noqa: E402

words = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 31
print(json.dumps(bench.diag_at_scale(xpl, torch, words=words, reps=1)))
