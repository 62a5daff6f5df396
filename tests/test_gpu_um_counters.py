"""NEXT-4 (optional part): CUPTI unified-memory counters (libxplum.so) next to the
xpl page view of the same run (tools/um_faults.py, a fresh process, real managed
memory touched by CPU and GPU).  The page view must mark the alternating managed
allocation on every page and the CPU-only / device ones not at all.  Where the
platform's CUPTI enables UM counters, the alternating allocation must take GPU
faults and migrations both ways and the others none.  On the
round-1 B200 boxes (driver 580 / CUDA 13.0) every CUPTI build refuses to enable
the UM counter activity (INVALID_PARAMETER at cuptiActivityEnable, kernel
activity works: profiles/r1_cupti_probe.txt); the library must then report that
refusal as its documented code (2000 + CUptiResult), never crash."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_um_counters_match_page_view():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "um_faults.py")], capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    out = json.loads(r.stdout.strip().splitlines()[-1])
    pages = 8192  # 32 MiB / 4 KiB
    a, b, c = out["A_managed_alternating"], out["B_managed_cpu_only"], out["C_device"]
    assert a["pages"]["pages"] == pages and a["pages"]["alternating_pages"] == pages
    assert a["pages"]["shared_pages"] == pages and a["pages"]["false_shared_pages"] == 0
    assert a["diagnose"]["alternating"] == pages and a["diagnose"]["flags"] & 1
    assert b["pages"]["gpu_pages"] == 0 and b["pages"]["cpu_pages"] == pages and b["diagnose"]["gpu_acc"] == 0
    assert c["pages"]["cpu_pages"] == 0 and c["pages"]["gpu_pages"] == pages
    if not out["um_available"]:
        assert 2000 < out["um_enable_status"] < 3000, out["um_enable_status"]  # enable refused, reported
        return
    k = set(out["kinds"])  # the counter kinds this platform's CUPTI accepted
    assert {"htod_bytes", "dtoh_bytes"} <= k, out["kinds"]
    assert a["um"]["htod_bytes"] > 0 and a["um"]["dtoh_bytes"] > 0
    if "gpu_page_fault_groups" in k:
        assert a["um"]["gpu_page_fault_groups"] > 0 and b["um"]["gpu_page_fault_groups"] == 0
    assert b["um"]["htod_bytes"] == 0
    assert c["um"]["records"] == 0
    assert out.get("dropped", 0) == 0
