"""NEXT-4 (optional part): CUPTI unified-memory counters (libxplum.so) agree with
the xpl page view of the same run (tools/um_faults.py, a fresh process): the
managed allocation the page view marks alternating on every page takes GPU page
faults and migrations both ways; the CPU-only managed allocation and the device
allocation take no GPU faults and no host-to-device migration."""
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
    k = set(out["kinds"])  # the counter kinds this platform's CUPTI accepted
    assert {"htod_bytes", "dtoh_bytes"} <= k, out["kinds"]
    assert a["um"]["htod_bytes"] > 0 and a["um"]["dtoh_bytes"] > 0
    if "gpu_page_fault_groups" in k:
        assert a["um"]["gpu_page_fault_groups"] > 0 and b["um"]["gpu_page_fault_groups"] == 0
    assert b["um"]["htod_bytes"] == 0
    assert c["um"]["records"] == 0
    assert out["dropped"] == 0
