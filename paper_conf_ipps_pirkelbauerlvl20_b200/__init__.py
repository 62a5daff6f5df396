"""B200-native XPlacer recording + diagnosis runtime (Pirkelbauer et al., IPDPS 2020).

The product is the C-ABI library libxpl.so (include/xpl.h, include/xpl_device.cuh)
built from csrc/ for sm_100a.  This package is the thin Python binding the tests
and bench.py use: argument marshalling only, every step runs in CUDA kernels.
There is no CPU fallback: importing `xpl` without the built library raises.
"""
import os

PKG_DIR = os.path.dirname(os.path.abspath(__file__))
# (XPL_LIB_PATH: an alternative build of the same library, for A/B tuning runs)
LIB_PATH = os.environ.get("XPL_LIB_PATH") or os.path.join(PKG_DIR, "libxpl.so")
WORK_PATH = os.environ.get("XPL_WORK_PATH") or os.path.join(PKG_DIR, "libxplwork.so")


def build(verbose=False):
    """Compile libxpl.so + libxplwork.so for sm_100a in-tree (make in csrc/)."""
    import subprocess
    cmd = ["make", "-C", os.path.join(PKG_DIR, "csrc"), "-j4"]
    if not verbose:
        cmd.append("-s")
    subprocess.run(cmd, check=True)
