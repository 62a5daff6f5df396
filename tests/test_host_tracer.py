"""CPU check of the inline coalescing host tracer (include/xpl_host.h): random
interleaved access streams (several arrays, adjacent/overlapping, mixed kinds
and sizes); the emitted ranges, expanded per 32-bit word, must give every word
the same access sequence as the raw accesses (repeats of R or W collapsed,
RW = R then W) -- DESIGN.md D28."""
import os
import subprocess
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_host_tracer_coalescing_is_exact():
    src = os.path.join(ROOT, "tests", "native", "host_tracer_check.cpp")
    with tempfile.TemporaryDirectory() as d:
        exe = os.path.join(d, "t")
        subprocess.run(["g++", "-O2", "-std=c++17", "-I", os.path.join(ROOT, "include"), src, "-o", exe],
                       check=True)
        out = subprocess.run([exe], capture_output=True, text=True)
        assert out.returncode == 0, out.stdout + out.stderr
        assert "tracer ok" in out.stdout
