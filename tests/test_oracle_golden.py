"""Pins for the oracle: hand-built traces whose reports follow from the paper's
definitions by hand (SURVEY.md §8(c) T1-T15 + D-readings), independent of any
code.  Expected values are written here as numbers or closed forms; each trace
file in tests/golden/ carries its citation.
"""
import os

import pytest

from oracle import run_trace
from xplgen.trace import parse_text

ALT, LOWD, H2DF, D2HF, UNUSED = 1, 2, 4, 8, 16


def run(golden_dir, name):
    with open(os.path.join(golden_dir, name)) as f:
        return run_trace(parse_text(f.read()))


def check(row, **exp):
    bad = {k: (row[k], v) for k, v in exp.items() if row[k] != v}
    assert not bad, f"row {row['id']}: (got, expected) {bad}"


def test_t1_alternating(golden_dir):
    (d,) = run(golden_dir, "T01_alternating.trace")
    check(d[0], w_c=4, w_g=0, r_cc=1, r_cg=3, r_gc=0, r_gg=0, alternating=2, any_acc=5,
          gpu_acc=3, density_pct_any=62, density_pct_gpu=37, low_density_blocks=1,
          low_density_words=8, h2d_unused_runs=0, d2h_unneeded_runs=0, flags=ALT | LOWD,
          ever_accessed=1, words=8, kind=1, live=1)


def test_t1b_runs(golden_dir):
    (d,) = run(golden_dir, "T01b_alternating_runs.trace")
    check(d[0], h2d_unused_runs=1, h2d_unused_words=2, d2h_unneeded_runs=1,
          d2h_unneeded_words=1, flags=ALT | LOWD)


def test_fig4_dom(golden_dir):
    # Fig. 4: C=27, G=0, C>C=680, density 9 %, 18 alternating.
    (d,) = run(golden_dir, "T01dom_fig4.trace")
    check(d[0], words=934, w_c=27, w_g=0, r_cc=680, r_cg=85, alternating=18,
          density_pct_gpu=9, gpu_acc=85, any_acc=27 + 680 + 67,
          density_pct_any=(100 * 774) // 934, d2h_unneeded_runs=1, d2h_unneeded_words=680,
          flags=ALT | LOWD)


def test_fig4_mp(golden_dir):
    # Fig. 4: C=0, G=1024, C>C=0, G>G=1024, density 100 %, 0 alternating.
    d0, d1 = run(golden_dir, "T02_mp_fig4.trace")
    check(d0[0], w_c=0, w_g=1024, r_cc=0, r_cg=0, r_gc=0, r_gg=0, density_pct_gpu=100)
    check(d1[0], w_c=0, w_g=1024, r_cc=0, r_cg=0, r_gc=0, r_gg=1024, density_pct_gpu=100,
          alternating=0, flags=0)


def test_t3_gaussian(golden_dir):
    (d,) = run(golden_dir, "T03_gaussian.trace")
    n = 1000
    check(d[0], w_c=n, w_g=n, r_cg=0, r_gg=n, h2d_unused_runs=1, h2d_unused_words=n,
          d2h_unneeded_runs=0, flags=H2DF, low_density_blocks=0)


def test_t4_backprop_input(golden_dir):
    (d,) = run(golden_dir, "T04_backprop_input.trace")
    n = 1000
    check(d[0], w_c=n, r_cg=n, r_cc=n, w_g=0, d2h_unneeded_runs=1, d2h_unneeded_words=n,
          h2d_unused_runs=0, flags=D2HF)


def test_t5_unused(golden_dir):
    (d,) = run(golden_dir, "T05_backprop_unused.trace")
    check(d[0], any_acc=0, flags=UNUSED, low_density_blocks=0, ever_accessed=0, words=17)
    check(d[1], w_c=16, r_cg=16, flags=0, ever_accessed=1)


def test_t6_lud(golden_dir):
    (d,) = run(golden_dir, "T06_lud.trace")
    n = 32
    check(d[0], w_c=n * n, r_cg=n * n, w_g=n * n - n, r_cc=n, r_gc=n * n - n,
          d2h_unneeded_runs=1, d2h_unneeded_words=n, h2d_unused_runs=0, flags=D2HF)


def test_t7_pathfinder(golden_dir):
    ds = run(golden_dir, "T07_pathfinder.trace")
    r, c, p = 100, 64, 20
    assert len(ds) == r // p
    for t, d in enumerate(ds):
        check(d[0], density_pct_gpu=100 * p // r, gpu_acc=p * c, r_cg=p * c)
        assert d[0]["flags"] & LOWD
    check(ds[0][0], w_c=r * c, h2d_unused_runs=1, h2d_unused_words=(r - p) * c, flags=LOWD | H2DF)
    for d in ds[1:]:
        check(d[0], w_c=0, flags=LOWD)


def test_t8_smith_waterman(golden_dir):
    (d,) = run(golden_dir, "T08_smith_waterman.trace")
    n, m = 7, 5
    check(d[0], words=(n + 1) * (m + 1), w_c=(n + 1) * (m + 1), w_g=n * m, r_cg=n + m + 1,
          r_gg=n * m - 1, h2d_unused_words=n * m, h2d_unused_runs=n,
          alternating=(n + 1) * (m + 1), density_pct_gpu=100, flags=ALT)


def test_t9_tie(golden_dir):
    (d,) = run(golden_dir, "T09_density_tie.trace")
    check(d[0], low_density_blocks=1, low_density_words=10, r_cg=5, w_g=6, gpu_acc=11,
          density_pct_gpu=1100 // 30, flags=LOWD)


def test_t10_snapshot_rw(golden_dir):
    d0, d1 = run(golden_dir, "T10_snapshot_rw.trace")
    check(d0[0], w_c=1, w_g=1, r_cg=1, r_gg=0, alternating=1, flags=ALT)
    check(d1[0], r_gc=1, r_cc=0, w_c=0, w_g=0, alternating=0, flags=0)


def test_t11_order(golden_dir):
    (d,) = run(golden_dir, "T11_epoch_order.trace")
    check(d[0], w_g=2, r_cg=2, r_gg=0)


def test_t12_delayed_free(golden_dir):
    d0, d1 = run(golden_dir, "T12_delayed_free.trace")
    assert [r["id"] for r in d0] == [0, 1]
    check(d0[0], live=0, w_c=2, any_acc=2, r_cg=0, words=16, flags=0)
    check(d0[1], live=1, r_cg=8, w_c=0, words=8, kind=0, flags=0)
    assert [r["id"] for r in d1] == [1]
    check(d1[0], any_acc=0, flags=UNUSED, ever_accessed=1)


def test_t13_reset(golden_dir):
    d0, d1 = run(golden_dir, "T13_reset_keeps_origin.trace")
    check(d0[0], w_c=1)
    check(d1[0], r_cg=1, w_c=0, alternating=0)


def test_t14_host_order(golden_dir):
    d0, d1, d2 = run(golden_dir, "T14_host_order.trace")
    check(d0[0], w_g=1)
    check(d1[0], r_gc=1, r_cc=1, w_c=1, w_g=0, alternating=0)
    check(d2[0], r_cg=1, r_gg=0)


def test_t15_untracked(golden_dir):
    (d,) = run(golden_dir, "T15_untracked.trace")
    for row in d:
        check(row, any_acc=0, flags=UNUSED, ever_accessed=0)


def test_t16_deferred_host(golden_dir):
    (d,) = run(golden_dir, "T16_deferred_host.trace")
    check(d[0], w_g=1, r_gc=1, r_cg=1, alternating=1, flags=ALT)


def test_t17_copies(golden_dir):
    (d,) = run(golden_dir, "T17_copies.trace")
    a, b, c = d
    check(a, r_cc=4, r_cg=8, w_g=4, w_c=0, alternating=0, d2h_unneeded_runs=1,
          d2h_unneeded_words=4, flags=D2HF)
    check(b, w_g=8, any_acc=8, flags=0)
    check(c, w_c=4, any_acc=4, density_pct_any=50, flags=0)


def test_t18_unaligned(golden_dir):
    (d,) = run(golden_dir, "T18_unaligned.trace")
    check(d[0], words=6, w_c=1, r_cg=5, any_acc=5, gpu_acc=5, alternating=1,
          density_pct_gpu=500 // 6, flags=ALT)


def test_names(golden_dir):
    # XplAllocData names: the first name inside a live row names it.
    ops = parse_text("REG 0x1000 16 M\nREG 0x2000 16 D\nREG 0x3000 16 H\n")
    ops.append(("DIAG", 50, 0, 1, 1, (0x2004, 0x5000, 0x1000, 0x2000)))
    (d,) = run_trace(ops)
    assert [r["name_idx"] for r in d] == [2, 0, 0xFFFFFFFF]


def test_all_golden_files_covered(golden_dir):
    files = sorted(f for f in os.listdir(golden_dir) if f.endswith(".trace"))
    assert len(files) >= 19
    for f in files:
        run(golden_dir, f)  # every fixture replays without a rejected event


def test_oracle_cli(golden_dir):
    import json
    import subprocess
    from oracle.oracle import HERE, build
    exe = os.path.join(HERE, "xpl_oracle")
    if not os.path.exists(exe):
        build()
    out = subprocess.run([exe, os.path.join(golden_dir, "T01_alternating.trace")],
                         capture_output=True, text=True, check=True).stdout
    row = json.loads(out.splitlines()[0])
    assert row["w_c"] == 4 and row["alternating"] == 2 and row["flags"] == 3


def test_t19_pages(golden_dir):
    """NEXT-3 page view, by hand from the definitions (T19's header)."""
    p1024, p1, pbig, adv, adv2, diag, after = run(golden_dir, "T19_pages.trace")
    FS, MISMATCH = 1, 2
    check(p1024[0], pages=4, cpu_pages=2, gpu_pages=3, shared_pages=2, false_shared_pages=1,
          alternating_pages=1, flags=FS, advice=0, words=3500, page_words=1024)
    check(p1024[1], pages=2, cpu_pages=1, gpu_pages=1, shared_pages=1, false_shared_pages=1,
          alternating_pages=0, flags=0)  # device: no page effects
    # one word per page: the per-word classes (CPU words 10 + 1, GPU words 8 + 1 + 3)
    check(p1[0], pages=3500, cpu_pages=11, gpu_pages=12, shared_pages=1, false_shared_pages=0,
          alternating_pages=1, flags=0)
    # one page for the whole allocation
    check(pbig[0], pages=1, cpu_pages=1, gpu_pages=1, shared_pages=1, false_shared_pages=0,
          alternating_pages=1, flags=0)
    # ReadMostly advised while a page alternates
    check(adv[0], advice=1, flags=FS | MISMATCH)
    # unset ReadMostly; PreferredLocation = CPU (device -1); AccessedBy GPU on B
    check(adv2[0], advice=4, flags=FS)
    check(adv2[1], advice=8, flags=0)
    # the resetting diagnose clears the interval: no page is used any more
    check(after[0], cpu_pages=0, gpu_pages=0, shared_pages=0, false_shared_pages=0, alternating_pages=0,
          advice=4, flags=0)
    assert diag[0]["alternating"] == 1 and diag[0]["any_acc"] == 10 + 1 + 8 + 3
