"""tracePrint output (NEXT-1): the Fig. 4 textual layout and the CSV form,
formatted by the library from report rows (no GPU: rows from the oracle)."""
import os

from oracle import run_trace
from xplgen.trace import parse_text


def test_fig4_text_and_csv(golden_dir):
    from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
    ops = parse_text(open(os.path.join(golden_dir, "T01dom_fig4.trace")).read())
    ops[-1] = ("DIAG", 50, 0, 256, 1, (0x200000,))
    (rows,) = run_trace(ops)
    txt = xpl.format_reports(rows, names=[(0x200000, "dom")], only_named=True)
    lines = txt.splitlines()
    assert lines[0] == "*** checking 1 named allocations"
    assert lines[1] == "dom"
    assert lines[4].split() == ["27", "0", "680", "85", "0", "0"]  # C G C>C C>G G>C G>G
    assert "access density (in %): 9" in txt
    assert "18 elements with alternating accesses" in txt
    csv = xpl.format_reports(rows, names=[(0x200000, "dom")], csv=True)
    head, row = csv.splitlines()[:2]
    rec = dict(zip(head.split(","), row.split(",")))
    assert rec["name"] == '"dom"' and rec["w_c"] == "27" and rec["alternating"] == "18"
