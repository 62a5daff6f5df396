"""TEST INFRASTRUCTURE ONLY: the plain CPU oracle (see xpl_oracle.cpp).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
--impl reference leg may import this package.  The product path
(paper_conf_ipps_pirkelbauerlvl20_b200) never does.
"""
from .oracle import Oracle, REPORT_FIELDS, run_trace, build  # noqa: F401
