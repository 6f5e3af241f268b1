"""CPU oracle for DyCuckoo (TEST INFRASTRUCTURE ONLY).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` leg may import this package.  The product path
(paper_conf_icde_lizlhs21_b200) never imports it and fails loudly without its
CUDA library.  See oracle/dyc_oracle.c for the paper citations and for which
outputs are pinned ("parity unpinned": placement positions, φ, eviction counts).
"""
from .oracle import FIRST_FIT, PAPER_WEIGHTED, OracleTable, build_oracle, oracle_lib  # noqa: F401
from .oracle_wide import OracleWideTable, build_oracle_wide, oracle_wide_lib  # noqa: F401,E402
from .brute import BruteMapCpp, build_brute  # noqa: F401,E402
