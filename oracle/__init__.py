"""TEST INFRASTRUCTURE -- the CPU fp64 oracle (see lmo_oracle.c header).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(paper_conf_ipps_wurypgll25_b200) never imports it.
"""
from .oracle import *  # noqa: F401,F403
