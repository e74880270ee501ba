"""fp64 CPU oracle of GRANII's hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  The product package
(paper_conf_cgo_lenadorasgytm26_b200) never imports it, and the two share no
code (see granii_oracle.c header).
"""
from .oracle import *  # noqa: F401,F403
