"""CPU oracle — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  The product package
(paper_conf_hpdc_wahibm15_b200) never imports it, and it imports nothing from
the product: its program loader, validation and evaluation are its own.

See oracle/oracle.h for what is computed and the PAPER.md passages it follows.
"""
from .oracle import OracleProgram, build_oracle, dense_arrays, load_library  # noqa: F401
