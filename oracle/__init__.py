"""CPU oracle for the SMIless co-optimisation hot path.

TEST INFRASTRUCTURE ONLY -- see oracle/smiless_oracle.c for what it computes.
Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline and
--impl reference) may import it.  The product path
(paper_conf_sc_luxl0y024_b200/) never does.

Parity pins: worked examples E1-E6 (tests/golden/),
the Eq. (5) closed form, Theorem 5.1, Lindley's recursion, the tandem-queue
recursion, longest path, the keep-alive billing closed form, SLA/price/time
scaling invariants, and cross-checks against an independent event-driven
simulator (oracle/des.py).  G3/G4/G5 are pinned only by that cross-check
("parity unpinned by the paper" for those three readings).
"""
from .oracle import OracleProblem, build  # noqa: F401
