"""CPU correctness oracle for CuART's hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import this package.  The product package
(``paper_conf_icpp_koppehelggp21_b200``) never imports it and shares no code with
it; the only common dependency is the seeded input generator ``workloads``.

Two oracles, both written from the paper (PAPER.md, cited P:<line>):

* ``ArtOracle``  — a plain single-threaded pointer ART (Leis et al. [17], the
  structure the paper defers to at P:47/P:74), compiled from ``art_oracle.c``.
  It follows the algorithm step by step: insert with path compression and lazy
  expansion, pessimistic prefix check on lookup, sequential batch update.
* ``MapOracle``  — the plain definition of what the method computes
  (SURVEY §8(c)): a finite map key -> value, ``lookup(q) = M[q]`` else MISS,
  updates applied in op order (highest op index wins per key).  Sorted
  arrays + binary search; used where the pointer ART would be too slow.

Pins (``tests/test_oracle_*.py``): brute force on tiny inputs (Python dict),
hand-derived closed-form trees (tests/golden/), ART invariants, insertion-order
independence, and an independent recursive-partition construction of the
canonical tree.  Parity pinned for every function here; nothing is "unpinned".
"""
from .art import ArtOracle, MapOracle, OART_MISS, build_oracle_lib, canonical_bytes  # noqa: F401
