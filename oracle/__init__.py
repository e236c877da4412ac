"""Oracle package -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything under ``oracle/``.  The product path
(``paper_conf_ppopp_moscovicicp17_b200``) never imports it, and the oracle never
imports the product path: they share no code.

* ``oracle.oracle_a`` -- Oracle-A, the plain definition of a batch's results and final
  set (a sequential Pugh skiplist in C, S1 snapshot-batch semantics).  See
  ``oracle_a.c``'s header for the cited passages.
* ``oracle.dat`` -- the direct-address-table checker: the same S1 definition vectorised
  over a presence bitmap, for the full-size configs; pinned against Oracle-A.
* ``oracle.oracle_b`` -- Oracle-B, the paper's GFSL algorithm step by step (Alg 4.1-4.12)
  as a sequential single-team Python model over the same chunk layout, pinned by the
  paper's worked examples.
"""
