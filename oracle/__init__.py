"""NASPipe CPU oracle — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct NumPy (float64) implementation of what the CSP pipelined
supernet-training hot path computes (PAPER.md = /root/reference/PAPER.md, cited "P:L<line>").

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything from this package.  The product path
(``paper_conf_asplos_zhaolcscwzlc22_b200``) never imports it, and this package imports
nothing from the product path: the two share no code.  Inputs come from ``synth`` (seeded
generators only).

Contents
--------
* ``mlp``, ``transformer``: per-candidate forward/backward of the block families
  (SURVEY §8c reading A17), written from their textbook definitions.
* ``train``: ``train_sequential`` — Def.1/P:L98 + P:L107: the result of CSP training is
  exactly the result of training each subnet "sequentially, one at a time, according to the
  order"; plain SGD (reading A3), MSE loss (A18).
* ``csp``: the dependency table (Def.2, Alg.2), Alg.2 verbatim, the
  logical-time CSP schedule (Alg.1 P:L170-197 under readings A5-A8), the access-order trace
  checker (Table 4) and the balanced partition (reading A12).
* ``residency``: Belady residency under an HBM budget with depth-2 lookahead (P:L156,
  P:L282; reading A9).

Parity status of each function is recorded in DESIGN.md ("Oracle pins").  Every function
here is pinned by a ``-m "not gpu"`` test in tests/test_oracle_*.py.
"""
