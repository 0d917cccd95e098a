"""EATSS oracle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``libeatss.so`` and ``paper_conf_cgo_jayaweerakwk24_b200``) never imports it and
shares no code with it.

Contents
  * ``numeric``  -- ctypes wrappers over ``oracle.c`` (plain fp64 loop nests).
  * ``model``    -- the EATSS tile-selection model (§IV, reading R of
                    DESIGN.md §2), evaluated by unpruned brute force.

Parity status per function is listed in DESIGN.md §2.4 ("pins").
"""
