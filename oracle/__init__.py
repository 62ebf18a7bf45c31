"""oracle -- TEST INFRASTRUCTURE ONLY (parity oracle for the spec-k FSM hot path).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import, call, link or execute anything under ``oracle/``.  The
product package (``paper_conf_ppopp_xiaja20_b200``) never imports it and has no CPU fallback.

Contents
* ``seq``   -- the plain sequential loop of PAPER.md Fig. 1c, in C
               (``fsm_oracle.c``) with a pure-Python twin for tiny cases.  This is the plain
               definition the spec-k method must reach exactly.
* ``speck`` -- a slow, step-by-step CPU model of the paper's spec-k method (Alg. 3 local
               processing, Alg. 1 / Alg. 2 runtime checks, Sec. 3.3 delayed re-execution,
               Fig. 4a sequential / Fig. 4b tree merge) used to pin the worked examples
                and the shard-map semantics.
Pins live in tests/test_oracle.py (``-m "not gpu"``).  Parity status per function is listed in
DESIGN.md "Oracle pins"; every function here is pinned (none is "parity unpinned").
"""
