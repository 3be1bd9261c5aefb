"""ORACLE — test infrastructure only.

Plain, slow, obviously-correct CPU (numpy fp64) implementation of what the
Mimose hot path computes (§IV, Algorithm 1; DESIGN.md readings).
Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import anything here.  It
shares no code with ``paper_conf_ipps_liaolysshfyctzlq23_b200/csrc`` and never
imports the product binding; the only shared module is the seeded input
generator ``paper_conf_ipps_liaolysshfyctzlq23_b200.workload``.

Modules:
  philox     Philox4x32-10 counter RNG + dropout keep masks   (DESIGN R-B)
  model      post-LN encoder forward/backward, heads, AdamW
  memsim     arena event model = definition of peak live bytes
  estimator  quadratic least-squares memory estimator
  planner    Algorithm 1 (our reading) + verify + brute force

Parity status of each function is stated in its docstring; DESIGN.md lists
every reading taken where the paper is silent or garbled.
"""
