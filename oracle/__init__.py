"""CPU ORACLE for the DyNN-Offload hot path — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct reference of what the B200 path computes:
  afm.py     operator signature, AFM, resolved path, block vector
  encode.py  pilot input features (readings R1-R3)
  pilot.py   pilot-model forward in float64
  decode.py  logits -> resolved control flow + execution blocks + tensor sets
  plan.py    double-buffered evict/prefetch plan (readings R7-R12)
  migrate.py byte-level execution of a plan (P:L180 evict-then-prefetch)
  brute.py   brute-force optimal retention on tiny instances
  invariants.py  I1-I7 of DESIGN.md

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
may import this package. It shares no code with paper_conf_hpca_renxyzlnwxl24_b200/
(the CUDA path) and never reads anything the CUDA path produced.

Parity pinning status: every function here is pinned by a `-m "not gpu"`
test against the paper's worked examples, hand-computed fixtures in tests/golden/,
closed forms, textbook routines or brute force — except where a module header says
"parity unpinned".
"""
