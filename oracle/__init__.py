"""DUET CPU oracle — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU reference for everything the DUET hot path computes
(Algorithm 1 at PAPER.md:86):

  oracle.ir         the IR text reader (independent of the C++ parser in libduet)
  oracle.forward    float64 NumPy forward pass of every op (C1: the plain definitions)
  oracle.partition  coarse-grained phased partitioner, step by step (C2)
  oracle.schedule   integer makespan model (C3), greedy-correction + fallback (C4, PAPER.md:81,
                    :86, :71, :90) and brute-force optimum (C5, "Ideal")

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this package.  It shares no code with the CUDA path (paper_conf_ipps_zhanghl21_b200/
and libduet.so) and imports nothing from it; inputs reach it as NumPy arrays.

Pins (tests/test_oracle_*.py): hand-computed toy MLP, closed-form LSTM/GRU/conv/join cases,
torch float64 modules, brute force on tiny inputs, the Table II and LPT fixtures.
"Parity unpinned" items are listed in DESIGN.md ("Oracle pins").
"""
