"""ORACLE -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation of what the HIOS hot path
computes (PAPER.md = /root/reference/PAPER.md, cited as P:<line>):

  infer.py  sequential DAG-CNN inference by the operators' definitions (fp64)
  sched.py  HIOS-LP step by step (Alg. 1 + Alg. 2), the cost-model simulator
            (§III), the feasibility validator and a brute-force optimum

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import, call or execute anything here.  The
product package (paper_conf_cluster_kundus23_b200) never imports it and shares
no code with it; the only shared module is ``workloads/`` (graph structure and
seeded random numbers, no arithmetic of the method).

Pins (tests/test_oracle_*.py, all ``-m "not gpu"``): textbook / library
routines (scipy.signal.correlate, torch CPU fp64, torchvision models with the
same weights), the Fig. 4 / Fig. 5 worked examples (fixtures in
tests/golden/), closed forms of the simulator, brute-force enumeration.
Parity unpinned: the C12 group-cost model (synthetic t(S)).
"""
