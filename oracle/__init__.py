"""ResCCL CPU oracle — TEST INFRASTRUCTURE ONLY.

This package is a plain, slow, obviously-correct CPU restatement of what the
paper's hot path computes (Liu et al., "ResCCL", SIGCOMM '25; PAPER.md line
numbers are cited as ``P:Lx-y``).  It shares NO code with the product path
(``paper_conf_sigcomm_liuhlgcwz025_b200``: C++ planner + CUDA kernels); the
two are independent restatements of the paper and are compared in ``tests/``.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything from here.  The product path never
does, and fails loudly when its CUDA extension is missing.

Modules
  ir          transfer model, text format, algorithm generators   (App. A/B)
  dag         global dependency analysis -> DAG G_A=(V_T,E)
  hpds        Alg. 1 HPDS and the round-robin baseline
  lower       task->primitive translation, state-based TB allocation, fusion
                                                                 (Eq. 7)
  definition  collective definitions (sum / concat / scatter)
  numerics    dtype rounding rules used by both definition and replay (R8)
  replay      symbolic + value replay under a blocking FIFO simulator, invariants I1-I6
  timeline    f2: alpha-beta + Eq. 1 contention timeline, Eq. 7 on wall-clock activity
  nvls        f3: the NVLS (multimem) schedule -- mred / mcast on the chunk layout (R28)

Parity-unpinned items: HPDS tie-breaks beyond ring/HM/DBT
(pinned only by readings R3/R4), the choice among equal-size TB colourings, and the
TB counts of synthesized schedules.
"""
