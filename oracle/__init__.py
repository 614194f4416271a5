"""oracle — CPU reference for the complex stencil sweep and the csTuner method.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The product
path (paper_conf_cluster_sunlyjldlq21_b200) never imports it and shares no code with
it; the only common module is the input generator ``cstgen``.

* ``oracle.stencil``  — ctypes wrapper of liboracle.so (oracle/oracle.cpp): the plain
  loop-nest definitions of the star / box / hypterm-like stencils.
* ``oracle.space``    — brute-force enumeration of the parameter space (Table I,
  P:129-151) under the rules of DESIGN.md.
* ``oracle.tuner``    — the csTuner method step by step (CV + Algorithm 1, PCC +
  Algorithm 2, PMNF, threshold sampling, re-indexing).
"""
