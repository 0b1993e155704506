"""CPU oracle for the FastZ hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (``cpu_baseline`` leg and ``--impl reference``)
may import this package.  The product path (``paper_conf_sc_gundaboluvt21_b200``) never imports it, and
the two share no code: this package holds its own scoring defaults, its own encoders and its own C source.

* ``oracle.fastz_oracle.c`` / ``oracle.core``: plain sequential LASTZ-style y-drop gapped extension with
  full traceback, row-major, int64.
* ``oracle.brute``: pure-Python full-matrix implementation of the same definitions and an exhaustive
  alignment-path enumerator, used to pin the C oracle on tiny inputs.
"""
