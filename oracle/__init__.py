"""PairHMM forward and Smith-Waterman ORACLES -- test infrastructure only.

Only ``tests/``, ``__graft_entry__.smoke()`` and the ``cpu_baseline`` /
``--impl reference`` legs of ``bench.py`` may import anything from this
package. The product path (``paper_conf_ipps_wangxc17_b200``) never does, and
the two share no code: see ``oracle/phmm_oracle.c`` for what is computed and
which passage of PAPER.md each step follows.

Modules:
  ``oracle.core``  -- ctypes binding of the plain-C double-precision oracle
                      (``phmm_oracle.c``), built with gcc on first use.
  ``oracle.brute`` -- explicit enumeration of every HMM path (Fractions or
                      mpmath), the independent pin for the DP on tiny inputs.
  ``oracle.sw``    -- ctypes binding of the plain-C Smith-Waterman oracle
                      (``sw_oracle.c``: Eq. 5 literally and in its running-max form,
                      end cell over the last row and column, traceback).
  ``oracle.sw_brute`` -- explicit enumeration of every Eq. 5 move path (tiny inputs).
"""
