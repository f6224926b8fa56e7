"""CPU ORACLE for the multifrontal factor-update hot path.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product path (``paper_conf_ipps_georgesgsc11_b200``) never
imports it, and this package never imports the product: the two share only
the seeded input generators in ``workloads/``.

Contents
  symbolic.c  plain-C symbolic analysis by definition (struct(L_j) sets,
              etree by definition, postorder, counts, fundamental supernodes,
              Appendix-B relaxed amalgamation, row lists).
  numeric.py  dense-per-front multifrontal factorization in fp64, following
              PAPER.md L27 (Sec. II-A) and Fig. 1 (L33-65) step by step: the
              Python driver builds each front (A entries, extend-add of the
              children in ascending order) and calls
  numeric.c   plain C + OpenMP, no BLAS/LAPACK: the F-U call (textbook column
              potrf, substitution trsm, syrk; cache-blocked loops), the
              extend-add, the supernodal triangular solves (PAPER.md L7:
              Ly = b, L^T x = y), and a long-double dense Cholesky used only
              as the higher-precision REFEREE of reading C11.

Every function cites the passage it follows.  Pins: tests/test_oracle_*.py.
Parity status of each function is listed in DESIGN.md "Oracle pins".
"""
from .numeric import (  # noqa: F401
    NotSPD, Symbolic, symbolic, assemble_B, factor, factor_stream, solve, panels_to_dense_L,
    dense_cholesky_longdouble,
    logdet, front_flops,
)
