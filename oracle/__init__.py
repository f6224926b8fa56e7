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
              PAPER.md L27 (Sec. II-A) and Fig. 1 (L33-65) step by step, with
              LAPACK/BLAS primitives (potrf, trsm, syrk) as the dense steps;
              supernodal triangular solves (Ly = b, L^T x = y).

Every function cites the passage it follows.  Pins: tests/test_oracle_*.py.
Parity status of each function is listed in DESIGN.md "Oracle pins".
"""
from .numeric import (  # noqa: F401
    NotSPD, Symbolic, symbolic, assemble_B, factor, solve, panels_to_dense_L,
    logdet, front_flops,
)
