"""oracle/ -- TEST INFRASTRUCTURE ONLY (not part of the product).

A plain, slow, single-threaded CPU Householder QR written from the paper
(Anderson, Ballard, Demmel, Keutzer, "Communication-Avoiding QR Decomposition
for GPUs", IPDPS 2011; /root/reference/PAPER.md) that the CUDA path is checked
against.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import anything from here.
The oracle shares no code with ``paper_conf_ipps_andersonbdk11_b200`` and never
imports it; the only module both sides use is the seeded input generator
``paper_conf_ipps_andersonbdk11_b200.workloads`` (random numbers only, none of
the method's arithmetic).

Contents
  householder.c   xGEQR2 / xORM2R / QR+ORG2R in double and long double (P:L212-224,
                  P:L694-711)
  householder.py  ctypes binding + sign normalisation
  cgs.py          classical Gram-Schmidt in mpmath at 50 digits, brute force for
                  tiny inputs (the independent pin of SURVEY 8(c))

Parity pins: every routine here is pinned by tests/test_oracle.py against closed
forms, LAPACK (numpy), Cholesky of A^T A, mpmath CGS and invariants.  No routine
is "parity unpinned".
"""
from .householder import (  # noqa: F401
    build,
    geqr2,
    orm2r,
    qr,
    normalize_signs,
    geqrf_flops,
)
