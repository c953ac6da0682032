"""CPU oracle for batched SS-HOPM — TEST INFRASTRUCTURE ONLY.

This package is the plain, slow, obviously-correct reference that the CUDA
path is checked against.  It is written from the paper
(/root/reference/PAPER.md, cited as ``P:L<line>``) and shares no code, tables
or constants with the CUDA library under ``paper_conf_ipps_ballardkp11_b200``;
neither side imports the other.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import it.  The product path
never routes through it.

Modules
-------
combinatorics  Sec. III literally: Fig. 4 UPDATEINDEX, MULTINOMIAL0/1,
               Fig. 2 / Fig. 3 compressed tensor-vector products (pure Python).
sshopm         FP64 full-tensor SS-HOPM (Fig. 1 with readings R1-R6 of
               DESIGN.md), Eq. 1/3/5 products, residuals.
dedup          Per-voxel greedy eigenpair clustering (reading R16).
pool           Process-pool wrapper used to time the oracle on host cores.

Parity status: every function is pinned by tests/test_oracle_*.py except
``sshopm.paper_flops_per_iter`` (reading R12) — "parity unpinned".
"""
