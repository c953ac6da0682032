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
               Fig. 2 / Fig. 3 compressed tensor-vector products and one Fig. 1
               update on them (pure Python scalar arithmetic).
sshopm         FP64 full-tensor SS-HOPM (Fig. 1 with readings R1-R6 of
               DESIGN.md), Eq. 1/3/5 products, residuals, the R12 flop count.
dedup          Per-voxel greedy eigenpair clustering (reading R16).
classify       Eigenpair type (local max / min / saddle) by the projected
               Hessian (reading R18).

(``bench.py`` times the oracle on the host cores with its own process pool.)

Parity status: every function is pinned by tests/test_oracle_*.py, including
``sshopm.paper_flops_per_iter`` (reading R12): tests/test_oracle_flops.py counts
the operations the literal Fig. 1-3 pseudocode executes.
"""
