"""ORACLE — test infrastructure only.

Plain, slow, obviously-correct CPU implementation of what the hot path of
Balaji et al., "Community-based Matrix Reordering for Sparse Linear Algebra
Optimization" (ISPASS'23) computes.  Citations "P:NN" are lines of
/root/reference/PAPER.md; "c-NN" are the readings of SURVEY.md §8(c), listed
again in DESIGN.md.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import, call, link or execute anything under
``oracle/``.  The product package never imports it, and the oracle never
imports the product package: the two share no code.  Inputs come from the
separate ``synth`` generator module.

Modules
-------
spmv      Alg. 1 as the exactly-summed, correctly-rounded row sum.
permute   B = P A P^T and vector relabel ("assigns ... consecutive IDs").
rabbit    RABBIT community detection + dendrogram DFS order (P:86, P:130,
          ref [1] P:259), read as SURVEY.md §8(c) c5-c10; RABBIT++ (P:162-189).
plan      Row classes / stream tiles / hub chunks / hot prefix H / partition
          bounds: build constants re-declared here (c23), not shared.
metrics   Compulsory traffic, insularity, skew,
          modularity [34], hub footprint.
power     Power-iteration recurrence (c22).
c/        Plain C fp64 CSR SpMV used as the timed CPU baseline and for
          large-size sampled parity.

Parity status: every function here is pinned by tests/test_oracle_*.py
against closed forms, brute force, library routines or invariants; none is
"parity unpinned" (see DESIGN.md §Oracle pins).
"""
