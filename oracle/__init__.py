"""CPU oracle for the MEGA GAT hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` legs may import, call, link or execute anything under
oracle/.  The product (paper_conf_icdcs_dengr24_b200/) never touches it and
shares no code, header, table or helper with it.

Contents (each function cites the PAPER.md passage or DESIGN.md reading it
follows; PAPER.md:L = line L of /root/reference/PAPER.md):
  gat.py       GAT forward/backward and the projection, fp64, per-edge
               (PAPER.md:49-55 for the layer skeleton).
  traverse.py  Traversal R: the deterministic reading of Algorithm 1
               (readings R1-R12).
  layout.py    The exact relabelled layout built from the traversal's
               permutation.
  gt.py        Graph Transformer attention (Q.K/sqrt(F) scores), fp64 — NEXT-3
               row, oracle only so far (DESIGN.md R-gt).
  c/oracle.c   The same definitions as plain C loops (fp64, OpenMP over
               destinations) for sizes numpy cannot reach in seconds;
               loaded through coracle.py.

Parity pins: tests/test_oracle_*.py check every function against something
other than itself (dense masked attention, torch autograd, finite
differences, closed forms, invariants, hand-derived traversal traces).
Parity unpinned: traversal R on the paper's own Fig. 3a/Fig. 7 example — the
figures are images in PAPER.md, so no value from
them can be recovered.
"""
