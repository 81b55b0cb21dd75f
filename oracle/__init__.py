"""CPU ORACLE — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct NumPy (fp64) implementation of what the hot
path computes, written from the paper (/root/reference/PAPER.md; citations are
"P:Lnnn" = line nnn) and the readings listed in DESIGN.md §Readings.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference leg may import anything under oracle/.  The product path
(paper_conf_sc_fernandonhzsgb22_b200) never imports it, and oracle/ never
imports the product path: they share no code, no tables and no constants.
Only synth/ (seeded inputs, no method arithmetic) serves both.

Modules:
  octree      — refinement rule, minimal 2:1 vertex balance, Morton order
  maps        — nodes, DOFs, hanging nodes, zip owners, padding sources
  unzip       — element reconstruction (interp_hanging) + octant-to-patch (Alg. 2)
  fd          — 6th-order D1, D2, mixed, Kreiss-Oliger
  bssn        — the 24-field BSSN RHS, eqs (1)-(19)
  rk4         — zip (patch-to-octant) + classic RK4                       (Alg. 1)
  constraints — Hamiltonian / momentum / Gamma constraints (diagnostic; not in the paper)
"""
