"""RHS code generators (the paper's Table II redone on
sm_100a).  `bssn_sym` builds the algebraic part A of the BSSN right-hand side
(§IV-B: 234 inputs -> 24 outputs) as SymPy expressions
from eqs (1)-(19); `gen` emits CUDA kernels for it in the paper's three
styles — SymPyGR-style global CSE, binary reduction over the expression DAG
(Alg. 3) and staged CSE — into csrc/gen/.
Build-time tooling only: the library ships the generated .cu files."""
