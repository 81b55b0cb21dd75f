"""CUDA code generators for the algebraic part A of the BSSN RHS (PAPER.md
§IV-B, the paper's Table II on sm_100a).

Three styles, each a kernel `k_alg_<variant>` that reads the 234 inputs of a
point (bssn_sym input order, [234][ld] SoA, coalesced), evaluates the 24
outputs and writes them ([24][ld]):

* ``sympygr_cse`` — the SymPyGR baseline: SymPy common
  sub-expression elimination over all 24 equations at once; every input is
  loaded first, then the temporaries, then the outputs (long live ranges).
* ``binary_reduce`` — Alg. 3: the 24 expression trees composed
  into one DAG G (hash-consed SymPy sub-expressions; networkx), traversed in
  the order of a topological sort of the line graph of G.  Visiting edge
  (u, v) reduces the operand u into v's accumulator (+ or *); u is dead once
  its last out-edge is reduced, v is complete once its last in-edge is; a
  completed output is stored.  Inputs are loaded right before their first
  use.  Every emitted statement is one binary operation.
* ``staged_cse`` — "staged + CSE": the equations are evaluated
  in stages, each as soon as its inputs are available, with CSE inside a
  stage only, so temporaries die at the end of their stage.  Stages follow
  the fused kernel's field order (alpha, chi, K, beta, B, Gt, gt, At).

`python -m paper_conf_sc_fernandonhzsgb22_b200.codegen.gen` writes
csrc/gen/rhs_alg.cu (committed; the library build compiles it).
"""
from __future__ import annotations

import os
import sys
from collections import defaultdict

import sympy as sp

from . import bssn_sym

HERE = os.path.dirname(os.path.abspath(__file__))
OUT = os.path.join(os.path.dirname(HERE), "csrc", "gen", "rhs_alg.cu")
OUT_PSI4 = os.path.join(os.path.dirname(HERE), "csrc", "gen", "psi4.cu")
VARIANTS = ["sympygr_cse", "binary_reduce", "staged_cse"]
STAGES = [[0], [1], [2], [6, 7, 8], [9, 10, 11], [3, 4, 5], list(range(12, 18)),
          list(range(18, 24))]
PARAM_C = {"eta": "p.eta", "lambda_f0": "p.lambda_f0", "lambda_f1": "p.lambda_f1"}


def _num(x):
    if x.is_Integer:
        return f"{int(x)}.0"
    if x.is_Rational:
        return f"({int(x.p)}.0 / {int(x.q)}.0)"
    return repr(float(x))


class Emitter:
    """C expression printer: Add/Mul keep SymPy's argument order (left to
    right), integer powers become products, negative powers a division."""

    def __init__(self, name_of):
        self.name_of = name_of          # Symbol / sub-expression -> C name or None

    def __call__(self, e):
        n = self.name_of(e)
        if n is not None:
            return n
        if e.is_Number:
            return _num(e)
        if e.is_Add:
            return "(" + " + ".join(self(a) for a in e.args) + ")"
        if e.is_Mul:
            num = [a for a in e.args if not (a.is_Pow and a.exp.is_negative)]
            den = [a.base ** -a.exp for a in e.args if a.is_Pow and a.exp.is_negative]
            if num and num[0] == -1:
                s = "-(" + (" * ".join(self(a) for a in num[1:]) or "1.0") + ")"
            else:
                s = "(" + " * ".join(self(a) for a in num) + ")" if num else "1.0"
            if den:
                s = f"({s} / ({' * '.join(self(d) for d in den)}))"
            return s
        if e.is_Pow:
            b, x = e.base, e.exp
            if x.is_Integer and x > 0:
                bs = self(b)
                return "(" + " * ".join([bs] * int(x)) + ")"
            if x.is_Integer and x < 0:
                bs = self(b)
                return "(1.0 / (" + " * ".join([bs] * int(-x)) + "))"
            if x.is_Rational and x.q == 2:          # half-integer powers: sqrt
                k = int(x.p)
                bs = f"sqrt({self(b)})"
                prod = " * ".join([bs] * abs(k))
                return f"({prod})" if k > 0 else f"(1.0 / ({prod}))"
        raise ValueError(f"cannot emit {e!r}")


def _sym_names(syms, prm):
    names = {s: f"v_{s.name}" for s in syms}
    names[prm["chi_e"]] = "chi_e"
    for k, c in PARAM_C.items():
        names[prm[k]] = c
    return names


def _load(s, idx):
    return f"const double v_{s.name} = in[{idx} * ld + i];"


def gen_cse(exprs, syms, prm):
    names = _sym_names(syms, prm)
    rep, red = sp.cse(exprs, symbols=sp.numbered_symbols("t"), optimizations=None, order="none")
    for t, _ in rep:
        names[t] = t.name
    em = Emitter(names.get)
    body = [_load(s, k) for k, s in enumerate(syms)]
    body.append("const double chi_e = fmax(v_chi, p.chi_floor);")
    body += [f"const double {t.name} = {em(x)};" for t, x in rep]
    body += [f"out[{f} * ld + i] = {em(x)};" for f, x in enumerate(red)]
    return body, len(rep)


def gen_staged(exprs, syms, prm):
    names = _sym_names(syms, prm)
    idx = {s: k for k, s in enumerate(syms)}
    body = [_load(syms[1], 1), "const double chi_e = fmax(v_chi, p.chi_floor);"]
    loaded = {syms[1]}
    ntemp = 0
    for st, fields in enumerate(STAGES):
        rep, red = sp.cse([exprs[f] for f in fields], symbols=sp.numbered_symbols(f"s{st}_"),
                          optimizations=None, order="none")
        need = set()
        for _, x in rep:
            need |= x.free_symbols
        for x in red:
            need |= x.free_symbols
        # this stage's inputs, loaded when the stage starts ("as soon as its
        # derivatives are ready"), visible to the later stages
        for s in sorted((need & set(syms)) - loaded, key=idx.get):
            body.append(_load(s, idx[s]))
            loaded.add(s)
        local = dict(names)
        for t, _ in rep:
            local[t] = t.name
        em = Emitter(local.get)
        body.append(f"{{  // stage {st}: fields {fields}")
        body += [f"  const double {t.name} = {em(x)};" for t, x in rep]
        body += [f"  out[{f} * ld + i] = {em(x)};" for f, x in zip(fields, red)]
        body.append("}")
        ntemp += len(rep)
    return body, ntemp


def gen_binary_reduce(exprs, syms, prm):
    """Alg. 3 over the composed DAG of the 24 expression trees."""
    import networkx as nx
    names = _sym_names(syms, prm)
    idx = {s: k for k, s in enumerate(syms)}
    G = nx.DiGraph()
    node_id = {}

    def nid(x):
        if x not in node_id:
            node_id[x] = len(node_id)
        return node_id[x]

    def build(x):
        if x.is_Atom or x in node_id:
            return
        v = nid(x)
        G.add_node(v)
        for a in x.args:
            if not a.is_Atom:
                build(a)
                G.add_edge(node_id[a], v)     # operand u -> operation v

    for x in exprs:
        build(x)
    expr_of = {v: x for x, v in node_id.items()}
    outputs = defaultdict(list)
    for f, x in enumerate(exprs):
        outputs[node_id[x]].append(f)
    L = nx.line_graph(G)
    order = list(nx.topological_sort(L))
    acc_name = {v: f"r{v}" for v in G.nodes}
    started, remaining_in = set(), {v: G.in_degree(v) for v in G.nodes}
    remaining_out = {v: G.out_degree(v) for v in G.nodes}
    body, loaded = [], set()
    maxlive, live = 0, set()

    def atom(a):
        if a.is_Number:
            return _num(a)
        if a in idx and a not in loaded:
            body.append(_load(a, idx[a]))
            loaded.add(a)
        return names[a]

    def op_of(x):
        return "+" if x.is_Add else "*"

    def init(v):
        """start v's accumulator from its atomic operands (constants, inputs)"""
        x = expr_of[v]
        if x.is_Pow:
            return None
        atoms = [a for a in x.args if a.is_Atom]
        if not atoms:
            return None
        s = atoms[0] if not atoms[0].is_Number else atoms[0]
        parts = [atom(a) for a in atoms]
        return f" {op_of(x)} ".join(parts)

    def finish_pow(v, u):
        x = expr_of[v]
        b = acc_name[u] if not x.base.is_Atom else atom(x.base)
        e = int(x.exp)
        if e > 0:
            return "(" + " * ".join([b] * e) + ")"
        return "(1.0 / (" + " * ".join([b] * (-e)) + "))"

    def complete(v):
        for f in outputs.get(v, []):
            body.append(f"out[{f} * ld + i] = {acc_name[v]};")

    def ensure_leafop(v):
        """nodes with no non-atomic operand have no in-edge: compute at first use"""
        if v in started:
            return
        x = expr_of[v]
        if x.is_Pow:
            body.append(f"double {acc_name[v]} = {finish_pow(v, None)};")
        else:
            body.append(f"double {acc_name[v]} = {init(v)};")
        started.add(v)
        live.add(v)
        complete(v)

    for (u, v) in order:
        ensure_leafop(u) if G.in_degree(u) == 0 else None
        x = expr_of[v]
        if x.is_Pow:
            body.append(f"double {acc_name[v]} = {finish_pow(v, u)};")
            started.add(v)
        elif v not in started:
            i0 = init(v)
            rhs = acc_name[u] if i0 is None else f"{i0} {op_of(x)} {acc_name[u]}"
            body.append(f"double {acc_name[v]} = {rhs};")
            started.add(v)
        else:
            body.append(f"{acc_name[v]} = {acc_name[v]} {op_of(x)} {acc_name[u]};")
        live.add(v)
        remaining_in[v] -= 1
        remaining_out[u] -= 1
        if remaining_out[u] == 0:
            live.discard(u)          # evict(u, B)
        if remaining_in[v] == 0:
            complete(v)
        maxlive = max(maxlive, len(live))
    for v in G.nodes:                # (an output that is a leaf operation)
        if G.in_degree(v) == 0 and G.out_degree(v) == 0:
            ensure_leafop(v)
    body.insert(0, "const double chi_e = fmax(v_chi, p.chi_floor);")
    body.insert(0, _load(syms[1], 1))
    loaded.add(syms[1])
    body = [l for k, l in enumerate(body) if k < 2 or l != _load(syms[1], 1)]
    return body, maxlive, G.number_of_nodes(), G.number_of_edges()


HEADER = """// GENERATED by paper_conf_sc_fernandonhzsgb22_b200/codegen/gen.py — do not edit.
// Algebraic part A of the BSSN RHS (PAPER.md eqs 1-19, §IV-B P:L313-374) in the
// paper's three code-generation styles (Table II), for sm_100a, fp64.
// in: [234][ld] inputs of codegen/bssn_sym.py's order, out: [24][ld] (field order).
#include <cuda_runtime.h>
#include <stdint.h>

#include "../device.cuh"

namespace dgr {
"""


def kernel(variant, body, bounds):
    lb = f"__launch_bounds__({bounds[0]}, {bounds[1]})" if bounds[1] else f"__launch_bounds__({bounds[0]})"
    tag = "" if not bounds[1] else f"_occ{bounds[1]}"
    lines = [f"__global__ void {lb}",
             f"k_alg_{variant}{tag}(const double* __restrict__ in, double* __restrict__ out, "
             "int64_t n, int64_t ld, AlgParams p) {",
             "  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n;",
             "       i += int64_t(gridDim.x) * blockDim.x) {"]
    lines += ["    " + l for l in body]
    lines += ["  }", "}", ""]
    return "\n".join(lines)


def main(out_path=None):
    exprs, syms, prm = bssn_sym.rhs_exprs()
    parts = [HEADER]
    stats = {}
    b_cse, n_cse = gen_cse(exprs, syms, prm)
    b_st, n_st = gen_staged(exprs, syms, prm)
    b_br, maxlive, nn, ne = gen_binary_reduce(exprs, syms, prm)
    stats = {"sympygr_cse": f"{n_cse} CSE temporaries",
             "staged_cse": f"{n_st} CSE temporaries over {len(STAGES)} stages",
             "binary_reduce": f"DAG {nn} nodes / {ne} edges, max {maxlive} live accumulators"}
    bodies = {"sympygr_cse": b_cse, "staged_cse": b_st, "binary_reduce": b_br}
    for v in VARIANTS:
        parts.append(f"// {v}: {stats[v]}")
        # natural register allocation, and the paper's occupancy-constrained
        # build (Table II: __launch_bounds__(343, 3) on A100 = 56 registers;
        # here 256 threads x 4 CTAs = 64 registers per thread)
        parts.append(kernel(v, bodies[v], (128, 0)))
        parts.append(kernel(v, bodies[v], (256, 4)))
    parts.append("""
void launch_rhs_alg(int variant, int occ, const double* in, double* out, int64_t n, int64_t ld,
                    const AlgParams& p, cudaStream_t s) {
  if (n <= 0) return;
  const int threads = occ ? 256 : 128;
  int64_t blocks = (n + threads - 1) / threads;
  const int64_t cap = int64_t(sm_count()) * (occ ? 4 : 8);
  if (blocks > cap) blocks = cap;
  switch (variant * 2 + (occ ? 1 : 0)) {""")
    for k, v in enumerate(VARIANTS):
        parts.append(f"    case {2 * k}: k_alg_{v}<<<int(blocks), threads, 0, s>>>(in, out, n, ld, p); break;")
        parts.append(f"    case {2 * k + 1}: k_alg_{v}_occ4<<<int(blocks), threads, 0, s>>>(in, out, n, ld, p); break;")
    parts.append("""    default: break;
  }
}

}  // namespace dgr
""")
    out_path = out_path or OUT
    os.makedirs(os.path.dirname(out_path), exist_ok=True)
    with open(out_path, "w") as f:
        f.write("\n".join(parts))
    for v in VARIANTS:
        print(f"{v}: {stats[v]}, {len(bodies[v])} statements")
    print("wrote", out_path)
    return stats


PSI4_HEADER = """// GENERATED by paper_conf_sc_fernandonhzsgb22_b200/codegen/gen.py — do not edit.
// The Weyl scalar Psi_4 (PAPER.md P:L159; readings R33-R34, codegen/psi4_sym.py)
// at n points: in [234][ld] (the inputs of dgr_rhs_inputs), xyz [3][ld] the
// points' positions relative to the extraction centre -> out [2][ld] (Re, Im).
// SymPy CSE over both outputs (the generator's second workload).
#include <cuda_runtime.h>
#include <stdint.h>

#include "../device.cuh"

namespace dgr {
"""


def gen_psi4(out_path=None):
    from . import psi4_sym
    exprs, syms, prm, (px, py, pz) = psi4_sym.psi4_exprs()
    names = _sym_names(syms, prm)
    names.update({px: "v_px", py: "v_py", pz: "v_pz"})
    rep, red = sp.cse(exprs, symbols=sp.numbered_symbols("t"), optimizations=None, order="none")
    for t, _ in rep:
        names[t] = t.name
    em = Emitter(names.get)
    need = set()
    for _, x in rep:
        need |= x.free_symbols
    for x in red:
        need |= x.free_symbols
    idx = {s_: k for k, s_ in enumerate(syms)}
    body = [_load(s_, idx[s_]) for s_ in sorted(need & set(syms), key=idx.get)]
    if syms[1] not in need:
        body.append(_load(syms[1], 1))
    body += ["const double v_px = xyz[0 * ld + i];", "const double v_py = xyz[1 * ld + i];",
             "const double v_pz = xyz[2 * ld + i];",
             "const double chi_e = fmax(v_chi, p.chi_floor);"]
    body += [f"const double {t.name} = {em(x)};" for t, x in rep]
    body += [f"out[{f} * ld + i] = {em(x)};" for f, x in enumerate(red)]
    lines = [PSI4_HEADER, f"// {len(rep)} CSE temporaries",
             "__global__ void __launch_bounds__(128)",
             "k_psi4(const double* __restrict__ in, const double* __restrict__ xyz, "
             "double* __restrict__ out, int64_t n, int64_t ld, AlgParams p) {",
             "  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n;",
             "       i += int64_t(gridDim.x) * blockDim.x) {"]
    lines += ["    " + l for l in body]
    lines += ["  }", "}", "",
              "void launch_psi4(const double* in, const double* xyz, double* out, int64_t n, "
              "int64_t ld, const AlgParams& p, cudaStream_t s) {",
              "  if (n <= 0) return;",
              "  int64_t blocks = (n + 127) / 128;",
              "  const int64_t cap = int64_t(sm_count()) * 8;",
              "  if (blocks > cap) blocks = cap;",
              "  k_psi4<<<int(blocks), 128, 0, s>>>(in, xyz, out, n, ld, p);",
              "}", "", "}  // namespace dgr", ""]
    out_path = out_path or OUT_PSI4
    with open(out_path, "w") as f:
        f.write("\n".join(lines))
    print(f"psi4: {len(rep)} CSE temporaries; wrote {out_path}")


if __name__ == "__main__":
    main()
    gen_psi4()
