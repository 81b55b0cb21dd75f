"""libdgr host builder vs the oracle: bit-exact octree and index maps (CPU).

The C ABI library builds the octree (dgr_octree_build) and every map inside
dgr_mesh_create on the host; dgr_mesh_export_maps returns them in canonical
global form.  They must equal the oracle's maps exactly (BASELINE.json
north_star: "bit-exactly for octree, unzip and zip index maps").  No device
call is made here (host-only meshes).
"""
import ctypes as C
import os
import subprocess

import numpy as np
import pytest

import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from oracle import octree
from oracle.maps import OracleMesh
from synth import configs

HDR = os.path.join(os.path.dirname(os.path.dirname(__file__)), "include", "dgr.h")


def test_library_exports_every_declared_symbol():
    import re
    decl = set(re.findall(r"^\s*(?:dgr_status|const char\*|int64_t)\s+(dgr_\w+)\s*\(",
                          open(HDR).read(), flags=re.M))
    assert len(decl) >= 15
    L = dgr.lib()
    for name in decl:
        assert hasattr(L, name), name
    assert set(dgr.EXPORTED) == decl
    out = subprocess.run(["nm", "-D", "--defined-only", dgr.LIB_PATH], capture_output=True,
                         text=True).stdout
    for name in decl:
        assert f" T {name}" in out, name
    assert dgr.lib().dgr_version().decode().startswith("dgr-b200")


def _degenerate(name, periodic, level_min):
    return configs.MeshConfig(name=name, xmin=(-0.5,) * 3, width=1.0, periodic=periodic,
                              level_min=level_min)


def _cfgs():
    # + the degenerate meshes: one octant (all padding extrapolated) and 8
    # periodic octants (+x and -x reach the same neighbour)
    return [configs.c1_uniform(), configs.small_adaptive(lmax=5, rho=0.5),
            configs.small_bbh(lmax=6, rho=0.5), configs.c2_schwarzschild(),
            _degenerate("one", False, 0), _degenerate("p8", True, 1)]


@pytest.mark.parametrize("cfg", _cfgs(), ids=lambda c: c.name)
def test_octree_bitexact(cfg):
    oc = dgr.octree_build(cfg)
    a, l = octree.build_octree(cfg)
    assert np.array_equal(oc[:, :3].astype(np.int64), a)
    assert np.array_equal(oc[:, 3].astype(np.int64), l)


@pytest.mark.parametrize("name", ["c3", "c4"])
def test_octree_bitexact_full_configs(name):
    cfg = configs.get(name)
    oc = dgr.octree_build(cfg)
    a, l = octree.build_octree(cfg)
    assert np.array_equal(oc[:, :3].astype(np.int64), a)
    assert np.array_equal(oc[:, 3].astype(np.int64), l)


@pytest.mark.parametrize("cfg", _cfgs(), ids=lambda c: c.name)
def test_maps_bitexact(cfg):
    m = dgr.Mesh(cfg, device=False)
    om = OracleMesh(cfg)
    om.build_dofs()
    mp = m.maps()
    assert m.info["n_dof_global"] == om.n_dof
    assert np.array_equal(mp["octants"][:, :3], om.anchors)
    assert np.array_equal(mp["o2n"], om.o2n)
    assert np.array_equal(mp["hanging"], om.hanging_table())
    assert np.array_equal(mp["zip"], np.stack([om.zip_leaf, om.zip_node], 1))
    assert np.array_equal(mp["dof_gid"], np.arange(om.n_dof))
    assert np.array_equal(m.dof_xyz_host(), om.dof_coords())
    # padding sources on a sample of octants (all of them for the small meshes)
    n = om.n_oct
    octs = np.arange(n) if n <= 700 else np.random.default_rng(0).choice(n, 400, replace=False)
    src, kind = om.padding_sources(octs)
    assert np.array_equal(mp["pad_src"][octs], src)
    assert np.array_equal(mp["pad_kind"][octs], kind)


@pytest.mark.slow
def test_maps_bitexact_c3_sampled():
    """Full-size q=1 mesh: DOF numbering for every octant, padding on a sample."""
    cfg = configs.c3_bbh_q1()
    m = dgr.Mesh(cfg, device=False)
    om = OracleMesh(cfg)
    om.build_dofs()
    mp = m.maps()
    assert np.array_equal(mp["o2n"], om.o2n)
    assert np.array_equal(mp["zip"], np.stack([om.zip_leaf, om.zip_node], 1))
    assert np.array_equal(mp["hanging"], om.hanging_table())
    octs = np.random.default_rng(1).choice(om.n_oct, 300, replace=False)
    src, kind = om.padding_sources(octs)
    assert np.array_equal(mp["pad_src"][octs], src)
    assert np.array_equal(mp["pad_kind"][octs], kind)


# ------------------------------------------------------------ tree validation

def _mesh_status(cfg, oc):
    try:
        dgr.Mesh(cfg, oc, device=False)
        return 0
    except dgr.DgrError as e:
        return e.status


def test_rejects_bad_trees():
    cfg = configs.small_adaptive(lmax=4, rho=0.5)
    oc = dgr.octree_build(cfg)
    assert _mesh_status(cfg, oc) == 0
    # unsorted
    bad = oc.copy()
    bad[[3, 4]] = bad[[4, 3]]
    assert _mesh_status(cfg, bad) == -2
    # incomplete
    assert _mesh_status(cfg, oc[:-1]) == -2
    # overlapping: duplicate an octant
    assert _mesh_status(cfg, np.concatenate([oc[:5], oc[4:]])) == -2
    # unbalanced: coarsen the whole tree around a fine leaf to level 1 except one
    D = cfg.max_depth
    a, l = octree.refine(cfg.__class__(**{**cfg.__dict__, "punctures": (), "level_min": 1}))
    a1, l1 = octree.children(a[:1], l[:1], D)
    a2, l2 = octree.children(a1[7:8], l1[7:8], D)
    A = np.concatenate([a[1:], a1[:7], a2])
    Lv = np.concatenate([l[1:], l1[:7], l2])
    A, Lv = octree.sort_morton(A, Lv, D)
    ub = np.concatenate([A, Lv[:, None]], 1).astype(np.uint32)
    assert _mesh_status(cfg, ub) == -2
    # the balanced closure of the same tree is accepted
    B, Lb = octree.balance(A, Lv, D, False)
    assert _mesh_status(cfg, np.concatenate([B, Lb[:, None]], 1).astype(np.uint32)) == 0


def test_rejects_single_periodic_octant():
    """A periodic domain of one octant (level 0) is its own neighbour across
    every face; both the library and the oracle refuse it (levels >= 1)."""
    cfg = _degenerate("p1", True, 0)
    oc = dgr.octree_build(cfg)
    assert oc.shape[0] == 1
    assert _mesh_status(cfg, oc) == -2
    with pytest.raises(AssertionError):
        OracleMesh(cfg)


def test_host_mesh_rejects_device_calls():
    cfg = configs.c1_uniform()
    m = dgr.Mesh(cfg, device=False)
    st = dgr.lib().dgr_rk4_step(m._h, C.c_double(0.1), C.c_void_p(16), None, None)
    assert st == -6          # DGR_ERR_STATE: host-only mesh
    st = dgr.lib().dgr_unzip(None, None, None, 24, None)
    assert st == -1          # DGR_ERR_ARG


def test_host_only_mesh_refuses_device_calls():
    """Device entry points (dgr_rk4_step_host included) on a host-only mesh
    return DGR_ERR_STATE before touching any buffer; a mismatched host-state
    list is rejected by the binding."""
    import torch
    cfg = configs.small_adaptive(lmax=4, rho=0.5)
    m = dgr.Mesh(cfg, device=False)
    h = torch.zeros((24, m.dof_stride), dtype=torch.float64)
    with pytest.raises(dgr.DgrError) as e:
        m.rk4_step_host([h], [h], 1e-3)
    assert e.value.status == -6
    with pytest.raises(ValueError):
        m.rk4_step_host([h], [], 1e-3)
    with pytest.raises(ValueError):
        m.rk4_step_host([h[:, :-1].contiguous()], [h], 1e-3)


def test_round2_entry_points_validate_without_gpu():
    """The round-2 C ABI (group, regrid, Psi_4, code-generation study) rejects
    null / host-only arguments synchronously, before any CUDA call."""
    L = dgr.lib()
    cfg = configs.c1_uniform()
    m = dgr.Mesh(cfg, device=False)
    vp = C.c_void_p
    p16 = vp(16)
    c3 = (C.c_double * 3)(0.0, 0.0, 0.0)
    # host-only mesh -> DGR_ERR_STATE
    assert L.dgr_regrid_indicator(m._h, p16, 0xFFFFFF, p16, None) == -6
    assert L.dgr_regrid_transfer(m._h, p16, m._h, p16, None) == -6
    assert L.dgr_psi4(m._h, p16, c3, p16, None, None) == -6
    assert L.dgr_psi4_modes(m._h, p16, c3, C.c_double(1.0), 4, 8, 2, p16, None, None, None) == -6
    assert L.dgr_rhs_inputs(m._h, p16, p16, 10, None, None) == -6
    # null / out-of-range arguments -> DGR_ERR_ARG
    assert L.dgr_rhs_algebra(3, 0, p16, p16, 1, 1, None, None) == -1
    assert L.dgr_rhs_algebra(0, 0, p16, p16, 5, 4, None, None) == -1
    n = C.c_int64(0)
    assert L.dgr_regrid_octree(None, None, C.c_double(1.0), C.c_double(0.5), 0, 3, None,
                               C.byref(n)) == -1
    arr = (vp * 1)(m._h.value)
    g = vp()
    assert L.dgr_group_create(arr, 1, C.byref(g)) == -1        # host-only mesh in a group
    assert L.dgr_group_create(None, 2, C.byref(g)) == -1
    # regrid octree works on host-only meshes: eps between all w -> the same tree
    w = np.full(m.info["n_oct_global"], 0.5)
    octs = m.regrid_octree(w, 1.0, 0.1, 0, 18)
    assert np.array_equal(octs, m.octants)
    # with every octant above eps_refine: one level finer everywhere
    octs = m.regrid_octree(w, 0.25, 0.1, 0, 18)
    assert len(octs) == 8 * m.info["n_oct_global"] and np.all(octs[:, 3] == m.octants[0, 3] + 1)
