"""Multi-rank CUDA path on ONE GPU (SURVEY §4 invariant 1, §8e).

Only one B200 is available to this build, so the partitioned path is checked
by running R rank-meshes of the same octree side by side in one process in
external-exchange mode (dgr_mesh_desc.nccl_id = NULL): between stages the test
moves each rank's owned DOFs to the peers' ghost slices using the library's
own send lists / receive counts (the same [peer][field][dof] blocks the NCCL
path sends).  After RK4 steps every rank's owned DOFs must be BIT-IDENTICAL to
the single-rank run: all kernels are per-octant deterministic and ghosts are
exact copies.
"""
import numpy as np
import pytest

import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from oracle import rk4 as ork4
from oracle.maps import OracleMesh
from synth import configs, initial

from .gpu_util import need_gpu, to_dev, torch

pytestmark = pytest.mark.gpu
NF = 24


def _exchange(meshes, states, lists):
    """Ghost refresh for all ranks (device copies following libdgr's lists)."""
    world = len(meshes)
    for r in range(world):
        send, scount, _, _ = lists[r]
        off = 0
        for peer in range(world):
            n = int(scount[peer])
            if n == 0:
                continue
            ids = send[off:off + n]
            off += n
            # where these land on the peer: its ghost block from rank r
            _, _, rcount_p, no_p = lists[peer]
            goff = no_p + int(rcount_p[:r].sum())
            states[peer][:, goff:goff + n] = states[r][:, ids]


@pytest.mark.parametrize("world,phases", [(2, 0), (3, 0), (2, 1)])
def test_multirank_bit_identical(world, phases):
    need_gpu()
    cfg = configs.small_bbh(lmax=6, rho=0.5)
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords())
    dt = ork4.dt_courant(om)
    ref = dgr.Mesh(cfg)
    ur = to_dev(u, ref.dof_stride)
    meshes, states, lists, gids = [], [], [], []
    for r in range(world):
        m = dgr.Mesh(cfg, rank=r, nranks=world)
        m.set_phases(phases)   # 1: interior octants first, then the boundary ones
        gid = m.export(dgr.MAP_DOF_GID, np.int64)
        st = torch.zeros((NF, m.dof_stride), dtype=torch.float64, device="cuda")
        st[:, :len(gid)] = torch.from_numpy(u[:, gid])
        send = torch.from_numpy(m.export(dgr.MAP_SEND, np.int32).astype(np.int64)).cuda()
        lists.append((send, m.export(dgr.MAP_SEND_COUNTS, np.int64),
                      m.export(dgr.MAP_RECV_COUNTS, np.int64), m.info["n_dof_owned"]))
        meshes.append(m)
        states.append(st)
        gids.append(gid)
        assert m.info["n_oct_ghost"] > 0
    us = [torch.zeros_like(s) for s in states]
    acc = [torch.zeros_like(s) for s in states]
    for step in range(2):
        ref.rk4_step(ur, dt)
        for s in range(4):
            cur = states if s == 0 else us
            if s == 0:
                for r in range(world):
                    us[r].copy_(states[r])
            _exchange(meshes, cur, lists)
            for r in range(world):
                meshes[r].rk4_stage(s, dt, states[r], us[r], acc[r])
        for r in range(world):
            states[r].copy_(acc[r])
    torch.cuda.synchronize()
    full = ur[:, :om.n_dof].cpu().numpy()
    for r in range(world):
        no = meshes[r].info["n_dof_owned"]
        got = states[r][:, :no].cpu().numpy()
        assert np.array_equal(got, full[:, gids[r][:no]]), f"rank {r} differs"


@pytest.mark.parametrize("world", [2, 3])
def test_interior_octants_need_no_ghost_values(world):
    """The octants the fused path runs while the ghost exchange is in flight
    (SURVEY §8e overlap) must not read any ghost value: with every ghost DOF set
    to NaN and only the interior phase executed (DGR_OPT_PHASES = 2), the RHS at
    every DOF whose zip owner is an interior octant is finite and bit-identical
    to the single-rank RHS."""
    need_gpu()
    cfg = configs.small_bbh(lmax=6, rho=0.5)
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords())
    ref = dgr.Mesh(cfg)
    rfull = ref.rhs(to_dev(u, ref.dof_stride))[:, :om.n_dof].cpu().numpy()
    for r in range(world):
        m = dgr.Mesh(cfg, rank=r, nranks=world)
        no_oct, ni = m.info["n_oct_local"], m.info["n_oct_interior"]
        order = m.rhs_order()
        assert sorted(order.tolist()) == list(range(no_oct))
        assert 0 < ni < no_oct, (ni, no_oct)
        gid = m.export(dgr.MAP_DOF_GID, np.int64)
        n_own = m.info["n_dof_owned"]
        st = torch.full((NF, m.dof_stride), float("nan"), dtype=torch.float64, device="cuda")
        st[:, :n_own] = torch.from_numpy(u[:, gid[:n_own]])
        m.set_phases(2)
        got = m.rhs(st)[:, :n_own].cpu().numpy()
        # zip owner (global leaf) of each owned DOF -> local octant id
        g2l = {g: l for l, g in enumerate(m.export(dgr.MAP_LOCAL_OCTS, np.int32).tolist())}
        owner = np.array([g2l[g] for g in m.export(dgr.MAP_ZIP, np.int32).reshape(-1, 2)[:, 0]])
        sel = np.isin(owner, order[:ni])
        assert sel.sum() > 0
        assert np.isfinite(got[:, sel]).all(), f"rank {r}: an interior octant read a ghost value"
        assert np.array_equal(got[:, sel], rfull[:, gid[:n_own]][:, sel]), f"rank {r} differs"


# ------------------------------------------------ libdgr's own exchange (group)

def _rank_meshes(cfg, world, u):
    meshes, states, gids = [], [], []
    for r in range(world):
        m = dgr.Mesh(cfg, rank=r, nranks=world)
        gid = m.export(dgr.MAP_DOF_GID, np.int64)
        st = torch.zeros((NF, m.dof_stride), dtype=torch.float64, device="cuda")
        st[:, :m.info["n_dof_owned"]] = torch.from_numpy(u[:, gid[:m.info["n_dof_owned"]]])
        meshes.append(m)
        states.append(st)
        gids.append(gid)
    return meshes, states, gids


@pytest.mark.parametrize("world", [2, 3])
def test_group_exchange_pack_and_ghosts(world):
    """libdgr's exchange code path (k_pack -> peer copies -> k_unpack, the
    buffers and offsets the NCCL transport uses): the packed send buffer equals
    u[f][DGR_MAP_SEND] laid out peer-major ([24][n_p] per peer), and after the
    exchange every ghost DOF holds its owner's value (DGR_MAP_DOF_GID)."""
    need_gpu()
    cfg = configs.small_bbh(lmax=6, rho=0.5)
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords(), kind="random", seed=4)
    meshes, states, gids = _rank_meshes(cfg, world, u)
    g = dgr.Group(meshes)
    g.ghost_exchange(states)
    torch.cuda.synchronize()
    for r, m in enumerate(meshes):
        send = m.export(dgr.MAP_SEND, np.int32)
        sc = m.export(dgr.MAP_SEND_COUNTS, np.int64)
        buf = m.export(dgr.MAP_SENDBUF, np.float64)
        host = states[r].cpu().numpy()
        want, off = [], 0
        for p in range(world):
            ids = send[off:off + sc[p]]
            off += sc[p]
            want.append(host[:, ids].reshape(-1))      # [24][n_p] block
        want = np.concatenate(want) if want else np.zeros(0)
        assert np.array_equal(buf, want), f"rank {r}: packed send buffer"
        no, nd = m.info["n_dof_owned"], m.n_dof
        assert np.array_equal(host[:, no:nd], u[:, gids[r][no:nd]]), f"rank {r}: ghosts"
    g.close()


@pytest.mark.parametrize("world", [2, 4])
def test_group_rk4_bit_identical(world):
    """dgr_group_rk4_step (libdgr's exchange, overlapped with the interior
    octants on the mesh's exchange stream) gives owned DOFs bit-identical to
    the single-rank dgr_rk4_step after RK4 steps."""
    need_gpu()
    cfg = configs.small_bbh(lmax=6, rho=0.5)
    om = OracleMesh(cfg)
    om.build_dofs()
    u = initial.for_config(cfg, om.dof_coords())
    dt = ork4.dt_courant(om)
    ref = dgr.Mesh(cfg)
    ur = to_dev(u, ref.dof_stride)
    meshes, states, gids = _rank_meshes(cfg, world, u)
    assert any(0 < m.info["n_oct_interior"] < m.info["n_oct_local"] for m in meshes)
    g = dgr.Group(meshes)
    side = [torch.cuda.Stream() for _ in range(world)]   # one stream per rank
    for _ in range(2):
        ref.rk4_step(ur, dt)
        g.rk4_step(states, dt, streams=[s.cuda_stream for s in side])
    torch.cuda.synchronize()
    full = ur[:, :om.n_dof].cpu().numpy()
    for r, m in enumerate(meshes):
        no = m.info["n_dof_owned"]
        assert np.array_equal(states[r][:, :no].cpu().numpy(), full[:, gids[r][:no]]), r
    g.close()


def test_step_without_communicator_is_rejected():
    """on an external-exchange mesh dgr_rk4_step / dgr_rk4_step_host
    would read stale ghosts, so they return DGR_ERR_STATE (-6)."""
    need_gpu()
    cfg = configs.small_bbh(lmax=6, rho=0.5)
    m = dgr.Mesh(cfg, rank=0, nranks=2)
    st = m.new_state()
    with pytest.raises(dgr.DgrError) as e:
        m.rk4_step(st, 0.01)
    assert e.value.status == -6
    h = torch.zeros((NF, m.dof_stride), dtype=torch.float64)
    with pytest.raises(dgr.DgrError) as e:
        m.rk4_step_host([h], [h], 0.01)
    assert e.value.status == -6
    with pytest.raises(dgr.DgrError) as e:
        m.ghost_exchange(st)
    assert e.value.status == -6


def test_device_calls_validate_tensors():
    need_gpu()
    m = dgr.Mesh(configs.c1_uniform())
    with pytest.raises(ValueError):
        m.rhs(torch.zeros((NF, m.dof_stride), dtype=torch.float32, device="cuda"))
    with pytest.raises(ValueError):
        m.rhs(torch.zeros((NF, m.dof_stride), dtype=torch.float64))          # CPU
    with pytest.raises(ValueError):
        m.rk4_step(torch.zeros((NF, m.dof_stride - 32), dtype=torch.float64, device="cuda"), 0.1)
