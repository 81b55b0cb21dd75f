"""Multi-rank host logic on CPU (gloo, world size 2 and 3).

libdgr partitions the Morton-ordered leaves into contiguous ranges (P:L168
SFC partitioning), adds ghost octants (leaves touching owned ones, closed under
hanging sources), assigns each DOF to the rank owning its zip owner, and
builds per-peer send lists and receive counts.  Each rank
here builds its host-only mesh, exchanges its owned DOF values with gloo
following exactly those lists (the same peer-major [field][dof] blocks the
NCCL path sends), and checks that every local DOF (owned + ghost) then holds
the global value — i.e. each rank has everything its octant-to-patch needs.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import paper_conf_sc_fernandonhzsgb22_b200 as dgr
from synth import configs

NF = 24


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cfg(name):
    return {"small_bbh": lambda: configs.small_bbh(lmax=6, rho=0.5),
            "c1": configs.c1_uniform,
            "c2": configs.c2_schwarzschild}[name]()


def _worker(rank, world, port, name, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        cfg = _cfg(name)
        glob = dgr.Mesh(cfg, device=False)
        n_glob = glob.info["n_dof_global"]
        o2n_glob = glob.export(dgr.MAP_O2N, np.int32).reshape(-1, 343)
        rng = np.random.default_rng(42)
        u_glob = rng.standard_normal((NF, n_glob))

        m = dgr.Mesh(cfg, device=False, rank=rank, nranks=world)
        info = m.info
        no, ng = info["n_dof_owned"], info["n_dof_ghost"]
        gid = m.export(dgr.MAP_DOF_GID, np.int64)
        send = m.export(dgr.MAP_SEND, np.int32)
        scount = m.export(dgr.MAP_SEND_COUNTS, np.int64)
        rcount = m.export(dgr.MAP_RECV_COUNTS, np.int64)
        local_octs = m.export(dgr.MAP_LOCAL_OCTS, np.int32)
        o2n_loc = m.export(dgr.MAP_O2N_LOCAL, np.int32).reshape(-1, 343)
        zipm = m.export(dgr.MAP_ZIP, np.int32).reshape(-1, 2)
        assert len(gid) == no + ng and scount[rank] == 0 and rcount[rank] == 0
        assert int(rcount.sum()) == ng
        ob = info["oct_begin"]
        owned = np.arange(ob, ob + info["n_oct_local"])
        assert np.array_equal(local_octs[:len(owned)], owned)
        # owned DOFs have owned zip owners
        assert np.all((zipm[:, 0] >= ob) & (zipm[:, 0] < ob + len(owned)))
        # local O2N is the global O2N renumbered
        g = o2n_glob[local_octs]
        assert np.array_equal(np.where(o2n_loc >= 0, gid[np.maximum(o2n_loc, 0)], -1), g)

        # state: owned values set, ghosts poisoned
        u = np.full((NF, no + ng), np.nan)
        u[:, :no] = u_glob[:, gid[:no]]
        # pack peer-major [peer][field][n_peer]
        blocks, off = [], 0
        for peer in range(world):
            ids = send[off:off + scount[peer]]
            off += scount[peer]
            blocks.append(u[:, ids].reshape(-1))
        sbuf = torch.from_numpy(np.concatenate(blocks) if blocks else np.zeros(0))
        rbuf = torch.empty(int(rcount.sum()) * NF, dtype=torch.float64)
        dist.all_to_all_single(rbuf, sbuf, output_split_sizes=[int(c) * NF for c in rcount],
                               input_split_sizes=[int(c) * NF for c in scount])
        r = rbuf.numpy()
        off, goff = 0, no
        for peer in range(world):
            n = int(rcount[peer])
            u[:, goff:goff + n] = r[off:off + n * NF].reshape(NF, n)
            off += n * NF
            goff += n
        assert np.array_equal(u, u_glob[:, gid]), "ghost exchange incomplete"
        # owned DOF sets partition the global DOFs
        owned_ids = torch.from_numpy(np.bincount(gid[:no], minlength=n_glob).astype(np.int64))
        dist.all_reduce(owned_ids)
        assert torch.all(owned_ids == 1)
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, "ok", info["n_oct_ghost"], ng))
    except Exception as ex:  # noqa: BLE001
        import traceback
        q.put((rank, "fail: " + repr(ex) + traceback.format_exc(), 0, 0))


@pytest.mark.parametrize("world,name", [(2, "small_bbh"), (3, "small_bbh"), (2, "c1"),
                                        (2, "c2")])
def test_partition_and_exchange_gloo(world, name):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for r, status, nghost_oct, nghost_dof in res:
        assert status == "ok", status
        assert nghost_oct > 0 and nghost_dof > 0
