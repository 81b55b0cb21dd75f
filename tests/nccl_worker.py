"""Worker of tests/test_gpu_nccl.py (launched by torch.distributed.run, one
rank per GPU): the NCCL path of libdgr — dgr_mesh_create with an ncclUniqueId,
RK4 steps whose stages run the peer-major pack, one grouped ncclSend/ncclRecv
per peer and the unpack, overlapped with the interior octants — against a
single-rank run of the same octree on rank 0.  Exits non-zero on mismatch."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import paper_conf_sc_fernandonhzsgb22_b200 as dgr  # noqa: E402
from synth import configs, initial  # noqa: E402


def main():
    world = int(os.environ["WORLD_SIZE"])
    rank = int(os.environ["RANK"])
    local = int(os.environ.get("LOCAL_RANK", rank))
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    obj = [bytes(torch.cuda.nccl.unique_id()) if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    cfg = configs.small_bbh(lmax=6, rho=0.5)
    octs = dgr.octree_build(cfg)
    ref = dgr.Mesh(cfg, octs)                       # every rank: the one-rank result
    xyz = ref.dof_xyz_host()
    u = initial.for_config(cfg, xyz, kind="bl")
    m = dgr.Mesh(cfg, octs, rank=rank, nranks=world, nccl_id=obj[0])
    gid = m.export(dgr.MAP_DOF_GID, np.int64)
    no = m.info["n_dof_owned"]
    st = m.new_state()
    st[:, :no] = torch.from_numpy(u[:, gid[:no]]).cuda()
    ur = ref.new_state()
    ur[:, :u.shape[1]] = torch.from_numpy(u).cuda()
    dt = 0.25 * ref.info["h_min"]
    for _ in range(3):
        ref.rk4_step(ur, dt)
        m.rk4_step(st, dt)
    # the NCCL exchange alone: ghosts equal their owners' values
    m.ghost_exchange(st)
    _, norms = m.constraints(st)                    # all-reduced norms (NCCL)
    _, rnorms = ref.constraints(ur)
    torch.cuda.synchronize()
    full = ur[:, :ref.n_dof].cpu().numpy()
    got = st[:, :m.n_dof].cpu().numpy()
    ok = np.array_equal(got[:, :no], full[:, gid[:no]])
    ok_g = np.array_equal(got[:, no:], full[:, gid[no:]])
    ok_n = np.allclose(norms[:, 1], rnorms[:, 1], rtol=0, atol=0)
    print(f"rank {rank}: owned bit-identical {ok}, ghosts {ok_g}, max-norms {ok_n}", flush=True)
    flag = torch.tensor([int(ok and ok_g and ok_n)], device="cuda")
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    m.close()
    dist.destroy_process_group()
    sys.exit(0 if flag.item() == 1 else 1)


if __name__ == "__main__":
    main()
