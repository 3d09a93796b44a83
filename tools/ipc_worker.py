"""One rank of a two-process group on ONE GPU using the cross-process fused transport (CUDA IPC
windows + device barrier, no NCCL): used by tests/test_gpu_ipc.py.  Blobs and results travel over
torch.distributed gloo.

  RANK=r WORLD_SIZE=2 MASTER_ADDR=127.0.0.1 MASTER_PORT=p python tools/ipc_worker.py <model> <H> <W> <steps> <out.npz>
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch.distributed as dist

    import paper_conf_asplos_luhtlwm0c26_b200 as tsv
    model, H, W, steps, out = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), sys.argv[5]
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dist.init_process_group("gloo", rank=rank, world_size=world)
    eng = tsv.Engine(model, devices=[0], rank_base=rank, world_size=world)
    g = eng.group_create(list(range(world)))
    blob = eng.group_ipc_export(g, max_tokens=(H // 16) * (W // 16) + 512, max_evals=2)
    blobs = [None] * world
    dist.all_gather_object(blobs, blob)
    eng.group_ipc_import(g, blobs)
    req = eng.request_create(H, W, num_steps=steps + 1, seed=1600)
    for s in range(steps):
        eng.request_step(req, s, g)
    Li = (H // 16) * (W // 16)
    r0, r1 = tsv.shard_range(Li, world, rank)
    lat = eng.read_latent(req, r0, r1 - r0)
    vel = eng.read_velocity(req, r0, r1 - r0)
    parts = [None] * world
    dist.all_gather_object(parts, (lat, vel))
    if rank == 0:
        np.savez(out, x=np.concatenate([p[0] for p in parts]), v=np.concatenate([p[1] for p in parts]))
    dist.barrier()
    eng.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
