"""Probe torch symmetric memory on this box (world of one, NCCL) and run the
peer-buffer exchange path of dist.join_target_sharded once (C5-shaped, small)."""
import os
import socket
import sys
sys.path.insert(0, os.getcwd())
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402
import datagen  # noqa: E402
import paper_conf_icde_chends17_b200 as sknn  # noqa: E402
from paper_conf_icde_chends17_b200 import dist as sdist  # noqa: E402

s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
try:
    import torch.distributed._symmetric_memory as symm_mem
    b = symm_mem.empty((4,), dtype=torch.float32, device="cuda")
    h = symm_mem.rendezvous(b, dist.group.WORLD)
    h.barrier(channel=0)
    print("symmetric memory ok: buffer_ptrs", len(h.buffer_ptrs))
    Q, T, k, _ = datagen.workload("C5", 0.002)
    dQ, dT = torch.from_numpy(Q).cuda(), torch.from_numpy(T).cuda()
    i, d = sdist._exchange_peer(dQ, dT, k, 0, None, 1, 0, sknn.join, False, True, {})
    ri, rd = sknn.join(dQ, dT, k)
    torch.cuda.synchronize()
    print("peer path equals the join:", bool(torch.equal(i, ri) and torch.equal(d, rd)))
except Exception as e:  # noqa: BLE001
    print("symmetric memory unavailable:", type(e).__name__, str(e)[:300])
finally:
    dist.destroy_process_group()
