"""Probe: gsw's own NCCL communicator next to a torch NCCL process group (bench.py's sequence)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ppopp_menglts19_b200 as gsw  # noqa: E402

mode = sys.argv[1] if len(sys.argv) > 1 else "device_id"
os.environ.update(RANK="0", WORLD_SIZE="1", LOCAL_RANK="0", MASTER_ADDR="127.0.0.1", MASTER_PORT="29631")
dev = torch.device("cuda", 0)
torch.cuda.set_device(0)
if mode == "device_id":
    dist.init_process_group("nccl", device_id=dev)
elif mode == "plain":
    dist.init_process_group("nccl")
elif mode == "gloo":
    dist.init_process_group("gloo")
g = gen.rmat(12, seed=1)
uid = gsw.dist_unique_id()
obj = [uid]
if mode != "none":
    dist.broadcast_object_list(obj, src=0)
time.sleep(float(sys.argv[2]) if len(sys.argv) > 2 else 0.0)
off, col = gsw.owned_rows(g.off, g.col, 0, 1)
try:
    D = gsw.DistGraph(off, col, g.n, obj[0], 1, 0)
    s = gen.sources(g, 1)[0]
    d, _ = D.bfs(s)
    print(mode, "ok", np.array_equal(d.cpu().numpy(), oracle.bfs(g, s)), flush=True)
except Exception as e:  # noqa: BLE001
    print(mode, "FAILED", e, flush=True)
