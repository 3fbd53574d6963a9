#!/usr/bin/env python
"""Can two NCCL ranks share one GPU? (NCCL normally refuses: "Duplicate GPU detected".) If the
library's world_size=2 NCCL path (broadcast receive on the non-root rank) can run on one GPU,
tests/test_gpu_nccl2.py exercises it. Prints one JSON line per rank."""
import json
import os
import sys

import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def worker(rank, world, port, q):
    import ctypes

    import numpy as np
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import graphgen as gg
    import paper_conf_ipps_xia0ar22_b200 as apsp
    out = {"rank": rank}
    try:
        obj = [apsp.apsp_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        g = gg.erdos_renyi(1000, 5000, seed=3)
        cfg = apsp.apsp_config_default(device=0, world_size=world, rank=rank)
        buf = ctypes.create_string_buffer(obj[0], 128)
        cfg.nccl_unique_id = ctypes.cast(buf, ctypes.c_void_p)
        with apsp.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg) as h:
            apsp.apsp_fw_blocked(h)
            r0, rc = apsp.apsp_local_rows(h)
            d = apsp.apsp_get_dist(h, r0, rc)
        out.update(ok=True, rows=[r0, rc], checksum=int(np.asarray(d, np.int64).sum()))
    except Exception as e:  # noqa: BLE001
        out.update(ok=False, error=str(e)[:300])
    q.put(out)
    dist.destroy_process_group()


if __name__ == "__main__":
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(300)
    while not q.empty():
        print(json.dumps(q.get()))
