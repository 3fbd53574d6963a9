"""World-size-2 coverage of the multi-GPU (1-D block-row) path on CPU with gloo.

The CUDA kernels need a GPU, so these tests cover the host side of the N>1 path:
 * the C ABI's host-only partition (apsp_partition) gives every rank a disjoint block
   of rows whose union is [0, n), agreed on by all ranks;
 * the NCCL unique id is produced on rank 0 by the C ABI and reaches every rank
   through torch.distributed (the rendezvous bench.py uses);
 * the round schedule the library runs (owner of band k: phase 1 + row panel;
   broadcast of the b x n_pad band; every rank: its column-panel tiles, then its
   phase-3 tiles) reproduces the oracle when its steps are carried out here in
   numpy over two gloo ranks — a check of the decomposition itself (which rows a
   rank owns, which band it receives, which tiles it skips), not of the kernels.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen as gg
import oracle

B = 128
BIG = 1 << 40  # "infinity" for the numpy emulation (int64)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def minplus(C, A, Bm):
    """min(C, A (x) B) with A: r x K, B: K x c (int64, BIG-saturated)."""
    out = C.copy()
    for kk in range(A.shape[1]):
        out = np.minimum(out, A[:, kk:kk + 1] + Bm[kk:kk + 1, :])
    return np.minimum(out, BIG)


def closure(T):
    T = T.copy()
    for kk in range(T.shape[0]):
        T = np.minimum(T, T[:, kk:kk + 1] + T[kk:kk + 1, :])
    return np.minimum(T, BIG)


def _worker(rank, world, port, n, seed, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_xia0ar22_b200 as lib
        # ---- partition agreed on by every rank --------------------------------
        n_pad, rb, rc = lib.apsp_partition(n, world, rank)
        parts = [None] * world
        dist.all_gather_object(parts, (n_pad, rb, rc))
        # ---- NCCL id rendezvous (bench.py's path) ------------------------------
        obj = [lib.apsp_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid_ok = isinstance(obj[0], bytes) and len(obj[0]) == 128
        # ---- the sharded round schedule, steps done in numpy ------------------
        g = gg.grid_2d(12, n // 12, seed=seed) if seed % 2 == 0 else gg.erdos_renyi(n, 4 * n, seed=seed)
        full = oracle.init_i64(g.row_ptr, g.col, g.w)
        full = np.where(full == oracle.INF_I64, BIG, full)
        Dp = np.full((n_pad, n_pad), BIG, dtype=np.int64)
        np.fill_diagonal(Dp, 0)
        Dp[:n, :n] = full
        R = n_pad // world
        r0 = rank * R
        D = Dp[r0:r0 + R].copy()  # this rank's rows only
        nb = n_pad // B
        for k in range(nb):
            owner = (k * B) // R
            band = np.empty((B, n_pad), dtype=np.int64)
            if rank == owner:
                lk = k * B - r0
                D[lk:lk + B, k * B:(k + 1) * B] = closure(D[lk:lk + B, k * B:(k + 1) * B])
                dkk = D[lk:lk + B, k * B:(k + 1) * B]
                for j in range(nb):
                    if j != k:
                        blk = D[lk:lk + B, j * B:(j + 1) * B]
                        D[lk:lk + B, j * B:(j + 1) * B] = minplus(blk, dkk, blk)
                band[:] = D[lk:lk + B]
            t = torch.from_numpy(band)
            dist.broadcast(t, src=owner)
            band = t.numpy()
            dkk = band[:, k * B:(k + 1) * B]
            for i in range(R // B):
                gi = (r0 // B) + i
                if gi == k:
                    continue
                rows = slice(i * B, (i + 1) * B)
                aik = D[rows, k * B:(k + 1) * B]
                D[rows, k * B:(k + 1) * B] = minplus(aik, aik, dkk)
            for i in range(R // B):
                gi = (r0 // B) + i
                if gi == k:
                    continue
                rows = slice(i * B, (i + 1) * B)
                aik = D[rows, k * B:(k + 1) * B]
                for j in range(nb):
                    if j != k:
                        D[rows, j * B:(j + 1) * B] = minplus(D[rows, j * B:(j + 1) * B], aik,
                                                             band[:, j * B:(j + 1) * B])
        shards = [None] * world
        dist.all_gather_object(shards, D)
        if rank == 0:
            got = np.concatenate(shards)[:n, :n]
            want, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
            want = np.where(want == oracle.INF_I64, BIG, want)
            q.put((parts, uid_ok, bool(np.array_equal(got, want))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n,seed", [(300, 0), (516, 1), (240, 3)])
def test_block_row_schedule_two_ranks_gloo(n, seed):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, seed, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    assert all(p.exitcode == 0 for p in procs)
    parts, uid_ok, equal = q.get(timeout=10)
    n_pad = parts[0][0]
    assert all(p[0] == n_pad for p in parts) and n_pad % (B * world) == 0
    rows = sorted(r for (_, rb, rc) in parts for r in range(rb, rb + rc))
    assert rows == list(range(n))
    assert uid_ok
    assert equal
