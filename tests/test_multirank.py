"""N>1 path on CPU: world_size-2 gloo process group.

Each rank takes its diagonal band from the C-ABI host scheduler (mp_plan_diagonals), builds
the partial profile of that band as merge keys (test-side brute force, the key format of
include/mp.h), and the ranks merge them with the product's MINLOC protocol
(mstamp.merge_partials) over gloo.  The merged profile must equal the FP64 oracle's -- i.e.
the bands cover every admissible diagonal exactly once and the exchange step is exact,
including the lowest-index tie rule.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import brute


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _band_keys(T, m, e, self_join, lo, hi, prec, Tr=None):
    """Partial keys of diagonals [lo, hi): FP32 -> int64 (float bits << 32 | j) over the SUM;
    FP64 -> two int64 planes (double bits of the SUM, index).  Layout [pos][rank]."""
    D = brute.dist_cube(T, m, Tr)   # d x n x n, D[k, i, j]
    d, n, _ = D.shape
    big = np.iinfo(np.int64).max
    if prec == "fp32":
        keys = np.full((n, d), (0x7F800000 << 32) | 0x7FFFFFFF, dtype=np.int64)
    else:
        kv = np.full((n, d), 0x7FF0000000000000, dtype=np.int64)
        ki = np.full((n, d), big, dtype=np.int64)

    def put(pos, other, S):
        for k in range(d):
            if prec == "fp32":
                v = np.float32(S[k]).view(np.uint32).astype(np.int64)
                key = (v << 32) | other
                if key < keys[pos, k]:
                    keys[pos, k] = key
            else:
                v = np.float64(S[k]).view(np.int64)
                if v < kv[pos, k] or (v == kv[pos, k] and other < ki[pos, k]):
                    kv[pos, k], ki[pos, k] = v, other

    for delta in range(lo, hi):
        for i in range(n):
            j = i + delta
            if j < 0 or j >= n:
                continue
            S = np.cumsum(np.sort(D[:, i, j]))
            put(i, j, S)
            if self_join:
                put(j, i, S)
    if prec == "fp32":
        return keys.reshape(-1)
    return np.concatenate([kv.reshape(-1), ki.reshape(-1)])


def _decode(keys, d, n, prec):
    P = np.full((d, n), np.inf)
    I = np.full((d, n), -1, dtype=np.int64)
    cnt = d * n
    for pos in range(n):
        for k in range(d):
            if prec == "fp32":
                key = int(keys[pos * d + k])
                if key >= (0x7F800000 << 32):
                    continue
                P[k, pos] = float(np.uint32(key >> 32).view(np.float32)) / (k + 1)
                I[k, pos] = key & 0xFFFFFFFF
            else:
                v, ix = int(keys[pos * d + k]), int(keys[cnt + pos * d + k])
                if v >= 0x7FF0000000000000 or ix == np.iinfo(np.int64).max:
                    continue
                P[k, pos] = float(np.int64(v).view(np.float64)) / (k + 1)
                I[k, pos] = ix
    return P, I


def _worker(rank, world, port, prec, self_join, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_juryl022_b200 import datagen, mstamp
    d, n, m = 3, 70, 8
    if self_join:
        T, Tr, e = datagen.random_walk(d, n, m, 41), None, 2
        T[:, 30:38] = T[:, 10:18]          # an exact repeat: ties in the index rule
    else:
        (T, Tr), e = datagen.random_walk_ab(d, n, m, 42), 0
    db = mstamp.plan_diagonals(d, n, m, prec, e, self_join, world)
    keys = torch.from_numpy(_band_keys(T, m, e, self_join, int(db[rank]), int(db[rank + 1]), prec, Tr))

    def cpu_mask(k, gv):   # the mp_key_mask_device step, for CPU tensors in this protocol test
        cnt = d * n
        k[cnt:] = torch.where(k[:cnt] != gv, torch.full_like(gv, torch.iinfo(torch.int64).max), k[cnt:])

    mstamp.merge_partials(None, keys, d, n, prec, mask=cpu_mask)
    if rank == 0:
        out.put((T, Tr, e, keys.numpy().copy(), db))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("prec", ["fp32", "fp64"])
@pytest.mark.parametrize("self_join", [True, False])
def test_two_rank_band_merge(oracle_mod, prec, self_join):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, prec, self_join, q)) for r in range(world)]
    for p in procs:
        p.start()
    T, Tr, e, keys, db = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    d, L = T.shape
    m = 8
    n = L - m + 1
    assert db[0] < db[1] < db[2]
    P, I = _decode(keys, d, n, prec)
    Po, Io, P2o = oracle_mod.mstamp(T, m, e, Tr=Tr)
    tol = 1e-5 if prec == "fp32" else 1e-12
    assert np.allclose(P, Po, rtol=tol, atol=1e-5)
    strict = (P2o - Po) > 1e-4
    assert np.array_equal(I[strict], Io[strict])
