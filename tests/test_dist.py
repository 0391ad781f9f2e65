"""Multi-GPU partition logic (dist.py) with the gloo backend, world size 2, on CPU.

The local per-rank kernels need a GPU, so the tests inject the CPU oracle as the
local computation (``local_fn``) and a uint32 sum as the int32 merge
(``merge_fn``); what is under test is the partitioning, the collectives and the
reassembly.  The NCCL path itself runs in bench.py under torchrun on GPUs.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_pldi_samadihmlm12_b200.dist import (combine_splitk, mv_rowshard, shard_range,
                                                    tmv_splitk, dot_splitk)


def test_shard_range_partitions():
    for n in (0, 1, 7, 8, 1000, 131072):
        for world in (1, 2, 3, 4, 8):
            parts = [shard_range(n, world, r) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            for (a, b), (c, d) in zip(parts, parts[1:]):
                assert b == c
            sizes = [b - a for a, b in parts]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        shard_range(10, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    res = {}
    err = None
    try:
        # ---- row shard (BJ:configs[3] in miniature): no collective unless gather
        R, C = 37, 53
        r0, r1 = shard_range(R, world, rank)
        A_loc = synth.matrix(R, C, "mv", np.float32, "uniform", 3, rows=(r0, r1))
        x = synth.vector(C, np.float32, "uniform", 4)
        loc = lambda A, xx: torch.from_numpy(oracle.mv(A.numpy(), xx.numpy())[0].astype(np.float32))
        y = mv_rowshard(torch.from_numpy(A_loc), torch.from_numpy(x), gather=True, local_fn=loc)
        res["rowshard"] = y.numpy()
        # ---- split-K fp32 (BJ:configs[4] in miniature): all_reduce(SUM)
        R2, C2 = 16, 1001
        c0, c1 = shard_range(C2, world, rank)
        B_loc = synth.matrix(R2, C2, "tmv", np.float32, "uniform", 5, cols=(c0, c1))
        x2 = synth.vector(C2, np.float32, "uniform", 6)
        loct = lambda B, xx: torch.from_numpy(oracle.tmv(B.numpy(), xx.numpy())[0].astype(np.float32))
        y2 = tmv_splitk(torch.from_numpy(B_loc), torch.from_numpy(x2[c0:c1]), local_fn=loct)
        res["splitk_f32"] = y2.numpy()
        # ---- split-K int32: all_gather + fixed-order uint32 merge (bit-exact)
        Bi = synth.matrix(R2, C2, "tmv", np.int32, "uniform", 7, cols=(c0, c1))
        xi = synth.vector(C2, np.int32, "uniform", 8)
        loci = lambda B, xx: torch.from_numpy(oracle.tmv(B.numpy(), xx.numpy()))
        merge = lambda P: torch.from_numpy(P.numpy().astype(np.uint32).sum(axis=0, dtype=np.uint32).astype(np.int32))
        y3 = tmv_splitk(torch.from_numpy(Bi), torch.from_numpy(xi[c0:c1]), local_fn=loci, merge_fn=merge)
        res["splitk_i32"] = y3.numpy()
        # ---- Sdot with N = 1 < world: split L
        L = 5000
        e0, e1 = shard_range(L, world, rank)
        a = synth.matrix(1, L, "mv", np.float32, "uniform", 9, cols=(e0, e1))
        b = synth.matrix(1, L, "mv", np.float32, "uniform", 10, cols=(e0, e1))
        locd = lambda p, q: torch.from_numpy(oracle.dot(p.numpy(), q.numpy())[0].astype(np.float32))
        res["dot"] = dot_splitk(torch.from_numpy(a), torch.from_numpy(b), local_fn=locd).numpy()
        # ---- combine_splitk rejects other dtypes
        try:
            combine_splitk(torch.zeros(3, dtype=torch.float64))
            res["dtype_error"] = False
        except TypeError:
            res["dtype_error"] = True
    except Exception as e:  # report instead of hanging the parent on q.get
        err = f"{type(e).__name__}: {e}"
    finally:
        dist.destroy_process_group()
    out_q.put((rank, res if err is None else {"error": err}))


def test_gloo_world2_partitions_and_collectives():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(world):
        assert "error" not in results[r], results[r]
    R, C = 37, 53
    A = synth.matrix(R, C, "mv", np.float32, "uniform", 3)
    x = synth.vector(C, np.float32, "uniform", 4)
    full = oracle.mv(A, x)[0].astype(np.float32)
    for r in range(world):
        assert np.array_equal(results[r]["rowshard"], full)          # P10: shards concatenate
    R2, C2 = 16, 1001
    B = synth.matrix(R2, C2, "tmv", np.float32, "uniform", 5)
    yref, S = oracle.tmv(B, synth.vector(C2, np.float32, "uniform", 6))
    for r in range(world):
        assert np.all(np.abs(results[r]["splitk_f32"] - yref) <= 1e-4 * S)   # P9 additivity
    Bi = synth.matrix(R2, C2, "tmv", np.int32, "uniform", 7)
    yi = oracle.tmv(Bi, synth.vector(C2, np.int32, "uniform", 8))
    for r in range(world):
        assert np.array_equal(results[r]["splitk_i32"], yi)
    a = synth.matrix(1, 5000, "mv", np.float32, "uniform", 9)
    b = synth.matrix(1, 5000, "mv", np.float32, "uniform", 10)
    yd, Sd = oracle.dot(a, b)
    for r in range(world):
        assert np.all(np.abs(results[r]["dot"] - yd) <= 1e-4 * Sd)
        assert results[r]["dtype_error"]


def test_partition_rule_is_rows_or_splitk():
    """Row blocks when every rank gets >= ROW_MIN outputs (no collective), else the
    reduction is split (P:480's merge across GPUs); the shares tile the problem."""
    from paper_conf_pldi_samadihmlm12_b200.dist import ROW_MIN, partition
    assert partition(8192, 8192, 8, 3)[0] == "rows"
    assert partition(1024, 1 << 24, 8, 3) == ("splitk", (0, 1024), (3 << 21, 4 << 21))
    assert partition(131072, 32768, 8, 7) == ("rows", (7 * 16384, 8 * 16384), (0, 32768))
    assert partition(5, 7, 1, 0) == ("rows", (0, 5), (0, 7))
    for R, C in [(8, 1 << 23), (1 << 23, 8), (4096, 16384), (2048, 32768), (1000, 1001)]:
        for G in (2, 3, 4, 8):
            kinds = {partition(R, C, G, g)[0] for g in range(G)}
            assert len(kinds) == 1
            kind = kinds.pop()
            assert kind == ("rows" if R >= G * ROW_MIN else "splitk")
            covered = sum((r1 - r0) * (c1 - c0) for _, (r0, r1), (c0, c1) in
                          (partition(R, C, G, g) for g in range(G)))
            assert covered == R * C
    with pytest.raises(ValueError):
        partition(4, 4, 2, 2)
