"""The multi-GPU data path of dist.py on the GPU, with the REAL per-rank kernels and
merges (no local_fn / merge_fn hooks) -- SURVEY 8(a) a6, 8(d) configs[3-4], 8(e).

One B200 is available per test box, so the ranks share cuda:0:
* gloo on CUDA tensors, world 2 and world 3 (the collectives stage through the host,
  the per-rank kernels and the int32 merge kernel are the library's);
* NCCL, world 1 (NCCL refuses two ranks on one GPU), which runs the same all_reduce /
  all_gather_into_tensor calls through NCCL itself.

Every rank generates its own share of the logical inputs on the device from the
global index (synth, no arithmetic of the method); the parent compares what every
rank returns with the oracle on the full problem: fp32 within 1e-4 * S_r, int32 and
integer-valued fp32 (P5 'smallint') bit-exact, for every shard count (P9, P10).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import oracle
import synth

pytestmark = pytest.mark.gpu

NP = {"f32": np.float32, "i32": np.int32}
TD = {"f32": torch.float32, "i32": torch.int32}

# (name, op, R, C, dtype, kind, entry): entry = how the rank computes its share
CASES = [
    ("rows_mv_f32", "mv", 2 * 1024 + 37, 333, "f32", "uniform", "rowshard"),
    ("rows_tmv_f32", "tmv", 3 * 1024 + 5, 129, "f32", "uniform", "rowshard"),
    ("rows_mv_i32", "mv", 4099, 77, "i32", "uniform", "rowshard"),
    ("rows_mv_p5", "mv", 3000, 4097, "f32", "smallint", "rowshard"),
    ("splitk_tmv_f32", "tmv", 1024, 40000, "f32", "uniform", "splitk"),
    ("splitk_tmv_p5", "tmv", 1000, 30001, "f32", "smallint", "splitk"),
    ("splitk_tmv_i32", "tmv", 1024, 50001, "i32", "uniform", "splitk"),
    ("splitk_mv_i32", "mv", 8, 1 << 20, "i32", "uniform", "splitk"),
    ("splitk_mv_f32", "mv", 64, 100003, "f32", "uniform", "splitk"),
    ("splitk_dot_f32", "dot", 1, 1 << 20, "f32", "uniform", "splitk"),
    ("splitk_dot_i32", "dot", 3, 333333, "i32", "uniform", "splitk"),
    ("part_mv_f32", "mv", 16, 65536, "f32", "uniform", "partitioned"),
    ("part_tmv_i32", "tmv", 8192, 512, "i32", "uniform", "partitioned"),
    ("part_tmv_p5", "tmv", 33, 200001, "f32", "smallint", "partitioned"),
]
BUCKET = [("mv", 8, 1 << 18, "uniform"), ("tmv", 100, 30000, "uniform"), ("dot", 2, 100000, "uniform"),
          ("tmv", 1000, 4001, "smallint")]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _local_inputs(op, R, C, dt, kind, rows, cols, seed, dev):
    """This rank's share of the logical problem, generated on the device."""
    (r0, r1), (c0, c1) = rows, cols
    if op == "dot":
        a = torch.empty(r1 - r0, c1 - c0, dtype=TD[dt], device=dev)
        b = torch.empty_like(a)
        synth.device_matrix(a, R, C, "mv", kind, synth.seed(seed, "A"), rows=rows, cols=cols)
        synth.device_matrix(b, R, C, "mv", kind, synth.seed(seed, "b"), rows=rows, cols=cols)
        return a, b
    shape = (r1 - r0, c1 - c0) if op == "mv" else (c1 - c0, r1 - r0)
    M = torch.empty(*shape, dtype=TD[dt], device=dev)
    synth.device_matrix(M, R, C, op, kind, synth.seed(seed, "A"), rows=rows, cols=cols)
    x = torch.empty(c1 - c0, dtype=TD[dt], device=dev)
    synth.device_vector(x, kind, synth.seed(seed, "x"), start=c0)
    return M, x


def _worker(rank, world, port, backend, out_q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    res, err = {}, None
    try:
        if backend == "nccl":
            dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
        else:
            dist.init_process_group("gloo", rank=rank, world_size=world)
        from paper_conf_pldi_samadihmlm12_b200 import dist as ad
        from paper_conf_pldi_samadihmlm12_b200 import _lib as L
        for i, (name, op, R, C, dt, kind, entry) in enumerate(CASES):
            seed = 40 + i
            if entry == "rowshard":
                rows, cols = ad.shard_range(R, world, rank), (0, C)
                M, X = _local_inputs(op, R, C, dt, kind, rows, cols, seed, dev)
                fn = ad.mv_rowshard if op == "mv" else ad.tmv_rowshard
                y = fn(M, X, gather=True)
            elif entry == "splitk":
                rows, cols = (0, R), ad.shard_range(C, world, rank)
                M, X = _local_inputs(op, R, C, dt, kind, rows, cols, seed, dev)
                fn = {"mv": ad.mv_splitk, "tmv": ad.tmv_splitk, "dot": ad.dot_splitk}[op]
                y = fn(M, X)
            else:
                _, rows, cols = ad.partition(R, C, world, rank)
                M, X = _local_inputs(op, R, C, dt, kind, rows, cols, seed, dev)
                y = ad.run_partitioned(op, M, X, R, C)
            res[name] = y.cpu().numpy()
        # a bucket of split-K problems: one collective for all of them (fp32 and int32)
        for dt in ("f32", "i32"):
            probs = [(op, R, C, k) for op, R, C, k in BUCKET if not (dt == "i32" and k == "smallint")]
            bucket = ad.SplitKBucket([R for _, R, _, _ in probs], TD[dt], dev)
            from paper_conf_pldi_samadihmlm12_b200 import ops
            for j, (op, R, C, kind) in enumerate(probs):
                cols = ad.shard_range(C, world, rank)
                M, X = _local_inputs(op, R, C, dt, kind, (0, R), cols, 90 + j, dev)
                {"mv": ops.mv, "tmv": ops.tmv, "dot": ops.dot}[op](M, X, out=bucket.views[j])
            bucket.combine()
            for j, v in enumerate(bucket.views):
                res[f"bucket_{dt}_{j}"] = v.cpu().numpy()
        torch.cuda.synchronize()
        res["_lib"] = L.LIB_PATH
    except Exception as e:  # report instead of hanging the parent on q.get
        import traceback
        err = f"{type(e).__name__}: {e}\n{traceback.format_exc()[-1500:]}"
    finally:
        try:
            dist.destroy_process_group()
        except Exception:
            pass
    out_q.put((rank, res if err is None else {"error": err}))


def _expected(op, R, C, dt, kind, seed):
    if op == "dot":
        a = synth.matrix(R, C, "mv", NP[dt], kind, synth.seed(seed, "A"))
        b = synth.matrix(R, C, "mv", NP[dt], kind, synth.seed(seed, "b"))
        return oracle.dot(a, b)
    M = synth.matrix(R, C, op, NP[dt], kind, synth.seed(seed, "A"))
    x = synth.vector(C, NP[dt], kind, synth.seed(seed, "x"))
    return (oracle.mv if op == "mv" else oracle.tmv)(M, x)


def _check(y, ref, dt, kind, what):
    if dt == "i32":
        assert np.array_equal(y, ref), f"{what}: int32 mismatch at {np.nonzero(y != ref)[0][:8]}"
        return
    yr, S = ref
    if kind == "smallint":                       # P5: every partial sum exact -> bit-exact
        assert np.array_equal(y.astype(np.float64), yr), f"{what}: P5 data not exact"
        return
    bad = ~(np.abs(y.astype(np.float64) - yr) <= 1e-4 * S)
    assert not bad.any(), f"{what}: {bad.sum()} outputs out of tolerance"


def _spawn(world, backend):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, backend, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for r in range(world):
        assert "error" not in results[r], results[r]["error"] if "error" in results[r] else ""
    return results


@pytest.mark.parametrize("world,backend", [(2, "gloo"), (3, "gloo"), (1, "nccl")])
def test_dist_real_kernels_match_oracle(world, backend):
    results = _spawn(world, backend)
    fails = []
    for i, (name, op, R, C, dt, kind, entry) in enumerate(CASES):
        ref = _expected(op, R, C, dt, kind, 40 + i)
        for r in range(world):
            try:
                y = results[r][name]
                assert y.shape == (R,), f"{name}: rank {r} shape {y.shape}"
                _check(y, ref, dt, kind, f"{name} rank {r}/{world}")
            except AssertionError as e:
                fails.append(str(e))
    for dt in ("f32", "i32"):
        probs = [(op, R, C, k) for op, R, C, k in BUCKET if not (dt == "i32" and k == "smallint")]
        for j, (op, R, C, kind) in enumerate(probs):
            ref = _expected(op, R, C, dt, kind, 90 + j)
            for r in range(world):
                try:
                    _check(results[r][f"bucket_{dt}_{j}"], ref, dt, kind, f"bucket {dt} {op} {R}x{C} rank {r}")
                except AssertionError as e:
                    fails.append(str(e))
    assert not fails, "\n".join(fails)



def _bench(*args):
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), *args], capture_output=True, text=True,
                       timeout=900, env=env, cwd=root)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_partitioned_sweep_two_ranks_on_one_gpu():
    """The default workload at N = 2 (both ranks on cuda:0, gloo): every problem sharded by
    dist.partition, split-K partials combined by ONE collective per step."""
    line = _bench("--gpus", "2", "--backend", "gloo", "--share-gpu", "--steps", "3", "--warmup", "3",
                  "--no-e2e", "--no-cpu-baseline")
    assert line["n_gpus"] == 2 and line["scaling"] == "strong"
    assert line["config"]["shares"] == {"rows": 26, "splitk": 16}
    assert line["value"] > 0 and line["split"]["collective_us"] > 0
    assert line["config"]["collective_bytes_per_step"] == 4 * sum(
        R for k in range(3, 24) for R in [1 << k] if R < 2048) * 2


def test_bench_splitk_reports_compute_and_collective():
    line = _bench("--workload", "splitk", "--steps", "3", "--warmup", "3", "--no-e2e", "--no-cpu-baseline")
    assert line["n_gpus"] == 1 and line["split"]["compute_us"] > 0
