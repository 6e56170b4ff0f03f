"""Multi-GPU path over NCCL on real GPUs (reading R15).

The ranks are real processes with one GPU each, joined by NCCL (torch.distributed.run).  World
size 1 still runs every collective (exchange=True / --collectives), so the NCCL path executes
on a one-GPU box; world size 2 needs two GPUs and is skipped otherwise.  Expected values come
from the oracle over the concatenation of every rank's arrays in rank order.
"""
import json
import os
import subprocess
import sys

import numpy as np
import pytest
import torch

import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHUNK, EPS = 4096, 1e-6

pytestmark = pytest.mark.gpu


def _free_port():
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def _torchrun(n, args, timeout=900):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), *args]
    env = dict(os.environ, NCCL_DEBUG="INFO", NCCL_DEBUG_SUBSYS="INIT", NCCL_DEBUG_FILE="/dev/stderr")
    return subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=timeout)


@pytest.mark.parametrize("world", [1, 2])
def test_nccl_compare_runs_and_sharded_array_match_oracle(world, tmp_path):
    if torch.cuda.device_count() < world:
        pytest.skip(f"needs {world} GPUs (one NCCL rank per GPU)")
    r = _torchrun(world, [os.path.join(ROOT, "tests", "nccl_worker.py"), str(tmp_path)])
    assert r.returncode == 0, r.stderr[-4000:]
    assert "NCCL INFO" in r.stderr, "no NCCL communicator was created"
    ranks = [np.load(tmp_path / f"rank{k}.npz") for k in range(world)]
    assert all(int(z["world"]) == world for z in ranks)

    # per-rank checkpoints: the box is the concatenation of every rank's arrays in rank order
    a_list = [x for z in ranks for x in z["a"]]
    b_list = [x for z in ranks for x in z["b"]]
    A = oracle.build_checkpoint(a_list, CHUNK, EPS)
    B = oracle.build_checkpoint(b_list, CHUNK, EPS)
    ref_chunks = oracle.diff_checkpoint(A, B)
    ref_idx = oracle.verify_checkpoint(a_list, b_list, CHUNK, ref_chunks, EPS, A)
    assert np.array_equal(ref_idx, oracle.brute_checkpoint(a_list, b_list, EPS))
    got_chunks = np.concatenate([z["chunks"] for z in ranks])
    got_idx = np.concatenate([z["idx"] for z in ranks])
    assert np.array_equal(got_chunks, ref_chunks)
    assert np.array_equal(got_idx, ref_idx)
    for z in ranks:   # every rank holds the same box roots and global counts after C1/C2
        assert z["root_a"].tobytes() == A.root and z["root_b"].tobytes() == B.root
        assert z["counts"].tolist() == [ref_chunks.size, ref_idx.size]

    # one array sharded over the ranks: same root and ids as one GPU on the whole array
    big_a, big_b = ranks[0]["big_a"], ranks[0]["big_b"]
    la, lb = oracle.leaves(big_a, CHUNK, EPS), oracle.leaves(big_b, CHUNK, EPS)
    na, nb = oracle.levels(la), oracle.levels(lb)
    sc = oracle.diff(na, nb, la.shape[0])
    si = oracle.verify(big_a, big_b, CHUNK, sc, EPS)
    assert np.array_equal(np.concatenate([z["sh_chunks"] for z in ranks]), sc)
    assert np.array_equal(np.concatenate([z["sh_idx"] for z in ranks]), si)
    for z in ranks:
        assert z["sh_root_a"].tobytes() == na[-1].tobytes()
        assert z["sh_root_b"].tobytes() == nb[-1].tobytes()
        assert z["sh_counts"].tolist() == [sc.size, si.size]


@pytest.mark.parametrize("world", [1, 2])
def test_bench_runs_n_nccl_ranks(world):
    """bench.py --gpus N under a launcher: N NCCL ranks, the per-step all-gather, one JSON line."""
    if torch.cuda.device_count() < world:
        pytest.skip(f"needs {world} GPUs")
    args = [os.path.join(ROOT, "bench.py"), "--gpus", str(world), "--steps", "3", "--warmup", "3",
            "--no-e2e", "--no-cpu", "--elems", str(1 << 20), "--collectives"]
    r = _torchrun(world, args)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1 and lines[0].startswith("{"), r.stdout    # stdout = the JSON line only
    line = json.loads(lines[0])
    assert line["n_gpus"] == world
    assert line["dist"]["backend"] == "nccl" and line["dist"]["world"] == world
    assert line["value"] > 0 and line["gpu_launches"] > 0
    assert "NCCL INFO" in r.stderr


def test_bench_two_gloo_ranks_on_one_gpu():
    """The N > 1 bench step's logic with two ranks sharing the GPU over gloo (a functional test:
    timings are meaningless): the exchange of step i runs on its own stream beside step i+1, and
    bench.py asserts that the exchanged global counts equal an all-reduce of the local ones."""
    args = [os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "4", "--warmup", "3",
            "--no-e2e", "--no-cpu", "--elems", str(1 << 20)]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), *args]
    env = dict(os.environ, CKPT_DIST_BACKEND="gloo")
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1, r.stdout
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2 and line["dist"]["backend"] == "gloo" and line["value"] > 0


def test_bench_json_contract():
    """python bench.py at N = 1 (reduced size): stdout is exactly one JSON line carrying every key
    of the bench contract -- metric/value/unit, roofline (bound, achieved, peak, frac, traffic),
    cpu_baseline (the oracle at all cores and one thread), e2e with its copied bytes, clocks and
    the launch count -- with self-consistent numbers."""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "3", "--warmup", "3",
                        "--elems", str(1 << 20)], cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e",
              "clocks", "gpu_launches"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] >= 3 and d["higher_is_better"] is True
    cfg = d["config"]
    # value = pair bytes per step / step time
    assert abs(d["value"] - cfg["bytes_per_step_per_gpu"] / (d["ms_per_step"] / 1e3) / 1e9) < 0.01 * d["value"]
    rf = d["roofline"]
    assert rf["bound"] == "hbm" and rf["unit"] == "GB/s" and rf["peak"] > 0
    assert abs(rf["frac"] - rf["achieved"] / rf["peak"]) < 1e-3
    cpu = d["cpu_baseline"]
    assert cpu["kind"] == "oracle" and cpu["cores"] >= 1 and cpu["value"] > 0
    assert cpu["single_thread"]["cores"] == 1
    e2e = d["e2e"]
    assert e2e["value"] > 0 and e2e["h2d_bytes_per_step"] == cfg["bytes_per_step_per_gpu"]
    assert e2e["d2h_bytes_per_step"] > 0
    assert {"sm_mhz", "sm_max_mhz", "reasons"} <= set(d["clocks"])
    assert d["gpu_launches"] >= 3 * d["steps"]


def test_bench_spawns_ranks_itself_when_not_launched():
    """python bench.py --gpus N (no launcher) re-executes itself as N ranks."""
    n = torch.cuda.device_count()
    if n < 2:
        pytest.skip("needs 2 GPUs")
    env = {k: v for k, v in os.environ.items()
           if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3",
                        "--warmup", "3", "--no-e2e", "--no-cpu", "--elems", str(1 << 20)],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2 and line["dist"]["backend"] == "nccl"
