#!/usr/bin/env python
"""Checkpoint-pair compare throughput (build + diff + verify) on B200.

Metric (BASELINE.json): checkpoint-pair compare GB/s (build+diff+verify) at
1/2/4/8 B200, % HBM peak.  One step = the whole hot path on one pair of
checkpoints resident in HBM:
    tree_build(run A) + tree_build(run B) + tree_diff + verify
    (+ for N>1: NCCL all-gather of array roots -> top tree, all-reduce of counts)
GB/s = (bytes(A) + bytes(B)) summed over all ranks / step time (max over ranks).

Workload at N=1: BASELINE configs[1] -- HACC-shaped checkpoint, 2^26 particles
x 6 float32 arrays (x,y,z ~ U[0,256), v ~ N(0,300^2)) per GPU, 4 KiB chunks,
eps = 1e-6, 1% of particles perturbed in 64 clusters.  N>1: every rank holds its
own such checkpoint pair (weak scaling, arrays sharded by rank as HACC writes
per-rank checkpoints).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

--gpus N > 1 without a torch.distributed environment re-launches this script
as N ranks (one process per GPU, NCCL) through torch.distributed.run on
127.0.0.1; under an existing launcher (WORLD_SIZE set) the world size must
equal N.  Rank 0 prints the one JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "checkpoint-pair compare GB/s (build+diff+verify) at 1/2/4/8 B200, % HBM peak"
CHUNK = 4096
EPS = 1e-6
SEED = 2

# --config: the bench line is configs[1] (c2) by default; c5 (verify-heavy,
# BASELINE configs[4] per-GPU shard) and c3 (f64) are extra workloads.
CONFIGS = {
    "c2": dict(n=1 << 26, workload="configs[1]: HACC-shaped checkpoint pair, 2^26 particles x 6 "
               "float32 per GPU, 4 KiB chunks, eps=1e-6, 1% particles perturbed in 64 clusters"),
    "c5": dict(n=50 << 20, workload="configs[4] (one GPU's shard): 8 HACC ranks x 50*2^20 "
               "particles x 6 float32, 4 KiB chunks, eps=1e-6, 10% chunks with 8 above-eps + 8 "
               "below-eps changes, 1% chunks below-eps only"),
    "c3": dict(n=1 << 29, workload="configs[2] (C=4 KiB, eps=1e-6 point): 2^29 float64 ~ N(0,1), "
               "1024 geometric clusters (mean 4096) with |d|=10^U(-9,-2)"),
    "c4": dict(n=1 << 24, workload="configs[3]: intermediate snapshots of a 64-rank HACC run (one "
               "snapshot, default s=9, or --snapshots all = the 10-snapshot sequence), 2^30 particles "
               "x 6 float32 per run (2^24 per rank), ranks sharded over the GPUs (strong scaling), "
               "4 KiB chunks, eps=1e-6, clustered divergence 1e-6*4^(s-3)"),
}
SNAPSHOT = 9
C4_RANKS = 64
CFG = "c2"
HASH_BLOCK = 16
JSON_OUT = sys.stdout
N_PARTICLES = CONFIGS[CFG]["n"]
WORKLOAD = CONFIGS[CFG]["workload"]


def make_pair(cfg: str, n: int, seed: int, device: str):
    import synth
    if cfg == "c2":
        return synth.c2_pair(n_particles=n, seed=seed, device=device)
    if cfg == "c5":
        return synth.c5_pair(n_ranks=8 if n == CONFIGS["c5"]["n"] else 1, n_particles=n,
                             seed=seed, device=device)
    if cfg == "c3":
        return synth.c3_pair(n=n, seed=seed, device=device)
    if cfg == "c4":
        # full run: this rank's share of the 64 HACC ranks; oracle samples: one rank of n particles
        world = int(os.environ.get("WORLD_SIZE", "1"))
        rank = int(os.environ.get("RANK", "0"))
        if n == CONFIGS["c4"]["n"] and device != "cpu":
            per = C4_RANKS // world
            ranks = range(rank * per, (rank + 1) * per)
        else:
            ranks = [0]
        return synth.c4_snapshot(SNAPSHOT, ranks, n_particles=n, device=device)
    raise ValueError(cfg)

def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.dev = device_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.dev}", f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.06)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.thread.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


# ---------------------------------------------------------------------------
# oracle (CPU) legs: cpu_baseline and --impl reference
# ---------------------------------------------------------------------------

def oracle_pair_sample(n_particles: int, seed: int):
    pair = make_pair(CFG, n_particles, seed, "cpu")
    return [t.numpy() for t in pair.a], [t.numpy() for t in pair.b]


def oracle_step(a_list, b_list, threads: int):
    """The oracle as it stands: build A, build B, BFS diff, verify (all arrays)."""
    import oracle
    A = oracle.build_checkpoint(a_list, CHUNK, EPS, threads=threads, hash_block=HASH_BLOCK)
    B = oracle.build_checkpoint(b_list, CHUNK, EPS, threads=threads, hash_block=HASH_BLOCK)
    ch = oracle.diff_checkpoint(A, B)
    idx = oracle.verify_checkpoint(a_list, b_list, CHUNK, ch, EPS, A)
    return ch.size, idx.size


def calibrate_oracle(target_s: float, threads: int):
    """Particles per sample so one oracle step takes about target_s seconds."""
    n = 1 << 14
    while True:
        a, b = oracle_pair_sample(n, SEED)
        t0 = time.perf_counter()
        oracle_step(a, b, threads)
        dt = time.perf_counter() - t0
        if dt > 0.3 or n >= N_PARTICLES:
            break
        n *= 4
    scale = target_s / max(dt, 1e-6)
    n = int(min(N_PARTICLES, max(1 << 12, n * scale)))
    n = max(1024, (n // 1024) * 1024)
    return n


def _time_oracle(target_s: float, threads: int):
    n = calibrate_oracle(target_s, threads)
    a, b = oracle_pair_sample(n, SEED)
    t0 = time.perf_counter()
    oracle_step(a, b, threads)
    dt = time.perf_counter() - t0
    nbytes = 2 * sum(x.nbytes for x in a)
    return nbytes / dt / 1e9, (f"same recipe ({CFG}) at {n} elements per array ({nbytes / 1e6:.1f} MB "
                               f"pair), one full step (build A+B, BFS diff, verify) in {dt:.2f} s")


def cpu_baseline(target_s: float = 8.0):
    """The oracle as it stands on the host cores: all cores (value) and one thread."""
    import oracle
    oracle.build()
    threads = host_cores()
    v_all, s_all = _time_oracle(target_s, threads)
    v_one, s_one = _time_oracle(target_s, 1)
    return {"value": round(v_all, 4), "unit": "GB/s", "cores": threads, "kind": "oracle",
            "sample": s_all,
            "single_thread": {"value": round(v_one, 4), "unit": "GB/s", "cores": 1, "sample": s_one}}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    oracle.build()
    threads = host_cores()
    budget = 150.0
    per_step = min(2.0, budget / max(1, args.steps + args.warmup))
    n = calibrate_oracle(per_step, threads)
    a, b = oracle_pair_sample(n, SEED)
    nbytes = 2 * sum(x.nbytes for x in a)
    for _ in range(args.warmup):
        oracle_step(a, b, threads)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle_step(a, b, threads)
    dt = (time.perf_counter() - t0) / max(1, args.steps)
    value = nbytes / dt / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(dt * 1e3, 3), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64 (quantizer/predicate), u64 hash", "data": "synthetic",
        "config": {"workload": WORKLOAD + f" (bounded sample: {n} particles per run per step)",
                   "chunk_bytes": CHUNK, "eps": EPS, "parallelism": "host threads"},
        "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": threads,
                         "kind": "oracle",
                         "sample": f"{CFG} recipe, {n} elements per array ({nbytes / 1e6:.1f} MB pair) per step"},
        "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), file=JSON_OUT, flush=True)
    return 0


# ---------------------------------------------------------------------------
# our arm
# ---------------------------------------------------------------------------

def run_ours(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"bench.py --gpus {args.gpus} but the launcher started {world} ranks")
    # CKPT_DIST_BACKEND=gloo + more ranks than GPUs: a functional test of the N>1 path on one
    # GPU (ranks share it; timings are not meaningful).  Production: one rank per GPU, NCCL.
    backend = os.environ.get("CKPT_DIST_BACKEND", "nccl")
    if backend == "nccl" and world > torch.cuda.device_count():
        raise SystemExit(f"{world} NCCL ranks need {world} GPUs; this node has "
                         f"{torch.cuda.device_count()}")
    local = local % max(1, torch.cuda.device_count()) if backend != "nccl" else local
    torch.cuda.set_device(local)
    # the C1/C2 exchange runs for N > 1, and at N = 1 under a launcher with --collectives
    # (exercises the NCCL path on a one-GPU box)
    collect = world > 1 or args.collectives
    nccl_info = None
    if collect:
        for k, v in (("MASTER_ADDR", "127.0.0.1"), ("RANK", "0"), ("WORLD_SIZE", "1")):
            os.environ.setdefault(k, v)
        os.environ.setdefault("MASTER_PORT", str(free_port()))
        if backend == "nccl":
            # communicator-init log on stderr (stdout carries only the JSON line)
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
            v = torch.cuda.nccl.version()
            nccl_info = {"backend": "nccl", "version": ".".join(str(x) for x in v)
                         if isinstance(v, tuple) else str(v), "world": dist.get_world_size(),
                         "exchange": "one all_gather_into_tensor per step (C1 roots + C2 counts), on its "
                                     "own stream beside the next step's leaf kernel"}
        else:
            dist.init_process_group(backend)
            nccl_info = {"backend": backend, "world": dist.get_world_size()}
    import paper_conf_middleware_tanaabcrtn24_b200 as ck
    from paper_conf_middleware_tanaabcrtn24_b200 import dist as ckd
    import synth

    ck.lib()
    if CFG == "c4" and C4_RANKS % world:
        raise SystemExit("c4 shards 64 HACC ranks: the GPU count must divide 64")
    pair = make_pair(CFG, N_PARTICLES, SEED + 1000 * rank, "cuda")
    A, B = pair.a, pair.b
    bytes_pair = 2 * pair.nbytes
    n_elems = sum(t.numel() for t in A)
    L = sum(-(-t.numel() * t.element_size() // CHUNK) for t in A)
    chunks = torch.empty(L, dtype=torch.int64, device="cuda")
    # element-id output: every element for the per-GPU configs; c4 (6.4e9 elements at N=1) is
    # capped at 2^28 ids (the full count is still returned; ~2.6e7 expected at s=9)
    idx = torch.empty(min(n_elems, 1 << 28) if CFG == "c4" else n_elems, dtype=torch.int64,
                      device="cuda")
    counts = torch.zeros(2, dtype=torch.int64, device="cuda")
    n_arrays = len(A)
    send = torch.empty((2 * n_arrays + 1, 16), dtype=torch.uint8, device="cuda")
    recv = torch.empty((world, 2 * n_arrays + 1, 16), dtype=torch.uint8, device="cuda")
    keep = []

    saved_a, host_a = None, None
    if args.path == "saved":
        # run A stored: its tree serialised (as written at capture time) and its data in pinned
        # host memory; only B is hashed on the device and only A's flagged chunks cross PCIe
        ta0 = ck.tree_build(A, CHUNK, EPS, hash_block=args.hash_block)
        saved_a = torch.frombuffer(bytearray(ta0.serialize()), dtype=torch.uint8).pin_memory()
        del ta0
        host_a = [x.cpu().pin_memory() for x in A]

    # N > 1: the C1/C2 exchange of step i runs on its own stream X while step i+1's leaf kernel
    # runs on the compute stream (its kernels take the SM slots that free up in that kernel's
    # tail; the NCCL transfer needs no SM of the compute stream).  Step i writes its counts to
    # cnt2[i % 2]; before step i+2 overwrites them, the compute stream waits for exchange i.
    xs = torch.cuda.Stream() if collect else None
    cnt2 = [torch.zeros(2, dtype=torch.int64, device="cuda") for _ in range(2)] if collect else None
    x_done = [None, None]
    step_no = [0]
    exch = []        # the last two exchanges' outputs (kept until their stream work is done)

    def exchange(TA, TB, cnt):
        # C1 + C2 in ONE collective: every rank contributes [A roots | B roots | counts]
        # (2*n_arrays*16 + 16 bytes); the counts are summed locally and both top trees are
        # built by one levels launch
        TA.array_roots(out=send[:n_arrays], stream=xs)
        TB.array_roots(out=send[n_arrays:2 * n_arrays], stream=xs)
        send[2 * n_arrays].view(torch.int64).copy_(cnt)
        dist.all_gather_into_tensor(recv.view(-1), send.view(-1))
        roots = recv[:, :2 * n_arrays].reshape(world, 2, n_arrays, 16).transpose(0, 1)
        tops = ck.tree_from_digests_batch(roots.reshape(2 * world * n_arrays, 16),
                                          [world * n_arrays, world * n_arrays], stream=xs)
        tot = recv[:, 2 * n_arrays].view(torch.int64).sum(0)
        return [TA, TB, *tops, tot]

    def step():
        i = step_no[0]
        step_no[0] += 1
        cnt = cnt2[i % 2] if collect else counts
        cur = torch.cuda.current_stream()
        if collect and x_done[i % 2] is not None:
            cur.wait_event(x_done[i % 2])          # exchange i-2 has read cnt2[i % 2]
        if args.path == "saved":
            TA, TB = ck.compare_saved(saved_a, host_a, B, chunks, idx, cnt)
        elif args.path == "fused":
            # one leaf launch hashes both runs, compares the digests and marks the flagged chunks
            TA, TB = ck.compare_pair_async(A, B, CHUNK, EPS, chunks, idx, cnt,
                                           hash_block=args.hash_block)
        else:
            TA, TB = ck.tree_build_batch([A, B], CHUNK, EPS, hash_block=args.hash_block)
            ck.diff_verify_async(TA, TB, A, B, chunks, idx, cnt)   # BFS diff, then verify
        if collect:
            xs.wait_stream(cur)                    # after this step's verify
            with torch.cuda.stream(xs):
                exch.append(exchange(TA, TB, cnt))
                ev = torch.cuda.Event()
                ev.record(xs)
            x_done[i % 2] = ev
            del exch[:-2]
            keep[:] = [TA, TB]
        else:
            keep[:] = [TA, TB]
        TA.wait()          # the step ends when both trees are complete (K2 runs on a side stream)
        TB.wait()

    def join():
        # the timed region ends when every step's exchange has completed
        if collect:
            torch.cuda.current_stream().wait_stream(xs)

    # configs[3] as written (--snapshots all): the 10 intermediate snapshots, one at a time
    # (each generated into HBM before its timed region), every snapshot's trees kept; the
    # sequence's time is the sum of the snapshots' device times.  Otherwise one snapshot / pair.
    global SNAPSHOT
    snaps = list(range(10)) if (CFG == "c4" and args.snapshots == "all") else [SNAPSHOT]
    sampler = ClockSampler(torch.cuda.current_device())
    sampler.start()
    time.sleep(0.2)
    ms_max = host_ms = leaf_ms = 0.0
    leaf_n = launches = 0
    per_snap, kept_trees = [], []
    for si, snap in enumerate(snaps):
        if si > 0 or snap != SNAPSHOT:
            SNAPSHOT = snap
            A = B = pair = None
            pair = make_pair(CFG, N_PARTICLES, SEED + 1000 * rank, "cuda")
            A, B = pair.a, pair.b
        for _ in range(max(3, args.warmup)):
            step()
        torch.cuda.synchronize()
        join()
        torch.cuda.synchronize()
        local_counts = (cnt2[(step_no[0] - 1) % 2] if collect else counts).cpu().tolist()
        if collect:   # the exchange's global counts equal an all-reduce of the local ones
            chk = torch.tensor(local_counts, dtype=torch.int64, device="cuda")
            dist.all_reduce(chk)
            assert exch[-1][-1].tolist() == chk.tolist(), (exch[-1][-1].tolist(), chk.tolist())
        # timed region: no events between the kernels (an event after the leaf kernel would end
        # the programmatic-launch overlap of the next kernel with its tail); the leaf kernel's
        # own duration is timed in a separate pass below
        l0 = ck.launch_count()
        if collect:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        h0 = time.perf_counter()
        for _ in range(args.steps):
            step()
        join()
        host_ms += (time.perf_counter() - h0) * 1e3 / args.steps   # enqueue time per step (host)
        e1.record()
        torch.cuda.synchronize()
        launches += ck.launch_count() - l0
        ms = e0.elapsed_time(e1) / args.steps
        t = torch.tensor([ms], dtype=torch.float64, device="cuda")
        if collect:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dist.barrier()
        ms_max += float(t.item())
        # the roofline kernel: events around every leaf launch of another K steps
        ck.profile_reset()
        ck.profile_enable(["leaf"])
        for _ in range(args.steps):
            step()
        join()
        torch.cuda.synchronize()
        ck.profile_enable(False)
        lm, ln = ck.profile_read("leaf")
        leaf_ms += lm
        leaf_n += ln
        ck.profile_reset()
        if len(snaps) > 1:
            # all trees kept, without references to this snapshot's arrays
            for tr in keep:
                if isinstance(tr, ck.Tree):
                    tr.detach_inputs()
            kept_trees.append(list(keep))
            per_snap.append({"snapshot": snap, "ms": round(float(t.item()), 4),
                             "flagged_chunks_per_gpu": local_counts[0],
                             "diff_elems_per_gpu": local_counts[1]})
    clocks = sampler.stop()
    # per-phase device times from a separate profiled pass (events around every family)
    k_prof = max(3, min(args.steps, 20))
    ck.profile_enable(True)
    for _ in range(k_prof):
        step()
    join()
    torch.cuda.synchronize()
    ck.profile_enable(False)
    phases = {"steps": k_prof}
    for k in ("leaf", "levels", "diff", "verify"):
        pms, pn = ck.profile_read(k)
        phases[k] = {"ms_per_step": round(pms / k_prof, 4), "launches": pn}
    if phases["diff"]["launches"] == 0:
        phases["diff"]["note"] = ("fused path: the leaf-level diff and its ordered compaction run inside "
                                  "the leaf kernel (per tile), the chunk list is written by verify_mark")
    ck.profile_reset()
    # side reference K5: "Direct" on the device -- verify with every chunk
    # flagged, i.e. 2S bytes compared element-wise with no hashing and no tree
    all_chunks = torch.arange(L, dtype=torch.int64, device="cuda")
    n_all = torch.full((1,), L, dtype=torch.int64, device="cuda")
    k5_cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    for _ in range(2):
        ck.verify_async(A, B, all_chunks, n_all, CHUNK, EPS, idx, k5_cnt)
    torch.cuda.synchronize()
    k0, k1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    k0.record()
    for _ in range(5):
        ck.verify_async(A, B, all_chunks, n_all, CHUNK, EPS, idx, k5_cnt)
    k1.record()
    torch.cuda.synchronize()
    k5_ms = k0.elapsed_time(k1) / 5
    direct_k5 = {"value": round(bytes_pair / (k5_ms / 1e3) / 1e9, 1), "unit": "GB/s",
                 "ms": round(k5_ms, 4), "diff_elems": int(k5_cnt.item()),
                 "what": "verify kernels over every chunk (no hashing, no tree): reported, not targeted"}
    del all_chunks
    leaf_avg_s = leaf_ms / max(1, leaf_n) / 1e3
    runs_hashed = 1 if args.path == "saved" else 2
    # algorithmic per launch: read the hashed run(s), write their leaves
    leaf_bytes = runs_hashed * (pair.nbytes + 16 * L)
    peak, peak_src = peaks()
    achieved = leaf_bytes / leaf_avg_s / 1e9
    traffic = None
    traffic_src = None
    tp = os.path.join(ROOT, "profiles", "leaf_traffic.json")
    # the stored capture is of the default workload's pair launch (c2, 4 KiB, 16-byte blocks)
    same = CFG == "c2" and CHUNK == 4096 and args.hash_block == 16 and args.path != "saved"
    if same and os.path.exists(tp):
        try:
            tj = json.load(open(tp))
            traffic = tj.get("dram_bytes_per_launch")
            traffic_src = ("stored ncu --set full capture (profiles/leaf_traffic.json, commit "
                           f"{tj.get('captured_at_commit', '?')}), not measured in this run")
        except Exception:
            traffic = None

    value = bytes_pair * len(snaps) * world / (ms_max / 1e3) / 1e9

    # end-to-end through the public API with host buffers (pinned), H2D+D2H inside
    e2e = None
    if CFG == "c4" and not args.no_e2e:
        e2e = {"skipped": "c4 holds 48 GiB per GPU at N=1: pinned host copies are not staged"}
    elif not args.no_e2e:
        ha = [x.cpu().pin_memory() for x in A]
        hb = [x.cpu().pin_memory() for x in B]
        k_e2e = max(3, min(args.steps, 8))

        def timed(fn):
            fn()                                         # warm-up
            if collect:
                dist.barrier()
            t0 = time.perf_counter()
            for _ in range(k_e2e):
                out = fn()
            dt = (time.perf_counter() - t0) / k_e2e
            tt = torch.tensor([dt], dtype=torch.float64, device="cuda")
            if collect:
                dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            return float(tt.item()), out

        # streamed (copy of segment k+1 overlaps the compare of segment k) and staged-then-compare
        dt_s, out_s = timed(lambda: ck.compare_stream(ha, hb, CHUNK, EPS, segment_bytes=256 << 20,
                                                      hash_block=args.hash_block, chunks_cap=0))
        dt_h, out_h = timed(lambda: ck.compare_host(ha, hb, CHUNK, EPS))
        assert out_s[2] == out_h[1] and out_s[3] == out_h[2], "e2e paths disagree"
        n_diff = out_s[3]
        e2e = {"value": round(bytes_pair * world / dt_s / 1e9, 3), "unit": "GB/s",
               "h2d_bytes_per_step": bytes_pair,
               "d2h_bytes_per_step": 8 * n_diff + 16 + 32, "steps": k_e2e,
               "api": "ckpt_compare_stream (pinned host arrays, 256 MiB segments)",
               "compare_host": {"value": round(bytes_pair * world / dt_h / 1e9, 3), "unit": "GB/s",
                                "api": "ckpt_compare_host (stage both runs, then compare)"}}
        if args.path == "fused" and args.hash_block == 16:
            # the stored-tree workflow: run A was captured earlier
            # with its tree; per step run B is copied H2D from pinned memory, A's tree is uploaded
            # from its serialised bytes, and only A's flagged chunks are read (zero-copy, pinned)
            ta0 = ck.tree_build(A, CHUNK, EPS)
            blob = torch.frombuffer(bytearray(ta0.serialize()), dtype=torch.uint8).pin_memory()
            del ta0
            dB = [torch.empty_like(x) for x in B]
            cnt_s = torch.zeros(2, dtype=torch.int64, device="cuda")
            cnt_h = torch.zeros(2, dtype=torch.int64).pin_memory()

            def saved_step():
                for d, h in zip(dB, hb):
                    d.copy_(h, non_blocking=True)
                ck.compare_saved(blob, ha, dB, chunks, idx, cnt_s)
                cnt_h.copy_(cnt_s, non_blocking=True)
                torch.cuda.synchronize()
                nd = int(cnt_h[1])
                return [int(cnt_h[0]), nd, idx[:nd].cpu()]

            dt_v, out_v = timed(saved_step)
            assert out_v[0] == out_s[2] and out_v[1] == n_diff, "saved-tree path disagrees"
            e2e["saved_tree"] = {
                "value": round(bytes_pair * world / dt_v / 1e9, 3), "unit": "GB/s",
                "h2d_bytes_per_step": pair.nbytes + blob.numel() + out_v[0] * CHUNK,
                "d2h_bytes_per_step": 8 * n_diff + 16,
                "api": "H2D of run B (pinned) + ckpt_compare_saved: run A = its stored tree + pinned "
                       "host data, of which only the flagged chunks cross PCIe (reported beside the "
                       "headline e2e, where both runs cross PCIe)"}
            del dB, blob
        del ha, hb

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline()

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": max(3, args.warmup), "ms_per_step": round(ms_max, 4),
            "higher_is_better": True, "scaling": "strong" if CFG == "c4" else "weak",
            "vs_baseline": None,
            "dtype": f"{'f64' if A[0].dtype == torch.float64 else 'f32'} in, f64 quantize/compare, u64 hash",
            "data": f"synthetic (seeded, synth {CFG} recipe)",
            "config": {"workload": WORKLOAD, "name": CFG, "elements_per_array": N_PARTICLES,
                       **({"snapshots": snaps, "hacc_ranks_per_gpu": C4_RANKS // world}
                          if CFG == "c4" else {}),
                       "arrays_per_run": n_arrays,
                       "chunk_bytes": CHUNK, "eps": EPS, "bytes_per_step_per_gpu": bytes_pair * len(snaps),
                       "l2": f"inputs larger than L2 ({bytes_pair / 1e9:.1f} GB per GPU per step >> 126 MB)",
                       "parallelism": f"dp{world} (checkpoint arrays sharded by rank)",
                       "path": args.path,
                       "hash_block": args.hash_block if args.hash_block else "chunk"},
            "pct_hbm_peak": round(value / (world * peak), 4),
            "roofline": {"bound": "hbm", "kernel": "K1 (leaf_pair_kernel for f32 pairs, leaf_kernel otherwise: quantize + chained Murmur3F)",
                         "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "traffic_source": traffic_src,
                         "peak_source": peak_src,
                         "algorithmic_bytes_per_launch": leaf_bytes,
                         "avg_launch_ms": round(leaf_avg_s * 1e3, 4),
                         "timing": "CUDA events around every leaf launch of a second pass of the same "
                                   "K steps (events in the timed pass would end the launch overlap)"},
            "phases_profiled_pass": phases, "host_enqueue_ms_per_step": round(host_ms, 4),
            "flagged_chunks_per_gpu": local_counts[0], "diff_elems_per_gpu": local_counts[1],
            "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks, "gpu_launches": launches,
            "direct_k5": direct_k5, "dist": nccl_info,
        }
        if per_snap:
            line["snapshot_sequence"] = {
                "what": "one step = the 10-snapshot sequence; per-snapshot device ms summed, every "
                        "snapshot's trees kept", "per_snapshot": per_snap,
                "trees_kept": 2 * len(kept_trees)}
        print(json.dumps(line), file=JSON_OUT, flush=True)
    if collect:
        dist.destroy_process_group()
    return 0


def free_port() -> int:
    import socket
    with socket.socket(socket.AF_INET, socket.SOCK_STREAM) as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def spawn_ranks(n: int) -> int:
    """Re-launch this command as n ranks (one per GPU) through torch.distributed.run."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--collectives", action="store_true",
                    help="run the per-step C1/C2 exchange even at N=1 (under a launcher)")
    ap.add_argument("--config", default="c2", choices=sorted(CONFIGS))
    ap.add_argument("--path", default="fused", choices=["fused", "unfused", "saved"],
                    help="fused: ckpt_compare_pair_async; unfused: build_batch + diff_verify_async; "
                         "saved: ckpt_compare_saved (A = stored tree + pinned host data)")
    ap.add_argument("--snapshot", type=int, default=9, help="c4: snapshot index 0..9")
    ap.add_argument("--snapshots", default="one", choices=["one", "all"],
                    help="c4: 'all' = BASELINE configs[3] as written, the 10-snapshot sequence")
    ap.add_argument("--elems", type=int, default=0,
                    help="elements per array (0 = the config's full size; smaller sizes are for "
                         "tests and are marked REDUCED in the workload)")
    ap.add_argument("--chunk", type=int, default=4096, help="chunk bytes (configs[2] sweeps 512..65536)")
    ap.add_argument("--eps", type=float, default=1e-6)
    ap.add_argument("--hash-block", type=int, default=16,
                    help="bytes per chained Murmur3F call: 16 = the paper's 128-bit blocks "
                         "(P:610, default); 0 = whole chunk (P:615-618 variant, R23)")
    args = ap.parse_args()
    global CFG, N_PARTICLES, WORKLOAD, HASH_BLOCK, SNAPSHOT, CHUNK, EPS
    CFG = args.config
    CHUNK = args.chunk
    EPS = args.eps
    HASH_BLOCK = args.hash_block
    SNAPSHOT = args.snapshot
    N_PARTICLES = CONFIGS[CFG]["n"]
    WORKLOAD = CONFIGS[CFG]["workload"]
    if args.elems:
        N_PARTICLES = args.elems
        WORKLOAD = f"REDUCED ({args.elems} elements per array, not a bench line): " + WORKLOAD
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return spawn_ranks(args.gpus)
    # stdout carries only the JSON line: whatever native code prints (e.g. NCCL's version banner)
    # goes to stderr
    global JSON_OUT
    JSON_OUT = os.fdopen(os.dup(1), "w")
    sys.stdout.flush()
    os.dup2(2, 1)
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
