"""e2e probe: compare_stream segment sizes vs compare_host on the c2 pair (pinned host)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_middleware_tanaabcrtn24_b200 as ck
import synth
pair = synth.c2_pair(n_particles=1 << 26, seed=2, device="cuda")
ha = [x.cpu().pin_memory() for x in pair.a]
hb = [x.cpu().pin_memory() for x in pair.b]
nb = 2 * pair.nbytes
# raw H2D bandwidth of the same bytes (one stream)
dev = [torch.empty_like(x, device="cuda") for x in ha + hb]
for rep in range(2):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    for d, h in zip(dev, ha + hb):
        d.copy_(h, non_blocking=True)
    torch.cuda.synchronize(); dt = time.perf_counter() - t0
    print(f"raw H2D {nb / dt / 1e9:.1f} GB/s")
del dev
for seg in (32 << 20, 64 << 20, 128 << 20, 256 << 20):
    ck.compare_stream(ha, hb, 4096, 1e-6, segment_bytes=seg, chunks_cap=0)
    t0 = time.perf_counter()
    for _ in range(4):
        ck.compare_stream(ha, hb, 4096, 1e-6, segment_bytes=seg, chunks_cap=0)
    dt = (time.perf_counter() - t0) / 4
    print(f"stream seg={seg >> 20} MiB: {nb / dt / 1e9:.1f} GB/s")
ck.compare_host(ha, hb, 4096, 1e-6)
t0 = time.perf_counter()
for _ in range(4):
    ck.compare_host(ha, hb, 4096, 1e-6)
dt = (time.perf_counter() - t0) / 4
print(f"compare_host: {nb / dt / 1e9:.1f} GB/s")
