import sys, torch
sys.path.insert(0, '/root/repo')
import paper_conf_middleware_tanaabcrtn24_b200 as ck, synth
pair = synth.c2_pair(n_particles=1 << 16, seed=5, device="cuda")
TA, TB = ck.tree_build_batch([pair.a, pair.b], 4096, 1e-6)
chunks = torch.empty(TA.n_leaves, dtype=torch.int64, device="cuda")
cnt = torch.zeros(2, dtype=torch.int64, device="cuda")
idx = torch.empty(1 << 20, dtype=torch.int64, device="cuda")
for _ in range(4):
    ck.tree_diff_async(TA, TB, chunks, cnt[0:1])
    ck.verify_async(pair.a, pair.b, chunks, cnt[0:1], 4096, 1e-6, idx, cnt[1:2])
torch.cuda.synchronize()
