import sys, torch
sys.path.insert(0, '.')
from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, ops, shard, synth
N, G, T = 16384, 8, 4
u = synth.matrix(4, N, N, backend="torch", device="cuda")
slabs = []
for g in range(G):
    lo, hi, llo, lhi = shard.slab_range(N, G, g, 1)
    a = u[llo:lhi].clone()
    slabs.append(dict(a=a, b=torch.empty_like(a), ll=torch.zeros(cc.ll_words(N), dtype=torch.int64, device="cuda")))
nb = lambda h: slabs[h]["ll"].data_ptr() if 0 <= h < G else None
for s in range(T):
    for g, x in enumerate(slabs):
        src, dst = (x["a"], x["b"]) if s % 2 == 0 else (x["b"], x["a"])
        ops.jacobi5_halo(src, dst, 1, s, x["ll"], nb(g - 1), nb(g + 1), None, backend="identity")
        ops.jacobi5(src, dst, 1, backend="identity")
torch.cuda.synchronize()
