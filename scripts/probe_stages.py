import sys, numpy as np, torch
sys.path.insert(0, '/root/repo')
import oracle as O
from paper_conf_asplos_lis0l0c17_b200 import ops, synth
case = sys.argv[1]; st = int(sys.argv[2]); N = int(sys.argv[3]) if len(sys.argv) > 3 else 300
u0 = synth.matrix(4, N, N - 40)
a = torch.from_numpy(u0).cuda(); b = torch.zeros_like(a)
if case == "jac":
    out = ops.jacobi5(a, b, 6, backend="agent", order="row", stages=st)
elif case == "jacf":
    out = ops.jacobi5(a, b, 6, backend="agent", order="row", stages=st, fuse=3)
else:
    w = synth.uniform(6, 9).reshape(3, 3)
    out = ops.conv2d(a, w, backend="agent", order="row", stages=st)
torch.cuda.synchronize()
ref = O.jacobi5_f32(u0, 6) if case != "conv" and N <= 4096 else None
print(case, st, "ok" if ref is None or np.array_equal(out.cpu().numpy(), ref) else "MISMATCH")
