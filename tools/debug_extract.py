"""Debug driver: a papers-shaped workload at reduced N, extract/release schedule with
release lag Q, optional per-kernel sync trace (GD_DEBUG_KERNELS=1)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, numpy as np
import synth
import paper_conf_icpp_jiangj024_b200 as gd

N = int(sys.argv[1]) if len(sys.argv) > 1 else 11_100_000
E = int(N * 14.4)
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
B, fan, Q, R = 1000, [15, 10, 5], 4, 512
dev = torch.device("cuda", 0)
ip, ix = synth.chung_lu_csr(N, E, device=dev)
g = gd.Graph(ip, ix, validate=False)
nm, _ = g.bounds(B, fan)
n_max = nm[-1]
S = max(int(0.1 * N), min(N, Q * n_max))
feat = torch.empty((N, R), dtype=torch.uint8)
feat.view(torch.int32).random_()
buf = gd.FeatureBuffer(feat, S, Q, n_max)
order = synth.epoch_order(synth.train_nodes(N, 0.0109 if N > 1e7 else 0.1, device=dev))
pend = []
outs = [g.alloc_out(B, fan) for _ in range(Q + 1)]
print(f"N={N} S={S} n_max={n_max}", flush=True)
for j in range(steps):
    t0 = time.time()
    o = outs[j % (Q + 1)]
    g.sample(order[(j * B) % (len(order) - B):][:B].contiguous(), fan, 3, j, out=o)
    st = torch.zeros(2, dtype=torch.int64, device=dev)
    buf.extract(o.n_id, o.num_nodes_dev, n_max, stats=st)
    pend.append(o)
    if len(pend) == Q:
        r = pend.pop(0)
        buf.release(r.n_id, r.num_nodes_dev, n_max)
    torch.cuda.synchronize()
    print(f"step {j}: stats={st.cpu().tolist()} {time.time()-t0:.3f}s", flush=True)
print("status", buf.check(), g.check())
