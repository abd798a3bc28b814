import sys, statistics, torch
sys.path.insert(0, '.')
import __graft_entry__; __graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap, workloads
x = workloads.random_bits(8192, 8192, torch.float32, seed=0, device="cuda"); y = torch.empty_like(x)
hist = torch.zeros((5, 3, 33), dtype=torch.int64, device="cuda")
K = 20
ev = [[torch.cuda.Event(enable_timing=True, external=True) for _ in range(4)] for _ in range(K)]
s = torch.cuda.Stream()
rap.transpose(x, layout="rap", out=y); rap.congestion_sweep(151552, seed=1, first_trial=0, out=hist)
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    for k in range(K):
        ev[k][0].record(); rap.transpose(x, layout="rap", out=y); ev[k][1].record()
        ev[k][2].record(); rap.congestion_sweep(151552, seed=1, first_trial=k * 151552, out=hist); ev[k][3].record()
for r in range(3):
    g.replay(); torch.cuda.synchronize()
    t = [ev[k][0].elapsed_time(ev[k][1]) for k in range(K)]
    sw = [ev[k][2].elapsed_time(ev[k][3]) for k in range(K)]
    print("graph: transpose median us", statistics.median(t) * 1e3, "GB/s", 2 * x.nbytes / statistics.median(t) / 1e6, "sweep us", statistics.median(sw) * 1e3)
print("hist total", int(hist[0,0].sum()))
