import sys, torch
sys.path.insert(0, '.')
import __graft_entry__; __graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap
for i in range(3):
    rap.congestion_sweep(1 << 18, seed=1, w=256, first_trial=i << 18)
torch.cuda.synchronize()
