"""Per-kernel times of the Fig. 4 ablation arms (bench-only library) for one mode shape:
    ncu --metrics gpu__time_duration.sum --csv --log-file out.csv python tools/ablation_probe.py [I] [R] [passes]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icpp_sohksc24_b200 import ablation as AB  # noqa: E402

I = int(sys.argv[1]) if len(sys.argv) > 1 else 2_500_000
R = int(sys.argv[2]) if len(sys.argv) > 2 else 32
k = int(sys.argv[3]) if len(sys.argv) > 3 else 3
torch.cuda.set_device(0)
rng = np.random.default_rng(0)
A = rng.random((R, R))
S = torch.from_numpy(A @ A.T / R).cuda()
M = torch.rand(I, R, dtype=torch.float64, device="cuda")
H = torch.rand(I, R, dtype=torch.float64, device="cuda")
U = torch.zeros_like(H)
for name, arm in AB.ARMS.items():
    for rep in range(2):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record()
        st = AB.admm(arm, M, S, H, U, max_iter=k)
        b.record()
        torch.cuda.synchronize()
        print(f"{name}: {a.elapsed_time(b):.3f} ms ({st['calls']} calls)", flush=True)
