"""Probe: time cstf_hals_update / cstf_mu_update / cstf_admm_update (10 sweeps or passes,
R = 32) on I rows (default: Delicious mode 1, 17.3M) and report the FP64 rate of the
HALS / MU row loops.  python tools/hals_probe.py [I]"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icpp_sohksc24_b200 import binding as B  # noqa: E402


def timed(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    I = int(sys.argv[1]) if len(sys.argv) > 1 else 17_300_000
    R = 32
    g = torch.Generator(device="cuda").manual_seed(1)
    A = torch.rand(256, R, dtype=torch.float64, device="cuda", generator=g)
    S = A.T @ A
    M = torch.rand(I, R, dtype=torch.float64, device="cuda", generator=g)
    H = torch.rand(I, R, dtype=torch.float64, device="cuda", generator=g)
    U = torch.zeros(I, R, dtype=torch.float64, device="cuda")
    flops = 2.0 * R * R * I * 10
    t = timed(lambda: B.cstf_hals_update(M, S, H, sweeps=10))
    print(f"HALS  I={I} R={R} 10 sweeps: {t:.2f} ms, {flops / t / 1e9:.1f} TF/s (2 R^2 per row and sweep)")
    t = timed(lambda: B.cstf_mu_update(M, S, H, sweeps=10))
    print(f"MU    I={I} R={R} 10 sweeps: {t:.2f} ms, {flops / t / 1e9:.1f} TF/s")
    t = timed(lambda: B.cstf_admm_update(M, S, H, U, tol=0.0, max_iter=10))
    print(f"ADMM  I={I} R={R} 10 passes: {t:.2f} ms, {flops / t / 1e9:.1f} TF/s")


if __name__ == "__main__":
    main()
