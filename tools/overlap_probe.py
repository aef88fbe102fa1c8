"""Probe: can the MTTKRP of one row segment overlap the ADMM of another on the
same SMs?  Times, on Delicious mode 1 (17.3M rows), MTTKRP then ADMM on one
stream against the two on two streams with their grids capped so both fit
(CSTF_MTTKRP_CTAS_PER_SM / CSTF_ADMM_CTAS_PER_SM).  Run on the GPU box:
    python tools/overlap_probe.py [mode]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import datagen  # noqa: E402
from paper_conf_icpp_sohksc24_b200 import binding as B  # noqa: E402


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1
    cfg = datagen.CONFIGS["delicious"]
    idx, vals = cfg.generate()
    X = B.cstf_tensor_load_coo(cfg.dims, idx, vals)
    del idx, vals
    R = cfg.R
    F = [torch.from_numpy(f).cuda() for f in datagen.init_factors(cfg.dims, R, cfg.seed)]
    I = cfg.dims[n]
    M = torch.empty(I, R, dtype=torch.float64, device="cuda")
    M2 = torch.rand(I, R, dtype=torch.float64, device="cuda")
    H = torch.rand(I, R, dtype=torch.float64, device="cuda")
    U = torch.zeros_like(H)
    g = torch.rand(256, R, dtype=torch.float64, device="cuda")
    S = (g.T @ g) / 256 + torch.eye(R, dtype=torch.float64, device="cuda")
    sa = torch.cuda.Stream()
    sb = torch.cuda.Stream()

    def run(conc, mt_cap=None, ad_cap=None, reps=5):
        for k, v in (("CSTF_MTTKRP_CTAS_PER_SM", mt_cap), ("CSTF_ADMM_CTAS_PER_SM", ad_cap)):
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = str(v)
        ts = []
        for r in range(reps + 1):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(sa)
            sb.wait_event(e0)
            with torch.cuda.stream(sa):
                B.cstf_mttkrp(X, n, F, M)
            with torch.cuda.stream(sb if conc else sa):
                B.cstf_admm_update(M2, S, H, U, tol=0.0, max_iter=10)
            if conc:
                ev = torch.cuda.Event()
                ev.record(sb)
                sa.wait_event(ev)
            e1.record(sa)
            torch.cuda.synchronize()
            if r:
                ts.append(e0.elapsed_time(e1))
        return float(np.median(ts))

    print(f"mode {n} I={I}", flush=True)
    print(f"  mttkrp alone {run(False, ad_cap=None) and 0 or 0:.0f}", flush=True)
    for conc, mc, ac in ((False, None, None), (True, None, None), (True, 3, 1), (True, 2, 1), (True, 2, 2),
                         (True, 3, 2), (False, None, None)):
        print(f"  {'concurrent' if conc else 'sequential'} mttkrp_cap={mc} admm_cap={ac}: {run(conc, mc, ac):.3f} ms",
              flush=True)


if __name__ == "__main__":
    main()
