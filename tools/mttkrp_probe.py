"""Probe: time cstf_mttkrp per mode of a config under environment variants.
Run on the GPU box:  python tools/mttkrp_probe.py CONFIG 'ENV=V,ENV2=V' ...
(each argument after the config is one variant; '-' = no extra variables).
Every variant's output is compared with the first one (max normwise error)."""
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import datagen  # noqa: E402
from paper_conf_icpp_sohksc24_b200 import binding as B  # noqa: E402


REPS = int(os.environ.get("PROBE_REPS", "10"))
MODES = os.environ.get("PROBE_MODES")   # e.g. "1,3": only these modes


def timed(fn, reps=REPS):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def parse(v):
    if v == "-":
        return {}
    return dict(kv.split("=", 1) for kv in v.split(","))


def main():
    name = sys.argv[1]
    variants = sys.argv[2:] or ["-"]
    cfg = datagen.CONFIGS[name]
    idx, vals = cfg.generate()
    t0 = time.time()
    X = B.cstf_tensor_load_coo(cfg.dims, idx, vals)
    del idx, vals
    print(f"{name}: load {time.time() - t0:.1f}s", flush=True)
    F = [torch.from_numpy(f).cuda() for f in datagen.init_factors(cfg.dims, cfg.R, cfg.seed)]
    for n, I in enumerate(cfg.dims):
        if MODES and str(n) not in MODES.split(","):
            continue
        M = torch.empty(I, cfg.R, dtype=torch.float64, device="cuda")
        ref = None
        out = []
        for v in variants:
            env = parse(v)
            old = {k: os.environ.get(k) for k in env}
            os.environ.update(env)
            t = timed(lambda: B.cstf_mttkrp(X, n, F, M))
            for k, o in old.items():
                if o is None:
                    os.environ.pop(k)
                else:
                    os.environ[k] = o
            if ref is None:
                ref = M.clone()
                err = 0.0
            else:
                err = ((M - ref).abs().max() / ref.abs().max()).item()
            out.append(f"[{v}] {t:.3f} ms (err {err:.1e})")
        print(f"mode {n} I={I} nnz/row={X.info()['nnz'] / I:.0f}: " + ", ".join(out), flush=True)


if __name__ == "__main__":
    main()
