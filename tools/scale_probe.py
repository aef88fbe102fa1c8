import torch, sys, os
sys.path.insert(0, os.getcwd())
from paper_conf_icpp_sohksc24_b200 import binding as B
I, R = 17_300_000, 32
H = torch.rand(I, R, dtype=torch.float64, device="cuda")
H2 = torch.empty_like(H)
s = torch.rand(R, dtype=torch.float64, device="cuda") + 0.5
def t(fn, reps=5):
    fn(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / reps
gb = 2 * I * R * 8 / 1e9
for name, fn in [("torch inplace mul", lambda: H.mul_(s)), ("torch out-of-place mul", lambda: torch.mul(H, s, out=H2)),
                 ("torch copy", lambda: H2.copy_(H)), ("torch inplace div", lambda: H.div_(s))]:
    ms = t(fn); print(f"{name}: {ms:.3f} ms, {gb/ms:.2f} TB/s")
lam = torch.zeros(R, dtype=torch.float64, device="cuda"); G = torch.zeros(R, R, dtype=torch.float64, device="cuda")
ms = t(lambda: B.cstf_normalize(H, lam, G)); print(f"cstf_normalize (gram + scale): {ms:.3f} ms")

# the same pass on factors produced by a factorisation (Delicious-shaped, one outer iteration)
import datagen
cfg = datagen.CONFIGS["delicious"]
idx, vals = cfg.generate()
X = B.cstf_tensor_load_coo(cfg.dims, idx, vals)
F = [torch.from_numpy(f).cuda() for f in datagen.init_factors(cfg.dims, cfg.R, cfg.seed)]
lam = torch.zeros(cfg.R, dtype=torch.float64, device="cuda")
B.cstf_factorize(X, F, lam, B.make_opts(cfg.R, outer_iters=1, tol=0.0, max_iter=10))
H1 = F[1]
nz = H1[H1 != 0]
print("mode-1 factor: zeros %.3f, min nonzero %.3e, below 2^-900: %d, subnormal: %d" % (
    1 - nz.numel() / H1.numel(), nz.abs().min().item(), int((nz.abs() < 2.0 ** -900).sum()),
    int((nz.abs() < 2.2250738585072014e-308).sum())))
Hc = H1.clone()
lam2 = torch.zeros(cfg.R, dtype=torch.float64, device="cuda")
ms = t(lambda: (Hc.copy_(H1), B.cstf_normalize(Hc, lam2, G)))
print(f"copy + cstf_normalize on the factorised mode-1 factor: {ms:.3f} ms")
ms = t(lambda: Hc.copy_(H1))
print(f"copy alone: {ms:.3f} ms")
