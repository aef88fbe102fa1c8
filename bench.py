"""Benchmark of the cSTF hot path on B200 (driver contract, one JSON line on rank 0).

A step is one outer iteration of Alg. 1 over the whole
tensor: for every mode S / rho / Cholesky / inverse, MTTKRP, the fused ADMM
update (10 inner iterations, eps = 0: the paper's timing protocol L930-933),
normalisation and Gram, then the fit.  Inputs are the seeded synthetic tensor
of the chosen BASELINE.json config, already resident in HBM when the timed
region starts.  Default: configs[3], Delicious-4D-shaped -- the largest config
the metric is quoted on at 1/2/4/8 B200 that fits one GPU (and the
ADMM-update-bound one); configs[1] (nell2) and configs[2] (enron) are
`--config` choices, configs[4] (amazon, 1.7B nonzeros) fits one GPU too but
takes minutes to generate and load.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config delicious|nell2|enron|amazon]
                  [--impl ours|reference] [--no-cpu-baseline] [--comm nccl|host] [--ablation]

--gpus N > 1 without torchrun re-launches itself under torch.distributed.run
with N ranks (one per GPU over NCCL; --comm host lets the N ranks share one GPU
to validate the multi-rank path).

--impl reference times the FP64 CPU oracle (the reference arm of this tier) on
the host cores: one outer iteration of the same workload per step.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402
from paper_conf_icpp_sohksc24_b200 import costmodel as cm  # noqa: E402

METRIC = "cSTF outer-iteration time (s) and ADMM update HBM GB/s at 1/2/4/8 B200"
PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
FP64_PEAK_TFLOPS = 37.1      # fallback: measured on this pool's B200 (DFMA and DMMA alike), profiles/r01_microbench.txt
L2_GATHER_GBS = 19890.0      # measured L2->SM random 256-byte row gathers, 7.4 MB tables (same microbench)
L1_GATHER_GBS = 28855.0      # measured all-L1-hit 256-byte row gathers (16 lanes x 16 B, two 200-row tables):
                             # the on-chip ceiling of the MTTKRP access (tools/gather_probe.cu, profiles/r01_gather_probe.txt)


def load_peaks():
    try:
        with open(PEAKS_PATH) as f:
            p = json.load(f)
        return p, "measured (MEASURED_PEAKS.json)"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0}, "fallback (B200_PROFILING.md)"


def measured_traffic(workload):
    """ncu DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) per launch of the
    MTTKRP and ADMM kernels of every mode, from the committed capture
    profiles/r02_traffic.json (or None)."""
    try:
        with open(os.path.join(ROOT, "profiles", "r02_traffic.json")) as f:
            d = json.load(f)
        t = d.get(workload)
        if t is not None:
            t = dict(t, source="profiles/r02_traffic.json (ncu capture of " + d.get("source", "?") + "; " +
                     d.get("how", "") + ")")
        return t
    except Exception:
        return None


def env_rank():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            out, _ = self.proc.communicate(timeout=5)
        except Exception:
            self.proc.kill()
            out = ""
        sms, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sms.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sms) if sms else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sms)}


def oracle_outer_iteration(cfg, idx, vals, R, steps, warmup):
    """The FP64 oracle as it stands: one outer iteration (eps = 0, 10 inner) per step."""
    import oracle
    # all host cores of this process (torchrun sets OMP_NUM_THREADS=1 in every rank;
    # only rank 0 runs the oracle); the count reported is the one in effect
    cores = oracle.set_threads(len(os.sched_getaffinity(0)))
    t0 = time.time()
    X = oracle.coalesce(cfg.dims, idx, vals)
    t_coalesce = time.time() - t0
    F = datagen.init_factors(cfg.dims, R, cfg.seed)
    times = []
    for s in range(warmup + steps):
        t0 = time.perf_counter()
        oracle.factorize(X, F, outer_iters=1, tol=0.0, max_iter=10)
        dt = time.perf_counter() - t0
        if s >= warmup:
            times.append(dt)
    return float(np.mean(times)), cores, t_coalesce


def run_reference(args, cfg):
    rank, world, _ = env_rank()
    if rank != 0:
        return 0
    idx, vals = cfg.generate()
    # the reference arm: the oracle, on the host cores, one full outer iteration per step
    w = max(0, min(args.warmup, 1))     # a CPU has nothing to warm up; keep the run within minutes
    k = max(1, min(args.steps, 3))
    v, cores, tco = oracle_outer_iteration(cfg, idx, vals, cfg.R, k, w)
    line = {"metric": METRIC, "value": v, "unit": "s", "n_gpus": world, "steps": k, "warmup": w,
            "ms_per_step": v * 1e3, "higher_is_better": False, "scaling": "strong", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic (datagen recipe)", "impl": "reference",
            "config": config_dict(cfg),
            "cpu_baseline": {"value": v, "unit": "s", "cores": cores, "kind": "oracle",
                             "sample": f"{k} full outer iteration(s) of the {cfg.name} workload "
                                       f"(eps=0, 10 inner); coalesce {tco:.1f}s excluded"},
            "e2e": {"value": v, "unit": "s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def admm_ablation(B, cfg, R, stream, reps=3):
    """SURVEY f2 / Fig. 4 (Sec. 5.2) on this workload's mode shapes:
    one ADMM update (10 passes, eps = 0) per mode for every arm -- the paper's
    baseline (Alg. 2 as separate element-wise calls + two cuBLAS DTRSM per pass),
    operation fusion only (OF), pre-inversion only (PI), both (OF+PI, the paper's
    cuADMM shape), and libcstf's one-launch-per-pass (streaming) and row-resident
    kernels.  S = Hadamard of the Grams (cstf_gram) of seeded normalised factors."""
    import torch
    from paper_conf_icpp_sohksc24_b200 import ablation as AB
    N = len(cfg.dims)
    Gs = []
    for k in range(N):
        f = datagen.uniform(cfg.seed, 50 + k, 256 * R).reshape(256, R)
        f = f / np.linalg.norm(f, axis=0)                       # column-normalised (reading D6)
        g = torch.zeros(R, R, dtype=torch.float64, device="cuda")
        B.cstf_gram(torch.from_numpy(f).cuda(), g)
        Gs.append(g.cpu().numpy())
    out = {}

    def timed(fn):
        fn()                                                     # warm-up (also allocates workspaces)
        ts = []
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            a.record(stream)
            fn()
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return float(np.median(ts))

    for n, I in enumerate(cfg.dims):
        S_h = np.ones((R, R))
        for k in range(N):
            if k != n:
                S_h = S_h * Gs[k]
        S = torch.from_numpy(S_h).cuda()
        M = torch.rand(I, R, dtype=torch.float64, device="cuda")
        H0 = torch.rand(I, R, dtype=torch.float64, device="cuda")
        H, U = H0.clone(), torch.zeros_like(H0)
        res = {"rows": I}
        for name, arm in (("baseline", AB.BASELINE), ("of", AB.OF), ("pi", AB.PI), ("of_pi", AB.OF_PI)):
            res[name + "_ms"] = timed(lambda: AB.admm(arm, M, S, H, U, max_iter=10))
        for name, var in (("streaming", B.CSTF_ADMM_STREAMING), ("resident", B.CSTF_ADMM_RESIDENT)):
            res[name + "_ms"] = timed(lambda: B.cstf_admm_update(M, S, H, U, tol=0.0, max_iter=10, variant=var))
        for k in ("of", "pi", "of_pi", "streaming", "resident"):
            res["speedup_" + k] = res["baseline_ms"] / res[k + "_ms"]
        out[f"mode{n}"] = res
        del M, H0, H, U
        torch.cuda.empty_cache()
    return out


def admm_streaming_probe(B, cfg, R, stream, hbm_peak, reps=3):
    """The metric's literal "ADMM update HBM GB/s": libcstf's one-launch-per-pass
    ADMM kernel (v1: reads M, H, U and writes H, U every pass = 40 I R bytes per
    pass) on the largest mode of this workload, 10 passes, CUDA events.  The bench's
    own update is the row-resident kernel (FP64-bound; it moves those bytes once)."""
    import torch
    n = int(np.argmax(cfg.dims))
    I = cfg.dims[n]
    f = datagen.uniform(cfg.seed, 60, 256 * R).reshape(256, R)
    f = f / np.linalg.norm(f, axis=0)
    g = torch.zeros(R, R, dtype=torch.float64, device="cuda")
    B.cstf_gram(torch.from_numpy(f).cuda(), g)
    S = g * g                                                   # Hadamard of two unit-diagonal Grams
    M = torch.rand(I, R, dtype=torch.float64, device="cuda")
    H = torch.rand(I, R, dtype=torch.float64, device="cuda")
    U = torch.zeros_like(H)
    B.cstf_admm_update(M, S, H, U, tol=0.0, max_iter=10, variant=B.CSTF_ADMM_STREAMING)
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(stream)
        B.cstf_admm_update(M, S, H, U, tol=0.0, max_iter=10, variant=B.CSTF_ADMM_STREAMING)
        b.record(stream)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ms = float(np.median(ts))
    byts = 10 * cm.admm_bytes(I, R)
    del M, H, U
    torch.cuda.empty_cache()
    return {"mode": n, "rows": I, "passes": 10, "ms": ms, "gbs": byts / (ms * 1e-3) / 1e9,
            "frac_of_hbm": byts / (ms * 1e-3) / 1e9 / hbm_peak,
            "note": "k_admm_dmma with one launch per pass (CSTF_ADMM_STREAMING), 40 I R bytes per pass"}


def relaunch_under_torchrun(n):
    """--gpus N > 1 without a torchrun environment: run this command again as N ranks
    (one process per GPU, rendezvous on 127.0.0.1)."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    os.execv(sys.executable, cmd)


def config_dict(cfg):
    return {"workload": cfg.name, "dims": list(cfg.dims), "nnz_generated": cfg.nnz, "R": cfg.R,
            "seed": cfg.seed, "admm": "eps=0, max_iter=10 (PAPER.md L930-933)",
            "warm_start": "scaled (D4)", "l2": "inputs larger than L2 (nonzero store >> 126 MB)"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="delicious", choices=sorted(datagen.CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-streaming-probe", action="store_true",
                    help="skip timing the one-launch-per-pass ADMM kernel on the largest mode")
    ap.add_argument("--comm", choices=["nccl", "host"], default="nccl",
                    help="N > 1 transport: nccl (one GPU per rank, the product path) or host (gloo "
                         "host callbacks; ranks may share one GPU -- validates the multi-rank path, "
                         "not a performance number)")
    ap.add_argument("--ablation", action="store_true",
                    help="also time one ADMM update per mode with the streaming (one launch per inner "
                         "iteration, the paper's fused shape) and the row-resident variants (SURVEY f2)")
    args = ap.parse_args()
    cfg = datagen.CONFIGS[args.config]
    if args.impl == "reference":
        return run_reference(args, cfg)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return relaunch_under_torchrun(args.gpus)

    import torch
    from paper_conf_icpp_sohksc24_b200 import binding as B

    rank, world, local = env_rank()
    if world != args.gpus:
        raise SystemExit(f"bench.py: {world} ranks but --gpus {args.gpus}")
    host_comm = world > 1 and args.comm == "host"
    if world > 1 and not host_comm and torch.cuda.device_count() < world:
        raise SystemExit(f"bench.py: --gpus {world} over NCCL needs {world} GPUs, found "
                         f"{torch.cuda.device_count()} (--comm host validates the multi-rank path on one GPU)")
    if host_comm:                            # validation: N ranks may share one GPU
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dist = None
    comm = None
    if world > 1:
        import torch.distributed as dist
        if host_comm:
            dist.init_process_group("gloo")
            comm = B.cstf_comm_create_host()
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
            comm = B.cstf_comm_create_nccl()     # rows of every mode partitioned over the ranks
    R = cfg.R
    t0 = time.time()
    idx, vals = cfg.generate()
    t_gen = time.time() - t0
    t0 = time.time()
    X = B.cstf_tensor_load_coo(cfg.dims, idx, vals, comm=comm)
    torch.cuda.synchronize()
    t_load = time.time() - t0
    info = X.info()
    F0 = datagen.init_factors(cfg.dims, R, cfg.seed)
    F = [torch.from_numpy(f).cuda() for f in F0]
    lam = torch.zeros(R, dtype=torch.float64, device="cuda")
    stream = torch.cuda.current_stream()

    def opts(n, timing=False):
        return B.make_opts(R, outer_iters=n, tol=0.0, max_iter=10, timing=timing)

    # nvidia-smi needs a few hundred ms before its first sample: start it now, so
    # it samples the (identical) warm-up work and the timed region
    # the ADMM roofline denominator, measured live on this box: the FP64
    # tensor-path (DMMA) peak from the bench-only library, before the timed region
    try:
        from paper_conf_icpp_sohksc24_b200 import ablation as AB
        fp64_peak, fp64_src = AB.fp64_peak(stream), ("measured live on this box: chain-only DMMA.8x8x4 kernel "
                                                     "(cstf_ablation_fp64_peak, best of 3)")
    except Exception as e:                   # keep the committed microbench figure
        fp64_peak, fp64_src = FP64_PEAK_TFLOPS, (f"tools/microbench.cu -> profiles/r01_microbench.txt "
                                                 f"(live measurement failed: {e})")
    clocks = ClockSampler(local)
    clocks.start()
    # warm-up: W outer iterations
    B.cstf_factorize(X, F, lam, opts(max(args.warmup, 3)), comm=comm)
    torch.cuda.synchronize()
    # timed: K outer iterations in one call (each call starts with the init pass: included)
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = B.cstf_kernel_launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    rep = B.cstf_factorize(X, F, lam, opts(args.steps, timing=True), comm=comm)
    e1.record(stream)
    torch.cuda.synchronize()
    launches = B.cstf_kernel_launch_count() - l0
    if dist:
        dist.barrier()
    clk = clocks.stop()
    ms_total = e0.elapsed_time(e1)
    if dist:
        t = torch.tensor([ms_total], device="cpu" if host_comm else "cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t.item())
    ms_step = ms_total / args.steps
    K = args.steps
    N = len(cfg.dims)
    mp = rep["mode_phase_ms"]             # [N][5], summed over K steps
    ml = rep["mode_launches"]
    phase_ms = {k: v / K for k, v in rep["phase_ms"].items()}
    # roofline of the dominant kernel: algorithmic bytes / flops per launch
    # over the CUDA-event time of that kernel's phase in the timed region
    peaks, peak_src = load_peaks()
    nnz = info["nnz"]
    mtt_ms = mp[:, 1].sum() / K
    upd_ms = mp[:, 2].sum() / K
    traffic = measured_traffic(cfg.name)          # ncu, one capture per kernel and mode (or None)
    # SURVEY s8(d) MTTKRP lower bound per launch: nnz (8 + 4N) + sum_k I_k R 8 (every
    # factor once, M included); our store's own compulsory bytes (no i_n per nonzero,
    # an int64 row pointer instead) are reported beside it
    bound_bytes = N * (nnz * (8 + 4 * N) + sum(I * R * 8 for I in cfg.dims))
    mtt_bytes = [cm.mttkrp_bytes(nnz, cfg.dims, n, R) for n in range(N)]
    roof_mtt = {"kernel": "mttkrp (k_mttkrp_fast + carry fix-up)", "bound": "hbm",
                "achieved": bound_bytes / (mtt_ms * 1e-3) / 1e9, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "peak_source": peak_src,
                "algorithmic_bytes_per_launch": bound_bytes / N,
                "algorithmic_bytes_def": "SURVEY s8(d): nnz*(8+4N) + sum_k I_k*R*8",
                "store_bytes_per_launch": sum(mtt_bytes) / N, "avg_launch_ms": mtt_ms / N,
                "per_mode_ms": (mp[:, 1] / K).tolist(),
                "traffic": None, "traffic_per_mode": None, "traffic_source": None}
    roof_mtt["frac"] = roof_mtt["achieved"] / peaks["hbm_gbs"]
    if traffic and "mttkrp" in traffic:
        tm = traffic["mttkrp"]["per_mode_bytes"]
        tg = sum(tm) / (mtt_ms * 1e-3) / 1e9
        roof_mtt.update(traffic=sum(tm) / len(tm), traffic_per_mode=tm, traffic_source=traffic["source"],
                        traffic_gbs=tg, traffic_frac=tg / peaks["hbm_gbs"],
                        traffic_note="measured DRAM bytes (ncu) per launch: the gathers of factor rows that "
                                     "miss L2 move several times the algorithmic bytes; traffic_frac = HBM "
                                     "utilisation by measured traffic")
    # the ADMM update (the paper's cuADMM, row-resident, FP64 tensor path): executed flops
    # (DMMA products + the element-wise ops the FNN passes really run; not Eq. 3) against
    # the measured FP64 peak, the ncu pipe fraction beside it
    fl_exec = sum(cm.admm_flops_executed(I, R, 10, fnn=True, gram=R <= 32) for I in cfg.dims)
    fl_eq3 = sum(10 * cm.admm_flops_per_row_iter(R) * I for I in cfg.dims)
    roof_admm = {"kernel": "admm (k_admm_dmma, row-resident, FNN passes)", "bound": "fp64",
                 "achieved": fl_exec / (upd_ms * 1e-3) / 1e12 if upd_ms > 0 else None,
                 "peak": fp64_peak, "unit": "TFLOP/s",
                 "peak_source": fp64_src + " (MEASURED_PEAKS.json has no FP64 figure)",
                 "flops": "executed: DMMA products 2 RP^2 + FNN element-wise 3R per pass + 13R last pass + "
                          "fused Gram tiles, per row (costmodel.admm_flops_executed)",
                 "eq3_flops_achieved": fl_eq3 / (upd_ms * 1e-3) / 1e12 if upd_ms > 0 else None,
                 "per_mode_ms": (mp[:, 2] / K).tolist()}
    roof_admm["frac"] = roof_admm["achieved"] / fp64_peak if upd_ms > 0 else None
    if traffic and "admm" in traffic:
        ta = traffic["admm"]
        roof_admm["ncu_fp64_datapath_frac"] = ta.get("fp64_datapath_frac")
        roof_admm["ncu_source"] = traffic["source"]
    # "ADMM update HBM GB/s" (BASELINE metric): measured DRAM bytes per ADMM launch (ncu)
    # over the CUDA-event ADMM time; the paper's streaming byte model beside it, labelled
    admm_gbs = {"model_40kIR_gbs": sum(10 * cm.admm_bytes(I, R) for I in cfg.dims) / (upd_ms * 1e-3) / 1e9
                if upd_ms > 0 else None,
                "model_note": "40 I R bytes per inner iteration (v1 streaming model), k = 10: NOT traffic",
                "measured_gbs": None, "measured_bytes_per_step": None}
    if traffic and "admm" in traffic and upd_ms > 0:
        tb = sum(traffic["admm"]["per_mode_bytes"])
        admm_gbs.update(measured_gbs=tb / (upd_ms * 1e-3) / 1e9, measured_bytes_per_step=tb,
                        measured_source=traffic["source"],
                        measured_frac_of_hbm=tb / (upd_ms * 1e-3) / 1e9 / peaks["hbm_gbs"])
    roof = roof_mtt if mtt_ms >= upd_ms else dict(roof_admm, bound="fp64")
    line = {"metric": METRIC, "value": ms_step / 1e3, "unit": "s", "n_gpus": world, "steps": K,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": False,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (datagen recipe, shapes of PAPER.md Table 2)",
            "config": dict(config_dict(cfg), **({"parallelism": f"rows of every mode partitioned over {world} ranks",
                                                 "comm": "host callbacks (validation, shared GPU)" if host_comm
                                                 else "NCCL + CUDA-IPC peer stores"} if world > 1 else {})),
            "gpu_launches": int(launches),
            "roofline": roof, "roofline_admm": roof_admm, "admm_update_gbs": admm_gbs,
            "phases_ms_per_step": phase_ms, "clocks": clk,
            "setup": {"generate_s": t_gen, "load_coo_s": t_load, "nnz_coalesced": nnz,
                      "layout": [dict(zip(("nblk", "blk_rows", "blk_mode"), X.layout(n)),
                                      record_bytes=X.record_bytes(n)) for n in range(N)]}}
    # end to end through the public API with HOST buffers (pinned), one outer iteration per step
    if not args.no_e2e:
        hf = [torch.from_numpy(f.copy()).pin_memory() for f in F0]
        hl = torch.zeros(R, dtype=torch.float64).pin_memory()
        B.cstf_factorize_host(X, hf, hl, opts(1), comm=comm)
        ts = []
        for _ in range(K):
            for h, f in zip(hf, F0):
                h.numpy()[...] = f
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            a.record(stream)
            B.cstf_factorize_host(X, hf, hl, opts(1), comm=comm)
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        fac_bytes = sum(I * R * 8 for I in cfg.dims)
        e2e_s = float(np.mean(ts)) / 1e3
        if dist:                              # max over ranks, like the device-timed value
            t = torch.tensor([e2e_s], device="cpu" if host_comm else "cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_s = float(t.item())
        line["e2e"] = {"value": e2e_s, "unit": "s", "h2d_bytes_per_step": fac_bytes,
                       "d2h_bytes_per_step": fac_bytes + R * 8 + 8,
                       "note": "cstf_factorize_host: initial factors H2D, 1 outer iteration, factors+lambda+fit D2H"}
        # context: one K-iteration factorisation job through the same call (factors cross
        # PCIe once per job, the K fits are read back at the end), per outer iteration
        for h, f in zip(hf, F0):
            h.numpy()[...] = f
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(stream)
        B.cstf_factorize_host(X, hf, hl, opts(K), comm=comm)
        b.record(stream)
        torch.cuda.synchronize()
        job_s = a.elapsed_time(b) / 1e3
        if dist:
            t = torch.tensor([job_s], device="cpu" if host_comm else "cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            job_s = float(t.item())
        line["e2e_job"] = {"value": job_s / K, "unit": "s", "outer_iterations": K, "job_s": job_s,
                           "h2d_bytes_per_job": fac_bytes, "d2h_bytes_per_job": fac_bytes + R * 8 + 8 * K,
                           "note": "context, not the e2e key: cstf_factorize_host with outer_iters=K, per outer iteration"}
    if world == 1 and not args.no_streaming_probe:
        line["admm_update_gbs"]["streaming_v1"] = admm_streaming_probe(B, cfg, R, stream, peaks["hbm_gbs"])
    if args.ablation and world == 1:
        line["ablation"] = admm_ablation(B, cfg, R, stream)
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, cores, tco = oracle_outer_iteration(cfg, idx, vals, R, 1, 0)
        line["cpu_baseline"] = {"value": v, "unit": "s", "cores": cores, "kind": "oracle",
                                "sample": f"1 full outer iteration of {cfg.name} (eps=0, 10 inner), "
                                          f"FP64 C/OpenMP oracle; coalesce {tco:.1f}s excluded"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
