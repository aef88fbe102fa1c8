#!/usr/bin/env bash
# Profiling recipe used for profiles/ (run under gpurun on one B200, from the repo root).
# Numbers printed by runs under ncu are never bench values.
set -euo pipefail
mkdir -p gpurun_out
CFG=${1:-nell2}
# 1. every launch with its device time (cold-cache, serialised: compare shares)
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${CFG}.csv \
    python bench.py --config "$CFG" --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null
# 2. full capture of the dominant kernels (skip the first launches of the warm-up)
ncu --set full --clock-control none --import-source on -k regex:k_mttkrp_fast -s 3 -c 1 \
    -o gpurun_out/prof_mttkrp_${CFG} \
    python bench.py --config "$CFG" --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null
ncu --set full --clock-control none --import-source on -k regex:k_admm_dmma -s 3 -c 1 \
    -o gpurun_out/prof_admm_${CFG} \
    python bench.py --config "$CFG" --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null
# here (no GPU): python tools/ncu_summary.py gpurun_out/prof_*.ncu-rep
