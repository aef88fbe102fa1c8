#!/usr/bin/env bash
# Per-mode MTTKRP / update times inside cstf_factorize (the bench path) under
# environment variants; one bench process per variant (load-time knobs apply).
# Usage (GPU box): tools/bench_variants.sh CONFIG "ENV=V ENV2=V" "ENV=W" ...
cfg=$1; shift
for v in "$@"; do
  env $v python bench.py --config "$cfg" --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-streaming-probe 2>/dev/null |
    python -c "
import json, sys
d = json.loads(sys.stdin.read().strip().splitlines()[-1])
r = d['roofline']['per_mode_ms']; u = d['roofline_admm']['per_mode_ms']
print('%-40s step %.2f ms  mttkrp %s  update %s  layout %s  clk %s' % ('$v', d['ms_per_step'],
      ' '.join('%.2f' % x for x in r), ' '.join('%.2f' % x for x in u),
      [l['nblk'] for l in d['setup']['layout']], d['clocks']['sm_mhz']))"
done
