# Round-end evidence on one B200 (run from the repo root under gpurun): GPU suite,
# bench line, ncu launch list and the per-kernel DRAM traffic capture (summarised on the box;
# the .ncu-rep itself stays in /tmp).
mkdir -p gpurun_out
[ -n "$SKIP_TESTS" ] || { (time python -m pytest tests -m gpu -x -q) > gpurun_out/gputest.log 2>&1; tail -6 gpurun_out/gputest.log; }
# (compute-sanitizer: tools/sanitize_cases.py; the tool was closed on this pool late in round 2,
#  see DESIGN.md section 13)
python bench.py --steps 20 --warmup 3 > gpurun_out/bench_final.log 2>&1; tail -c 300 gpurun_out/bench_final.log
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02b_launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /tmp/ncu_launch.log 2>&1; echo launches rc=$?
ncu --set full --clock-control none -k regex:'k_mttkrp_fast|k_admm_dmma' -s 24 -c 8 -o /tmp/r02b_traffic python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /tmp/ncu_full.log 2>&1; echo full rc=$?
python tools/traffic_json.py /tmp/r02b_traffic.ncu-rep delicious gpurun_out/r02b_traffic.json "ncu --set full --clock-control none -k regex:'k_mttkrp_fast|k_admm_dmma' -s 24 -c 8 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e (packed records)"; echo traffic rc=$?
python tools/ncu_summary.py /tmp/r02b_traffic.ncu-rep > gpurun_out/r02b_ncu_delicious.txt 2>&1; echo summary rc=$?
ls -la gpurun_out
