mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do timeout 900 compute-sanitizer --tool $tool --error-exitcode 7 python tests/sanitize_cases.py > gpurun_out/r2p_sanitize_$tool.log 2>&1; echo "sanitize $tool rc=$?"; tail -3 gpurun_out/r2p_sanitize_$tool.log; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2p_launches.csv python bench.py --steps 3 --warmup 3 --ooc off --no-schedules --no-naive --no-cpu > gpurun_out/r2p_ncu_bench.log 2>&1; echo "ncu-list rc=$?"
timeout 600 python tools/triad_probe.py --diag --reps 20 > gpurun_out/r2p_triad_diag.jsonl 2> gpurun_out/r2p_triad_diag.err; echo "triad rc=$?"
