mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu -x -p no:cacheprovider > gpurun_out/r2o_pytest_gpu.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/r2o_pytest_gpu.log
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2o_launches.csv python bench.py --steps 3 --warmup 3 --ooc-steps 1 --ooc-verify last > gpurun_out/r2o_ncu_bench.log 2>&1; echo "ncu-list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:stencil7_tma -s 3 -c 1 -o gpurun_out/r2o_prof_stencil -f python bench.py --steps 3 --warmup 3 --ooc off --no-cpu --no-naive --no-schedules --no-triad --verify 0 > gpurun_out/r2o_ncu_full.log 2>&1; echo "ncu-full rc=$?"
