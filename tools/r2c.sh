mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu -x -p no:cacheprovider > gpurun_out/r2c_pytest_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r2c_pytest_gpu.log
for d in f32 f64; do timeout 300 python tools/kernel_probe.py --kernel conv3d --paths tma --chunks 510,8 --dtype $d; done > gpurun_out/r2c_conv_probe.jsonl 2>&1; cat gpurun_out/r2c_conv_probe.jsonl
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv3d_tma -s 3 -c 1 -o gpurun_out/r2c_conv32 -f python tools/kernel_probe.py --kernel conv3d --paths tma --chunks 510 --dtype f32 > gpurun_out/r2c_ncu_conv32.log 2>&1; echo "ncu rc=$?"
