# A/B of conv3d kernel builds (build/ab/*.so) on resident 512^3, interleaved; then conv parity tests
mkdir -p gpurun_out
LIBS=${LIBS:-"base fma pair"}
for rep in 1 2; do for lib in $LIBS; do for d in f32 f64; do
  PP_LIBPPIPE=${LIBDIR:-build/ab}/$lib.so timeout 300 python tools/kernel_probe.py --kernel conv3d --paths tma --chunks 510,8 --dtype $d | sed "s/^/{\"lib\": \"$lib\", \"dtype\": \"$d\", \"rep\": $rep, \"r\": /; s/$/}/"
done; done; done > gpurun_out/${TAG:-r2}_conv_ab.jsonl 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "conv3d or halo" > gpurun_out/${TAG:-r2}_pytest_conv.log 2>&1; echo "conv/halo tests rc=$?"; tail -2 gpurun_out/${TAG:-r2}_pytest_conv.log
