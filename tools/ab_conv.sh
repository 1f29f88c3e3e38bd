# A/B of conv3d kernel builds (abl/*.so via PP_LIBPPIPE) on resident 512^3, interleaved; then the conv parity tests
# usage (under gpurun): TAG=x LIBS="a b" DTYPES="f32 f64" TLIBS="b" bash tools/ab_conv.sh
mkdir -p gpurun_out
for rep in 1 2 3; do for lib in ${LIBS:-base new}; do for d in ${DTYPES:-f32}; do
  PP_LIBPPIPE=abl/$lib.so timeout 300 python tools/kernel_probe.py --kernel conv3d --paths tma --chunks 510 --dtype $d | sed "s/^/{\"lib\": \"$lib\", \"dtype\": \"$d\", \"rep\": $rep, \"r\": /; s/$/}/"
done; done; done > gpurun_out/${TAG}_conv_ab.jsonl 2>&1
for lib in ${TLIBS:-}; do PP_LIBPPIPE=abl/$lib.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_oracle.py -q -x -k "conv" -p no:cacheprovider > gpurun_out/${TAG}_pytest_conv_$lib.log 2>&1; echo "conv tests $lib rc=$?"; tail -1 gpurun_out/${TAG}_pytest_conv_$lib.log; done
