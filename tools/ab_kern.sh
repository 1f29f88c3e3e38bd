# A/B of kernel builds (abl/*.so, PP_LIBPPIPE) on resident 512^3, interleaved; then the stencil parity tests
# usage (under gpurun): TAG=x LIBS="a b" KERNELS="stencil7" DTYPES="f64 f32" TLIBS="b" bash tools/ab_kern.sh
mkdir -p gpurun_out
for rep in 1 2 3; do for lib in ${LIBS:-base new}; do for k in ${KERNELS:-stencil7}; do for d in ${DTYPES:-f64 f32}; do
  PP_LIBPPIPE=${LIBDIR:-abl}/$lib.so timeout 300 python tools/kernel_probe.py --kernel $k --paths tma --chunks 510,6 --dtype $d | sed "s/^/{\"lib\": \"$lib\", \"k\": \"$k\", \"dtype\": \"$d\", \"rep\": $rep, \"r\": /; s/$/}/"
done; done; done; done > gpurun_out/${TAG:-r2}_kern_ab.jsonl 2>&1
for lib in ${TLIBS:-}; do PP_LIBPPIPE=${LIBDIR:-abl}/$lib.so timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "${TESTK:-stencil or tma or chain or sweeps}" -p no:cacheprovider > gpurun_out/${TAG:-r2}_pytest_$lib.log 2>&1; echo "tests $lib rc=$?"; tail -1 gpurun_out/${TAG:-r2}_pytest_$lib.log; done
