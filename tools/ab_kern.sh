# A/B of kernel builds (build/ab/*.so) on resident 512^3: conv3d and stencil7, both dtypes, interleaved
mkdir -p gpurun_out
LIBS=${LIBS:-"cfg0 hint"}
for rep in 1 2; do for lib in $LIBS; do for k in conv3d stencil7; do for d in f32 f64; do
  PP_LIBPPIPE=${LIBDIR:-build/ab}/$lib.so timeout 300 python tools/kernel_probe.py --kernel $k --paths tma --chunks 510,6 --dtype $d | sed "s/^/{\"lib\": \"$lib\", \"dtype\": \"$d\", \"rep\": $rep, \"r\": /; s/$/}/"
done; done; done; done > gpurun_out/${TAG:-r2}_kern_ab.jsonl 2>&1
