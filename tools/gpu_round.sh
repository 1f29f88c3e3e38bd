#!/bin/bash
# One GPU session: parity tests, smoke, bench, sweep, ncu launch list + full capture of the stencil.
# usage (under gpurun): bash tools/gpu_round.sh <tag> [sections...]
set -u
TAG=${1:-r}
shift || true
SECTIONS=${@:-"smoke tests bench sweep ncu"}
mkdir -p gpurun_out
for s in $SECTIONS; do
  case $s in
    smoke) timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" ;;
    tests) timeout 1500 python -m pytest tests -q -m gpu -x -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/${TAG}_pytest_gpu.log ;;
    bench) timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"; cat gpurun_out/${TAG}_bench.json | head -c 3000; echo ;;
    sweep) timeout 900 python tools/sweep.py --reps 3 --chunks 1,2,4,8,16,32,64 --streams 2,3,4,6 --policies 0,1,2 --graphs 0 > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err; echo "sweep rc=$?" ;;
    ooc64) timeout 900 python tests/ooc_run.py --gb 64 > gpurun_out/${TAG}_ooc64.json 2> gpurun_out/${TAG}_ooc64.err; echo "ooc64 rc=$?"; cat gpurun_out/${TAG}_ooc64.json ;;
    oocfull) timeout 1500 python tests/ooc_run.py --gb auto > gpurun_out/${TAG}_ooc.json 2> gpurun_out/${TAG}_ooc.err; echo "ooc rc=$?"; cat gpurun_out/${TAG}_ooc.json ;;
    sweep34) timeout 900 python tools/sweep.py --reps 3 --chunks 1,2,4,8,16 --streams 2,3,4,6 --policies 0,1,3,4 --graphs 0 > gpurun_out/${TAG}_sweep34.jsonl 2> gpurun_out/${TAG}_sweep34.err; echo "sweep34 rc=$?" ;;
    torchrun) timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu --no-schedules > gpurun_out/${TAG}_torchrun1.json 2> gpurun_out/${TAG}_torchrun1.err; echo "torchrun rc=$?"; head -c 600 gpurun_out/${TAG}_torchrun1.json; echo;
         PP_BENCH_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu --no-schedules --no-naive > gpurun_out/${TAG}_torchrun2share.json 2> gpurun_out/${TAG}_torchrun2share.err; echo "torchrun2 (shared gpu) rc=$?"; head -c 700 gpurun_out/${TAG}_torchrun2share.json; echo;
         timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_reference.json 2>&1; echo "reference rc=$?"; head -c 800 gpurun_out/${TAG}_reference.json; echo ;;
    sanitize) for tool in memcheck racecheck synccheck; do timeout 900 compute-sanitizer --tool $tool --error-exitcode 7 python tests/sanitize_cases.py > gpurun_out/${TAG}_sanitize_$tool.log 2>&1; echo "sanitize $tool rc=$?"; tail -3 gpurun_out/${TAG}_sanitize_$tool.log; done ;;
    temporal) timeout 900 python tools/temporal.py > gpurun_out/${TAG}_temporal.jsonl 2> gpurun_out/${TAG}_temporal.err; echo "temporal rc=$?"; cat gpurun_out/${TAG}_temporal.jsonl | cut -c1-400 ;;
    cupti) for cfg in "6 1 1 0" "2 3 1 0" "16 3 1 0"; do set -- $cfg;
         timeout 300 python tools/cupti_timeline.py --c $1 --S $2 --policy $3 --graph $4 --out gpurun_out/${TAG}_cupti_c$1S$2p$3g$4.json > gpurun_out/${TAG}_cupti_c$1S$2p$3g$4.jsonl 2>/dev/null; echo "cupti c=$1 S=$2 rc=$?"; done ;;
    timeline) for cfg in "6 1 1" "2 3 1" "16 3 1"; do set -- $cfg;
         timeout 300 python tools/timeline.py --c $1 --S $2 --policy $3 --out gpurun_out/${TAG}_timeline_c$1S$2p$3.json; done ;;
    ncu) timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu --no-naive --no-schedules --no-triad --no-temporal --ooc off --verify 0 > gpurun_out/${TAG}_ncu_bench.log 2>&1; echo "ncu-list rc=$?";
         timeout 900 ncu --set full --clock-control none --import-source on -k regex:stencil7_tma -s 3 -c 1 -o gpurun_out/${TAG}_prof -f python bench.py --steps 3 --warmup 3 --no-cpu --no-naive --no-schedules --no-triad --no-temporal --ooc off --verify 0 > gpurun_out/${TAG}_ncu_full.log 2>&1; echo "ncu-full rc=$?" ;;
    triad) timeout 600 python tools/triad_probe.py > gpurun_out/${TAG}_triad.jsonl 2> gpurun_out/${TAG}_triad.err; echo "triad rc=$?"; cut -c1-600 gpurun_out/${TAG}_triad.jsonl ;;
    ncu_kernels) timeout 600 ncu --set full --clock-control none --import-source on -k regex:triad -s 3 -c 1 -o gpurun_out/${TAG}_prof_triad -f python tools/triad_probe.py --reps 1 > gpurun_out/${TAG}_ncu_triad.log 2>&1; echo "ncu triad rc=$?";
         timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv3d_tma -s 1 -c 1 -o gpurun_out/${TAG}_prof_conv_tma -f python tools/kernel_probe.py --kernel conv3d --paths tma --chunks 510 --dtype f64 > gpurun_out/${TAG}_ncu_conv_tma.log 2>&1; echo "ncu conv tma rc=$?";
         timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv3d_generic -s 1 -c 1 -o gpurun_out/${TAG}_prof_conv_gen -f python tools/kernel_probe.py --kernel conv3d --paths generic --chunks 510 --dtype f64 > gpurun_out/${TAG}_ncu_conv_gen.log 2>&1; echo "ncu conv generic rc=$?";
         timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv3d_tma -s 1 -c 1 -o gpurun_out/${TAG}_prof_conv_tma32 -f python tools/kernel_probe.py --kernel conv3d --paths tma --chunks 510 --dtype f32 > gpurun_out/${TAG}_ncu_conv_tma32.log 2>&1; echo "ncu conv tma f32 rc=$?" ;;
  esac
done
