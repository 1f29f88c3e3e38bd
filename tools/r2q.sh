mkdir -p gpurun_out
timeout 600 python tools/triad_probe.py --diag --reps 20 > gpurun_out/r2q_triad_diag.jsonl 2> gpurun_out/r2q_triad_diag.err; echo "triad rc=$?"
python3 - <<'PY'
import json
for l in open('gpurun_out/r2q_triad_diag.jsonl'):
    d=json.loads(l)
    if d['case']!='diag': continue
    print(d['policy'],d['graph'],d['sm_copy'],d['chunk'],d['streams'],round(d['events_median_ms']*1e3,1),round(d['lib_median_ms']*1e3,1))
PY
