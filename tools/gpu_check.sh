#!/bin/bash
# gpurun: all GPU tests, time-to-optimal of C2/C3/C5(pinned 7,0) and the default bench line.
#   gpurun -- 'bash tools/gpu_check.sh TAG'
TAG=${1:-chk}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || { tail -20 $O/${TAG}_build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1
echo "pytest exit $?"; tail -3 $O/${TAG}_pytest_gpu.log
for cfg in C2 C3; do
  timeout 300 python tools/time_to_optimal.py $cfg > $O/${TAG}_tto_${cfg}.json 2>$O/${TAG}_tto_${cfg}.err
  echo "$cfg: $(python -c "import json,sys; d=json.load(open(sys.argv[1])); print({k: d[k] for k in ['time_to_optimal_s','device_ms','evaluator_ms','n_full_evals','cost','oracle_check']})" $O/${TAG}_tto_${cfg}.json 2>&1 | tail -1)"
done
timeout 300 python tools/time_to_optimal.py C5 --fixed 7,0 > $O/${TAG}_tto_C5p.json 2>&1
echo "C5p: $(python -c "import json,sys; d=json.load(open(sys.argv[1])); print({k: d[k] for k in ['time_to_optimal_s','device_ms','evaluator_ms','n_full_evals','cost','oracle_check']})" $O/${TAG}_tto_C5p.json 2>&1 | tail -1)"
timeout 900 python bench.py > $O/${TAG}_bench.log 2>&1; echo "bench exit $?"
python -c "
import json,sys
d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1])
print('value %.4g frac %.3f e2e %.4g' % (d['value'], d['roofline']['frac'], d['e2e']['value']), 'pruned', d['pruned'])
print({k: (v['time_to_optimal_s'], v.get('oracle_check')) for k, v in d['time_to_optimal_full_space'].items()})
print('c4', d['c4_sla_sweep_replanning']['replans_per_s'], 'launches', d['gpu_launches'], 'share', d['kernel_share_of_step'])
" $O/${TAG}_bench.log || tail -20 $O/${TAG}_bench.log
# per-kernel launch list of the C2 time-to-optimal plan (cold-cache, serialised: shares only)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file $O/${TAG}_tto_C2_launches.csv \
    python tools/time_to_optimal.py C2 > $O/${TAG}_tto_C2_ncu.log 2>&1; echo "ncu tto exit $?"
python tools/ncu_summary.py launches $O/${TAG}_tto_C2_launches.csv 2>&1 | head -20
