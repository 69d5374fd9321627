#!/bin/bash
# smiless_plan_digits: parity tests, C5 time-to-optimal in one call vs one call per digit
TAG=${1:-dg}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
timeout 900 python -m pytest tests -m gpu -q -x -k "plan_digits or pinned or heavy_subplan" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -3 $O/${TAG}_pytest.log
for c in C5 C5s; do
  for m in "" "--per-digit"; do
    for rep in 1 2; do
      timeout 300 python tools/tto_full.py $c $m > $O/${TAG}_tmp.json 2>$O/${TAG}_tmp.err
      python -c "import json,sys; d=json.load(open(sys.argv[1])); print('$c', '$m', round(d['time_to_optimal_s']*1e3,1), 'ms', d['cost'], d.get('digit0'), d['oracle_check']['cost_bits_equal'], d['decided'], d['launches'])" $O/${TAG}_tmp.json || tail -3 $O/${TAG}_tmp.err
    done
  done
done
SMILESS_BENCH_FULL=C5,C5s timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-c4 --no-extra --no-pruned > $O/${TAG}_bench.log 2>&1; echo "bench exit $?"
python -c "
import json
d=json.loads([l for l in open('$O/${TAG}_bench.log') if l.startswith('{')][-1])
print({k: (round(v['time_to_optimal_s']*1e3,1), v['oracle_check'], v['digits'], v['candidates']) for k, v in d['time_to_optimal_full_space'].items()})"
