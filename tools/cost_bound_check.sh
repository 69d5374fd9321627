#!/bin/bash
# gpurun: cost-bound pruning check -- GPU parity of the pruned paths + time-to-optimal with the
# cost bound on and off.   gpurun -- 'bash tools/cost_bound_check.sh TAG'
TAG=${1:-cb}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || { tail -20 $O/${TAG}_build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q -k "cost or c1_plan or bench_configuration or branch_and_bound or plan_parity or ties or stream_compaction or derived or top1 or decompose or random_dags_exhaustive" > $O/${TAG}_pytest.log 2>&1
echo "pytest exit $?"; tail -3 $O/${TAG}_pytest.log
for cfg in C2 C3; do
  for cp in 0 1; do
    SMILESS_COST_PRUNE=$cp timeout 300 python tools/time_to_optimal.py $cfg > $O/${TAG}_tto_${cfg}_cp${cp}.json 2>$O/${TAG}_tto_${cfg}_cp${cp}.err
    echo "$cfg cp=$cp: $(python -c "import json,sys; d=json.load(open(sys.argv[1])); print(round(d['time_to_optimal_s'],4), d['n_full_evals'], d['cost'], d.get('oracle_check'))" $O/${TAG}_tto_${cfg}_cp${cp}.json 2>&1 | tail -1)"
  done
done
for cp in 0 1; do
  SMILESS_COST_PRUNE=$cp timeout 300 python tools/time_to_optimal.py C5 --fixed 7,0 > $O/${TAG}_tto_C5p_cp${cp}.json 2>&1
  echo "C5 pinned 7,0 cp=$cp: $(python -c "import json,sys; d=json.load(open(sys.argv[1])); print(round(d['time_to_optimal_s'],4), d['n_full_evals'], d['cost'], d.get('oracle_check'))" $O/${TAG}_tto_C5p_cp${cp}.json 2>&1 | tail -1)"
done
