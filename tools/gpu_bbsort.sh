#!/bin/bash
TAG=${1:-bs}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
for srt in 0 1; do
  for c in "C2" "C2 --sla 4000000" "C2 --sla 8000000" "C3" "C5"; do
    for rep in 1 2; do
      SMILESS_BB_SORT=$srt timeout 300 python tools/tto_full.py $c > $O/${TAG}_tmp.json 2>/dev/null
      python -c "import json,sys; d=json.load(open(sys.argv[1])); print('sort=$srt', '$c', 'rep $rep', round(d['time_to_optimal_s']*1e3,1), 'ms', d['cost'], d['oracle_check']['cost_bits_equal'], d['full_evals'])" $O/${TAG}_tmp.json
    done
  done
done
timeout 1200 python -m pytest tests -m gpu -q -x -k "branch_and_bound or cost_bound or cost_cap or full_space or heavy_subplan or window0" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -3 $O/${TAG}_pytest.log
