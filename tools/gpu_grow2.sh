#!/bin/bash
TAG=${1:-gr2}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
for g in 16 64 256; do
  for c in "C2" "C2 --sla 4000000" "C2 --sla 8000000" "C3"; do
    for rep in 1 2 3; do
      SMILESS_BB_GROW=$g timeout 300 python tools/tto_full.py $c > $O/${TAG}_tmp.json 2>/dev/null
      python -c "import json,sys; d=json.load(open(sys.argv[1])); print('grow=$g', '$c', round(d['time_to_optimal_s']*1e3,1), 'ms', d['oracle_check']['cost_bits_equal'], d['full_evals'])" $O/${TAG}_tmp.json
    done
  done
done
