#!/bin/bash
TAG=${1:-dg2}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
for c in C5 C5s; do
  for cfg in "def def" "3 6" "3 5" "3 def"; do set -- $cfg
    E=""; [ $1 != def ] && E="$E SMILESS_BB_DEPTH_A=$1"; [ $2 != def ] && E="$E SMILESS_BB_DEPTH_M=$2"
    for rep in 1 2; do
      env $E timeout 300 python tools/tto_full.py $c > $O/${TAG}_tmp.json 2>$O/${TAG}_tmp.err
      python -c "import json,sys; d=json.load(open(sys.argv[1])); print('$c', 'DA=$1 DM=$2', round(d['time_to_optimal_s']*1e3,1), 'ms', d['oracle_check']['cost_bits_equal'], d['full_evals'])" $O/${TAG}_tmp.json || tail -3 $O/${TAG}_tmp.err
    done
  done
done
SMILESS_PROFILE_HOST=1 timeout 300 python tools/tto_full.py C5 > $O/${TAG}_prof.json 2> $O/${TAG}_prof.err
