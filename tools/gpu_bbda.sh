#!/bin/bash
# shallow-level depth sweep with the middle level (C5/C5s pinned digits, C3)
TAG=${1:-bbda}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
for c in C5 C5s C3; do
  for cfg in "def def" "3 def" "3 5" "3 6" "2 def" "2 4"; do set -- $cfg
    E=""; [ $1 != def ] && E="$E SMILESS_BB_DEPTH_A=$1"; [ $2 != def ] && E="$E SMILESS_BB_DEPTH_M=$2"
    env $E timeout 300 python tools/tto_full.py $c > $O/${TAG}_tmp.json 2>$O/${TAG}_tmp.err
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print('$c', 'DA=$1 DM=$2', round(d['time_to_optimal_s']*1e3,1), 'ms', d['cost'], d['oracle_check']['cost_bits_equal'], d['full_evals'], d.get('per_digit_ms'))" $O/${TAG}_tmp.json 2>/dev/null || { echo "$c $cfg failed"; tail -2 $O/${TAG}_tmp.err; }
  done
done
