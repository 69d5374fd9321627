#!/bin/bash
# anatomy of the live-window instance C2 at SLA 8 s: host stages + kernel launch list
TAG=${1:-c2s8}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
for rep in 1 2 3; do
  SMILESS_PROFILE_HOST=1 timeout 300 python tools/tto_full.py C2 --sla 8000000 > $O/${TAG}_tto$rep.json 2> $O/${TAG}_tto$rep.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(round(d['time_to_optimal_s']*1e3,1), 'ms', d['full_evals'], d['launches'])" $O/${TAG}_tto$rep.json
  grep "smiless host" $O/${TAG}_tto$rep.err | tail -1 | cut -c1-600
done
for first in 16 256 4096; do
  SMILESS_BB_FIRST=$first timeout 300 python tools/tto_full.py C2 --sla 8000000 > $O/${TAG}_f.json 2>/dev/null
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print('first $first', round(d['time_to_optimal_s']*1e3,1), 'ms', d['full_evals'])" $O/${TAG}_f.json
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file $O/${TAG}_launches.csv \
    python tools/tto_full.py C2 --sla 8000000 > $O/${TAG}_ncu.log 2>&1; echo "ncu exit $?"
