#!/bin/bash
# three-level B&B: parity tests, then time-to-optimal with and without the middle level
TAG=${1:-bb3}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
for dm in auto 0; do
  for c in "C5" "C3" "C5s" "C3s" "C2 --sla 8000000"; do
    if [ $dm = auto ]; then E=""; else E="SMILESS_BB_DEPTH_M=0"; fi
    env $E timeout 300 python tools/tto_full.py $c > $O/${TAG}_tmp.json 2>$O/${TAG}_tmp.err
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print('dm=$dm', '$c', round(d['time_to_optimal_s']*1e3,1), 'ms', d['cost'], d['oracle_check']['cost_bits_equal'], d['full_evals'])" $O/${TAG}_tmp.json || tail -3 $O/${TAG}_tmp.err
  done
done
timeout 1800 python -m pytest tests -m gpu -q -x -k "branch_and_bound or full_space or heavy_subplan or cost_bound or cost_cap or window0 or scale_out or derived_window_c2 or decompose_plan or fused" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -3 $O/${TAG}_pytest.log
SMILESS_PROFILE_HOST=1 timeout 300 python tools/tto_full.py C5 > $O/${TAG}_c5.json 2> $O/${TAG}_c5.err; echo "c5 prof exit $?"
