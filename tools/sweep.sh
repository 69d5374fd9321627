#!/bin/bash
# tuning sweep of the evaluator's launch/shape knobs on the bench workload (run under gpurun)
for cfg in "1 1 4" "1 2 4" "2 1 4" "2 2 4" "2 1 2" "2 2 2"; do
  set -- $cfg
  SMILESS_G=$1 SMILESS_MINB=$2 SMILESS_UNROLL=$3 timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-pruned > gpurun_out/sweep_G$1_M$2_U$3.log 2>&1
  python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[1], '%.4g' % d['value'], 'frac %.3f' % d['roofline']['frac'], d['winner']['index'])" gpurun_out/sweep_G$1_M$2_U$3.log
done
