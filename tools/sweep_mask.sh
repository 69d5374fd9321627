#!/bin/bash
for m in 0 1 2 3 4 5 6 7; do
  SMILESS_MASK=$m timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-pruned --no-full-space --no-c4 > gpurun_out/sweep_mask$m.log 2>&1
  python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[1], '%.4g' % d['value'], 'frac %.3f' % d['roofline']['frac'], d['winner']['index'])" gpurun_out/sweep_mask$m.log
done
