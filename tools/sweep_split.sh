#!/bin/bash
# split-cost (SMILESS_SPLITCOST) on/off on the bench slice + the memoisation parity tests
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for sc in 1 0 1 0; do
  SMILESS_SPLITCOST=$sc timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-pruned --no-full-space --no-c4 > gpurun_out/sws_$sc.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print('SPLITCOST', sys.argv[2], '%.4g' % d['value'], 'frac %.3f' % d['roofline']['frac'], d['winner']['index'], d['winner']['cost'], 'launches', d['gpu_launches'])" gpurun_out/sws_$sc.log $sc || tail -5 gpurun_out/sws_$sc.log
done
timeout 900 python -m pytest tests -m gpu -q -x -k "memo or bench_configuration or sla_sweep or derived" 2>&1 | tail -1
