#!/bin/bash
for cfg in "0 256" "1 256" "1 384" "1 320"; do
  set -- $cfg
  SMILESS_MEMO=$1 SMILESS_VTHREADS=$2 timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-pruned --no-full-space --no-c4 > gpurun_out/sweep_memo$1_t$2.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[1], '%.4g' % d['value'], 'frac %.3f' % d['roofline']['frac'], d['winner']['index'], d['winner']['cost'])" gpurun_out/sweep_memo$1_t$2.log || tail -5 gpurun_out/sweep_memo$1_t$2.log
done
