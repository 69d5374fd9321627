#!/bin/bash
# Launch-shape / pipe-balance sweep of the memoised variants kernel on the bench workload
# (run under gpurun): G (configs per lane), CTA size, min CTAs/SM, select mask.
mkdir -p gpurun_out
for cfg in "$@"; do
  set -- $cfg
  tag="G$1_T$2_M$3_S$4"
  SMILESS_G=$1 SMILESS_VTHREADS=$2 SMILESS_VMINB=$3 SMILESS_SELMASK=$4 timeout 300 python bench.py --steps 3 --warmup 3 \
      --no-cpu-baseline --no-pruned --no-full-space --no-c4 > gpurun_out/sweepv_$tag.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[2], '%.4g' % d['value'], 'frac %.3f' % d['roofline']['frac'], d['winner']['index'], d['winner']['cost'])" gpurun_out/sweepv_$tag.log $tag || tail -5 gpurun_out/sweepv_$tag.log
done
