#!/bin/bash
# ALU-pinned add sweep of the variants kernel (SMILESS_ALUG / SMILESS_ALUSUL masks), bench slice
mkdir -p gpurun_out
for cfg in "$@"; do
  set -- $cfg
  tag="ALUG$1_ALUSUL$2_S$3"
  SMILESS_ALUG=$1 SMILESS_ALUSUL=$2 SMILESS_SELMASK=$3 timeout 300 python bench.py --steps 3 --warmup 3 \
      --no-cpu-baseline --no-pruned --no-full-space --no-c4 > gpurun_out/sweepa_$tag.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[2], '%.4g' % d['value'], 'frac %.3f' % d['roofline']['frac'], d['winner']['index'], d['winner']['cost'])" gpurun_out/sweepa_$tag.log $tag || tail -5 gpurun_out/sweepa_$tag.log
done
