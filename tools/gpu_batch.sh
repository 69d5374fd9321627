#!/bin/bash
# memo batch-size and split-cost sweep on the bench slice (C2, 2^28 candidates)
TAG=${1:-mb}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
run() {  # label, env...
  local lab=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-pruned --no-full-space --no-c4 --no-extra > $O/${TAG}_bench_$lab.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[2], 'value %.4g frac %.3f ms %.1f' % (d['value'], d['roofline']['frac'], d['ms_per_step']), d['clocks']['sm_mhz'], d['gpu_launches'])" $O/${TAG}_bench_$lab.log $lab 2>&1 | tail -1
}
run base SMILESS_NOP=1
for b in 32768 131072 262144 524288; do run b$b SMILESS_MEMO_BATCH=$b; done
run split0 SMILESS_SPLITCOST=0
run split0_b262144 SMILESS_SPLITCOST=0 SMILESS_MEMO_BATCH=262144
