#!/bin/bash
TAG=${1:-fs}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
B="--no-cpu-baseline --no-pruned --no-full-space --no-c4 --no-extra"
run() {
  local lab=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 $B > $O/${TAG}_bench_$lab.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[2], 'value %.4g frac %.3f ms %.1f' % (d['value'], d['roofline']['frac'], d['ms_per_step']), d['clocks']['sm_mhz'])" $O/${TAG}_bench_$lab.log $lab 2>&1 | tail -1
}
run default SMILESS_NOP=1
run slots3 SMILESS_FSLOTS=3
run slots6 SMILESS_FSLOTS=6
run slots8 SMILESS_FSLOTS=8
run fpw2 SMILESS_FPW=2 SMILESS_FTHREADS=576
run default2 SMILESS_NOP=1
for rep in 1 2; do
  SMILESS_PROFILE_HOST=1 timeout 300 python tools/tto_full.py C3 > $O/${TAG}_c3.json 2> $O/${TAG}_c3.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print('C3', round(d['time_to_optimal_s']*1e3,1), 'ms', d['full_evals'])" $O/${TAG}_c3.json
  grep "smiless host" $O/${TAG}_c3.err | tail -1 | cut -c1-400
done
