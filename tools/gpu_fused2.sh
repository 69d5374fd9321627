#!/bin/bash
# fused kernel: launch list + full ncu capture; two-kernel memo batch sweep
TAG=${1:-fu2}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
B="--no-cpu-baseline --no-pruned --no-full-space --no-c4 --no-extra"
run() {  # label, env...
  local lab=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 $B > $O/${TAG}_bench_$lab.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[2], 'value %.4g frac %.3f ms %.1f' % (d['value'], d['roofline']['frac'], d['ms_per_step']), d['clocks']['sm_mhz'], d['gpu_launches'], d['winner']['index'])" $O/${TAG}_bench_$lab.log $lab 2>&1 | tail -1
}
for b in 131072 262144 524288 1048576 2097152; do run two_b$b SMILESS_FUSED=0 SMILESS_MEMO_BATCH=$b; done
run fused SMILESS_FUSED=1
SMILESS_FUSED=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/${TAG}_launches_fused.csv \
    python bench.py --steps 2 --warmup 1 $B > $O/${TAG}_ncu_launch.log 2>&1; echo "ncu launches exit $?"
SMILESS_FUSED=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"smiless_(fused|plan)_kernel" -c 2 \
    -o $O/${TAG}_prof_fused -f python bench.py --steps 1 --warmup 0 $B > $O/${TAG}_ncu_full.log 2>&1; echo "ncu full exit $?"
