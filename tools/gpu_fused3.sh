#!/bin/bash
# fused kernel occupancy sweep (CTAs/SM, ring depth, CTA size) against the two-kernel path
TAG=${1:-fu3}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
B="--no-cpu-baseline --no-pruned --no-full-space --no-c4 --no-extra"
run() {  # label, env...
  local lab=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 $B > $O/${TAG}_bench_$lab.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[2], 'value %.4g frac %.3f ms %.1f' % (d['value'], d['roofline']['frac'], d['ms_per_step']), d['clocks']['sm_mhz'], d['gpu_launches'], d['winner']['index'])" $O/${TAG}_bench_$lab.log $lab 2>&1 | tail -1
}
run f256x3s3 SMILESS_FUSED=1 SMILESS_FMINB=3 SMILESS_FSLOTS=3
run f256x3s2 SMILESS_FUSED=1 SMILESS_FMINB=3 SMILESS_FSLOTS=2
run f288x3s3 SMILESS_FUSED=1 SMILESS_FMINB=3 SMILESS_FSLOTS=3 SMILESS_VTHREADS=288
run f288x3s2 SMILESS_FUSED=1 SMILESS_FMINB=3 SMILESS_FSLOTS=2 SMILESS_VTHREADS=288
run f288x2s4 SMILESS_FUSED=1 SMILESS_FMINB=2 SMILESS_FSLOTS=4 SMILESS_VTHREADS=288
run f256x2s4 SMILESS_FUSED=1
run two_b1M SMILESS_FUSED=0 SMILESS_MEMO_BATCH=1048576
SMILESS_FUSED=1 SMILESS_FMINB=3 SMILESS_FSLOTS=3 SMILESS_FPROF=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"smiless_fused_kernel" -c 1 \
    -o $O/${TAG}_prof_fused -f python bench.py --steps 1 --warmup 0 $B > $O/${TAG}_ncu_full.log 2>&1; echo "ncu full exit $?"
