#!/bin/bash
# fused kernel with several producer warps (SMSP balance): parity under each shape, then bench
TAG=${1:-fu4}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
B="--no-cpu-baseline --no-pruned --no-full-space --no-c4 --no-extra"
for cfg in "640 1 4" "576 1 2"; do set -- $cfg
  SMILESS_VTHREADS=$1 SMILESS_FMINB=$2 SMILESS_FPW=$3 timeout 600 python -m pytest tests -m gpu -q -x -k "fused" > $O/${TAG}_pytest_$1_$3.log 2>&1; echo "pytest $cfg exit $?"; tail -2 $O/${TAG}_pytest_$1_$3.log
done
run() {  # label, env...
  local lab=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 $B > $O/${TAG}_bench_$lab.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[2], 'value %.4g frac %.3f ms %.1f' % (d['value'], d['roofline']['frac'], d['ms_per_step']), d['clocks']['sm_mhz'], d['gpu_launches'], d['winner']['index'])" $O/${TAG}_bench_$lab.log $lab 2>&1 | tail -1
}
run f640x1p4 SMILESS_FUSED=1 SMILESS_VTHREADS=640 SMILESS_FMINB=1 SMILESS_FPW=4
run f576x1p2 SMILESS_FUSED=1 SMILESS_VTHREADS=576 SMILESS_FMINB=1 SMILESS_FPW=2
run f512x1p2 SMILESS_FUSED=1 SMILESS_VTHREADS=512 SMILESS_FMINB=1 SMILESS_FPW=2
run f320x2p2 SMILESS_FUSED=1 SMILESS_VTHREADS=320 SMILESS_FMINB=2 SMILESS_FPW=2
run f640x1p4s3 SMILESS_FUSED=1 SMILESS_VTHREADS=640 SMILESS_FMINB=1 SMILESS_FPW=4 SMILESS_FSLOTS=3
run f256x2p1 SMILESS_FUSED=1
run two_b1M SMILESS_FUSED=0 SMILESS_MEMO_BATCH=1048576
SMILESS_FUSED=1 SMILESS_VTHREADS=640 SMILESS_FMINB=1 SMILESS_FPW=4 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"smiless_fused_kernel" -c 1 \
    -o $O/${TAG}_prof_fused -f python bench.py --steps 1 --warmup 0 $B > $O/${TAG}_ncu_full.log 2>&1; echo "ncu full exit $?"
