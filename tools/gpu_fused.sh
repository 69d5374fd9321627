#!/bin/bash
# fused producer/consumer memo kernel: parity tests, then bench fused vs two-kernel paths
TAG=${1:-fu}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
SMILESS_FUSED=1 timeout 900 python -m pytest tests -m gpu -q -x -k "fused or memo or throughput_mode or split_cost or bench_configuration" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -4 $O/${TAG}_pytest.log
run() {  # label, env...
  local lab=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-pruned --no-full-space --no-c4 --no-extra > $O/${TAG}_bench_$lab.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print(sys.argv[2], 'value %.4g frac %.3f ms %.1f' % (d['value'], d['roofline']['frac'], d['ms_per_step']), d['clocks']['sm_mhz'], d['gpu_launches'], d['winner']['index'], d['winner']['cost'])" $O/${TAG}_bench_$lab.log $lab 2>&1 | tail -1
}
run fused SMILESS_FUSED=1
run two SMILESS_FUSED=0
run fused_split0 SMILESS_FUSED=1 SMILESS_SPLITCOST=0
run two_split0 SMILESS_FUSED=0 SMILESS_SPLITCOST=0
run two_b262144 SMILESS_FUSED=0 SMILESS_MEMO_BATCH=262144
run fused_vt288 SMILESS_FUSED=1 SMILESS_VTHREADS=288
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"smiless_(fused|plan)_kernel" -c 2 \
    -o $O/${TAG}_prof -f python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-full-space --no-c4 --no-pruned --no-extra \
    > $O/${TAG}_ncu.log 2>&1; echo "ncu exit $?"
