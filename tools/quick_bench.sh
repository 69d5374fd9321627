#!/bin/bash
# quick check under gpurun: throughput-mode bench line + one ncu --set full capture of the
# variants kernel.  usage: bash tools/quick_bench.sh TAG [extra bench args]
TAG=${1:-q}; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -20 gpurun_out/${TAG}_build.log; exit 1; }
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-pruned --no-full-space --no-c4 "$@" > gpurun_out/${TAG}_bench.log 2>&1
python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print('value %.4g' % d['value'], 'frac %.3f' % d['roofline']['frac'], d['winner'])" gpurun_out/${TAG}_bench.log || tail -5 gpurun_out/${TAG}_bench.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"smiless_(variants|upstream)_kernel" -c 2 \
    -o gpurun_out/${TAG}_prof -f python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-full-space --no-c4 --no-pruned \
    > gpurun_out/${TAG}_ncu.log 2>&1; echo "ncu exit $?"
