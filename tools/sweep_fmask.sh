#!/bin/bash
# gpurun: bench throughput line for several positive-time variant masks (SMILESS_FMASK)
O=gpurun_out; TAG=${1:-fm}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || { tail -20 $O/${TAG}_build.log; exit 1; }
for m in 0 0x54 0xaa 0x14 0x56 0xfe; do
  SMILESS_FMASK=$m timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-pruned --no-full-space --no-c4 --no-extra > $O/${TAG}_bench_$m.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print('FMASK', sys.argv[2], 'value %.4g frac %.3f' % (d['value'], d['roofline']['frac']), d['clocks']['sm_mhz'])" $O/${TAG}_bench_$m.log $m || tail -3 $O/${TAG}_bench_$m.log
done
