#!/bin/bash
# development GPU pass: build, FMASK sweep, a test selection, scale-out time-to-optimal.
#   gpurun --timeout 2700 -- 'bash tools/gpu_dev.sh TAG "pytest -k expr"'
TAG=${1:-dev}; K=${2:-}
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
for m in 0 0x54 0xaa 0x14 0x56 0xfe; do
  SMILESS_FMASK=$m timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-pruned --no-full-space --no-c4 --no-extra > $O/${TAG}_bench_$m.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print('FMASK', sys.argv[2], 'value %.4g frac %.3f' % (d['value'], d['roofline']['frac']), d['clocks']['sm_mhz'])" $O/${TAG}_bench_$m.log $m 2>&1 | tail -1
done
for c in C3 C5; do
  timeout 400 python tools/tto_full.py $c > $O/${TAG}_tto_$c.json 2> $O/${TAG}_tto_$c.err; echo "tto $c exit $?"; tail -c 700 $O/${TAG}_tto_$c.json; tail -3 $O/${TAG}_tto_$c.err
done
if [ -n "$K" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -k "$K" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -6 $O/${TAG}_pytest.log
fi
