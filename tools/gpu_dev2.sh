#!/bin/bash
# gpurun: scale-out time-to-optimal + a test selection
TAG=${1:-dev}; K=${2:-}
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
for c in C3 C5; do
  SMILESS_PROFILE_HOST=1 timeout 300 python tools/tto_full.py $c ${3:-} > $O/${TAG}_tto_$c.json 2> $O/${TAG}_tto_$c.err; echo "tto $c exit $?"; tail -c 900 $O/${TAG}_tto_$c.json; tail -2 $O/${TAG}_tto_$c.err | cut -c1-300
done
if [ -n "$K" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -x -k "$K" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -6 $O/${TAG}_pytest.log
fi
