#!/bin/bash
# C5 time-to-optimal anatomy: host stage profile + kernel launch list; new fused tests
TAG=${1:-c5p}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
timeout 600 python -m pytest tests -m gpu -q -x -k "fused" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -2 $O/${TAG}_pytest.log
SMILESS_PROFILE_HOST=1 timeout 300 python tools/tto_full.py C5 > $O/${TAG}_tto.json 2> $O/${TAG}_tto.err; echo "tto exit $?"; tail -c 300 $O/${TAG}_tto.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv --log-file $O/${TAG}_launches.csv \
    python tools/tto_full.py C5 > $O/${TAG}_ncu.log 2>&1; echo "ncu exit $?"
