#!/bin/bash
TAG=${1:-r02g}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
bash tools/sanitize.sh 2>&1 | tee $O/${TAG}_sanitize_summary.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval_exact -c 1 -o $O/${TAG}_exact -f \
    python tools/tto_full.py C3 > $O/${TAG}_ncu_exact.log 2>&1; echo "ncu exact exit $?"
for c in C2 C3; do SMILESS_PROFILE_HOST=1 timeout 300 python tools/tto_full.py $c > $O/${TAG}_tto_$c.json 2> $O/${TAG}_tto_$c.err; tail -1 $O/${TAG}_tto_$c.err; done
