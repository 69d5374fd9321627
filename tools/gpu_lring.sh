#!/bin/bash
TAG=${1:-lr}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
timeout 1500 python -m pytest tests -m gpu -q -x -k "scale_out" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -4 $O/${TAG}_pytest.log
for l in 0 1; do SMILESS_LRING=$l timeout 300 python tools/tto_full.py C5 > $O/${TAG}_tto_C5_$l.json 2> $O/${TAG}_tto_C5_$l.err; echo "C5 lring=$l"; tail -c 400 $O/${TAG}_tto_C5_$l.json; done
SMILESS_LRING=1 timeout 600 python -c "
import bench, torch, json
from paper_conf_sc_luxl0y024_b200 import smiless as S
dev = torch.device('cuda:0'); st = torch.cuda.current_stream(dev)
print(json.dumps(bench.throughput_slice('C5', S, dev, st, 0)))
" > $O/${TAG}_slice_C5.json 2>&1; tail -c 600 $O/${TAG}_slice_C5.json
