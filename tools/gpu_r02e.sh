#!/bin/bash
TAG=${1:-r02e}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); print('build ok')" > $O/${TAG}_build.log 2>&1; tail -1 $O/${TAG}_build.log
timeout 1500 python -m pytest tests -m gpu -q -k "decompose or evaluate or exact or device_view or c1_ or golden or window0 or smoke or top1" > $O/${TAG}_pytest.log 2>&1; echo "pytest exit $?"; tail -4 $O/${TAG}_pytest.log
for c in C2 C3; do SMILESS_PROFILE_HOST=1 timeout 300 python tools/tto_full.py $c > $O/${TAG}_tto_$c.json 2> $O/${TAG}_tto_$c.err; tail -c 300 $O/${TAG}_tto_$c.json; tail -1 $O/${TAG}_tto_$c.err; done
timeout 900 python tools/next_compare.py C1 C2 C3 C5 C4_4 > $O/${TAG}_next_vs_opt.jsonl 2> $O/${TAG}_next.err; echo "next exit $?"; tail -3 $O/${TAG}_next.err
SMILESS_BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --no-cpu-baseline --no-c4 --no-extra > $O/${TAG}_bench_2rank.log 2>&1
echo "2-rank exit $?"; python -c "
import json,sys
d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1])
print('2rank value %.4g' % d['value'], {k: (round(v['time_to_optimal_s'],4), v.get('oracle_check',{}).get('cost_bits_equal'), v['decided_per_rank'], v.get('digits')) for k, v in d['time_to_optimal_full_space'].items()})
" $O/${TAG}_bench_2rank.log || tail -20 $O/${TAG}_bench_2rank.log
