#!/bin/bash
# round-2 GPU pass: build, new sharding tests first, then the whole GPU suite, smoke, bench,
# and the 2-rank same-GPU flow.   gpurun --timeout 2400 -- 'bash tools/gpu_r02.sh TAG [pytest -k expr]'
TAG=${1:-r02}
K=${2:-}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || { tail -20 $O/${TAG}_build.log; exit 1; }
if [ -n "$K" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q -k "$K" > $O/${TAG}_pytest_sel.log 2>&1; echo "pytest sel exit $?"; tail -5 $O/${TAG}_pytest_sel.log
fi
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest gpu exit $?"; tail -5 $O/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke exit $?"; tail -2 $O/${TAG}_smoke.log
timeout 900 python bench.py > $O/${TAG}_bench.log 2>&1; echo "bench exit $?"
python -c "
import json,sys
d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1])
print('value %.4g frac %.3f e2e %.4g' % (d['value'], d['roofline']['frac'], d['e2e']['value']), 'pruned', d['pruned'])
print({k: (v['time_to_optimal_s'], v.get('oracle_check'), v['cost']) for k, v in d['time_to_optimal_full_space'].items()})
" $O/${TAG}_bench.log || tail -20 $O/${TAG}_bench.log
SMILESS_BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --no-cpu-baseline --no-c4 > $O/${TAG}_bench_2rank.log 2>&1
echo "2-rank exit $?"; python -c "
import json,sys
d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1])
print('2rank value %.4g' % d['value'], {k: (v['time_to_optimal_s'], v.get('oracle_check'), v['cost'], v['decided_per_rank']) for k, v in d['time_to_optimal_full_space'].items()})
" $O/${TAG}_bench_2rank.log || tail -20 $O/${TAG}_bench_2rank.log
