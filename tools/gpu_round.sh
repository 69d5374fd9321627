#!/bin/bash
# One gpurun pass: build, GPU parity tests, smoke, bench (ours + reference arm),
# ncu launch list of the bench command and one full capture of the hot kernels.
#   gpurun --timeout 2400 -- 'bash tools/gpu_round.sh TAG'
TAG=${1:-rXX}
O=gpurun_out
mkdir -p $O
nvidia-smi > $O/${TAG}_nvidia_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || { tail -20 $O/${TAG}_build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest gpu exit $?"; tail -3 $O/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke exit $?"; tail -2 $O/${TAG}_smoke.log
timeout 900 python bench.py > $O/${TAG}_bench.log 2>&1; echo "bench exit $?"; tail -c 600 $O/${TAG}_bench.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/${TAG}_bench_ref.log 2>&1; echo "ref exit $?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/${TAG}_launches.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-full-space --no-c4 --no-pruned --no-extra > $O/${TAG}_ncu_launch_bench.log 2>&1
echo "ncu launches exit $?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"smiless_(fused|plan|variants|upstream)_kernel" -c 2 \
    -o $O/${TAG}_prof_eval -f python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-full-space --no-c4 --no-pruned --no-extra \
    > $O/${TAG}_ncu_full.log 2>&1
echo "ncu full exit $?"
ls -la $O | tail -20
# multi-rank flow on the one GPU (gloo collectives, SMILESS_BENCH_SAME_GPU): sharded slice,
# full-space plans and the C5 cross-rank incumbent exchange, oracle-checked winners
SMILESS_BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --no-cpu-baseline --no-c4 --no-extra > $O/${TAG}_bench_2rank.log 2>&1
echo "2-rank exit $?"; python -c "
import json,sys
d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1])
print('2rank value %.4g' % d['value'], {k: (v['time_to_optimal_s'], v.get('oracle_check'), v['cost']) for k, v in d['time_to_optimal_full_space'].items()})
" $O/${TAG}_bench_2rank.log || tail -20 $O/${TAG}_bench_2rank.log
