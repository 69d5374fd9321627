python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for u in 4 8 4 8; do
  SMILESS_VUNROLL=$u timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-pruned --no-full-space --no-c4 > gpurun_out/swu_$u.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1]); print('VUNROLL', sys.argv[2], '%.4g' % d['value'], 'frac %.3f' % d['roofline']['frac'], d['winner']['index'], d['winner']['cost'])" gpurun_out/swu_$u.log $u
done
SMILESS_VUNROLL=8 timeout 600 python -m pytest tests -m gpu -q -x -k "memoisation or memo_variants or bench_configuration" 2>&1 | tail -1
