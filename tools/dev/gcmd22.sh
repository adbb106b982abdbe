python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -5 gpurun_out/gpu_tests.log
for i in 1 2; do
GS_NO_CLUSTER_SORT=1 python bench.py --no-cpu-baseline --no-extras --steps 200 > gpurun_out/bench_cub.log 2>>gpurun_out/bench.err
python bench.py --no-cpu-baseline --no-extras --steps 200 > gpurun_out/bench.log 2>>gpurun_out/bench.err
for f in bench_cub bench; do python -c "
import json; d=json.loads(open('gpurun_out/$f.log').read().splitlines()[-1]); r=d['roofline']
print('$f', 'step', d['ms_per_step'], 'frac', round(r['frac'],4), {k: round(v,4) for k,v in d['phases_ms'].items()}, d['gpu_launches'])"; done
done
