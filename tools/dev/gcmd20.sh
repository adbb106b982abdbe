python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2; do
python tools/bench_detect.py --lib tools/libgs_nopdl.so --cpu-scale 0.001 2>&1 | tail -1 | cut -c1-160
python tools/bench_detect.py --cpu-scale 0.001 2>&1 | tail -1 | cut -c1-160
done
for i in 1 2; do
python bench.py --lib tools/libgs_nopdl.so --no-cpu-baseline --no-extras --steps 200 > gpurun_out/bench_nopdl.log 2>>gpurun_out/bench.err
python bench.py --no-cpu-baseline --no-extras --steps 200 > gpurun_out/bench.log 2>>gpurun_out/bench.err
for f in bench_nopdl bench; do python -c "
import json; d=json.loads(open('gpurun_out/$f.log').read().splitlines()[-1]); r=d['roofline']
print('$f', 'step', d['ms_per_step'], 'frac', round(r['frac'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"; done
done
