python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_hist.py -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2 3; do
python tools/time_hist.py --lib tools/libgs_nopdl.so --iters 20 2>&1 | grep "ms," | tail -1
python tools/time_hist.py --iters 20 2>&1 | grep "ms," | tail -1
done
python bench.py --no-cpu-baseline --no-extras > gpurun_out/bench.log 2>gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); r=d['roofline']
print('step', d['ms_per_step'], 'value', d['value'], 'frac', r['frac'], 'kernel_ms', r['kernel_ms'], d['phases_ms'], d['clocks'])"
