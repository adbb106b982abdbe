python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo SMOKE $? >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
python bench.py > gpurun_out/bench.log 2>gpurun_out/bench.err
tail -3 gpurun_out/gpu_tests.log; tail -2 gpurun_out/smoke.log
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); r=d['roofline']
print('step', d['ms_per_step'], 'value', d['value'], 'frac', r['frac'], d['phases_ms'], d.get('clocks'))"
