python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo SMOKE $? >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
python bench.py > gpurun_out/bench.log 2>gpurun_out/bench.err
python bench.py --order shuffled --no-cpu-baseline --no-extras > gpurun_out/bench_shuf.log 2>>gpurun_out/bench.err
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.log 2>>gpurun_out/bench.err
GS_TIMING=1 python tools/bench_detect.py --cpu-scale 0.001 > gpurun_out/detect.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-extras > gpurun_out/ncu_bench.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_hist_window" -c 1 -o gpurun_out/hist_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-extras > gpurun_out/ncu_hist.log 2>&1
tail -3 gpurun_out/gpu_tests.log; tail -2 gpurun_out/smoke.log
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); r=d['roofline']
print('step', d['ms_per_step'], 'value', d['value'], 'frac', r['frac'], d.get('clocks'))"
