python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
GS_TIMING=1 python tools/bench_detect.py --cpu-scale 0.001 > gpurun_out/detect.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_" -c 12 --csv --log-file gpurun_out/det_launch5.csv python tools/bench_detect.py --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det.log 2>&1
python bench.py --no-cpu-baseline --no-extras > gpurun_out/bench.log 2>gpurun_out/bench.err
tail -3 gpurun_out/gpu_tests.log; grep gs_load gpurun_out/detect.log; tail -1 gpurun_out/detect.log | cut -c1-200
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); r=d['roofline']
print('step', d['ms_per_step'], 'value', d['value'], 'frac', r['frac'], 'kernel_ms', r['kernel_ms'], 'call_ms', r['call_ms'], d['phases_ms'])"
