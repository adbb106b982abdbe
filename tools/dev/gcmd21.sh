python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2; do
python tools/bench_detect.py --lib tools/libgs_nopdl.so --cpu-scale 0.001 2>&1 | tail -1 | cut -c1-140
python tools/bench_detect.py --cpu-scale 0.001 2>&1 | tail -1 | cut -c1-140
done
python bench.py --no-cpu-baseline --no-extras --steps 200 > gpurun_out/bench.log 2>>gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); r=d['roofline']
print('bench', 'step', d['ms_per_step'], 'frac', round(r['frac'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:"k_resolve|k_summary" -c 4 --csv --log-file gpurun_out/det_launch.csv python tools/bench_detect.py --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det.log 2>&1
