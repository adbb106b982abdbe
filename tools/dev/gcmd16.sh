python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2; do
python tools/time_hist.py --lib tools/libgs_old.so --iters 20 2>&1 | grep "ms," | tail -1
python tools/time_hist.py --iters 20 2>&1 | grep "ms," | tail -1
python tools/time_hist.py --order shuffled --mode 4 --iters 10 2>&1 | grep "ms," | tail -1
done
python tools/time_c5.py 2>&1 | tail -1
python tools/bench_detect.py --cpu-scale 0.001 > gpurun_out/detect.log 2>&1; tail -1 gpurun_out/detect.log | cut -c1-250
python bench.py --no-cpu-baseline --no-extras > gpurun_out/bench.log 2>gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); r=d['roofline']
print('step', d['ms_per_step'], 'value', d['value'], 'frac', r['frac'], 'kernel_ms', r['kernel_ms'], d['phases_ms'], d['clocks'])"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_" -c 14 --csv --log-file gpurun_out/det_launch.csv python tools/bench_detect.py --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:"k_pscatter" -c 1 -o gpurun_out/psc_full6 python tools/time_hist.py --order shuffled --mode 4 --iters 1 > gpurun_out/ncu_part6.log 2>&1
