python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_hist.py tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
for i in 1 2 3; do
python tools/time_hist.py --lib tools/libgs_base.so --iters 20 >> gpurun_out/th.log 2>&1
python tools/time_hist.py --iters 20 --check >> gpurun_out/th.log 2>&1
done
python tools/attr_ctx_probe.py >> gpurun_out/th.log 2>&1
python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>gpurun_out/bench.err
tail -3 gpurun_out/gpu_tests.log; cat gpurun_out/th.log | grep -v Warn
python tools/bench_detect.py --cpu-scale 0.001 > gpurun_out/detect.log 2>&1; tail -1 gpurun_out/detect.log | cut -c1-200
