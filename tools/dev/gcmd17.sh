python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2 3; do
python tools/time_hist.py --lib tools/libgs_head.so --iters 20 2>&1 | grep "ms," | tail -1
python tools/time_hist.py --lib tools/libgs_vplan.so --iters 20 2>&1 | grep "ms," | tail -1
done
python tools/bench_detect.py --lib tools/libgs_head.so --cpu-scale 0.001 2>&1 | tail -1 | cut -c1-200
python tools/bench_detect.py --cpu-scale 0.001 2>&1 | tail -1 | cut -c1-200
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_" -c 14 --csv --log-file gpurun_out/det_launch.csv python tools/bench_detect.py --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det.log 2>&1
