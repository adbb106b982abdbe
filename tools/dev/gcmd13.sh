python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_hist.py tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2; do
python tools/time_hist.py --order shuffled --mode 4 --iters 10 2>&1 | grep "ms," | tail -1
python tools/time_hist.py --iters 20 2>&1 | grep "ms," | tail -1
done
python tools/time_c5.py 2>&1 | tail -3
python tools/bench_detect.py --cpu-scale 0.001 > gpurun_out/detect.log 2>&1; tail -1 gpurun_out/detect.log | cut -c1-250
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_p" -c 4 --csv --log-file gpurun_out/part_launch.csv python tools/time_hist.py --order shuffled --mode 4 --iters 1 > gpurun_out/ncu_part.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:"k_pscatter" -c 1 -o gpurun_out/psc_full4 python tools/time_hist.py --order shuffled --mode 4 --iters 1 > gpurun_out/ncu_part4.log 2>&1
