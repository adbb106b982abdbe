python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_hist.py -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2; do
python tools/time_hist.py --lib tools/libgs_old.so --order shuffled --mode 4 --iters 10 2>&1 | grep -v Warn | tail -1
python tools/time_hist.py --order shuffled --mode 4 --iters 10 --check 2>&1 | grep -v Warn | tail -1
python tools/time_hist.py --lib tools/libgs_pb14.so --order shuffled --mode 4 --iters 10 2>&1 | grep -v Warn | tail -1
done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_p" -c 8 --csv --log-file gpurun_out/part_launch.csv python tools/time_hist.py --order shuffled --mode 4 --iters 1 > gpurun_out/ncu_part.log 2>&1
