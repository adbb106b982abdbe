python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_hist.py -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2; do
for l in tools/libgs_old.so paper_conf_sc_senvs23_b200/libgpuscout_b200.so tools/libgs_pst1024.so tools/libgs_pst256.so; do
python tools/time_hist.py --lib $l --order shuffled --mode 4 --iters 10 2>&1 | grep "ms," | tail -1
done
done
python tools/time_hist.py --order shuffled --mode 4 --iters 3 --check 2>&1 | grep -i "check\|ms,"
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_p" -c 4 --csv --log-file gpurun_out/part_launch.csv python tools/time_hist.py --order shuffled --mode 4 --iters 1 > gpurun_out/ncu_part.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:"k_pscatter" -c 1 -o gpurun_out/psc_full python tools/time_hist.py --order shuffled --mode 4 --iters 1 > gpurun_out/ncu_part2.log 2>&1
