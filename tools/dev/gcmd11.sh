python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2; do
for l in paper_conf_sc_senvs23_b200/libgpuscout_b200.so tools/libgs_gs_pst512.so tools/libgs_gs_pv16dgs_pst512.so tools/libgs_gs_pv16.so; do
python tools/time_hist.py --lib $l --order shuffled --mode 4 --iters 10 2>&1 | grep "ms," | tail -1
done
done
python tools/bench_detect.py --cpu-scale 0.001 > gpurun_out/detect.log 2>&1; tail -1 gpurun_out/detect.log | cut -c1-250
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_" -c 14 --csv --log-file gpurun_out/det_launch.csv python tools/bench_detect.py --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:"k_pscatter" -c 1 -o gpurun_out/psc_full2 python tools/time_hist.py --order shuffled --mode 4 --iters 1 > gpurun_out/ncu_part2.log 2>&1
