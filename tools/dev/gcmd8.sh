python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_" -c 14 --csv --log-file gpurun_out/det_launch.csv python tools/bench_detect.py --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_resolve|k_trace|k_summary|k_write|k_carry" -c 6 -o gpurun_out/det_full python tools/bench_detect.py --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det_full.log 2>&1
echo done
