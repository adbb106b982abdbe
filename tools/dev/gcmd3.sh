python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,smsp__inst_executed.sum --clock-control none -k regex:"k_" -c 12 --csv --log-file gpurun_out/det_launch2.csv python tools/bench_detect.py --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_resolve|k_summary|k_carry" -c 3 -o gpurun_out/det_src3 python tools/bench_detect.py --scale 0.35 --steps 1 --cpu-scale 0.001 > gpurun_out/ncu_det3.log 2>&1
