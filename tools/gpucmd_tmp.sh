nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1 || tail -20 gpurun_out/build.txt
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/t_all.txt 2>&1; tail -3 gpurun_out/t_all.txt; grep -E "FAILED|Error" gpurun_out/t_all.txt | head -5
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; tail -1 gpurun_out/smoke.txt
timeout 300 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
timeout 300 python bench.py --hist-row32 --no-cpu-baseline > gpurun_out/bench_row32.json 2>> gpurun_out/bench.err; cat gpurun_out/bench_row32.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_ncu.log 2>&1; tail -2 gpurun_out/b_ncu.log
