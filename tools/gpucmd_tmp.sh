python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1 || tail -20 gpurun_out/build.txt
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/t_all.txt 2>&1; tail -3 gpurun_out/t_all.txt; grep -E "FAILED|Error|assert" gpurun_out/t_all.txt | head -20
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
