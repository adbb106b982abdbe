python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout -s KILL 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; tail -1 gpurun_out/gpu_tests.log
timeout -s KILL 300 python bench.py > gpurun_out/bench_r01d.json 2> gpurun_out/bench_r01d.err; tail -1 gpurun_out/bench_r01d.json | cut -c1-300
timeout -s KILL 300 python bench.py --order shuffled --no-cpu-baseline > gpurun_out/bench_r01d_shuffled.json 2>/dev/null
timeout -s KILL 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_r01d_reference.json 2>/dev/null
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01d.csv python tools/prof_step.py --steps 3 > /dev/null 2>&1
timeout -s KILL 400 ncu --set full --clock-control none --import-source on -k regex:k_hist_window -s 2 -c 1 -o gpurun_out/hist_r01d python tools/prof_step.py --only hist --steps 3 > gpurun_out/ncu_hist.log 2>&1
echo done
