python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout -s KILL 900 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; tail -1 gpurun_out/gpu_tests.log
timeout -s KILL 300 python bench.py > gpurun_out/bench_r01e.json 2> gpurun_out/bench_r01e.err; tail -1 gpurun_out/bench_r01e.json | cut -c1-200
timeout -s KILL 300 python bench.py --order shuffled --no-cpu-baseline > gpurun_out/bench_r01e_shuffled.json 2>/dev/null
timeout -s KILL 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_r01e_reference.json 2>/dev/null
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01e.csv python tools/prof_step.py --steps 3 > /dev/null 2>&1
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01e_shuffled.csv python tools/prof_step.py --steps 2 --order shuffled --mode 4 > /dev/null 2>&1
echo done
