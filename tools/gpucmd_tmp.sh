python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout -s KILL 900 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; tail -1 gpurun_out/gpu_tests.log
timeout -s KILL 300 python bench.py > gpurun_out/bench_r01f.json 2> gpurun_out/bench_r01f.err; tail -1 gpurun_out/bench_r01f.json | cut -c1-200
timeout -s KILL 300 python bench.py --order shuffled --no-cpu-baseline > gpurun_out/bench_r01f_shuffled.json 2>/dev/null
timeout -s KILL 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_r01f_reference.json 2>/dev/null
timeout -s KILL 400 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches_r01f_bench.csv python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
echo done
