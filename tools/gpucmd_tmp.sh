python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout -s KILL 900 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; tail -1 gpurun_out/gpu_tests.log
GS_NO_GRAPH=1 timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py -q -k "graph or rank or flow" > gpurun_out/gpu_tests_nograph.log 2>&1; tail -1 gpurun_out/gpu_tests_nograph.log
timeout -s KILL 300 python bench.py > gpurun_out/bench_r01g.json 2> gpurun_out/bench_r01g.err; tail -1 gpurun_out/bench_r01g.json | cut -c1-200
timeout -s KILL 300 python bench.py --order shuffled --no-cpu-baseline > gpurun_out/bench_r01g_shuffled.json 2>/dev/null
timeout -s KILL 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_r01g_reference.json 2>/dev/null
timeout -s KILL 400 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches_r01g_bench.csv python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
timeout -s KILL 400 ncu --set full --clock-control none --import-source on -k regex:k_hist_window -s 2 -c 1 -o gpurun_out/hist_r01g python tools/prof_step.py --only hist --steps 3 > gpurun_out/ncu_hist.log 2>&1
echo done
