python -c "import __graft_entry__ as g; g.build()"
timeout 300 python bench.py > gpurun_out/bench_r01c.json 2> gpurun_out/bench_r01c.err
timeout 300 python bench.py --order shuffled --no-cpu-baseline > gpurun_out/bench_r01c_shuffled.json 2>/dev/null
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01c.csv python tools/prof_step.py --steps 3 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_hist_window -s 2 -c 1 -o gpurun_out/hist_r01c python tools/prof_step.py --only hist --steps 3 > gpurun_out/ncu_hist.log 2>&1
timeout 300 python tools/time_hist.py --iters 1 --lib tools/libgs_diag11.so > gpurun_out/diag11.txt 2>&1
tail -1 gpurun_out/bench_r01c.json; tail -3 gpurun_out/ncu_hist.log
