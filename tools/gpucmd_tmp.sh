timeout 300 python -m pytest tests/test_gpu_hist.py -x -q -m gpu > gpurun_out/t_hist.txt 2>&1; tail -1 gpurun_out/t_hist.txt
export GS_HIST_NO_TMA=1
for b in 16 32; do
  timeout 120 python bench.py --steps 30 --warmup 3 --hist-bits $b --no-cpu-baseline --e2e-steps 1 2> gpurun_out/b10_$b.err > gpurun_out/b10_$b.json
  python -c "import json; d=json.load(open('gpurun_out/b10_$b.json')); print('$b', d['value']/1e9, d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'])"
done
