python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "cluster_sort or c4_full_size_flow or rank" > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for i in 1 2 3; do
for l in tools/libgs_head.so paper_conf_sc_senvs23_b200/libgpuscout_b200.so; do
python bench.py --lib $l --no-cpu-baseline --no-extras --steps 200 > gpurun_out/bench.log 2>>gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); r=d['roofline']
print('$l', 'step', d['ms_per_step'], 'frac', round(r['frac'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
done
done
