python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "cupti" > gpurun_out/gpu_tests.log 2>&1; echo TESTS $? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
for l in tools/libgs_head.so paper_conf_sc_senvs23_b200/libgpuscout_b200.so; do
python bench.py --lib $l --no-cpu-baseline --steps 50 > gpurun_out/bench.log 2>>gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); print('$l', json.dumps(d['extra']['cupti_C4']))"
done
