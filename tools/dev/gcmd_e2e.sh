python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
for l in paper_conf_sc_senvs23_b200/libgpuscout_b200.so tools/libgs_stage4.so tools/libgs_stage64.so; do
python bench.py --lib $l --no-cpu-baseline --no-extras --steps 50 --e2e-steps 8 > gpurun_out/bench.log 2>>gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); print('$l', round(d['e2e']['value']/1e9,3), round(d['e2e']['ms_per_step'],2))"
done
done
