python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
for l in paper_conf_sc_senvs23_b200/libgpuscout_b200.so tools/libgs_cs7.so tools/libgs_cs8.so; do
python bench.py --lib $l --no-cpu-baseline --no-extras --steps 200 > gpurun_out/bench.log 2>>gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.log').read().splitlines()[-1]); r=d['roofline']
print('$l', 'step', d['ms_per_step'], 'frac', round(r['frac'],4), {k: round(v,4) for k,v in d['phases_ms'].items()})"
done
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_cluster_sort|k_emit|k_join|k_ktot" -c 8 --csv --log-file gpurun_out/rank_launch.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-extras > gpurun_out/ncu_rank.log 2>&1
