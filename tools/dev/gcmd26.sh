python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
for l in paper_conf_sc_senvs23_b200/libgpuscout_b200.so tools/libgs_gsresminb4.so tools/libgs_gsresminb6.so tools/libgs_gssumminb6.so; do
echo "$l $(python tools/bench_detect.py --lib $l --steps 20 --cpu-scale 0.001 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["ms_per_detect"],4))')"
done
done
