python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for lib in tools/libgs_old.so paper_conf_sc_senvs23_b200/libgpuscout_b200.so; do
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/rk.csv python tools/prof_step.py --only rank --steps 3 --lib $lib > /dev/null 2>&1
echo $lib; python tools/ncu_summary.py launches gpurun_out/rk.csv 3 | grep -v k_expand | head -12
done
