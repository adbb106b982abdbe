python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in shuffled trace; do
timeout -s KILL 200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/pt.csv python tools/prof_step.py --only hist --steps 2 --mode 4 --order $o > /dev/null 2>&1
echo $o; grep -E "k_p" gpurun_out/pt.csv | awk -F'","' '{print $5, $NF}' | sed 's/(.*)//' | tail -4
done
