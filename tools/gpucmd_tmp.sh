python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for o in shuffled trace; do
timeout -s KILL 100 python tools/time_hist.py --iters 10 --check --order $o --mode 4 2>&1 | tail -2
for v in pst512 pst256; do timeout -s KILL 100 python tools/time_hist.py --iters 10 --check --order $o --mode 4 --lib tools/libgs_$v.so 2>&1 | tail -2; done
done
