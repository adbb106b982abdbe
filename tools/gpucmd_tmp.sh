python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in r64 r56 r48; do timeout -s KILL 100 python tools/time_hist.py --iters 20 --check --lib tools/libgs_$v.so 2>&1 | tail -2; timeout -s KILL 200 python tools/overlap.py --lib tools/libgs_$v.so 2>&1 | tail -4; done
