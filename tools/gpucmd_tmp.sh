python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do for v in i2 i4 i8; do timeout 200 python tools/time_hist.py --iters 40 --lib tools/libgs_$v.so 2>&1 | tail -1; done; done
