python -c "import __graft_entry__ as g; g.build()"
timeout 200 python tools/time_hist.py --iters 20 --synthetic 2>&1 | tail -1; timeout 200 python tools/time_hist.py --iters 20 --check 2>&1 | tail -2;
timeout 200 python tools/time_hist.py --iters 5 --check --order shuffled 2>&1 | tail -2;
for v in k4 k12 k16 k8_t768; do timeout 200 python tools/time_hist.py --iters 20 --synthetic --lib tools/libgs_$v.so 2>&1 | tail -1; timeout 200 python tools/time_hist.py --iters 20 --check --lib tools/libgs_$v.so 2>&1 | tail -2; done
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
