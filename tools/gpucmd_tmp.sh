for v in s1x4 s2x2 s4x1; do GS_HIST_TMA=1 timeout 200 python tools/time_hist.py --iters 20 --lib tools/libgs_$v.so; done
