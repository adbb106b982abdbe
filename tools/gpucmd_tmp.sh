timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/t_all.txt 2>&1; tail -1 gpurun_out/t_all.txt; grep -E "FAILED|Error" gpurun_out/t_all.txt | head -5
python tools/time_hist.py; python tools/time_hist.py --lib tools/libgs_d7.so --iters 1; python tools/time_hist.py --lib tools/libgs_d8.so --iters 1
