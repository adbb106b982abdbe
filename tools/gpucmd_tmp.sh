timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/t_all.txt 2>&1; tail -1 gpurun_out/t_all.txt; grep -E "FAILED|Error" gpurun_out/t_all.txt | head -5
timeout 120 python tools/time_hist.py; timeout 120 python tools/time_hist.py --bits 32
