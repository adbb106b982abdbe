python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2 3 4 5; do
timeout 600 python -m pytest -x -q -m gpu tests/test_gpu_parity.py -k "cluster_sort or async_detect or c4_full_size_flow or rank_graph or rank_repeated" >> gpurun_out/stress.log 2>&1; echo "RUN $i $?" >> gpurun_out/stress.log
timeout 600 python -m pytest -x -q -m gpu tests/test_gpu_hist.py -k "c5 or single_bin or small_and_ragged or partition or unaligned" >> gpurun_out/stress.log 2>&1; echo "HIST $i $?" >> gpurun_out/stress.log
done
grep -E "RUN|HIST|passed|failed" gpurun_out/stress.log | tail -20
