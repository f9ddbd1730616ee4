python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; tail -3 gpurun_out/gpu_tests.log
python bench.py --steps 10 --sweep "group_size=2;group_size=4;group_size=8;group_size=2,smem_levels=-1;group_size=4,smem_levels=-1;group_size=2,window=16777216;group_size=4,window=16777216;group_size=2,flags=4;group_size=8,flags=4" > gpurun_out/sweep5.jsonl 2>&1; cat gpurun_out/sweep5.jsonl
