python -m pytest tests/test_gpu_search.py -m gpu -x -q -k "range or edge" > gpurun_out/gpu_tests.log 2>&1; tail -2 gpurun_out/gpu_tests.log
python tools/bench_extras.py --what range 2>&1 | grep range_batch > gpurun_out/extras_range_r1.jsonl; cat gpurun_out/extras_range_r1.jsonl
