set -x
timeout 900 python -m pytest tests/test_gpu_search.py -x -q -k "range" > gpurun_out/t_range.log 2>&1; tail -3 gpurun_out/t_range.log; grep -E "Error|assert" gpurun_out/t_range.log | head -5
timeout 600 python tools/bench_extras.py --what range,range_group,update > gpurun_out/range.jsonl 2>&1; cat gpurun_out/range.jsonl | cut -c1-260
