set -x
timeout 900 python -m pytest tests/test_ntg_model.py tests/test_gpu_search.py -x -q -m gpu > gpurun_out/t_tune.log 2>&1; tail -3 gpurun_out/t_tune.log
timeout 1200 python tools/ablation.py --what ablation > gpurun_out/ablation.jsonl 2> gpurun_out/ablation.err; tail -3 gpurun_out/ablation.err
timeout 1500 python tools/ablation.py --what ntg_model --reps 3 > gpurun_out/ntg_model.jsonl 2> gpurun_out/ntg_model.err; tail -3 gpurun_out/ntg_model.err
