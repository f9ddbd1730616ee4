python tools/bench_extras.py --what update,range > gpurun_out/extras_r1.jsonl 2> gpurun_out/extras_r1.err; cat gpurun_out/extras_r1.jsonl; tail -3 gpurun_out/extras_r1.err
timeout 900 python tools/bench_extras.py --what sweep > gpurun_out/sweep_c3_r1.jsonl 2> gpurun_out/sweep_c3.err; tail -3 gpurun_out/sweep_c3.err
