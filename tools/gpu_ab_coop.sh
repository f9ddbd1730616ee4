set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_search.py -x -q > gpurun_out/t_search.log 2>&1; tail -3 gpurun_out/t_search.log
for f in 0 1024; do python bench.py --no-e2e --no-cpu --steps 20 --flags $f > gpurun_out/ab_$f.json 2>gpurun_out/ab_$f.err; python -c "
import json
d=json.loads(open('gpurun_out/ab_$f.json').read().strip().splitlines()[-1]); kb=d['kernel_breakdown']
print('$f', round(d['value'],2), round(d['ms_per_step'],3), {k:round(x['ms_per_step'],3) for k,x in kb.items()})"; done
for c in 3 4; do for f in 0 1024; do python bench.py --config $c --no-e2e --no-cpu --steps 10 --flags $f > gpurun_out/ab_c${c}_$f.json 2>&1; python -c "
import json
d=json.loads(open('gpurun_out/ab_c${c}_$f.json').read().strip().splitlines()[-1]); kb=d['kernel_breakdown']
print('c$c $f', round(d['value'],2), round(d['ms_per_step'],3), {k:round(x['ms_per_step'],3) for k,x in kb.items()})"; done; done
