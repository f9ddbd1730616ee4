set -x
timeout 900 python -m pytest tests/test_gpu_peer.py -x -q > gpurun_out/t_peer.log 2>&1; tail -15 gpurun_out/t_peer.log
for m in partitioned peer; do timeout 600 torchrun --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --mode $m --steps 10 --no-cpu > gpurun_out/b_$m.json 2> gpurun_out/b_$m.err; tail -2 gpurun_out/b_$m.err; tail -1 gpurun_out/b_$m.json | cut -c1-400; done
