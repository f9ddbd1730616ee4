# Level-2 chunk (4096 vs 8192) across tree sizes; parity of the search suite.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_search.py -m gpu -x -q 2>&1 | tail -3
S="sort_chunk=4096;sort_chunk=8192"
for k in 23 24 25 26; do
  echo "== uniform T=2^$k"; timeout 300 python bench.py --keys $k --no-e2e --no-cpu --steps 10 --sweep "$S" 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); print(d.get('sweep'), round(d.get('gqs',0),2))"
done
echo "== c3 zipf"; timeout 300 python bench.py --config 3 --no-e2e --no-cpu --steps 10 --sweep "$S" 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); print(d.get('sweep'), round(d.get('gqs',0),2))"
echo "== c4"; timeout 600 python bench.py --config 4 --no-e2e --no-cpu --steps 5 --sweep "$S" 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); print(d.get('sweep'), round(d.get('gqs',0),2))"
timeout 600 python bench.py --no-cpu --no-e2e > gpurun_out/chunk_bench_c2.json 2>/dev/null; head -c 300 gpurun_out/chunk_bench_c2.json
