# sort_chunk 4096 vs 8192 across tree sizes (current kernels), + carveout variant A/B
S="sort_chunk=4096;sort_chunk=8192"
for cfg in "--keys 24" "--keys 25" "--keys 26" "--keys 25 --dist zipf" "--config 3" "--config 3 --fanout 32" "--config 3 --fanout 128"; do
  echo "== $cfg"; timeout 300 python bench.py $cfg --no-e2e --no-cpu --steps 10 --sweep "$S" 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); print(d.get('sweep',{}).get('sort_chunk'), round(d.get('gqs',0),2))"
done
echo "== carveout A/B"; bash tools/ab_psa.sh 2>/dev/null; bash tools/ab_psa.sh --config 3 2>/dev/null
