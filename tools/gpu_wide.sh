# WIDE (11-bit level-1) vs default per config
S="flags=0;flags=512"
for cfg in "--config 3 --dist uniform" "--config 3" "--config 4" "--keys 25" "--keys 24"; do
  echo "== $cfg"; timeout 600 python bench.py $cfg --no-e2e --no-cpu --steps 5 --sweep "$S" 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); print(d.get('sweep',{}).get('flags'), round(d.get('gqs',0),2), d.get('plan',{}).get('sort_chunk'))"
done
