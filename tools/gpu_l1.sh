# shared-memory staging vs L1 capacity: smem_levels sweep (0 = auto, -1 = nothing staged)
for cfg in "" "--config 3" "--config 3 --dist uniform" "--config 4 --steps 5"; do
  echo "== $cfg"; timeout 600 python bench.py $cfg --no-e2e --no-cpu --steps 10 --sweep "smem_levels=0;smem_levels=-1;smem_levels=1;sort_chunk=4096,smem_levels=-1;sort_chunk=8192,smem_levels=-1" 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l); p=d.get('plan',{}); s=d.get('sweep',{})
  print(s.get('smem_levels'), s.get('sort_chunk'), round(d.get('gqs',0),2), 'plan:', p.get('smem_levels'), p.get('ps_in_smem'), p.get('smem_bytes'), p.get('sort_chunk'))"
done
