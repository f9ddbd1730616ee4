for v in lib_1024_1 lib_512_3 lib_1024_2 lib_256_6; do
  echo "== $v"
  HARMONIA_LIB=/root/repo/gpurun_variants/$v/libharmonia.so python bench.py --steps 10 --sweep "reuse_run=1;reuse_run=4;reuse_run=8;reuse_run=4,flags=16" 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    l=l.strip()
    if l.startswith('{'):
        d=json.loads(l); s=d['sweep']; print(s['reuse_run'], s['flags'], round(d['gqs'],2), {k:round(v,2) for k,v in d['kernels_ms_per_step'].items()})
    else: print(l[:200])
"
done
