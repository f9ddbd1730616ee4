python bench.py --steps 10 --sweep "group_size=1;group_size=1,window=16777216" 2>&1 | grep sweep
HARMONIA_LIB=/root/repo/gpurun_variants/s1024/libharmonia.so python bench.py --steps 10 --sweep "group_size=1;group_size=1,window=16777216" 2>&1 | grep sweep
