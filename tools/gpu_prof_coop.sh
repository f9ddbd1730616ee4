# ncu --set full of the G=1 staged search kernel, warp-shared (default) vs per-lane (QF_PER_LANE)
for f in 0 1024; do
ncu --set full --import-source on --clock-control none -k regex:k_lane_search_c -c 1 -s 1 \
  -o gpurun_out/prof_coop_$f -f python tools/prof_search.py --calls 3 --flags $f > gpurun_out/prof_coop_$f.log 2>&1
done
ls -la gpurun_out
