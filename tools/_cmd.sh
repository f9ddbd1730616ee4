python -m pytest tests -m gpu -x -q 2>&1 | tail -4
ncu --set full --clock-control none --import-source on -k regex:"k_lane_search_c|k_psa2_unmove|k_psa2_move" -c 3 -o gpurun_out/ret_full python tools/prof_search.py --calls 1 > gpurun_out/ncu_ret.log 2>&1; tail -2 gpurun_out/ncu_ret.log
