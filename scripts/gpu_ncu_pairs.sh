# ncu --set full of the one-per-lane and the pair-per-lane pass 1 (C2, DH1, no field)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 4 -c 1 -o gpurun_out/prof_base python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --field 0 > /dev/null 2>&1; echo ncu1 $?
cp variants/libopp_p4.so paper_conf_icpp_lantra0m24_b200/libopp.so
OPP_PAIRS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pmd_pairs -s 4 -c 1 -o gpurun_out/prof_pairs python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --field 0 > /dev/null 2>&1; echo ncu2 $?
