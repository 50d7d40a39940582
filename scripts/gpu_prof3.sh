python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
export OPP_TILE_GROUP=16
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit -s 6 -c 1 -o gpurun_out/prof_tmaout python bench.py --steps 4 --warmup 1 --no-e2e --no-cpu --sort 5 --deposit 1 > /dev/null 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit -s 6 -c 1 -o gpurun_out/prof_direct python bench.py --steps 4 --warmup 1 --no-e2e --no-cpu --sort 5 --deposit 1 --direct > /dev/null 2>&1; echo ncu $?
