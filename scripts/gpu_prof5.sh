python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 4 -c 1 -o gpurun_out/prof_dh python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu $?
