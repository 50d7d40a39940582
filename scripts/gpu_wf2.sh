M=gpu__time_duration.sum,l1tex__data_pipe_lsu_wavefronts_mem_lgds.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed,smsp__inst_executed.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_red.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active
for cfg in "3 --mh" "4 --mh" "3" "0" "0 --ov 0.25"; do
  set -- $cfg; d=$1; shift
  OPP_PMD_DEBUG=$d timeout 600 ncu --metrics $M --clock-control none --csv -k regex:k_push_move_deposit_tiled -s 4 -c 1 python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>/dev/null | grep -v "^==" > "gpurun_out/wf2_dbg${d}$*.csv"; echo "dbg $d $* $?"
done
