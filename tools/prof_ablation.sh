#!/bin/bash
# F1 ncu evidence: one --set full capture per staging variant and size (run on the GPU box).
mkdir -p gpurun_out/ablate
for case in config1_n4096 config5_p8; do
  for v in small 0 1 2 3 4 5 6; do
    if [ $v = small ] && [ $case = config5_p8 ]; then continue; fi
    if [ $v = 6 ] && [ $case = config5_p8 ]; then continue; fi
    timeout 900 ncu --set full --clock-control none --profile-from-start off -k regex:force \
        -o gpurun_out/ablate/${case}_v${v} -f python tools/prof_ablation.py $case $v > gpurun_out/ablate/${case}_v${v}.log 2>&1
    echo "$case $v rc=$?"
  done
done
# summaries only (the .ncu-rep files of 15 full captures exceed what gpurun brings back)
python tools/ncu_summary.py gpurun_out/ablate/*.ncu-rep > gpurun_out/ablate/ncu_ablation_summary.json
for f in gpurun_out/ablate/*.ncu-rep; do
  ncu -i $f --page raw --csv --metrics l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,lts__t_sectors_srcunit_tex_op_read.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,l1tex__t_sector_hit_rate.pct,lts__t_sector_hit_rate.pct,sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active,gpu__time_duration.sum,smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio,smsp__average_warp_latency_issue_stalled_short_scoreboard.ratio,l1tex__t_sectors_pipe_lsu_mem_global_op_ld_lookup_hit.sum,idc__requests.sum > ${f%.ncu-rep}.raw.csv 2>&1
done
rm -f gpurun_out/ablate/*.ncu-rep
