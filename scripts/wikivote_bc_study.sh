#!/bin/bash
# BC template study on the Wiki-vote-shaped graph (PAPER.md P5@13172-13524, Fig. 6 BC bars and
# the Table II BC row; inlgen.wikivote_like): timings, then the ncu warp-execution / gld / gst
# efficiencies of the BC kernels per variant (scripts/ncu_efficiency.py 'k_bc|k_bct').
mkdir -p gpurun_out
M=gpu__time_duration.sum,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct,smsp__sass_average_data_bytes_per_sector_mem_global_op_st.pct
timeout 900 python scripts/template_study_bc.py > gpurun_out/ts_bc_wikivote.jsonl 2> gpurun_out/ts_bc_wikivote.err
for v in thread_only dual_queue:32 dbuf_global:32 dbuf_shared:32 dbuf_shared:64 dbuf_shared:256 dbuf_shared:1024 default source; do
  f=$(echo $v | tr ':' '_')
  timeout 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/eff_bc_$f.csv python scripts/template_study_bc.py --sources 4 --only $v > /dev/null 2>&1
done
for f in gpurun_out/eff_bc_*.csv; do python scripts/ncu_efficiency.py $f 'k_bc|k_bct' $(basename $f .csv); done > gpurun_out/eff_bc_summary.txt 2>&1
echo wikivote bc study done
