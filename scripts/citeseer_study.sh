#!/bin/bash
# NEXT-2 on the CiteSeer-shaped graph (PAPER.md P5@12491-13052; inlgen.citeseer_like): the
# template study (SpMV Fig. 4/6, SSSP Fig. 5 analogs) and the ncu Table I / II analogs.
mkdir -p gpurun_out
M=gpu__time_duration.sum,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct,smsp__sass_average_data_bytes_per_sector_mem_global_op_st.pct
timeout 900 python scripts/template_study.py --graph citeseer > gpurun_out/ts_spmv_citeseer.jsonl 2> gpurun_out/ts_spmv_citeseer.err
timeout 900 python scripts/template_study_sssp.py --graph citeseer --sources 3 > gpurun_out/ts_sssp_citeseer.jsonl 2> gpurun_out/ts_sssp_citeseer.err
for v in thread_only dual_queue:32 dbuf_shared:32 dbuf_shared:64 dbuf_shared:256 dbuf_shared:1024 dbuf_global:32 dbuf_global:128 default; do
  f=$(echo $v | tr ':' '_')
  timeout 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/eff_sssp_$f.csv python scripts/template_study_sssp.py --graph citeseer --sources 1 --only $v > /dev/null 2>&1
done
for v in thread_only dual_queue:32:64 dbuf_global:32:64 dbuf_shared:32:64 dbuf_shared:64:64 dbuf_shared:256:64 dbuf_shared:1024:64 "fused (default kernel):8:None"; do
  f=$(echo $v | tr ': ()' '____')
  timeout 600 ncu --metrics $M --clock-control none --csv --log-file "gpurun_out/eff_spmv_$f.csv" python scripts/template_study.py --graph citeseer --only "$v" --reps 1 > /dev/null 2>&1
done
for v in thread_only dual_queue:32 dbuf_shared:32 dbuf_shared:64 dbuf_shared:256 dbuf_shared:1024 default; do
  f=$(echo $v | tr ":" "_")
  timeout 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/eff_pr_$f.csv python scripts/template_study_pr.py --graph citeseer --only $v --iterations 3 > /dev/null 2>&1
done
timeout 900 python scripts/template_study_pr.py --graph citeseer > gpurun_out/ts_pr_citeseer.jsonl 2> gpurun_out/ts_pr_citeseer.err
echo citeseer study done
