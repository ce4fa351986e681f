mkdir -p gpurun_out
export INL_SSSP_LOOP=dyn INL_SSSP_DYN_BITS=1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ll_sssp_dynbits.csv python scripts/sssp_steps.py --no-warmup > gpurun_out/ll_sssp_dynbits.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_expand_ -s 4 -c 8 -o gpurun_out/prof_sssp_bits -f python scripts/sssp_steps.py --no-warmup > gpurun_out/ncu_sssp_bits.log 2>&1
echo done >> gpurun_out/ncu_sssp_bits.log
