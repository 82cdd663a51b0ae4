timeout 900 ncu --set full --clock-control none --import-source on -k regex:"add_ln|splitk|attn_decode" -s 3 -c 3 -o gpurun_out/ncu_small python tools/ncu_small.py > gpurun_out/ncu_small.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:"gemm_tc" -s 3 -c 2 -o gpurun_out/ncu_gemm_small python tools/ncu_small.py >> gpurun_out/ncu_small.log 2>&1
for f in ncu_small ncu_gemm_small; do
  ncu -i gpurun_out/$f.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed,launch__grid_size,sm__warps_active.avg.pct_of_peak_sustained_active > gpurun_out/$f.raw.csv 2>&1
done
