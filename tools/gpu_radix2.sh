mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none --csv --log-file gpurun_out/radix_launches.csv python tools/prof_any.py radix 256 > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none -k regex:radix_scatter -s 5 -c 1 -o gpurun_out/prof_radix_scatter -f python tools/prof_any.py radix 256 > /dev/null 2>&1
echo done
