# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize.py (T1 sizes)
mkdir -p gpurun_out
for t in memcheck synccheck racecheck; do
  timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool $t --error-exitcode 9 \
      python tools/sanitize.py > gpurun_out/sanitizer_${t}_${1:-r2}.log 2>&1
  echo "$t rc=$?"
done
NCU="ncu --set full --clock-control none --import-source on -s 2 -c 1"
timeout 600 $NCU -k regex:pure_kernel -o gpurun_out/prof_purenew_k32_${1:-r2} -f python tools/prof_any.py pure 32 > gpurun_out/ncu_pn32.log 2>&1
echo prof rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:radix -s 16 -c 16 --csv --log-file gpurun_out/radix_launches_${1:-r2}.csv python tools/prof_any.py radix 256 > gpurun_out/ncu_radix.log 2>&1
echo radix rc=$?
