# round-2 ncu captures (one launch each, --set full) + launch list of the bench command
mkdir -p gpurun_out
R=${1:-r2}
NCU="ncu --set full --clock-control none --import-source on -s 3 -c 1"
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_select_k256_$R -f python tools/prof_any.py select 256 > /dev/null 2>&1; echo sel256 $?
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_select_k1024_$R -f python tools/prof_any.py select 1024 > /dev/null 2>&1; echo sel1024 $?
timeout 600 $NCU -k regex:pure_kernel -o gpurun_out/prof_purenew_k32_$R -f python tools/prof_any.py pure 32 > /dev/null 2>&1; echo pure32 $?
timeout 600 $NCU -k regex:pure64_kernel -o gpurun_out/prof_pure64_k256_$R -f python tools/prof_any.py pure 256 > /dev/null 2>&1; echo pure256 $?
timeout 600 $NCU -k regex:select_kernel -o gpurun_out/prof_kkk_$R -f python tools/prof_any.py kkk 64 > /dev/null 2>&1; echo kkk $?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'select_kernel|merge_kernel|pure' -c 80 --csv --log-file gpurun_out/launches_$R.csv python bench.py --steps 20 --warmup 3 --no-sweep --no-cpu-baseline --no-big --no-ncu > /dev/null 2>&1; echo launches $?
# summaries on the box (the reports themselves are too large to bring back)
mkdir -p gpurun_out/prof_md
cp tools/prof_meta_r2.json gpurun_out/prof_meta.json
PROF_OUT=gpurun_out/prof_md python tools/summarize_profiles.py $R > gpurun_out/prof_md/traffic_$R.txt 2>&1; echo summarize $?
rm -f gpurun_out/*.ncu-rep
