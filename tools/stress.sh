# repeat the GPU parity suite to surface rare races
for i in $(seq 1 ${STRESS_N:-3}); do
  timeout 600 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/stress_$i.log 2>&1; echo "run $i rc=$?"; tail -2 gpurun_out/stress_$i.log
done
