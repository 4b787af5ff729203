# A/B the compile-time knob variants in paper_conf_sigmod_shanbhagpm18_b200/variants/ (dev tool)
for run in 1 2; do
for lib in base paper_conf_sigmod_shanbhagpm18_b200/variants/libtopk_*.so; do
  if [ "$lib" = base ]; then L=""; else L="TOPK_LIB=$lib"; fi
  echo "== $lib run $run"
  env $L timeout 200 python tools/quick_time.py $((1<<29)) uniform filter 32,128,256,512,1024 2>&1 | python -c "
import sys, json
print(' '.join(f\"k{d['k']}={d['ms']*1e3:.1f}\" for d in map(json.loads, (l for l in sys.stdin if l.startswith('{')))))"
done
done
