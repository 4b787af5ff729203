set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_radix.py tests/test_gpu_query.py -x -q > gpurun_out/r_tests.log 2>&1; echo rtests rc=$?
tail -25 gpurun_out/r_tests.log
timeout 300 python - > gpurun_out/radix_time.log 2>&1 <<'PY'
import torch, json
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
n = 1 << 29
x = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device="cuda")
for name, f in (("radix", tk.topk_radix), ("bitonic", tk.topk)):
    for k in (32, 256, 1024):
        for _ in range(3): f(x, k)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10): f(x, k)
        e1.record(); torch.cuda.synchronize()
        print(json.dumps({"impl": name, "k": k, "us": e0.elapsed_time(e1) / 10 * 1e3}))
PY
cat gpurun_out/radix_time.log
