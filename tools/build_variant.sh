#!/bin/bash
# build_variant.sh NAME "-DMACRO=.. ..." [sel_f32_m0_f1_q0,...]
#   -> paper_conf_sigmod_shanbhagpm18_b200/variants/libtopk_NAME.so
# (load it with TOPK_LIB=<path>; dev tool for A/B runs of compile-time knobs)
set -e
cd "$(dirname "$0")/.."
python - "$1" "$2" "${3:-}" <<'PY'
import os, sys
from paper_conf_sigmod_shanbhagpm18_b200 import _build
name, flags = sys.argv[1], sys.argv[2].split()
only = [x for x in sys.argv[3].split(",") if x] or None
vdir = os.path.join(_build.PKG, "variants")
os.makedirs(vdir, exist_ok=True)
print(_build.build(force=True, extra_flags=flags, lib=os.path.join(vdir, f"libtopk_{name}.so"),
                   objdir=os.path.join(vdir, f"build_{name}"), only=only))
PY
