#!/bin/bash
# A/B the experiment builds: tools/ab.sh "cfgs" lib1 lib2 ...   (lib "-" = the default build)
cfgs=$1; shift
for lib in "$@"; do
  for c in $cfgs; do
    if [ "$lib" = "-" ]; then L=""; else L="paper_conf_iiswc_choilkha22_b200/$lib"; fi
    SR_MHA_LIB=$L timeout 150 python bench.py --config $c --no-all-configs --cpu-seconds 0.05 --steps 30 > gpurun_out/ab_${lib}_$c.json 2>gpurun_out/ab_${lib}_$c.err
    python - "$lib" "$c" <<'PY'
import json, sys
lib, c = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/ab_{lib}_{c}.json"))
except Exception:
    print(lib, c, "FAILED", open(f"gpurun_out/ab_{lib}_{c}.err").read()[-400:]); sys.exit()
k = {n: round(v["us"], 2) for n, v in d["kernels"].items()}
v = d.get("variants") or {}
fi = v.get("fused_ir", {}).get("ms_per_step")
g1 = v.get("ir_kernel", {})
kg = {n: round(x["us"], 2) for n, x in (g1.get("kernels") or {}).items()}
print(f"{lib:22s} C{c} ms={d['ms_per_step']:.4f} fir={fi} irk={g1.get('ms_per_step')} {k} irk_k={kg}")
PY
  done
done
