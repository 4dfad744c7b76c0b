#!/bin/bash
# quick per-config summary: tools/bench_quick.sh TAG [configs...]
tag=$1; shift
for c in "$@"; do
  timeout 300 python bench.py ${BQ_ARGS} --config $c --no-all-configs --cpu-seconds 0.2 --steps 30 > gpurun_out/q_${tag}_$c.json 2>gpurun_out/q_${tag}_$c.err
  python - "$tag" "$c" <<'PY'
import json, sys
tag, c = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/q_{tag}_{c}.json"))
except Exception as e:
    print(tag, c, "FAILED", open(f"gpurun_out/q_{tag}_{c}.err").read()[-500:]); sys.exit()
k = {n: (v["us"], v["GB/s"]) for n, v in d["kernels"].items()}
u = d["unfused"]["ms_per_step"] if d["unfused"] else None
v = d.get("variants") or {}
vs = {n: x["ms_per_step"] for n, x in v.items()}
kg = {n: x["us"] for n, x in (v.get("ir_kernel", {}).get("kernels") or {}).items()}
print(f"{tag} C{c} ms={d['ms_per_step']:.4f} unf={u} frac={d['roofline']['frac']} {k} variants={vs} irk_kernels={kg}")
PY
done
