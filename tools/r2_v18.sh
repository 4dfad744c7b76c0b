set -u
mkdir -p gpurun_out
python - <<'PY'
import math, torch, numpy as np
import paper_conf_iiswc_choilkha22_b200 as sr, workloads as W, oracle
from tests.gpu_util import qkv, oracle_mask
import os
# quick correctness of the rounds variant
os.environ["SR_CHUNKS"]="3"
PY
for c in 3 4 5; do
for ch in 1 2 3 4; do
  echo "chunks=$ch $(SR_CHUNKS=$ch timeout 300 python tools/sustained_ab.py $c 2 2>&1 | tail -1)"
done; done > gpurun_out/r2_v18.txt 2>&1
cat gpurun_out/r2_v18.txt
SR_CHUNKS=3 timeout 900 python -m pytest tests/test_gpu_full_layers.py -m gpu -q -x -k "default" > gpurun_out/r2_v18_pytest.log 2>&1; tail -3 gpurun_out/r2_v18_pytest.log
