set -u
mkdir -p gpurun_out
for c in 3 2 4; do timeout 300 python tools/headline_ab.py $c 20; done > gpurun_out/r2_v11.txt 2>&1
cat gpurun_out/r2_v11.txt
