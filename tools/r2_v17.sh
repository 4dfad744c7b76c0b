set -u
mkdir -p gpurun_out
for c in 3 4 5 2; do
for v in "P2 0 2" "P1 1 2" "P1 1 3" "P1 1 4"; do set -- $v
  echo "$1 keep=$3 $(SR_P1_REVERSE=$2 SR_X_KEEP=$3 timeout 300 python tools/sustained_ab.py $c 2 2>&1 | tail -1)"
done; done > gpurun_out/r2_v17.txt 2>&1
cat gpurun_out/r2_v17.txt
