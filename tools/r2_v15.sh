set -u
mkdir -p gpurun_out
for c in 3 4 5; do
for cfgv in "0 0" "0 1" "1 1" "2 1" "3 1"; do set -- $cfgv
  echo "keep=$1 rev=$2 $(SR_X_KEEP=$1 SR_P2_REVERSE=$2 timeout 300 python tools/sustained_ab.py $c 2 2>&1 | tail -1)"
done; done > gpurun_out/r2_v15.txt 2>&1
cat gpurun_out/r2_v15.txt
