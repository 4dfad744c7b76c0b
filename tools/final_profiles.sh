#!/bin/bash
# A round's evidence captures on the GPU box (then, here: python tools/make_profiles.py ROUND):
# ncu launch lists of short bench runs per config (DRAM bytes per kernel -> profiles/ncu_traffic.json),
# --set full of the one-launch kernel (C3, C4), and the compute-sanitizer pass.
set -u
mkdir -p gpurun_out
for c in 2 3 4 5 6; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --csv --log-file gpurun_out/launches_c$c.csv \
    python bench.py --config $c --steps 2 --warmup 3 --no-all-configs --no-shard-model --no-sweep --cpu-seconds 0.05 \
    > gpurun_out/launches_c$c.log 2>&1
  timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --csv --log-file gpurun_out/launches_train_c$c.csv python tools/run_layer.py $c train 3 > /dev/null 2>&1
done
for c in 3 4; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_fused -s 1 -c 1 \
    -o gpurun_out/full_c${c}_tc_fused -f python tools/run_layer.py $c fused 3 > /dev/null 2>&1
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:row_softmax -s 1 -c 1 \
    -o gpurun_out/full_c${c}_softmax -f python tools/run_layer.py $c unfused 3 > /dev/null 2>&1
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:ir_kernel -s 1 -c 1 \
    -o gpurun_out/full_c${c}_ir_kernel -f python tools/run_layer.py $c ir_kernel 3 > /dev/null 2>&1
done
[ "${SKIP_SANITIZE:-0}" = 1 ] || bash tools/sanitize.sh
ls gpurun_out
