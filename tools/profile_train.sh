#!/bin/bash
# GPU box: ncu launch list of a training step (forward + backward) per config and --set full of the
# backward's tensor-core kernels.  Then, here: python tools/make_profiles.py rN
set -u
NCU=${NCU:-ncu}
mkdir -p gpurun_out
for c in ${CFGS:-2 3 4 5}; do
  timeout 300 $NCU --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --csv --log-file gpurun_out/launches_train_c$c.csv python tools/run_layer.py $c train 3 > /dev/null 2>&1
  timeout 300 $NCU --set full --clock-control none --import-source on -k regex:tc_bwd_ds -s 1 -c 1 \
    -o gpurun_out/full_c${c}_tc_bwd_ds -f python tools/run_layer.py $c train 3 > /dev/null 2>&1
  timeout 300 $NCU --set full --clock-control none --import-source on -k regex:tc_bwd_kv -s 1 -c 1 \
    -o gpurun_out/full_c${c}_tc_bwd_dkdv -f python tools/run_layer.py $c train 3 > /dev/null 2>&1
done
ls gpurun_out/
