#!/bin/bash
# GPU box: ncu launch lists (bench.py per config) + --set full of each kernel of tools/run_layer.py.
# Then, here: python tools/make_profiles.py rN
set -u
NCU=${NCU:-ncu}
mkdir -p gpurun_out
for c in ${CFGS:-2 3 4 5}; do
  timeout 300 $NCU --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --csv --log-file gpurun_out/launches_c$c.csv \
    python bench.py --config $c --steps 2 --warmup 3 --no-all-configs --cpu-seconds 0.05 > gpurun_out/launches_c$c.log 2>&1
  timeout 300 $NCU --set full --clock-control none --import-source on -k regex:tc_fused -s 1 -c 1 \
    -o gpurun_out/full_c${c}_tc_fused -f python tools/run_layer.py $c fused 3 > /dev/null 2>&1
  for k in tc_gemm1 tc_gemm2; do
    timeout 300 $NCU --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
      -o gpurun_out/full_c${c}_$k -f python tools/run_layer.py $c two_kernels 3 > /dev/null 2>&1
  done
  timeout 300 $NCU --set full --clock-control none --import-source on -k regex:tc_gemm2 -s 1 -c 1 \
    -o gpurun_out/full_c${c}_tc_gemm2_fi -f python tools/run_layer.py $c fused_ir 3 > /dev/null 2>&1
  timeout 300 $NCU --set full --clock-control none --import-source on -k regex:ir_kernel -s 1 -c 1 \
    -o gpurun_out/full_c${c}_ir_kernel -f python tools/run_layer.py $c ir_kernel 3 > /dev/null 2>&1
done
ls gpurun_out/
