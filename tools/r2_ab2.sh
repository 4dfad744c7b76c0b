set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
for c in 2 3 4 5; do
  for lib in libsr_r1.so libsr_mha.so libsr_noblob.so libsr_ldg.so; do
    SR_MHA_LIB=$P/$lib timeout 300 python tools/ab_time.py $c 20 default,two_kernels,unfused 2>&1 | tail -3
  done
done > gpurun_out/r2_ab2.txt
cat gpurun_out/r2_ab2.txt
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r2_ncu2_c4.csv python tools/run_layer.py 4 ir_kernel 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r2_ncu2_u3.csv python tools/run_layer.py 3 unfused 3 > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ir_kernel -s 1 -c 1 \
    -o gpurun_out/r2_full_c4_ir -f python tools/run_layer.py 4 ir_kernel 3 > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:row_softmax -s 1 -c 1 \
    -o gpurun_out/r2_full_c3_softmax -f python tools/run_layer.py 3 unfused 3 > /dev/null 2>&1
ls gpurun_out | grep r2_
