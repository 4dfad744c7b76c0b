set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
for rep in 1 2; do
for c in 2 3 4 5; do
  for lib in libsr_r1.so libsr_mha.so libsr_noblob.so; do
    SR_MHA_LIB=$P/$lib timeout 300 python tools/ab_time.py $c 20 default,two_kernels,ir_kernel,unfused 2>&1 | tail -4
  done
done
done > gpurun_out/r2_ab.txt
cat gpurun_out/r2_ab.txt
# kernel durations (ncu) of the new default and the IR kernel variant at C2-C5
for c in 2 3 4 5; do
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/r2_ncu_c$c.csv python tools/run_layer.py $c ir_kernel 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r2_ncu_def_c$c.csv python tools/run_layer.py $c fused 3 > /dev/null 2>&1
done
ls gpurun_out | grep r2_ncu
