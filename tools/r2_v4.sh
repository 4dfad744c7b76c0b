set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
for c in 2 5 4 3; do
  for lib in libsr_r1.so libsr_mha.so libsr_noblob.so; do
    SR_MHA_LIB=$P/$lib timeout 300 python tools/ab_time.py $c 20 default,two_kernels,ir_kernel 2>&1 | tail -3
  done
done > gpurun_out/r2_v4_ab.txt
cat gpurun_out/r2_v4_ab.txt
timeout 900 python bench.py --steps 20 --warmup 5 --cpu-seconds 3 > gpurun_out/r2_v4_bench.json 2> gpurun_out/r2_v4_bench.err
tail -3 gpurun_out/r2_v4_bench.err
