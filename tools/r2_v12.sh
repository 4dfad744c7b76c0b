set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
for rep in 1 2; do for c in 3 4; do for lib in libsr_mha.so libsr_susp.so; do
  SR_MHA_LIB=$P/$lib timeout 300 python tools/sustained_ab.py $c 3
done; done; done > gpurun_out/r2_v12.txt 2>&1
cat gpurun_out/r2_v12.txt
