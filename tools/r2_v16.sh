set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2_v16_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_v16_pytest.log
tail -3 gpurun_out/r2_v16_pytest.log
for c in 2 3 4 5 6; do
  for lib in libsr_r1.so libsr_mha.so; do SR_MHA_LIB=$P/$lib timeout 300 python tools/ab_time.py $c 20 default 2>&1 | tail -1; done
done > gpurun_out/r2_v16_ab.txt 2>&1
cat gpurun_out/r2_v16_ab.txt
