set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2_v19_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_v19_pytest.log
tail -3 gpurun_out/r2_v19_pytest.log
for c in 2 3 4 5 6; do
  for lib in libsr_base.so libsr_mha.so; do
    SR_MHA_LIB=$P/$lib timeout 300 python tools/ab_time.py $c 20 default 2>&1 | tail -1
  done
done > gpurun_out/r2_v19_ab.txt
for c in 3 6; do
  for lib in libsr_base.so libsr_mha.so; do
    echo "$lib C$c $(SR_MHA_LIB=$P/$lib timeout 300 python tools/sustained_ab.py $c 3 2>&1 | tail -1)"
  done
done >> gpurun_out/r2_v19_ab.txt
cat gpurun_out/r2_v19_ab.txt
