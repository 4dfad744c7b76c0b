set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
timeout 2400 python -m pytest tests -m gpu -q -x -k "unfused or full_layer or pins or window or block" > gpurun_out/r2_v8_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_v8_pytest.log
tail -3 gpurun_out/r2_v8_pytest.log
for c in 2 3 4 5 6; do
  for lib in libsr_r1.so libsr_mha.so; do
    SR_MHA_LIB=$P/$lib timeout 300 python tools/ab_time.py $c 20 unfused 2>&1 | tail -1
  done
done > gpurun_out/r2_v8_ab.txt
cat gpurun_out/r2_v8_ab.txt
for c in 3 4 5; do
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/r2_v8_ncu_unf_c$c.csv python tools/run_layer.py $c unfused 3 > /dev/null 2>&1
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:row_softmax -s 1 -c 1 \
    -o gpurun_out/r2_full_c3_softmax_v3 -f python tools/run_layer.py 3 unfused 3 > /dev/null 2>&1
ls gpurun_out | grep r2_v8
