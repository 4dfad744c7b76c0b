set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2_v5_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_v5_pytest.log
tail -3 gpurun_out/r2_v5_pytest.log
for c in 2 5 4 3; do
  for lib in libsr_r1.so libsr_mha.so; do
    SR_MHA_LIB=$P/$lib timeout 300 python tools/ab_time.py $c 20 default,two_kernels,ir_kernel,unfused 2>&1 | tail -4
  done
done > gpurun_out/r2_v5_ab.txt
cat gpurun_out/r2_v5_ab.txt
for c in 3 4 5; do SR_MHA_LIB=$P/libsr_ph.so timeout 300 python tools/diag_phases.py $c; done > gpurun_out/r2_v5_phases.txt 2>&1
cat gpurun_out/r2_v5_phases.txt
for c in 2 3 4 5; do
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/r2_v5_ncu_irk_c$c.csv python tools/run_layer.py $c ir_kernel 3 > /dev/null 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_fused -s 1 -c 1 \
    -o gpurun_out/r2_full_c3_tc_fused -f python tools/run_layer.py 3 fused 3 > /dev/null 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 --cpu-seconds 3 > gpurun_out/r2_v5_bench.json 2> gpurun_out/r2_v5_bench.err
tail -3 gpurun_out/r2_v5_bench.err
ls gpurun_out | grep r2_v5
