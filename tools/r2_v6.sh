set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
for c in 3 4 5; do
  for pair in 0 1; do for fx in 1 3 6; do
    echo "pair=$pair fixed=$fx $(SR_G1_PAIR=$pair SR_LPT_FIXED=$fx timeout 300 python tools/ab_time.py $c 20 default 2>&1 | tail -1)"
  done; done
done > gpurun_out/r2_v6_ab.txt 2>&1
cat gpurun_out/r2_v6_ab.txt
timeout 900 python bench.py --steps 20 --warmup 5 --cpu-seconds 3 > gpurun_out/r2_v6_bench.json 2> gpurun_out/r2_v6_bench.err
tail -3 gpurun_out/r2_v6_bench.err
