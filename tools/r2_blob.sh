set -u
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ptest tools/ubench_param_generic.cu && /tmp/ptest > gpurun_out/r2_param_generic.txt 2>&1
cat gpurun_out/r2_param_generic.txt
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2_blob.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_blob.log
tail -5 gpurun_out/r2_blob.log
for c in 2 3 4; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 5 --cpu-seconds 1 --no-all-configs > gpurun_out/r2_blob_bench_c$c.json 2> gpurun_out/r2_blob_bench_c$c.err
done
