set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full_layers.py -m gpu -q -x -k "split" > gpurun_out/r2_v13_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_v13_pytest.log
tail -15 gpurun_out/r2_v13_pytest.log
timeout 600 python tools/shard_split_ab.py 3 1 2 4 8 > gpurun_out/r2_v13_split.txt 2>&1
for c in 2 4 5 6; do timeout 600 python tools/shard_split_ab.py $c 1 8 >> gpurun_out/r2_v13_split.txt 2>&1; done
cat gpurun_out/r2_v13_split.txt
