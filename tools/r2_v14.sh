set -u
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2_v14_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_v14_pytest.log
tail -3 gpurun_out/r2_v14_pytest.log
for c in 3 4 5 2; do timeout 600 python tools/shard_split_ab.py $c 1 8; done > gpurun_out/r2_v14_split.txt 2>&1
cat gpurun_out/r2_v14_split.txt
