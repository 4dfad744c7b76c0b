set -u
mkdir -p gpurun_out
export SR_PARITY_REPORT=gpurun_out/parity_report2.jsonl
rm -f $SR_PARITY_REPORT
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2_own.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_own.log
tail -5 gpurun_out/r2_own.log
for c in 2 3; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 5 --cpu-seconds 1 --no-all-configs > gpurun_out/r2_own_bench_c$c.json 2> gpurun_out/r2_own_bench_c$c.err
done
bash tools/sanitize.sh
