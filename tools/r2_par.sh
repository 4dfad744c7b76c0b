set -u
mkdir -p gpurun_out
export SR_PARITY_REPORT=gpurun_out/parity_report.jsonl
rm -f $SR_PARITY_REPORT
timeout 2000 python -m pytest tests/test_gpu_full_layers.py tests/test_gpu_pins.py tests/test_gpu_backward.py -m gpu -q -x -s -k "not separate_dq" > gpurun_out/r2_par.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_par.log
tail -5 gpurun_out/r2_par.log
bash tools/sanitize.sh
