#!/bin/bash
# compute-sanitizer over the small runs of tools/sanitize_case.py (VERDICT r1 missing #5).
# GPU box: bash tools/sanitize.sh  -> gpurun_out/sanitize_<tool>.log ; summary in gpurun_out/sanitize_summary.txt
set -u
mkdir -p gpurun_out
CS=${CS:-/usr/local/cuda/bin/compute-sanitizer}
: > gpurun_out/sanitize_summary.txt
for tool in memcheck racecheck synccheck initcheck; do
  extra=""; which=default
  [ $tool = memcheck ] && which=all
  [ $tool = memcheck ] && extra="--leak-check full"
  [ $tool = racecheck ] && extra="--racecheck-report all"
  timeout 900 $CS --tool $tool $extra --print-limit 5000 --target-processes all \
      python tools/sanitize_case.py $which > gpurun_out/sanitize_$tool.log 2>&1
  rc=$?
  echo "$tool rc=$rc :: $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|LEAK SUMMARY' gpurun_out/sanitize_$tool.log | tr '\n' ' ') :: $(grep -c 'sanitize_case ok' gpurun_out/sanitize_$tool.log) ok" >> gpurun_out/sanitize_summary.txt
done
# racecheck on a textbook mbarrier handoff (tools/ubench_racecheck_mbar.cu): does the tool model
# mbarrier parity waits at all?
nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -o /tmp/ubench_rc tools/ubench_racecheck_mbar.cu && \
  timeout 300 $CS --tool racecheck --racecheck-report all --print-limit 20 /tmp/ubench_rc > gpurun_out/sanitize_racecheck_mbar_ubench.log 2>&1
echo "racecheck on the textbook mbarrier handoff: $(grep -E 'RACECHECK SUMMARY|handoff' gpurun_out/sanitize_racecheck_mbar_ubench.log | tr '\n' ' ')" >> gpurun_out/sanitize_summary.txt
# unique hazard sites of the library run (first 5000 reports)
grep -E "Write Thread|Read Thread" gpurun_out/sanitize_racecheck.log | sed -E 's/.*(Write|Read) Thread.*in ([a-z0-9_]+\.cuh?:[0-9]+).*/\1 \2/' | paste - - | sort | uniq -c >> gpurun_out/sanitize_summary.txt
cat gpurun_out/sanitize_summary.txt
