set -u
mkdir -p gpurun_out
P=paper_conf_iiswc_choilkha22_b200
for c in 3 4 5 2; do SR_MHA_LIB=$P/libsr_ph.so timeout 300 python tools/diag_phases.py $c gpurun_out/r2_v7_cta_c$c.txt; done > gpurun_out/r2_v7_phases.txt 2>&1
cat gpurun_out/r2_v7_phases.txt
