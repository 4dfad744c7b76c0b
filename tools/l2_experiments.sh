# L2-policy experiments on the C3 one-launch kernel: ncu DRAM / L2 counters per setting (GPU box; see profiles/r2_experiments.txt)
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum
run() { echo "== $1"; shift; env "$@" timeout 120 ncu --metrics $M --clock-control none -k regex:tc_fused -s 1 -c 1 --csv python tools/run_layer.py 3 fused 2 2>/dev/null | grep '^"' | python3 -c "
import csv,sys
for row in csv.reader(sys.stdin):
    if row[0]!='ID': print('   ', row[12], row[14])"; }
run default X=1
run xkeep0 SR_X_KEEP=0
run xkeep4 SR_X_KEEP=4
run nokhint SR_MHA_LIB=paper_conf_iiswc_choilkha22_b200/lib_nokhint.so
run nog2hint SR_MHA_LIB=paper_conf_iiswc_choilkha22_b200/lib_nog2hint.so
run nopair SR_G1_PAIR=0
run xef0 SR_X_EVICT_FIRST=0
