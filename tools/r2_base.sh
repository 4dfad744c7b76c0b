set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2b_smi.txt 2>&1
timeout 600 python bench.py --config 3 --steps 20 --warmup 5 --cpu-seconds 2 > gpurun_out/r2b_bench_c3.json 2> gpurun_out/r2b_bench_c3.err
# LTS / DRAM counters of the one-launch kernel at C3/C4 (VERDICT weak #6)
for c in 3 4; do
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,lts__t_sectors.sum,lts__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors_srcunit_tex.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,sm__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__m_xbar2l1tex_read_bytes.sum,lts__d_sectors_fill_device.sum,lts__t_sectors_srcnode_gpc.sum --clock-control none -k regex:tc_fused -s 1 -c 1 --csv --log-file gpurun_out/r2b_lts_c$c.csv python tools/run_layer.py $c fused 3 > gpurun_out/r2b_lts_c$c.log 2>&1
done
ls gpurun_out
