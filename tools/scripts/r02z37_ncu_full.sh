# ncu --set full of the dominant kernels at the C3 shapes on the final code (tensor-pipe %, DRAM)
set -x
N="ncu --set full --clock-control none --import-source on -s 3 -c 1"
$N -k regex:attn_tc3 -o gpurun_out/r02z37_attn_masked python tools/attn_probe.py 1331 4608 24 128 1 > /dev/null 2>&1
$N -k regex:attn_tc3 -o gpurun_out/r02z37_attn_dense python tools/attn_probe.py 4608 4608 24 128 1 > /dev/null 2>&1
$N -k regex:gemm_tc -o gpurun_out/r02z37_gemm_w1_masked python tools/gemm_probe.py 1331 21504 3072 0 4 > /dev/null 2>&1
$N -k regex:gemm_tc -o gpurun_out/r02z37_gemm_qkv_dense python tools/gemm_probe.py 4608 9216 3072 0 4 > /dev/null 2>&1
$N -k regex:gemm_tc -o gpurun_out/r02z37_gemm_w2_masked python tools/gemm_probe.py 1331 3072 15360 0 4 > /dev/null 2>&1
for f in attn_masked attn_dense gemm_w1_masked gemm_qkv_dense gemm_w2_masked; do
ncu -i gpurun_out/r02z37_$f.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__cycles_elapsed.avg.per_second,lts__throughput.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size,launch__registers_per_thread > gpurun_out/r02z37_$f.csv
done
rm -f gpurun_out/r02z37_*.ncu-rep
