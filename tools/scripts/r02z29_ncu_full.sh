# ncu --set full: attn_tc5 vs attn_tc3 at the C2A masked shape (d = 64), and attn_tc3 at C3 masked
set -x
N="ncu --set full --clock-control none --import-source on -s 3 -c 1"
$N -k regex:attn_tc5 -o gpurun_out/r02z29_tc5_c2a python tools/attn_probe.py 1229 4096 10 64 4 0 > gpurun_out/r02z29_a1.log 2>&1
$N -k regex:attn_tc3 -o gpurun_out/r02z29_tc3_c2a python tools/attn_probe.py 1229 4096 10 64 4 65536 > gpurun_out/r02z29_a2.log 2>&1
for f in tc5_c2a tc3_c2a; do
ncu -i gpurun_out/r02z29_$f.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__cycles_elapsed.avg.per_second,smsp__issue_active.avg.pct_of_peak_sustained_active,launch__grid_size > gpurun_out/r02z29_$f.csv
done
ls -la gpurun_out/ | grep r02z29
