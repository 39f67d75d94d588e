# round 2: ncu launch list of the C2A bench's timed region (SDXL-scale kernels) + default C3 bench with plan refinement
set -x
FPS_PROFILE_RANGE=1 timeout 1500 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active --clock-control none --csv --log-file gpurun_out/r02q_c2a_launches.csv python bench.py --config C2A --steps 2 --warmup 1 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02q_c2a.json 2> gpurun_out/r02q_c2a.err; tail -2 gpurun_out/r02q_c2a.err
timeout 900 python bench.py --steps 10 --warmup 3 --no-extras --no-cpu > gpurun_out/r02q_c3.json 2> gpurun_out/r02q_c3.err; grep "refinement" gpurun_out/r02q_c3.err | tail -1
