# Y-mode C3 on the final code: ncu launch list of the timed region
set -x
FPS_PROFILE_RANGE=1 timeout 1500 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r02z42_y_launches.csv python bench.py --mode y --steps 2 --warmup 1 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02z42_y.json 2> gpurun_out/r02z42_y.err
tail -1 gpurun_out/r02z42_y.err
