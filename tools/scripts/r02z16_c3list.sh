# C3 default: ncu launch list of the timed region (per-kernel times incl. the dense prefix)
set -x
FPS_PROFILE_RANGE=1 timeout 1500 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg.per_second,launch__grid_size --clock-control none --csv --log-file gpurun_out/r02z16_c3_launches.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02z16_c3.json 2> gpurun_out/r02z16_c3.err
tail -2 gpurun_out/r02z16_c3.err; wc -l gpurun_out/r02z16_c3_launches.csv
