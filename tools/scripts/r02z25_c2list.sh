# C2A / C2B (Y-mode default): ncu launch lists of the timed region
set -x
for c in C2A C2B; do
FPS_PROFILE_RANGE=1 timeout 1500 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size --clock-control none --csv --log-file gpurun_out/r02z25_${c}_launches.csv python bench.py --config $c --steps 2 --warmup 1 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02z25_$c.json 2> gpurun_out/r02z25_$c.err
done
