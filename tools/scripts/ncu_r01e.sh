# launch lists (per-kernel device time) of the SDXL-scale C2A bench and the Flux-stack C3 bench
set -x
ncu --metrics gpu__time_duration.sum --clock-control none -c 2500 --csv --log-file gpurun_out/ncu_c2a_sdxl.csv python bench.py --config C2A --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/ncu_c2a.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 2500 --csv --log-file gpurun_out/ncu_c3_flux.csv python bench.py --block flux --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/ncu_c3f.log 2>&1
timeout 300 python bench.py --config C2B --no-cpu > gpurun_out/c2b_sdxl.json 2> gpurun_out/c2b_sdxl.err
head -c 1500 gpurun_out/c2b_sdxl.json
