# round 2: the serving loop on the real engine (one GPU) vs the simulator; 2-rank C3 functional rechecks
set -x
timeout 2400 python tools/serve_real.py 0.5,0.8 60 > gpurun_out/r02_serving_real.json 2> gpurun_out/r02_serving_real.err; tail -4 gpurun_out/r02_serving_real.err
for i in 1 2; do
FPS_BENCH_TIMEOUT=600 timeout 900 python bench.py --gpus 2 --no-extras --no-cpu > gpurun_out/r02_c3_2ranks_$i.json 2> gpurun_out/r02_c3_2ranks_$i.err; echo rc=$?; head -c 300 gpurun_out/r02_c3_2ranks_$i.json
done
