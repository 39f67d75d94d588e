# round 2: new GPU tests (shared arena), full default bench line, the 2-rank path on one GPU,
# and the ncu launch list (time + DRAM bytes) of the timed region of the default command
set -x
timeout 600 python -m pytest tests/test_gpu_shared_arena.py -q -m gpu 2>&1 | tail -3
timeout 1200 python bench.py > gpurun_out/r02i_c3.json 2> gpurun_out/r02i_c3.err; tail -2 gpurun_out/r02i_c3.err
timeout 1200 python bench.py --gpus 2 --no-extras --no-cpu > gpurun_out/r02i_c3_n2.json 2> gpurun_out/r02i_c3_n2.err; tail -3 gpurun_out/r02i_c3_n2.err
FPS_PROFILE_RANGE=1 timeout 1500 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r02i_launches.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu > gpurun_out/r02i_ncu_bench.json 2> gpurun_out/r02i_ncu_bench.err; tail -2 gpurun_out/r02i_ncu_bench.err
python tools/ncu_classes.py gpurun_out/r02i_launches.csv C3 2 > /dev/null; cp -r profiles/ncu gpurun_out/ncu_r02i
