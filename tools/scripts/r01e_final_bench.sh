# round-end style runs: default bench (C3, Flux stack), reference arm, C4, C2A/C2B (SDXL), 2-rank
timeout 600 python bench.py > gpurun_out/r01e2_c3.json 2> gpurun_out/r01e2_c3.err; echo c3=$?
timeout 300 python bench.py --impl reference > gpurun_out/r01e2_ref.json 2> gpurun_out/r01e2_ref.err; echo ref=$?
timeout 900 python bench.py --config C4 --no-cpu > gpurun_out/r01e2_c4.json 2> gpurun_out/r01e2_c4.err; echo c4=$?
timeout 400 python bench.py --config C2A --no-cpu > gpurun_out/r01e2_c2a.json 2> gpurun_out/r01e2_c2a.err; echo c2a=$?
timeout 600 python bench.py --config C2B --no-cpu > gpurun_out/r01e2_c2b.json 2> gpurun_out/r01e2_c2b.err; echo c2b=$?
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 4 --warmup 3 --no-extras --no-cpu > gpurun_out/r01e2_2rank.json 2> gpurun_out/r01e2_2rank.err; echo 2rank=$?
