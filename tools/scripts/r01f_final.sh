# round evidence after the KV-mode transition block (R28): bench lines for every config, reference arm, 2-rank, launch list of the default bench command
timeout 600 python bench.py > gpurun_out/r01f_c3.json 2> gpurun_out/r01f_c3.err; echo c3=$?
timeout 400 python bench.py --impl reference > gpurun_out/r01f_ref.json 2> gpurun_out/r01f_ref.err; echo ref=$?
timeout 900 python bench.py --config C4 --no-cpu > gpurun_out/r01f_c4.json 2> gpurun_out/r01f_c4.err; echo c4=$?
timeout 400 python bench.py --config C2A --no-cpu > gpurun_out/r01f_c2a.json 2> gpurun_out/r01f_c2a.err; echo c2a=$?
timeout 600 python bench.py --config C2B --no-cpu > gpurun_out/r01f_c2b.json 2> gpurun_out/r01f_c2b.err; echo c2b=$?
timeout 600 python bench.py --block seq --no-cpu > gpurun_out/r01f_c3_seq.json 2> gpurun_out/r01f_c3_seq.err; echo c3seq=$?
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 4 --warmup 3 --no-extras --no-cpu > gpurun_out/r01f_2rank.json 2> gpurun_out/r01f_2rank.err; echo 2rank=$?
ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base function -k regex:"gemm|attn|ln_|copy_rows|euler|mask_|combine" --csv --log-file gpurun_out/r01f_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/r01f_ncu.log 2>&1; echo ncu=$?
