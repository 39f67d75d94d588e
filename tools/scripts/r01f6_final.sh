# round evidence, final code (copy_method 2 default on both tiers after the per-run DMA change): bench lines, reference arm, 2-rank, launch list
timeout 600 python bench.py > gpurun_out/r01f6_c3.json 2> gpurun_out/r01f6_c3.err; echo c3=$?
timeout 400 python bench.py --impl reference > gpurun_out/r01f6_ref.json 2> gpurun_out/r01f6_ref.err; echo ref=$?
timeout 900 python bench.py --config C4 --no-cpu > gpurun_out/r01f6_c4.json 2> gpurun_out/r01f6_c4.err; echo c4=$?
timeout 400 python bench.py --config C2A --no-cpu > gpurun_out/r01f6_c2a.json 2> gpurun_out/r01f6_c2a.err; echo c2a=$?
timeout 600 python bench.py --config C2B --no-cpu > gpurun_out/r01f6_c2b.json 2> gpurun_out/r01f6_c2b.err; echo c2b=$?
timeout 600 python bench.py --block seq --no-cpu > gpurun_out/r01f6_c3_seq.json 2> gpurun_out/r01f6_c3_seq.err; echo c3seq=$?
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 2 --steps 4 --warmup 3 --no-extras --no-cpu > gpurun_out/r01f6_2rank.json 2> gpurun_out/r01f6_2rank.err; echo 2rank=$?
ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base function -k regex:"gemm|attn|ln_|copy_rows|euler|mask_|combine" --csv --log-file gpurun_out/r01f6_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/r01f6_ncu.log 2>&1; echo ncu=$?
python - <<P
import json,glob
for f in sorted(glob.glob("gpurun_out/r01f6_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1]); print(f, d.get("ms_per_step"), d.get("value"), (d.get("e2e") or {}).get("value"), (d.get("roofline") or {}).get("frac"))
    except Exception as e: print(f, "ERR", e)
P
