# round 2: C4 / C2B with the plan refinement, whole-entry DMA vs TMA row gather
set -x
for cfg in C4 C2B; do for cm in 2 3; do
timeout 1500 python bench.py --config $cfg --copy-method $cm --steps 6 --warmup 3 --no-extras --no-cpu > gpurun_out/r02z_${cfg}_m$cm.json 2> gpurun_out/r02z_${cfg}_m$cm.err
python -c "import json;d=json.load(open('gpurun_out/r02z_${cfg}_m$cm.json'));print('$cfg', $cm, round(d['ms_per_step'],1), d['plan']['cached_blocks'], d['plan']['refinement'])"
done; done
