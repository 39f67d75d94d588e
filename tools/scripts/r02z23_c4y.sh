# configs[3] cache mode: Y caching with whole-entry DMA vs the KV-mode default (TMA row gather)
set -x
timeout 2400 python bench.py --config C4 --mode y --copy-method 2 --steps 6 --no-extras --no-cpu > gpurun_out/r02z23_c4_y_m2.json 2> gpurun_out/r02z23_c4_y_m2.err
timeout 2400 python bench.py --config C4 --mode y --copy-method 3 --copy-ctas 8 --steps 6 --no-extras --no-cpu > gpurun_out/r02z23_c4_y_m3.json 2> gpurun_out/r02z23_c4_y_m3.err
timeout 2400 python bench.py --config C4 --mode kv --steps 6 --no-extras --no-cpu > gpurun_out/r02z23_c4_kv.json 2> gpurun_out/r02z23_c4_kv.err
for c in y_m2 y_m3 kv; do python -c "import json;d=json.load(open('gpurun_out/r02z23_c4_$c.json'));print('c4 $c', round(d['ms_per_step'],1), d['plan']['cached_blocks'], d['plan']['refinement'].get('measured_ms'))"; done
