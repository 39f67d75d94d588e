# configs[1] lines on the final code (after the y_split grouped launch): C2A, C2B, two-level step
set -x
timeout 1500 python bench.py --config C2A --no-cpu > gpurun_out/r02h_c2a.json 2> gpurun_out/r02h_c2a.err
timeout 1500 python bench.py --config C2B --no-cpu > gpurun_out/r02h_c2b.json 2> gpurun_out/r02h_c2b.err
timeout 1500 python tools/c2_step.py 10 3 y > gpurun_out/r02h_c2_two_level.json 2> gpurun_out/r02h_c2_two_level.err
for c in c2a c2b; do python -c "import json;d=json.load(open('gpurun_out/r02h_$c.json'));print('$c', round(d['ms_per_step'],3), d['value'], d['e2e']['ms_per_step'], d['extras']['time_fraction_of_dense'], d['extras']['dense_ms_per_step'], d['extras']['kv_mode_host_ms_per_step'], d['extras']['exposed_load_ms_per_step'], d['extras']['load_overlap_frac'], d['roofline']['frac'], d['step_roofline']['frac'])"; done
python -c "import json;d=json.load(open('gpurun_out/r02h_c2_two_level.json'));print('two-level', d['ms_per_step'], d['dense_ms_per_step'], d['time_fraction_of_dense'], d['images_per_s'])"
