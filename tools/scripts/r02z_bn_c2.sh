# round 2: 1-SM GEMM tile width at ties (epilogue-aware choice) on the SDXL shapes; C2 bench
# lines; ncu launch lists of the C2 timed regions (per-class split)
set -x
for s in "4916 640 640" "4916 640 2560" "4916 1920 640" "1228 1280 1280" "1331 3072 3072" "1228 1280 5120"; do
  for f in 0 8192 16384; do python tools/gemm_probe.py $s $f 1 bias; done
done
timeout 900 python bench.py --config C2A --no-cpu --no-extras > gpurun_out/r02z_c2a.json 2> gpurun_out/r02z_c2a.err
timeout 900 python bench.py --config C2B --no-cpu --no-extras > gpurun_out/r02z_c2b.json 2> gpurun_out/r02z_c2b.err
for c in C2A C2B; do
  FPS_PROFILE_RANGE=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r02z_launches_$c.csv python bench.py --config $c --steps 2 --warmup 1 --no-extras --no-cpu > /dev/null 2>&1
  python tools/ncu_classes.py gpurun_out/r02z_launches_$c.csv $c 2
done
cp -r profiles/ncu gpurun_out/ncu_r02z
python - <<'P'
import json
for f in ['r02z_c2a','r02z_c2b']:
    d=json.load(open(f'gpurun_out/{f}.json')); print(f, d['ms_per_step'], d['value'], d['roofline']['frac'], d['roofline']['avg_launch_ms'])
P
