# copy-method A/B per config after the batched-copy call was closed (decides per-config defaults)
for cfg in C4 C2A C2B; do for m in 1 0; do
  timeout 900 python bench.py --config $cfg --copy-method $m --no-cpu --no-extras > gpurun_out/r01f7_${cfg}_m$m.json 2> gpurun_out/r01f7_${cfg}_m$m.err; echo $cfg m$m=$?
done; done
python - <<P
import json,glob
for f in sorted(glob.glob("gpurun_out/r01f7_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1]); print(f, d.get("ms_per_step"), d.get("value"), (d.get("e2e") or {}).get("value"), d.get("clocks"))
    except Exception as e: print(f, "ERR", e)
P
