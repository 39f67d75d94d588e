# final code of the round (per-run DMA for copy_method 1): GPU suite, smoke, default bench line,
# and the copy-method A/B that decides the pinned-host default
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01f5_gpu_tests.log 2>&1; echo tests=$?
tail -3 gpurun_out/r01f5_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r01f5_smoke.log 2>&1; echo smoke=$?
tail -1 gpurun_out/r01f5_smoke.log
timeout 600 python bench.py > gpurun_out/r01f5_c3.json 2> gpurun_out/r01f5_c3.err; echo c3=$?
tail -c 600 gpurun_out/r01f5_c3.json
for m in 2 0; do
  timeout 600 python bench.py --copy-method $m --no-cpu > gpurun_out/r01f5_c3_m$m.json 2> gpurun_out/r01f5_c3_m$m.err; echo m$m=$?
done
python - <<'P'
import json
for f in ["r01f5_c3", "r01f5_c3_m2", "r01f5_c3_m0"]:
    try:
        d = json.loads(open(f"gpurun_out/{f}.json").read().strip().splitlines()[-1])
        print(f, d["ms_per_step"], d["value"], d.get("e2e", {}).get("value"))
    except Exception as e:
        print(f, "ERR", e)
P
