# HEAD sanity at the end of the round: GPU suite, smoke, default bench line
set -x
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1500 python bench.py > gpurun_out/r02z36_c3.json 2> gpurun_out/r02z36_c3.err
python -c "import json;d=json.load(open('gpurun_out/r02z36_c3.json'));print('c3', round(d['ms_per_step'],3), d['extras']['time_fraction_of_dense'], d['extras'].get('y_mode_host_ms_per_step'), d['roofline']['frac'], d['cpu_baseline']['value'])"
