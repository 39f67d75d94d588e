# TMA row gather in the step: bytes in flight (FPS_BULK_INFLIGHT) and CTAs, high-priority load stream
set -x
run() { # cfg inflight ctas tag
FPS_BULK_INFLIGHT=$2 timeout 1500 python bench.py --config $1 --copy-method 3 --copy-ctas $3 --load-priority -5 --steps 6 --warmup 3 --no-extras --no-cpu > gpurun_out/r02z6_$4.json 2> gpurun_out/r02z6_$4.err
python -c "import json;d=json.load(open('gpurun_out/r02z6_$4.json'));print('$4', round(d['ms_per_step'],1), d['plan']['cached_blocks'], round(d['plan']['predicted_ms_per_step'],1), round(d['plan']['fit'].get('load_gbs'),1), d['plan']['refinement'].get('measured_ms'), {k:round(v['ms_per_step'],1) for k,v in d['kernels'].items() if v['ms_per_step']>1})"
}
run C4 393216 4 C4_384k_4
run C4 786432 4 C4_768k_4
run C4 786432 8 C4_768k_8
run C3 393216 4 C3_384k_4
run C3 786432 8 C3_768k_8
