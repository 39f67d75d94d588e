# TMA row gather, second sweep around C4's 8 CTAs x 768 KB; C3 with 4 CTAs and a deeper ring
set -x
run() { # cfg inflight ctas prio tag
FPS_BULK_INFLIGHT=$2 timeout 1500 python bench.py --config $1 --copy-method 3 --copy-ctas $3 --load-priority $4 --steps 6 --warmup 3 --no-extras --no-cpu > gpurun_out/r02z7_$5.json 2> gpurun_out/r02z7_$5.err
python -c "import json;d=json.load(open('gpurun_out/r02z7_$5.json'));print('$5', round(d['ms_per_step'],1), d['plan']['cached_blocks'], round(d['plan']['predicted_ms_per_step'],1), round(d['plan']['fit'].get('load_gbs'),1), d['plan']['refinement'].get('measured_ms'), {k:round(v['ms_per_step'],1) for k,v in d['kernels'].items() if v['ms_per_step']>1})"
}
run C4 786432 8 0 C4_768k_8_p0
run C4 393216 8 -5 C4_384k_8
run C4 1572864 8 -5 C4_1536k_8
run C4 1179648 12 -5 C4_1152k_12
run C4 786432 6 -5 C4_768k_6
run C3 786432 4 -5 C3_768k_4
