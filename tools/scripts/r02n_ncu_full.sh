# round 2: ncu --set full of the dominant kernels at the C3 shapes (tensor-pipe %, DRAM, stalls)
set -x
N="ncu --set full --clock-control none --import-source on -s 3 -c 1"
$N -k regex:attn_tc3 -o gpurun_out/r02n_attn_masked python tools/attn_probe.py 1331 4608 24 128 1 > gpurun_out/r02n_a1.log 2>&1
$N -k regex:attn_tc3 -o gpurun_out/r02n_attn_dense python tools/attn_probe.py 4608 4608 24 128 1 > gpurun_out/r02n_a2.log 2>&1
$N -k regex:gemm_tc -o gpurun_out/r02n_gemm_w1_masked python tools/gemm_probe.py 1331 21504 3072 0 4 > gpurun_out/r02n_g1.log 2>&1
$N -k regex:gemm_tc -o gpurun_out/r02n_gemm_qkv_dense python tools/gemm_probe.py 4608 9216 3072 0 4 > gpurun_out/r02n_g2.log 2>&1
$N -k regex:gemm_tc -o gpurun_out/r02n_gemm_w2_masked python tools/gemm_probe.py 1331 3072 15360 0 4 > gpurun_out/r02n_g3.log 2>&1
python tools/attn_probe.py 1331 4608 24 128 1; python tools/attn_probe.py 4608 4608 24 128 1
python tools/gemm_probe.py 1331 21504 3072 0 4; python tools/gemm_probe.py 4608 9216 3072 0 4; python tools/gemm_probe.py 1331 3072 15360 0 4
python tools/gemm_probe.py 1331 21504 3072 12 4; python tools/gemm_probe.py 1331 3072 15360 12 4
ls -la gpurun_out/
