# launch list of the default bench command (C3 on the Flux stack) and full captures of the
# single-stream (parallel) block's GEMMs for the roofline traffic figure
ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base function -k regex:"gemm|attn|ln_|copy_rows|euler|mask_|combine" --csv --log-file gpurun_out/r01e2_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/r01e2_ncu_bench.log 2>&1
echo launches=$?
ncu --set full --clock-control none -k regex:gemm_tc --launch-skip 16 --launch-count 4 -o gpurun_out/r01e2_par_gemm python tools/block_probe.py C3 0 par > /dev/null 2>&1
echo par=$?
ncu --set full --clock-control none -k regex:gemm_tc --launch-skip 32 --launch-count 8 -o gpurun_out/r01e2_dbl_gemm python tools/block_probe.py C3 0 flux > /dev/null 2>&1
echo dbl=$?
