# r01e evidence: launch lists of one SDXL C2A block stack and one Flux double-stream stack
# (tools/block_probe.py), and ncu --set full of the SDXL block's GEMMs and attentions.
set -x
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01e_c2a_launches.csv python tools/block_probe.py C2A > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01e_flux_launches.csv python tools/block_probe.py C3 0 flux > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:gemm_tc --launch-skip 48 --launch-count 6 -o gpurun_out/r01e_c2a_gemm python tools/block_probe.py C2A > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:attn --launch-skip 16 --launch-count 3 -o gpurun_out/r01e_c2a_attn python tools/block_probe.py C2A > /dev/null 2>&1
ncu --set full --clock-control none -k regex:gemm_tc --launch-skip 80 --launch-count 10 -o gpurun_out/r01e_flux_gemm python tools/block_probe.py C3 0 flux > /dev/null 2>&1
ls -la gpurun_out/
