# round 2: launch timelines of the C3 step, TMA row gather vs whole-entry DMA, planner plan and k=42
set -x
for a in "3 -1" "3 42" "2 -1"; do
  set -- $a
  TRACE_OUT=gpurun_out/r02c_trace_m$1_k$2.npz timeout 600 python tools/step_trace.py C3 $1 $2 4 > gpurun_out/r02c_trace_m$1_k$2.json 2> gpurun_out/r02c_trace_m$1_k$2.err
  cat gpurun_out/r02c_trace_m$1_k$2.json
done
FPS_SM_RESERVE=0 timeout 600 python tools/step_probe.py C3 3 40 6 > gpurun_out/r02c_probe_res0.jsonl 2> gpurun_out/r02c_probe_res0.err
cat gpurun_out/r02c_probe_res0.jsonl
