# round 2: planner accuracy -- calibration with clock-settling bursts (FPS_CALIB_SETTLE s per fit point)
set -x
for st in 0 0.5; do
FPS_CALIB_SETTLE=$st timeout 900 python tools/step_probe.py C3 2 37,38,39,40 6 > gpurun_out/r02m_settle$st.jsonl 2> gpurun_out/r02m_settle$st.err
cat gpurun_out/r02m_settle$st.jsonl
done
