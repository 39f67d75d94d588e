# measured plan optima with the transition block: C2A (SDXL blocks) and C3 (Flux stack)
timeout 600 python tools/sweep_plan.py --config C2A --block sdxl --steps 20 5 6 7 8 6 7 2>&1 | grep "k="
timeout 300 python tools/sweep_plan.py --config C2A --block sdxl --steps 20 --kv-transition 0 6 7 2>&1 | grep "k="
timeout 900 python tools/sweep_plan.py --config C3 --block flux --steps 10 41 42 43 44 42 2>&1 | grep "k="
