"""Run a few engine steps of the bench workload (for ncu). Usage:
   python tools/profile_step.py [--config C3] [--mode kv] [--policy 1] [--steps 2]"""
import argparse, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import bench, synth
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3"); ap.add_argument("--mode", default="kv")
ap.add_argument("--policy", type=int, default=1); ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--location", type=int, default=0)
a = ap.parse_args()
w = bench.WORKLOADS[a.config]
dev = torch.device("cuda", 0)
layers, mod, cache = bench.build_engine_inputs(F, w, a.mode, dev, 2 * (w["layers"] + 1), a.location)
pool = bench.make_requests(w, w["batch"], bench.SEED)
L = w["L_img"] + w["L_txt"]
reqs = [dict(template_id=i, step=0, n_steps=w["steps"], mask=torch.as_tensor(p["mask_np"]).to(dev),
             x=torch.randn(L, w["H"], device=dev).to(torch.bfloat16)) for i, p in enumerate(pool)]
eng = F.Engine(layers, w["heads"], F.MODE_CODE[a.mode], F.FPS_BF16, w["L_img"], w["L_txt"], len(reqs),
               w["steps"], synth.delta_table(w["steps"]), cache, mod_table=mod, slots=4,
               plan_policy=a.policy)
ls = torch.cuda.Stream()
eng.run_batch(reqs, a.steps, load_stream=ls)
torch.cuda.synchronize()
print("done", eng.last_plan()[0].count(1), "cached")
