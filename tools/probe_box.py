"""Probe the GPU box: host cores/RAM, pinned H2D bandwidth, small-copy rate, SM count."""
import os, subprocess, json, time, torch
out = {}
out["nproc"] = os.cpu_count()
out["affinity"] = len(os.sched_getaffinity(0))
try:
    out["cpu_model"] = [l.split(":",1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name")][0]
except Exception as e: out["cpu_model"] = str(e)
out["mem_total_gb"] = int([l for l in open("/proc/meminfo") if l.startswith("MemTotal")][0].split()[1]) / 1e6
out["mem_avail_gb"] = int([l for l in open("/proc/meminfo") if l.startswith("MemAvailable")][0].split()[1]) / 1e6
out["nvsmi"] = subprocess.run(["nvidia-smi", "--query-gpu=name,memory.total,clocks.max.sm,pcie.link.gen.current,pcie.link.width.current", "--format=csv"], capture_output=True, text=True).stdout
p = torch.cuda.get_device_properties(0)
out["sms"] = p.multi_processor_count
out["cc"] = f"{p.major}.{p.minor}"
res = {}
for mb in (4, 20, 40, 256, 1024):
    n = mb << 20
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True); h.fill_(1)
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(3): d.copy_(h, non_blocking=True)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        it = 10
        for _ in range(it): d.copy_(h, non_blocking=True)
        e1.record(s)
    torch.cuda.synchronize()
    res[f"h2d_{mb}MB_GBs"] = n * it / (e0.elapsed_time(e1) * 1e-3) / 1e9
    with torch.cuda.stream(s):
        e0.record(s)
        for _ in range(it): h.copy_(d, non_blocking=True)
        e1.record(s)
    torch.cuda.synchronize()
    res[f"d2h_{mb}MB_GBs"] = n * it / (e0.elapsed_time(e1) * 1e-3) / 1e9
out["link"] = res
# small copies: 6 KB rows, 660 copies
h = torch.empty(4096 * 6144, dtype=torch.uint8, pin_memory=True)
d = torch.empty(4096 * 6144, dtype=torch.uint8, device="cuda")
for rb in (6144, 12288, 61440):
    cnt = (4096 * 6144) // rb // 2
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(cnt):
        o = 2 * i * rb
        d[o:o+rb].copy_(h[o:o+rb], non_blocking=True)
    e1.record()
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    out[f"small_copy_{rb}B"] = {"count": cnt, "gpu_ms": e0.elapsed_time(e1), "host_ms": (t1-t0)*1e3, "GBs": cnt*rb/(e0.elapsed_time(e1)*1e-3)/1e9}
# zero-copy SM gather over mapped pinned memory (torch can't do UVA directly); skipped
print(json.dumps(out, indent=1))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/probe_box.json", "w"), indent=1)
