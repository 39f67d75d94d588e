"""Summarise ncu outputs from gpurun_out/ into profiles/ (committed evidence)."""
import csv, collections, json, subprocess, sys, os

def launch_table(src, dst_csv):
    rows = list(csv.reader(open(src)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[h]
    ki, vi, ui, ii = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit"), hdr.index("ID")
    out = []
    for r in rows[h + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        u = r[ui]
        us = v / 1e3 if u in ("ns", "nsecond") else v * 1e3 if u in ("ms", "msecond") else v
        out.append((int(r[ii]), r[ki], us))
    with open(dst_csv, "w") as f:
        w = csv.writer(f)
        w.writerow(["id", "kernel", "gpu_time_us"])
        for t in out:
            if "fps::" in t[1]:
                w.writerow([t[0], t[1][:120], f"{t[2]:.3f}"])
    agg = collections.defaultdict(lambda: [0, 0.0])
    for _, k, us in out:
        if "fps::" not in k:
            continue
        name = k.split("(")[0].replace("void ", "")
        agg[name][0] += 1
        agg[name][1] += us
    return agg

def raw_metrics(rep, wanted):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    hdr = rows[0]
    res = []
    for r in rows[2:]:
        res.append({w: (r[hdr.index(w)] if w in hdr else None) for w in wanted})
    return res

if __name__ == "__main__":
    tag = sys.argv[1]
    src = sys.argv[2]
    agg = launch_table(f"gpurun_out/{src}", f"profiles/{tag}_launches.csv")
    tot = sum(v[1] for v in agg.values())
    lines = [f"| kernel | launches | total us | avg us | share |", "|---|---|---|---|---|"]
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append(f"| `{k}` | {n} | {t:.1f} | {t/n:.2f} | {t/tot:.3f} |")
    print("\n".join(lines))
    wanted = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
              "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
              "sm__throughput.avg.pct_of_peak_sustained_elapsed",
              "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
              "launch__grid_size", "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
              "lts__throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second"]
    for rep in sys.argv[3:]:
        print(f"\n### {rep}")
        for m in raw_metrics(f"gpurun_out/{rep}.ncu-rep", wanted):
            print(json.dumps(m))
