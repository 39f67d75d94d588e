"""Per-class summary of an ncu launch list of the bench's timed region (bench.py with
FPS_PROFILE_RANGE=1 under `ncu --profile-from-start off --metrics gpu__time_duration.sum,
dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv`).  ncu serialises the
launches and runs them cold-cache, so per-class SHARES (not absolute times) are what compare
with the live step; DRAM bytes per launch are per kernel and need no such care.

  python tools/ncu_classes.py gpurun_out/launches.csv C3 <timed steps>
writes profiles/ncu/<config>_classes.json and profiles/ncu/<config>_traffic.json."""
import collections
import csv
import json
import os
import sys

CLASSES = [("gemm_tcgen05", ("gemm_tc",)), ("attention", ("attn_",)), ("rownorm", ("ln_mod", "ln_affine", "ln_")),
           ("row_copy", ("copy_rows", "gather_rows", "scatter_rows")), ("cache_prefetch", ("prefetch", "bulk_gather")),
           ("sampler", ("euler", "flow_blend")), ("mask_index", ("mask_index", "mask_pool")),
           ("gemm_simt", ("gemm_simt", "simt"))]


def cls(name):
    """Library kernels by their (demangled, namespace-less in ncu's list) names; the rest are
    torch / driver kernels."""
    base = name.split("(")[0].replace("void ", "").replace("fps::", "").strip()
    if base.startswith(("at::", "cub", "cutlass", "sm90", "sm100", "nvjet", "ampere", "void at::")):
        return "other (torch / driver)"
    for c, keys in CLASSES:
        if any(base.startswith(k) or ("::" + k) in base for k in keys):
            return c
    return "other (torch / driver)"


def main():
    src, config, steps = sys.argv[1], sys.argv[2], int(sys.argv[3])
    rows = list(csv.reader(open(src)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[h]
    ki, mi, vi, ui, ii = (hdr.index(k) for k in ("Kernel Name", "Metric Name", "Metric Value",
                                                  "Metric Unit", "ID"))
    per = collections.defaultdict(dict)
    names = {}
    for r in rows[h + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        u = r[ui]
        if r[mi] == "gpu__time_duration.sum":
            v = v / 1e3 if u in ("ns", "nsecond") else v * 1e3 if u in ("ms", "msecond") else v
        elif u in ("Kbyte", "KB"):
            v *= 1e3
        elif u in ("Mbyte", "MB"):
            v *= 1e6
        elif u in ("Gbyte", "GB"):
            v *= 1e9
        per[int(r[ii])][r[mi]] = v
        names[int(r[ii])] = r[ki]
    agg = collections.defaultdict(lambda: {"launches": 0, "us": 0.0, "dram_bytes": 0.0})
    for i, m in per.items():
        a = agg[cls(names[i])]
        a["launches"] += 1
        a["us"] += m.get("gpu__time_duration.sum", 0.0)
        a["dram_bytes"] += m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
    tot = sum(a["us"] for c, a in agg.items() if c != "cache_prefetch")
    classes = {"source": f"ncu launch list of bench.py's timed region ({steps} steps, {src.split('/')[-1]}; "
                         "gpu__time_duration.sum, --clock-control none; serialised cold-cache launches: "
                         "compare shares)", "steps": steps,
               "compute_stream_ms_per_step_serialised": tot / 1e3 / steps,
               "classes": {c: {"launches_per_step": a["launches"] / steps,
                               "ms_per_step_serialised": a["us"] / 1e3 / steps,
                               "share_of_compute_stream": (a["us"] / tot if c != "cache_prefetch" else None)}
                           for c, a in sorted(agg.items(), key=lambda x: -x[1]["us"])}}
    traffic = {"source": f"dram__bytes_read.sum + dram__bytes_write.sum per launch, ncu over every launch "
                         f"of the bench's timed region ({steps} steps: dense-prefix, transition and "
                         f"masked blocks together -- the launch mix of roofline.achieved)"}
    for c, a in agg.items():
        if a["launches"]:
            traffic[c] = {"dram_bytes_per_launch": a["dram_bytes"] / a["launches"],
                          "launches": a["launches"]}
    os.makedirs("profiles/ncu", exist_ok=True)
    json.dump(classes, open(f"profiles/ncu/{config}_classes.json", "w"), indent=1)
    json.dump(traffic, open(f"profiles/ncu/{config}_traffic.json", "w"), indent=1)
    print(json.dumps(classes, indent=1))
    print(json.dumps(traffic, indent=1))


if __name__ == "__main__":
    main()
