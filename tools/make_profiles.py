"""Summarise gpurun_out/ckpt/* (ncu launch list, ncu full capture, bench lines)
into profiles/ (tracked).  Usage: python tools/make_profiles.py <round-tag>"""
import csv, io, json, os, re, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CK = os.path.join(ROOT, "gpurun_out", "ckpt")
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
P = os.path.join(ROOT, "profiles")
os.makedirs(P, exist_ok=True)
out = []

# 1. launch list: the last MxM step's kernels (ncu serialises launches: shares, not absolutes)
rows = list(csv.reader(open(os.path.join(CK, "launches.csv"))))
hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hi]
ki, vi, ui = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
seq = []
for r in rows[hi + 1:]:
    name = r[ki]
    v = float(r[vi].replace(',', ''))
    v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(r[ui], 1.0)
    m = re.search(r'(\w+_kernel)(<[^>]*>)?', name)
    seq.append(((m.group(1) + (m.group(2) or '')) if m else name[:60], v, 'spbla' in name))
# last step = from the last row_span_kernel (first launch of an MxM) to the end
last = max(i for i, s in enumerate(seq) if s[0].startswith(('row_span_kernel', 'row_info_kernel')))
step = [s for s in seq[last:] if s[2]]
tot = sum(v for _, v, _ in step)
out.append(f"# {tag}: ncu launch list of one bench.py step (configs[4], rmat22_ef32 A.A)\n")
out.append("`ncu --metrics gpu__time_duration.sum --clock-control none` over `bench.py --steps 1 --warmup 3`;"
           " serialised, cold-cache launches — compare shares, not absolutes.\n")
out.append("| kernel | us | share |\n|---|---:|---:|")
for name, v, _ in step:
    out.append(f"| `{name}` | {v:.1f} | {v / tot * 100:.1f}% |")
out.append(f"| **total (library kernels)** | {tot:.1f} | 100% |\n")

# 2. full captures of the dominant kernels (top_<group>.ncu-rep)
import glob
traffic = {}
for rep in sorted(glob.glob(os.path.join(CK, "top_*.ncu-rep"))):
    grp = os.path.basename(rep)[4:-8]
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(io.StringIO(raw)))
    if len(rr) < 3:
        continue
    hh, uu, vv = rr[0], rr[1], rr[2]
    def g(k):
        return (vv[hh.index(k)], uu[hh.index(k)]) if k in hh else ("n/a", "")
    kname = vv[hh.index("Kernel Name")]
    out.append(f"## ncu --set full ({grp}): `{kname[:110]}`\n")
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
            "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
            "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
            "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct", "launch__registers_per_thread",
            "launch__shared_mem_per_block_dynamic", "smsp__inst_executed.sum"]
    out.append("| metric | value |\n|---|---|")
    for k in keys:
        val, un = g(k)
        out.append(f"| `{k}` | {val} {un} |")
    stalls = [(hh[i], float(vv[i] or 0)) for i in range(len(hh))
              if 'pcsamp_warps_issue_stalled' in hh[i] and not hh[i].endswith('not_issued')]
    st = sum(s for _, s in stalls) or 1
    out.append("\nWarp-state samples (top):\n")
    for nm, sv in sorted(stalls, key=lambda x: -x[1])[:6]:
        out.append(f"- {nm.replace('smsp__pcsamp_warps_issue_stalled_', '')}: {sv / st * 100:.1f}%")
    def gb(k):
        val, un = g(k)
        return float(val) * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1}.get(un, 1)
    traffic[grp] = (gb("dram__bytes_read.sum") + gb("dram__bytes_write.sum"), kname)
    out.append("")

# 3. bench lines
for f in ("bench.json", "bench_ref.json", "bench_2rank_gloo.json", "bench_ewise_kron.json", "bench_closure18.json"):
    p = os.path.join(CK, f)
    if os.path.exists(p) and os.path.getsize(p):
        out.append(f"## {f}\n\n```json\n{open(p).read().strip()}\n```\n")
open(os.path.join(P, f"{tag}_summary.md"), "w").write("\n".join(out) + "\n")
if traffic:
    tp = os.path.join(P, "ncu_traffic.json")
    tj = json.load(open(tp)) if os.path.exists(tp) else {}
    for grp, (byt, kname) in traffic.items():
        tj.setdefault("ewise_kron" if grp.startswith("ewise") else "rmat22_ef32", {})[grp] = byt
        tj.setdefault("_source", {})[grp] = f"profiles/{tag}_summary.md: {kname[:80]}"
    json.dump(tj, open(tp, "w"), indent=1)
print(open(os.path.join(P, f"{tag}_summary.md")).read()[:3000])
