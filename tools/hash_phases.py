"""Per-phase SASS instruction and stall-sample breakdown of a hash-bin kernel
from an ncu --set full --import-source capture (source view), phases by line
ranges of rowsort.cu found from markers in the source.
usage: python tools/hash_phases.py <report.ncu-rep> <products in the launch>"""
import csv, io, os, re, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src = open(os.path.join(ROOT, "paper_conf_ipps_orachevkkg21_b200/csrc/rowsort.cu")).read().split("\n")


def line_of(pat, start=0):
    for i in range(start, len(src)):
        if pat in src[i]:
            return i + 1
    raise SystemExit(f"marker not found: {pat}")


k0 = line_of("hash_bin_kernel(SegSource src")
ins = line_of("const uint32_t d = c - clo;", line_of("const uint32_t W = P.W, l = P.l, M = P.M;", k0))
pa = line_of("// ---- pass A", k0)
ov = line_of("// ---- overflow buckets", k0)
ms = line_of("// ---- multi-scan", k0)
pb = line_of("// ---- pass B", k0)
fb = line_of("// ---- fallback: restore", k0)
kend = line_of("// ---- 4c.", k0)
phases = [  # (name, lo, hi) inclusive line ranges of rowsort.cu
    ("gather (segment staging + product loads)", line_of("__device__ __forceinline__ void stage_one"), line_of("// Block scan of per-warp counts") - 1),
    ("insert (bucket, atomic slot, 16-bit store)", ins, ins + 12),
    ("pass A (16x2 sort, duplicate count, compaction)", pa, ov - 1),
    ("sort network (cswap2 / sort16x2)", line_of("__device__ __forceinline__ void cswap2"), line_of("__device__ __forceinline__ uint32_t vadd2") - 1),
    ("overflow buckets", ov, ms - 1),
    ("multi-scan", ms, pb - 1),
    ("pass B (emission, st_if)", pb, fb - 1),
    ("predicated store helper (st_if)", line_of("__device__ __forceinline__ void st_if"), line_of("__device__ __forceinline__ void st_if") + 5),
    ("row pipeline / plan / prefetch / bitmap mode", k0, ins - 1),
    ("fallback restore, row end", fb, kend),
    ("plan (make_plan)", line_of("RowPlan make_plan(const RowRec& x)") - 2, line_of("RowPlan make_plan(const RowRec& x)") + 30),
]
rep, prods = sys.argv[1], float(sys.argv[2])
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
fname, agg = None, []
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0].isdigit() and len(r) > 8:
        try:
            agg.append((fname, int(r[0]), float(r[7] or 0), float(r[4] or 0)))
        except ValueError:
            pass
te = sum(a[2] for a in agg) or 1
ts = sum(a[3] for a in agg) or 1
res = {}
for f, ln, e, w in agg:
    name = "other (" + f + ")"
    if f == "rowsort.cu":
        for nm, lo, hi in phases:
            if lo <= ln <= hi:
                name = nm
                break
    x = res.setdefault(name, [0.0, 0.0])
    x[0] += e
    x[1] += w
print(f"| phase | warp-instr | share | thread-instr / product | stall samples |")
print(f"|---|---:|---:|---:|---:|")
for k, (e, w) in sorted(res.items(), key=lambda kv: -kv[1][0]):
    print(f"| {k} | {e / 1e9:.2f} G | {e / te * 100:.1f}% | {e * 32 / prods:.1f} | {w / ts * 100:.1f}% |")
print(f"| **total** | {te / 1e9:.2f} G | 100% | {te * 32 / prods:.1f} | 100% |")
