"""Instruction / stall-sample share of hash_bin_kernel phases (by source line ranges of rowsort.cu)."""
import csv, io, subprocess, sys, re
rep, kern = sys.argv[1], sys.argv[2]
src = open(sys.argv[3] if len(sys.argv) > 3 else "paper_conf_ipps_orachevkkg21_b200/csrc/rowsort.cu").read().splitlines()
def find(pat, start=0):
    for i in range(start, len(src)):
        if pat in src[i]: return i + 1
    raise SystemExit("marker not found: " + pat)
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "--kernel-name",
                      f"regex:{kern}", "--launch-count", "1"], capture_output=True, text=True).stdout
rows, fname, hdr = [], None, None
for r in csv.reader(io.StringIO(out)):
    if not r: continue
    if r[0] in ("File Path", "File Name"): fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr and r[0].isdigit():
        d = dict(zip(hdr, r))
        try: rows.append((fname, int(r[0]), float(d.get("Instructions Executed", 0) or 0), float(d.get("# Samples", 0) or 0)))
        except ValueError: pass
k0 = find("hash_bin_kernel(SegSource src")
marks = [("setup/meta", k0), ("bitmap-mode", find("if (P.mode == kPlanBitmap)", k0)), ("pre-insert", find("PROBE(1);", k0)),
         ("insert", find("const uint32_t b = __umulhi(d, M) >> l;", k0) - 3),
         ("passA", find("// ---- pass A", k0)), ("overflow", find("// ---- overflow buckets", k0)),
         ("scan", find("// ---- multi-scan", k0)), ("passB", find("// ---- pass B", k0)), ("end", find("// ---- fallback: restore", k0))]
agg = {}
ti = sum(r[2] for r in rows) or 1; ts = sum(r[3] for r in rows) or 1
for f, ln, ins, smp in rows:
    ph = "helpers(" + f + ")"
    if f == "rowsort.cu":
        if ln < k0: ph = "gather/stage helpers" if 150 < ln < 260 else "other helpers (sort, scan...)"
        else:
            for name, lo in marks:
                if ln >= lo: ph = name
    a = agg.setdefault(ph, [0, 0]); a[0] += ins; a[1] += smp
for k, (i, s) in sorted(agg.items(), key=lambda t: -t[1][0]):
    print(f"{k:32s} instr {i/ti*100:5.1f}%  samples {s/ts*100:5.1f}%")
print(f"total warp-instr {ti/1e9:.3f} G")
