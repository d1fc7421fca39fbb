"""Aggregate ncu per-source-line instructions / stall samples into line ranges (phases)."""
import csv, io, subprocess, sys
rep, kern, skip = sys.argv[1], sys.argv[2], sys.argv[3]
ranges = []
for a in sys.argv[4:]:  # file:lo-hi=name
    spec, nm = a.split("=")
    fn, rng = spec.split(":")
    lo, hi = rng.split("-")
    ranges.append((fn, int(lo), int(hi), nm))
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "--kernel-name",
                      f"regex:{kern}", "--launch-skip", skip, "--launch-count", "1"], capture_output=True, text=True).stdout
fname = None
agg = []
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] and r[0].isdigit():
        try:
            agg.append((float(r[7] or 0), float(r[4] or 0), fname, int(r[0])))
        except (ValueError, IndexError):
            pass
te = sum(a[0] for a in agg) or 1
tw = sum(a[1] for a in agg) or 1
print(f"total warp-instr {te/1e9:.2f}G samples {tw:.0f}")
res = {}
for e, w, f, ln in agg:
    name = "other:" + f
    for fn, lo, hi, nm in ranges:
        if f == fn and lo <= ln <= hi:
            name = nm
            break
    x = res.setdefault(name, [0, 0])
    x[0] += e
    x[1] += w
for k, (e, w) in sorted(res.items(), key=lambda kv: -kv[1][0]):
    print(f"{k:30s} instr {e/te*100:5.1f}%  ({e/1e9:6.2f}G)  stall-samples {w/tw*100:5.1f}%")
