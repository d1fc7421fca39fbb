"""Top SASS lines by stall samples / executed instructions of one kernel in an ncu report."""
import csv, subprocess, sys, io
rep, kern = sys.argv[1], sys.argv[2]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "--kernel-name",
                      f"regex:{kern}", "--launch-skip", sys.argv[5] if len(sys.argv) > 5 else "0", "--launch-count", "1"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(rows) if 'Source' in r and 'Warp Stall Sampling (All Samples)' in r][0]
h = rows[hi]
si, ei, wi = h.index('Source'), h.index('Instructions Executed'), h.index('Warp Stall Sampling (All Samples)')
data = []
for r in rows[hi + 1:]:
    try:
        e = float(r[ei] or 0); w = float(r[wi] or 0)
    except ValueError:
        continue
    data.append((e, w, r[si][:80]))
te = sum(d[0] for d in data); tw = sum(d[1] for d in data) or 1
print(f"total warp-instr {te/1e9:.2f} G, samples {tw:.0f}")
mode = sys.argv[4] if len(sys.argv) > 4 else "both"
idx = sorted(range(len(data)), key=lambda i: -data[i][1])[:n]
for i in sorted(idx):
    e, w, s = data[i]
    print(f"{i:5d} {e/1e6:9.1f}M {w/tw*100:5.1f}%  {s}")
# instruction-count heavy regions (blocks of 16)
print("--- heavy regions (by executed instructions)")
blk = 16
regs = sorted(range(0, len(data), blk), key=lambda i: -sum(d[0] for d in data[i:i + blk]))[:8]
for i in sorted(regs):
    s = sum(d[0] for d in data[i:i + blk])
    print(f"{i:5d}-{i+blk:5d} {s/te*100:5.1f}% instr  first: {data[i][2][:60]}")
