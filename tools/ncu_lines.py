"""Per-CUDA-source-line executed instructions and stall samples of one kernel (ncu cuda,sass view)."""
import csv, io, subprocess, sys
rep, kern = sys.argv[1], sys.argv[2]
skip = sys.argv[3] if len(sys.argv) > 3 else "0"
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
    if r[0] in ("Function Name", "Line No"):
        continue
    if r[0] and r[0].isdigit():
        try:
            agg.append((float(r[7] or 0), float(r[4] or 0), fname, int(r[0]), r[1][:90]))
        except (ValueError, IndexError):
            pass
te = sum(a[0] for a in agg) or 1
tw = sum(a[1] for a in agg) or 1
print(f"total warp-instr {te/1e9:.2f}G  samples {tw:.0f}")
for e, w, f, ln, src in sorted(agg, key=lambda a: -(a[0] / te + a[1] / tw))[:int(sys.argv[4]) if len(sys.argv) > 4 else 40]:
    print(f"{e/te*100:5.1f}%i {w/tw*100:5.1f}%s {f}:{ln:<4d} {src}")
